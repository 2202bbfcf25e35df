"""Copy the round's GPU evidence from gpurun_out/ into profiles/ (tracked):
bench line, ncu launch list (+ per-kernel summary), key metrics of the full
ncu capture of the dominant kernel, per-config sweeps, and traffic.json
(dram read+write bytes of the dominant kernel, read by bench.py)."""
from __future__ import annotations

import csv
import json
import shutil
import subprocess
import sys
from collections import defaultdict
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
OUT = ROOT / "gpurun_out"
PROF = ROOT / "profiles"
KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "sm__cycles_elapsed.avg.per_second",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__thread_inst_executed_per_inst_executed.ratio",
    "smsp__inst_executed.sum", "sm__warps_active.avg.pct_of_peak_sustained_active", "lts__t_sector_hit_rate.pct",
    "l1tex__t_sector_hit_rate.pct", "smsp__inst_executed_op_tma_ld.sum", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
]


def ncu_raw(rep: Path):
    txt = subprocess.run(["ncu", "-i", str(rep), "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(txt.splitlines()))
    return rows[0], rows[1], rows[2:]


def main(tag: str = "r01"):
    PROF.mkdir(exist_ok=True)
    if (OUT / "bench.json").exists():
        shutil.copy(OUT / "bench.json", PROF / f"{tag}_bench_c2.json")
    if (OUT / "bench_ref.json").exists():
        shutil.copy(OUT / "bench_ref.json", PROF / f"{tag}_bench_reference_c2.json")
    if (OUT / "launches.csv").exists():
        shutil.copy(OUT / "launches.csv", PROF / f"{tag}_ncu_launches_c2.csv")
        rows = list(csv.reader(open(OUT / "launches.csv")))
        hdr = [i for i, x in enumerate(rows) if "Kernel Name" in x][0]
        h = rows[hdr]
        ki, vi = h.index("Kernel Name"), h.index("Metric Value")
        agg = defaultdict(list)
        for x in rows[hdr + 1:]:
            if len(x) > vi:
                agg[x[ki].split("(")[0][:100]].append(float(x[vi].replace(",", "")) / 1e3)
        with open(PROF / f"{tag}_ncu_launches_c2_summary.md", "w") as f:
            f.write("# ncu launch list (gpu__time_duration.sum, --clock-control none), "
                    "`bench.py --steps 3 --warmup 1`, C2\n\n"
                    "Cold-cache, serialised per-launch times: compare SHARES with bench.py's live events.\n\n"
                    "| kernel | launches | mean us |\n|---|---|---|\n")
            for k, v in agg.items():
                f.write(f"| `{k}` | {len(v)} | {sum(v) / len(v):.1f} |\n")
    rep = OUT / "prof_c2_full.ncu-rep"
    if rep.exists():
        h, u, rows = ncu_raw(rep)
        caps = []
        for r in rows:
            caps.append({"kernel": r[h.index("Kernel Name")],
                         "metrics": {k: {"value": r[h.index(k)], "unit": u[h.index(k)]} for k in KEYS if k in h}})
        json.dump({"capture": "ncu --set full --clock-control none --import-source on, "
                              "scripts/prof_target.py --config c2 (list mode)", "launches": caps},
                  open(PROF / f"{tag}_ncu_full_c2_staged.json", "w"), indent=1)
        emit = [c for c in caps if ", 3, " in c["kernel"] or "3, 32" in c["kernel"]] or caps
        m = emit[-1]["metrics"]
        rd = float(m["dram__bytes_read.sum"]["value"]) * (1e6 if m["dram__bytes_read.sum"]["unit"] == "Mbyte" else 1e9)
        wr = float(m["dram__bytes_write.sum"]["value"]) * (1e6 if m["dram__bytes_write.sum"]["unit"] == "Mbyte" else 1e9)
        ia = float(m["smsp__issue_active.avg.pct_of_peak_sustained_active"]["value"]) / 100
        json.dump({"c2/list/k_scan_staged(emit1)": int(rd + wr),
                   "c2/list/k_scan_staged(emit1)/issue_active": round(ia, 4)}, open(PROF / "traffic.json", "w"), indent=1)
    rep = OUT / "prof_c2_list.ncu-rep"
    if rep.exists():  # the list-mode step's kernels (count scan, emitting scan, gather)
        h, u, rows = ncu_raw(rep)
        caps = [{"kernel": r[h.index("Kernel Name")],
                 "metrics": {k: {"value": r[h.index(k)], "unit": u[h.index(k)]} for k in KEYS if k in h}}
                for r in rows]
        json.dump({"capture": "ncu --set full --clock-control none --import-source on -k regex:'k_scan_staged|k_gather', "
                              "scripts/prof_target.py --config c2 --reps 2 (count scan, then list-mode steps)",
                   "launches": caps}, open(PROF / f"{tag}_ncu_list_c2.json", "w"), indent=1)
    sweeps = {}
    for p in sorted(OUT.glob("sweep_*.jsonl")):
        sweeps[p.stem] = [json.loads(l) for l in open(p) if l.strip()]
    if sweeps:
        json.dump(sweeps, open(PROF / f"{tag}_sweeps.json", "w"), indent=1)
    print("profiles updated:", sorted(x.name for x in PROF.iterdir()))


if __name__ == "__main__":
    main(*sys.argv[1:])
