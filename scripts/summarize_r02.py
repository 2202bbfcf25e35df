"""Copy the round's GPU evidence from gpurun_out/full/ into profiles/ (tracked):
the bench and reference-arm lines, the ncu launch list of the bench command
(+ per-kernel summary), key metrics of the full ncu capture of each config's
list-mode scan, the C5 grid, and traffic.json (DRAM bytes read + written per
launch and the binding unit of each dominant kernel, read by bench.py).

    python scripts/summarize_r02.py [tag]      # default tag r02
"""
from __future__ import annotations

import csv
import json
import shutil
import subprocess
import sys
from collections import defaultdict
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
OUT = ROOT / "gpurun_out" / "full"
PROF = ROOT / "profiles"
KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "sm__cycles_elapsed.avg.per_second",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "l1tex__m_xbar2l1tex_read_sectors_mem_global_op_tma_ld.sum",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__thread_inst_executed_per_inst_executed.ratio",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed_op_tma_ld.sum",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "sm__cycles_active.avg", "sm__cycles_active.max",
    "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
]
# unit utilisations compared to name the one that binds the kernel
UNITS = {
    "SM issue (warp instructions)": "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "shared-memory wavefronts": "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "L1TEX": "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "L2": "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "DRAM": "dram__throughput.avg.pct_of_peak_sustained_elapsed",
}


def ncu_raw(rep: Path):
    raw = rep.with_suffix(".raw.csv")
    if raw.exists() and raw.stat().st_size:
        txt = raw.read_text()
    else:
        txt = subprocess.run(["ncu", "-i", str(rep), "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(txt.splitlines()))
    return rows[0], rows[1], rows[2:]


def to_bytes(v: str, unit: str) -> float:
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    return float(v.replace(",", "")) * scale.get(unit, 1)


def last_json(p: Path):
    lines = [l for l in p.read_text().splitlines() if l.strip().startswith("{")]
    return json.loads(lines[-1]) if lines else None


def main(tag: str = "r02"):
    PROF.mkdir(exist_ok=True)
    for src, dst in (("bench.json", f"{tag}_bench.json"), ("bench_ref.json", f"{tag}_bench_reference.json"),
                     ("pytest_gpu.log", f"{tag}_gpu_tests.log"), ("host.txt", f"{tag}_host.txt"),
                     ("gpu.txt", f"{tag}_gpu.txt"),
                     *[(f"sanitize_{t}.log", f"{tag}_sanitize_{t}.log")
                       for t in ("memcheck", "racecheck", "synccheck", "initcheck")]):
        if (OUT / src).exists():
            shutil.copy(OUT / src, PROF / dst)
    if (OUT / "launches.csv").exists():
        shutil.copy(OUT / "launches.csv", PROF / f"{tag}_ncu_launches.csv")
        rows = list(csv.reader(open(OUT / "launches.csv")))
        hdr = [i for i, x in enumerate(rows) if "Kernel Name" in x][0]
        h = rows[hdr]
        ki, vi = h.index("Kernel Name"), h.index("Metric Value")
        agg = defaultdict(list)
        for x in rows[hdr + 1:]:
            if len(x) > vi:
                agg[x[ki].split("(")[0][:100]].append(float(x[vi].replace(",", "")) / 1e3)
        tot = sum(sum(v) for v in agg.values())
        with open(PROF / f"{tag}_ncu_launches_summary.md", "w") as f:
            f.write("# ncu launch list (gpu__time_duration.sum, --clock-control none) of "
                    "`bench.py --steps 3 --warmup 1 --no-e2e --no-cpu-baseline --extra ''` (C3)\n\n"
                    "Cold-cache, serialised per-launch times (the build and warm-up launches included): "
                    "compare SHARES with bench.py's live events.\n\n"
                    "| kernel | launches | mean us | share of listed time |\n|---|---|---|---|\n")
            for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
                f.write(f"| `{k}` | {len(v)} | {sum(v) / len(v):.1f} | {sum(v) / tot:.3f} |\n")
    traffic = {}
    for cfg in ("c3", "c2", "c4"):
        rep = OUT / f"prof_{cfg}_list.ncu-rep"
        if not rep.exists() and not rep.with_suffix(".raw.csv").exists():
            continue
        h, u, rows = ncu_raw(rep)
        r = rows[-1]
        m = {k: {"value": r[h.index(k)], "unit": u[h.index(k)]} for k in KEYS if k in h}
        util = {name: float(r[h.index(k)].replace(",", "")) for name, k in UNITS.items() if k in h}
        bind = max(util, key=util.get)
        json.dump({"capture": f"ncu --set full --clock-control none --import-source on -k regex:k_scan_staged "
                              f"-s 1 -c 1, scripts/prof_target.py --config {cfg} --mode list (the list-mode scan)",
                   "kernel": r[h.index("Kernel Name")], "metrics": m,
                   "unit_utilisation_pct": util, "binding_unit": bind},
                  open(PROF / f"{tag}_ncu_full_{cfg}_list.json", "w"), indent=1)
        rd = to_bytes(m["dram__bytes_read.sum"]["value"], m["dram__bytes_read.sum"]["unit"])
        wr = to_bytes(m["dram__bytes_write.sum"]["value"], m["dram__bytes_write.sum"]["unit"])
        traffic[f"{cfg}/list/k_scan_staged(emit1)"] = int(rd + wr)
        traffic[f"{cfg}/list/k_scan_staged(emit1)/binding"] = f"{bind} {util[bind]:.0f}% (ncu, {tag})"
    if traffic:
        json.dump(traffic, open(PROF / "traffic.json", "w"), indent=1)
    if (OUT / "sweep_c5.jsonl").exists():
        pts = [json.loads(l) for l in open(OUT / "sweep_c5.jsonl") if l.strip().startswith("{")]
        json.dump(pts, open(PROF / f"{tag}_sweep_c5.json", "w"), indent=1)
    print("profiles updated:", sorted(x.name for x in PROF.iterdir()))


if __name__ == "__main__":
    main(*sys.argv[1:])
