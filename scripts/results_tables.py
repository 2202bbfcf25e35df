"""Print the BASELINE.md "Results" tables (markdown) from the round's evidence
in profiles/: the bench line (C3 + other_configs), the reference arm, the
C5 grid and the ncu summaries.

    python scripts/results_tables.py [tag]
"""
from __future__ import annotations

import json
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
PROF = ROOT / "profiles"


def last_json(p: Path):
    lines = [l for l in p.read_text().splitlines() if l.strip().startswith("{")]
    return json.loads(lines[-1]) if lines else None


def main(tag: str = "r02"):
    b = last_json(PROF / f"{tag}_bench.json")
    ref = last_json(PROF / f"{tag}_bench_reference.json") if (PROF / f"{tag}_bench_reference.json").exists() else None
    print(f"bench.py (N=1, {b['steps']} steps, {b['warmup']} warm-up): **{b['value']:,.0f} Gbps** on "
          f"{b['config']['workload']} ({b['ms_per_step']:.3f} ms/step), tier {b['workload_info']['tier']}, "
          f"{b['workload_info']['matches_rank0']:,} matches; SM clock {b['clocks']['sm_mhz']:.0f} MHz, "
          f"reasons {b['clocks']['reasons']}.")
    r = b["roofline"]
    print(f"Dominant kernel `{r['kernel']}`: {r['achieved']:,.0f} Glookup/s = {r['frac']:.3f} of the "
          f"{r['peak']:,.0f} Glookup/s shared-memory lookup roof; HBM {r['hbm']['achieved']:,.0f} GB/s = "
          f"{r['hbm']['frac']:.3f} of {r['hbm']['peak']:,.1f} GB/s; DRAM traffic {r['traffic']} B per launch; "
          f"binding unit (ncu): {r.get('binding_unit_ncu')}.")
    print()
    print("| kernel | ms | share of step | stream |\n|---|---|---|---|")
    for k in b["kernels"]:
        print(f"| `{k['name']}` | {k['ms']:.4f} | {k['share']:.3f} | {k['stream']} |")
    print()
    e = b.get("e2e")
    if e:
        print(f"e2e through `{e['api']}`: {e['value']:,.0f} Gbps ({e['ms_per_step']:.2f} ms/step, "
              f"{e['h2d_bytes_per_step']:,} B in, {e['d2h_bytes_per_step']:,} B out per step).")
    c = b.get("cpu_baseline")
    if c:
        print(f"CPU oracle on the box ({c['cores']} × {c.get('cpu_model')}): {c['value']:.4f} Gbps "
              f"(1 thread: {c['single_thread']['value']:.4f}).")
    if ref:
        print(f"Reference arm (`--impl reference`, the oracle on {ref['cpu_baseline']['cores']} cores): "
              f"{ref['value']:.4f} Gbps.")
    print()
    print("| config | tier | list Gbps | ms/step | lookup-roof frac | HBM frac |\n|---|---|---|---|---|---|")
    print(f"| {b['config']['config']} | {b['workload_info']['tier']} | {b['value']:,.0f} | {b['ms_per_step']:.3f} | "
          f"{r['frac']:.3f} | {r['hbm']['frac']:.3f} |")
    for cfg, v in b.get("other_configs", {}).items():
        print(f"| {cfg} | {v['workload_info']['tier']} | {v['value']:,.0f} | {v['ms_per_step']:.3f} | "
              f"{v['roofline_frac']:.3f} | {v['hbm_frac']:.3f} |")
    sw = PROF / f"{tag}_sweep_c5.json"
    if sw.exists():
        print()
        print("| point | tier | states | matches | count Gbps | list Gbps | parity |\n|---|---|---|---|---|---|---|")
        for p in json.load(open(sw)):
            lg = f"{p['list_gbps']:,.0f}" if p.get("list_gbps") else "—"
            par = p.get("parity") or p.get("parity_closed_form") or p.get("list", "")
            if p.get("parity_closed_form"):
                par = f"closed form K·n − K(K−1)/2: {p['parity_closed_form']}"
            print(f"| {p['point']} | {p['tier']} | {p['states']:,} | {p['matches']:,} | {p['count_gbps']:,.0f} | "
                  f"{lg} | {par} |")


if __name__ == "__main__":
    main(*sys.argv[1:])
