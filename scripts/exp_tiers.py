"""Tier experiment on one GPU: count-mode scan time of the staged kernel for
several dictionaries and STT tiers (development tool; bench.py is the
contract).  One JSON line per (workload, tier, variant)."""
from __future__ import annotations

import argparse
import json
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))

import torch  # noqa: E402

import paper_conf_ipps_tranlhc13_b200 as ac  # noqa: E402
import synth  # noqa: E402

TIERS = {"auto": ac.TIER_AUTO, "global": ac.TIER_GLOBAL, "split": ac.TIER_SPLIT, "compact": ac.TIER_COMPACT}


def timeit(fn, reps=10, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--workloads", default="c3")
    p.add_argument("--n", type=int, default=1 << 28)
    p.add_argument("--tiers", default="global,split")
    p.add_argument("--variants", default="0")
    p.add_argument("--list", action="store_true")
    p.add_argument("--exact-cap", action="store_true", help="list buffer of exactly count records")
    p.add_argument("--policies", default="0", help="text L2 policies (0 auto, 1 evict-normal, 2 evict-first)")
    p.add_argument("--two-pass", default="0", help="ac_match_opts.two_pass values to time (0 auto, 1 two passes, 4 events)")
    a = p.parse_args()
    for name in a.workloads.split(","):
        w = synth.make(name, n=a.n)
        n = w.text.size
        text = torch.from_numpy(w.text).cuda()
        res = torch.zeros(2, dtype=torch.int64, device="cuda")
        for tname in a.tiers.split(","):
            try:
                stt = ac.build(w.patterns, tier=TIERS[tname])
            except ac.AcError as e:
                print(json.dumps({"workload": name, "tier": tname, "skipped": str(e)}), flush=True)
                continue
            cap = ac.count(stt, text) if a.exact_cap else n // 8 + 64
            out = torch.empty(max(1, cap), dtype=torch.int64, device="cuda") if a.list else None
            for v, pol, tpm in [(v, pol, tpm) for v in a.variants.split(",") for pol in a.policies.split(",")
                                for tpm in a.two_pass.split(",")]:
                tpol, prom, win = (pol + ":0:0").split(":")[:3]  # text policy[:promotion[:L2 window MiB]]
                knobs = dict(kernel=ac.KERNEL_STAGED, variant=int(v), text_policy=int(tpol), text_promotion=int(prom),
                             l2_window_mib=int(win), two_pass=int(tpm))
                try:
                    ac.match_async(stt, text, out, res, **knobs)
                except ac.AcError as e:
                    print(json.dumps({"workload": name, "tier": tname, "variant": v, "skipped": str(e)}), flush=True)
                    continue
                t = timeit(lambda: ac.match_async(stt, text, out, res, **knobs))
                print(json.dumps({"workload": name, "n": n, "tier": stt.tier_name, "variant": int(v),
                                  "policy": pol, "two_pass": int(tpm), "list": bool(a.list),
                                  "exact_cap": bool(a.exact_cap),
                                  "states": stt.info["n_states"], "split_dense": stt.info["split_dense"],
                                  "split_records": stt.info["split_records"], "ms": round(t, 4),
                                  "gbps": round(n * 8 / t / 1e6, 1), "matches": int(res[0]),
                                  "names": ac.last_launch_names()}), flush=True)
            del stt
        del text


if __name__ == "__main__":
    main()
