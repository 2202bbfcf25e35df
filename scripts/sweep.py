"""Variant sweep on one GPU: times the count and list passes of every staged
variant (and the global-only kernel) on a config, printing one JSON line per
setting.  Development tool -- bench.py is the contract."""
from __future__ import annotations

import argparse
import json
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_tranlhc13_b200 as ac  # noqa: E402
import synth  # noqa: E402


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
    p.add_argument("--config", default="c2")
    p.add_argument("--n", type=int, default=0)
    p.add_argument("--variants", default="1,2,3,4,5,6,7")
    p.add_argument("--tiers", default="auto")
    p.add_argument("--global-kernel", action="store_true")
    p.add_argument("--two-pass", default="0", help="list-mode placements to time: 0 single pass (block gather), "
                   "1 count+emit passes, 2 single pass via offset scan + k_gather")
    a = p.parse_args()
    w = synth.make(a.config, n=a.n or None)
    n = w.text.size
    text = torch.from_numpy(w.text).cuda()
    res = torch.zeros(2, dtype=torch.int64, device="cuda")
    tiers = {"auto": ac.TIER_AUTO, "smem": ac.TIER_SMEM, "hybrid": ac.TIER_HYBRID, "global": ac.TIER_GLOBAL,
             "compact": ac.TIER_COMPACT}
    for tname in a.tiers.split(","):
        stt = ac.build(w.patterns, tier=tiers[tname])
        cnt = ac.count(stt, text)
        out = torch.empty(max(1, cnt), dtype=torch.int64, device="cuda")
        settings = [(ac.KERNEL_STAGED, int(v), int(tp)) for v in a.variants.split(",") for tp in a.two_pass.split(",")]
        if a.global_kernel:
            settings.append((ac.KERNEL_GLOBAL, 0, 0))
        ref = None
        for kernel, v, tp in settings:
            knobs = dict(kernel=kernel, variant=v, two_pass=tp)
            try:
                ac.match_async(stt, text, None, res, **knobs)
            except ac.AcError as e:
                print(json.dumps({"config": a.config, "variant": v, "skipped": str(e)}), flush=True)
                continue
            t_count = timeit(lambda: ac.match_async(stt, text, None, res, **knobs))
            t_list = timeit(lambda: ac.match_async(stt, text, out, res, **knobs))
            torch.cuda.synchronize()
            assert int(res[0]) == cnt and int(res[1]) == 0
            h = int(torch.sum(out[:cnt] * 0x9E3779B1 % 1000003).item())
            ref = h if ref is None else ref
            print(json.dumps({"config": a.config, "n": n, "tier": stt.tier_name, "hot_rows": stt.info["hot_rows"],
                              "kernel": kernel, "variant": v, "two_pass": tp, "count_ms": round(t_count, 4),
                              "list_ms": round(t_list, 4), "count_gbps": round(n * 8 / t_count / 1e6, 1),
                              "list_gbps": round(n * 8 / t_list / 1e6, 1), "matches": cnt,
                              "same_list": h == ref}), flush=True)
        del stt


if __name__ == "__main__":
    main()
