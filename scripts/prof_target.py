"""Small ncu target: one config, a few list-mode (or count) scans.

    ncu ... python scripts/prof_target.py --config c2 --reps 2
"""
from __future__ import annotations

import argparse
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))

import torch  # noqa: E402

import paper_conf_ipps_tranlhc13_b200 as ac  # noqa: E402
import synth  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="c2")
    p.add_argument("--n", type=int, default=0)
    p.add_argument("--reps", type=int, default=2)
    p.add_argument("--mode", default="list")
    p.add_argument("--variant", type=int, default=0)
    p.add_argument("--kernel", type=int, default=0)
    a = p.parse_args()
    w = synth.make(a.config, n=a.n or None)
    stt = ac.build(w.patterns)
    text = torch.from_numpy(w.text).cuda()
    res = torch.zeros(2, dtype=torch.int64, device="cuda")
    cnt = ac.count(stt, text, variant=a.variant, kernel=a.kernel)
    out = torch.empty(max(1, cnt), dtype=torch.int64, device="cuda") if a.mode == "list" else None
    for _ in range(a.reps):
        ac.match_async(stt, text, out, res, variant=a.variant, kernel=a.kernel)
    torch.cuda.synchronize()
    print("matches", int(res[0]), "status", int(res[1]), "tier", stt.tier_name, "launches", ac.last_launch_names())


if __name__ == "__main__":
    main()
