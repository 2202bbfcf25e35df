"""C5 sweep on one GPU (BASELINE.json configs[4]): dictionary size x text size for the
English-like (C2) and Snort-like (C3) families, plus the high-match-rate adversarial texts.
One JSON line per point: count and list Gbps (CUDA events, text resident, STT built),
tier, states, matches, and a parity verdict against the CPU oracle (test infrastructure,
oracle/): the full count plus the multiset digest of the whole list (oracle windows on every
host core) up to --digest-max bytes of text, sampled windows beyond -- or the closed form
K*n - K(K-1)/2 for a^n with {a^1..a^K}, whose list does not fit in memory.
Development tool, like sweep.py; bench.py is the contract.

    python scripts/sweep_c5.py [--logn 26,28,30,34] [--patterns 1000,5000,10000,20000,50000]
                               [--big english-1000,snort-10000,adv-a]
"""
from __future__ import annotations

import argparse
import json
import sys
import time
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_tranlhc13_b200 as ac  # noqa: E402
import synth  # noqa: E402
from oracle import Oracle  # noqa: E402

sys.path.insert(0, str(ROOT / "tests"))
from test_gpu_parity import digest_keys_torch  # noqa: E402

DIGEST_MAX = 1 << 34


def timeit(fn, reps=5, warm=2):
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


def windows_ok(pats, text_np, recs, k=4, width=1 << 16, seed=7):
    """Oracle windows (first, last, random) against the device list `recs`."""
    o = Oracle(pats)
    n = text_np.size
    rng = np.random.default_rng(seed)
    los = [0, max(0, n - width)] + rng.integers(0, max(1, n - width), size=k - 2).tolist()
    s = recs >> 24
    for lo in los:
        hi = min(n, lo + width)
        ends, pids = o.match_window(text_np, lo, hi)
        want = ((ends.astype(np.int64) - o.lens[pids].astype(np.int64) + 1) << 24) | pids.astype(np.int64)
        a = int(torch.searchsorted(s, torch.tensor([lo], device=s.device)))
        b = int(torch.searchsorted(s, torch.tensor([hi], device=s.device)))
        if not np.array_equal(recs[a:b].cpu().numpy(), want):
            return False
    return True


def point(label, pats, text_np, list_budget=64 << 30, closed_form=None):
    t0 = time.time()
    stt = ac.build(pats)
    build_s = time.time() - t0
    text = torch.from_numpy(text_np).cuda()
    n = text_np.size
    res = torch.zeros(2, dtype=torch.int64, device="cuda")
    cnt = ac.count(stt, text)
    t_count = timeit(lambda: ac.match_async(stt, text, None, res))
    line = {"point": label, "n": n, "patterns": len(pats), "tier": stt.tier_name, "states": stt.info["n_states"],
            "classes": stt.info["n_classes"], "build_s": round(build_s, 2), "matches": cnt,
            "count_ms": round(t_count, 4), "count_gbps": round(n * 8 / t_count / 1e6, 1)}
    if cnt * 8 <= list_budget:
        out = torch.empty(max(1, cnt), dtype=torch.int64, device="cuda")
        t_list = timeit(lambda: ac.match_async(stt, text, out, res))
        assert int(res[0]) == cnt and int(res[1]) == 0
        line.update(list_ms=round(t_list, 4), list_gbps=round(n * 8 / t_list / 1e6, 1))
        recs = out[:cnt]
        if n <= DIGEST_MAX:
            # the list's digest on the device (test side), the oracle's on every host core
            t0 = time.time()
            ok = digest_keys_torch(recs) == Oracle(pats).digest_parallel(text_np)
            line["parity"] = f"whole-text count + digest ({time.time() - t0:.0f} s): " + ("ok" if ok else "MISMATCH")
        else:
            line["parity"] = ("oracle windows: ok" if windows_ok(pats, text_np, recs) else "oracle windows: MISMATCH")
        del out, recs
    else:
        line["list"] = f"skipped: {cnt} records > list budget"
    if closed_form is not None:
        line["parity_closed_form"] = "ok" if cnt == closed_form else f"MISMATCH (want {closed_form})"
    del text
    torch.cuda.empty_cache()
    print(json.dumps(line), flush=True)


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--logn", default="26,28")
    p.add_argument("--patterns", default="1000,5000,20000,50000")
    p.add_argument("--families", default="english,snort,adv")
    p.add_argument("--digest-max", type=int, default=DIGEST_MAX)
    p.add_argument("--big", default="english-1000,snort-10000,adv-a", help="points at log2 n > 30")
    a = p.parse_args()
    globals()["DIGEST_MAX"] = a.digest_max
    Ps = [int(x) for x in a.patterns.split(",")]
    fams = a.families.split(",")
    for logn in [int(x) for x in a.logn.split(",")]:
        n = 1 << logn
        if logn > 30:
            # 4-16 GiB texts: the dictionaries named by --big only (one oracle
            # digest over 16 GiB takes minutes on the host)
            for item in a.big.split(","):
                fam, P = item.split("-")
                if fam == "english":
                    voc = synth.english_vocabulary(5002)
                    text = synth.text_english(n, 5000, voc)
                    # the same dictionary as the smaller texts: substrings of their first 1 GiB
                    point(f"c5-english-{P}-{logn}", synth.patterns_substrings(text[:1 << 30], int(P), 4, 32, 5001),
                          text)
                elif fam == "snort":
                    pats = synth.patterns_snort(int(P), 5011)
                    text = synth.text_payload(n, 5010, pats)
                    point(f"c5-snort-{P}-{logn}", pats, text)
                elif fam == "adv" and P == "a":
                    w = synth.make(f"c5-adv-a-{logn}")
                    K = len(w.patterns)
                    point(f"c5-adv-a-{logn}", w.patterns, w.text, closed_form=K * n - K * (K - 1) // 2)
                    text = w.text
                del text
            continue
        if "english" in fams:
            voc = synth.english_vocabulary(5002)
            text = synth.text_english(n, 5000, voc)
            for P in Ps:
                point(f"c5-english-{P}-{logn}", synth.patterns_substrings(text, P, 4, 32, 5001), text)
            del text
        if "snort" in fams:
            for P in Ps:
                pats = synth.patterns_snort(P, 5011)
                point(f"c5-snort-{P}-{logn}", pats, synth.text_payload(n, 5010, pats))
    if "adv" in fams:
        n = 1 << 28
        w = synth.make("c5-adv-a-28")
        K = len(w.patterns)
        point("c5-adv-a-28", w.patterns, w.text, closed_form=K * n - K * (K - 1) // 2)
        w = synth.make("c5-adv-p-28")
        point("c5-adv-p-28", w.patterns, w.text)


if __name__ == "__main__":
    main()
