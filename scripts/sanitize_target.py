"""Small compute-sanitizer target: every scan kernel on small inputs, list and
count modes, checked against the oracle.  Run under
``compute-sanitizer --tool {memcheck,racecheck,synccheck,initcheck}``
(scripts/gpu_sanitize.sh); the logs go to profiles/.

Covers the staged kernel's mbarrier rings and TMA loads, its in-kernel
look-back (a ticketed decoupled look-back across CTAs, P:216 is the paper's
synchronisation step), the SMEM / COMPACT / SPLIT / GLOBAL tiers, k_offsets,
k_gather (record copy and EVENTS expansion), k_rewalk and the packet-batch
kernel."""
from __future__ import annotations

import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parents[1]
sys.path.insert(0, str(ROOT))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_tranlhc13_b200 as ac  # noqa: E402
import synth  # noqa: E402
from oracle import Oracle  # noqa: E402


def keys(o, text):
    ends, pids = o.match(text)
    starts = ends.astype(np.int64) - o.lens[pids].astype(np.int64) + 1
    return (starts << 24) | pids.astype(np.int64)


def check(name, stt, o, text_np, **kw):
    t = torch.from_numpy(np.ascontiguousarray(text_np)).cuda()
    want = keys(o, text_np)
    c, recs = ac.match(stt, t, **kw)
    assert c == want.size and np.array_equal(recs.cpu().numpy(), want), name
    assert ac.count(stt, t, **{k: v for k, v in kw.items() if k in ("kernel", "chain_bytes", "variant")}) == c
    print(f"ok {name}: {c} matches, tier {stt.tier_name}, launches {ac.last_launch_names()}", flush=True)


def main():
    w = synth.make("c1", n=(1 << 18) + 77)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    check("c1 global", stt, o, w.text)
    check("c1 staged", stt, o, w.text, kernel=ac.KERNEL_STAGED, chain_bytes=256)
    check("c1 staged overflow", stt, o, w.text, kernel=ac.KERNEL_STAGED, chain_bytes=256, scratch_slots=2)
    check("c1 staged two-pass", stt, o, w.text, kernel=ac.KERNEL_STAGED, chain_bytes=256, two_pass=True)

    w = synth.make("c2", n=(1 << 20) + 5, n_patterns=1000)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)  # COMPACT
    check("c2 compact staged", stt, o, w.text, kernel=ac.KERNEL_STAGED, chain_bytes=256)
    check("c2 compact staged k_offsets", stt, o, w.text, kernel=ac.KERNEL_STAGED, chain_bytes=256, two_pass=2)

    w = synth.make("c3", n=(1 << 20) + 9)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)  # SPLIT
    check("c3 split staged", stt, o, w.text, kernel=ac.KERNEL_STAGED, chain_bytes=256)
    check("c3 global-only", stt, o, w.text, kernel=ac.KERNEL_GLOBAL)
    check("c3 split staged events", stt, o, w.text, kernel=ac.KERNEL_STAGED, chain_bytes=256, two_pass=4)

    # dense outputs: the EVENTS single pass (GLOBAL tier, 32-bit table) and the
    # SPLIT two-pass re-walk with emit_coop
    voc = synth.english_vocabulary(5002)
    text = synth.text_english((1 << 18) + 11, 5000, voc)
    pats = synth.patterns_substrings(text, 5000, 4, 32, 5001)
    o = Oracle(pats)
    stt = ac.build(pats)
    check("english5k events", stt, o, text, kernel=ac.KERNEL_STAGED, chain_bytes=256, two_pass=4)
    stt = ac.build(pats, tier=ac.TIER_SPLIT)
    check("english5k split two-pass", stt, o, text, kernel=ac.KERNEL_STAGED, chain_bytes=256, two_pass=True)

    w = synth.make("c4", n=(1 << 20) + 3)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)  # GLOBAL + two-byte walk
    check("c4 stride2 staged", stt, o, w.text, kernel=ac.KERNEL_STAGED, chain_bytes=256)

    # packet batches
    w = synth.make("c1", n=(1 << 16) + 1)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    cuts = np.unique(np.concatenate([[0, w.text.size], np.random.default_rng(3).integers(0, w.text.size, 200)]))
    want = np.concatenate([keys(o, w.text[a:b]) + (a << 24) for a, b in zip(cuts[:-1], cuts[1:])])
    c, recs = ac.match_segments(stt, torch.from_numpy(w.text).cuda(),
                                torch.from_numpy(cuts.astype(np.int64)).cuda())
    assert c == want.size and np.array_equal(recs.cpu().numpy(), want)
    print(f"ok segments: {c} matches", flush=True)
    torch.cuda.synchronize()
    print("SANITIZE TARGET DONE", flush=True)


if __name__ == "__main__":
    main()
