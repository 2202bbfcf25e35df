"""GPU parity: libac's sm_100a scan against the CPU oracle, record by record.

Bar: bit-exact -- identical canonical lists (start, pattern) and counts
(integer work).  Inputs are the seeded synthetic workloads of synth/, at
oracle-sized scales that still span many CTA tiles and ragged tails, plus the
full BASELINE.json sizes in the launch configuration bench.py times, checked
on sampled windows (oracle.match_window) and closed forms.
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import paper_conf_ipps_tranlhc13_b200 as ac
import synth
from oracle import Oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    ac.build_library()
    ac.lib()


def oracle_keys(o: Oracle, text, lo=None, hi=None) -> np.ndarray:
    if lo is None:
        ends, pids = o.match(text)
    else:
        ends, pids = o.match_window(text, lo, hi)
    starts = ends.astype(np.int64) - o.lens[pids].astype(np.int64) + 1
    return (starts << 24) | pids.astype(np.int64)


def gpu_keys(stt, text_np: np.ndarray, **kw) -> np.ndarray:
    if not text_np.size:
        t = torch.empty(0, dtype=torch.uint8, device="cuda")
    else:
        # read-only views (np.frombuffer) are copied: torch.from_numpy wants a writable array
        a = text_np if text_np.flags.writeable and text_np.flags.c_contiguous else np.array(text_np, order="C")
        t = torch.from_numpy(a).cuda()
    c, recs = ac.match(stt, t, **kw)
    cnt = ac.count(stt, t, **{k: v for k, v in kw.items() if k in ("kernel", "chain_bytes", "variant")})
    if c:  # the two-pass list mode and a forced-overflow single pass agree bit for bit
        _, r2 = ac.match(stt, t, two_pass=True, **kw)
        _, r3 = ac.match(stt, t, scratch_slots=2, **kw)  # most chains overflow -> k_rewalk
        _, r4 = ac.match(stt, t, two_pass=2, **kw)  # single pass with the separate offset scan
        _, r5 = ac.match(stt, t, two_pass=3, **kw)  # single pass with wide scratch records
        _, r6 = ac.match(stt, t, two_pass=4, **kw)  # EVENTS single pass (32-bit tables; else as auto)
        assert torch.equal(r2, recs) and torch.equal(r3, recs) and torch.equal(r4, recs) and torch.equal(r5, recs)
        assert torch.equal(r6, recs)
    assert cnt == c
    return recs.cpu().numpy()


def assert_same(got: np.ndarray, want: np.ndarray):
    assert got.shape == want.shape, (got.shape, want.shape)
    if got.size:
        bad = np.nonzero(got != want)[0]
        assert bad.size == 0, f"first mismatch at {bad[0]}: got {got[bad[0]]:#x} want {want[bad[0]]:#x}"


KERNELS = [ac.KERNEL_STAGED, ac.KERNEL_GLOBAL]


# ----------------------------------------------------------------- examples
def test_worked_example():
    pats = [b"he", b"she", b"his", b"hers"]
    stt = ac.build(pats)
    for k in KERNELS:
        got = gpu_keys(stt, np.frombuffer(b"ushers", np.uint8), kernel=k)
        # she@1, he@2, hers@2 (north_star)
        assert [(int(x) >> 24, pats[int(x) & 0xFFFFFF]) for x in got] == [(1, b"she"), (2, b"he"), (2, b"hers")]
        e = ac.ends(torch.from_numpy(got), stt.lens).tolist()
        assert e == [3, 3, 5]


# ---------------------------------------------------------- configs (scaled)
@pytest.mark.parametrize("kernel", KERNELS)
def test_c1_full(kernel):
    w = synth.make("c1")
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    assert stt.tier_name == "smem"
    assert_same(gpu_keys(stt, w.text, kernel=kernel), oracle_keys(o, w.text))


@pytest.mark.parametrize("name,n", [("c2", 3 << 20), ("c3", 1 << 20), ("c4", 3 << 20)])
@pytest.mark.parametrize("kernel", KERNELS)
def test_configs_scaled(name, n, kernel):
    w = synth.make(name, n=n + 12345)  # ragged tail
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    assert_same(gpu_keys(stt, w.text, kernel=kernel), oracle_keys(o, w.text))


@pytest.mark.parametrize("tier,hot,eb", [(ac.TIER_SMEM, 0, 2), (ac.TIER_HYBRID, 37, 2), (ac.TIER_GLOBAL, 0, 2),
                                         (ac.TIER_SMEM, 0, 4), (ac.TIER_HYBRID, 5, 4), (ac.TIER_GLOBAL, 0, 4)])
def test_tiers_and_widths(tier, hot, eb):
    w = synth.make("c2", n=(1 << 20) + 77, n_patterns=60)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns, tier=tier, hot_rows=hot, entry_bytes=eb)
    assert stt.info["tier"] == tier and stt.info["entry_bytes"] == eb
    want = oracle_keys(o, w.text)
    for k in KERNELS:
        assert_same(gpu_keys(stt, w.text, kernel=k), want)


@pytest.mark.parametrize("variant", [0, 4, 7, 11])
@pytest.mark.parametrize("name,n,P", [("c2", 3 << 20, None), ("c1", 1 << 20, None), ("c2", 1 << 20, 60)])
def test_compact_tier(name, n, P, variant):
    w = synth.make(name, n=n + 999, n_patterns=P)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns, tier=ac.TIER_COMPACT)
    assert stt.tier_name == "compact"
    want = oracle_keys(o, w.text)
    try:
        got = gpu_keys(stt, w.text, kernel=ac.KERNEL_STAGED, variant=variant)
    except ac.AcError as e:  # a fat-ring variant cannot hold a big COMPACT table
        assert variant != 0 and "no room" in str(e) and stt.info["compact_bytes"] > 150_000
        return
    assert_same(got, want)
    if variant == 0:
        assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_GLOBAL), want)


@pytest.mark.parametrize("P,tier", [(1000, ac.TIER_AUTO), (5000, ac.TIER_AUTO), (5000, ac.TIER_SPLIT),
                                    (20000, ac.TIER_AUTO), (20000, ac.TIER_GLOBAL)])
def test_dense_outputs_english(P, tier):
    """C5 English dictionaries: 0.26-5.2 matches per byte, up to 78 patterns
    per output state -- the two-pass emission with the warp-cooperative
    writes of multi-output states (emit_coop) in every tier the family lands
    in (COMPACT 1K, GLOBAL 5K, SPLIT 20K), record by record."""
    voc = synth.english_vocabulary(5002)
    text = synth.text_english((2 << 20) + 4321, 5000, voc)
    pats = synth.patterns_substrings(text, P, 4, 32, 5001)
    o = Oracle(pats)
    stt = ac.build(pats, tier=tier)
    want = oracle_keys(o, text)
    assert want.size > text.size // 5
    assert_same(gpu_keys(stt, text, kernel=ac.KERNEL_STAGED), want)
    # one record short: the capacity status and the needed count, nothing written
    t = torch.from_numpy(text).cuda()
    out = torch.full((want.size - 1,), -1, dtype=torch.int64, device="cuda")
    for tp in (0, 1, 4):
        with pytest.raises(ac.CapacityError) as ei:
            ac.match(stt, t, out, two_pass=tp)
        assert ei.value.count == want.size
    assert bool((out == -1).all())


@pytest.mark.parametrize("tier", [ac.TIER_SMEM, ac.TIER_GLOBAL])
def test_saturated_output_counts(tier):
    """70,000 copies of one pattern (reading R5: every id reported): |output|
    exceeds the 16-bit row count (0xFFFF -> CSR offsets) and one event expands
    into more records than a gather chunk's rounds hold; every emission mode
    (gpu_keys: auto, two passes, overflow re-walk, EVENTS) against the oracle."""
    pats = [b"ab"] * 70000 + [b"b", b"zab"]
    rng = np.random.default_rng(5)
    text = rng.choice(np.frombuffer(b"abz", np.uint8), size=(1 << 12) + 3)
    o = Oracle(pats)
    stt = ac.build(pats, tier=tier)
    assert stt.info["entry_bytes"] == 2 and stt.info["tier"] == tier
    want = oracle_keys(o, text)
    assert want.size > 70000 * 100
    assert_same(gpu_keys(stt, text, kernel=ac.KERNEL_STAGED), want)
    assert_same(gpu_keys(stt, text, kernel=ac.KERNEL_GLOBAL), want)


def test_compact_is_auto_for_c2():
    w = synth.make("c2", n=1 << 20)
    stt = ac.build(w.patterns)
    assert stt.tier_name == "compact" and stt.info["n_states"] > 15000


def test_compact_edge_cases():
    pats = [b"he", b"she", b"his", b"hers", b"\x00\x00", b"a" * 40, b"ab" * 10]
    o = Oracle(pats)
    stt = ac.build(pats, tier=ac.TIER_COMPACT)
    rng = np.random.default_rng(9)
    text = rng.choice(np.frombuffer(b"hersia\x00b", np.uint8), size=(1 << 20) + 3)
    text[5000:5040] = ord("a")
    for k in KERNELS:
        assert_same(gpu_keys(stt, text, kernel=k), oracle_keys(o, text))


@pytest.mark.parametrize("variant", [0, 4, 7, 3])
def test_stride2_dna(variant):
    """NEXT-4: two bytes per lookup -- matches at odd and even offsets,
    middle and final positions, chains and halos of both parities."""
    pats = [b"A", b"AC", b"CAG", b"GTTA", b"T" * 9, b"ACGTACGTAC", b"NN", b"GATTACA"]
    o = Oracle(pats)
    stt = ac.build(pats, tier=ac.TIER_GLOBAL, entry_bytes=4, stride=2)
    assert stt.info["stride"] == 2
    rng = np.random.default_rng(21)
    text = np.frombuffer(b"ACGT", np.uint8)[rng.integers(0, 4, size=(1 << 20) + 7)].copy()
    text[1000:1010] = ord("T")
    text[77777:77784] = np.frombuffer(b"GATTACA", np.uint8)
    text[5:7] = ord("N")
    want = oracle_keys(o, text)
    got = gpu_keys(stt, text, kernel=ac.KERNEL_STAGED, variant=variant)
    assert_same(got, want)
    assert_same(gpu_keys(stt, text, kernel=ac.KERNEL_STAGED, variant=variant, chain_bytes=80), want)
    assert_same(gpu_keys(stt, text, kernel=ac.KERNEL_STAGED, stride=1), want)


def test_stride2_is_auto_for_c4():
    w = synth.make("c4", n=(2 << 20) + 3)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    assert stt.tier_name == "global" and stt.info["stride"] == 2
    assert_same(gpu_keys(stt, w.text), oracle_keys(o, w.text))


def test_c3_hybrid_and_global_tiers():
    w = synth.make("c3", n=(1 << 20) + 5)
    o = Oracle(w.patterns)
    want = oracle_keys(o, w.text)
    assert ac.build(w.patterns).tier_name == "split"  # AUTO for a 131K-state byte dictionary
    for tier in (ac.TIER_AUTO, ac.TIER_HYBRID, ac.TIER_GLOBAL, ac.TIER_SPLIT):
        stt = ac.build(w.patterns, tier=tier)
        assert_same(gpu_keys(stt, w.text), want)
        assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_STAGED), want)


# SPLIT tier: hot rows + records in shared memory, cold states via L1/L2
@pytest.mark.parametrize("name,n,P", [("c3", (3 << 20) + 11, None), ("c5-english-5000-22", None, None),
                                      ("c5-english-20000-22", None, None), ("c1", (1 << 20) + 3, None),
                                      ("c5-snort-1000-21", None, None)])
def test_split_tier(name, n, P):
    w = synth.make(name, n=n, n_patterns=P)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns, tier=ac.TIER_SPLIT)
    assert stt.tier_name == "split" and stt.info["entry_bytes"] == 4 and stt.info["split_bytes"] > 0
    want = oracle_keys(o, w.text)
    assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_STAGED), want)
    assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_STAGED, chain_bytes=112), want)
    assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_GLOBAL), want)


def test_split_tier_escapes_and_cold_records():
    # a 50K-pattern English dictionary (624K states): children ids past 32766
    # (escaped entries) and states with more than four children (cold
    # records) -- both must fall back to the global table
    w = synth.make("c5-english-50000-22")
    stt = ac.build(w.patterns, tier=ac.TIER_SPLIT)
    T = ac.compile_table(w.patterns, split=True)
    assert T.info["split_cold_records"] > 0
    o = Oracle(w.patterns)
    assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_STAGED), oracle_keys(o, w.text))


@pytest.mark.parametrize("variant", [1, 3, 4, 7, 9, 10, 11])
def test_split_tier_variants(variant):
    # a smaller byte dictionary so the split part also fits the fat-ring variants
    w = synth.make("c3", n=(2 << 20) + 4321, n_patterns=1500)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns, tier=ac.TIER_SPLIT)
    want = oracle_keys(o, w.text)
    assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_STAGED, variant=variant), want)


@pytest.mark.parametrize("variant", [1, 2, 3, 4, 5, 6, 7, 8, 9, 10, 11])
@pytest.mark.parametrize("name,tier", [("c1", ac.TIER_AUTO), ("c2", ac.TIER_GLOBAL), ("c2s", ac.TIER_COMPACT)])
def test_staged_variants(variant, name, tier):
    P = {"c1": None, "c2": 400, "c2s": 80}[name]
    w = synth.make(name[:2], n=(2 << 20) + 4321, n_patterns=P)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns, tier=tier)
    want = oracle_keys(o, w.text)
    assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_STAGED, variant=variant), want)
    assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_STAGED, variant=variant, chain_bytes=96), want)


@pytest.mark.parametrize("chain", [64, 128, 320, 1024, 4096, 65536])
def test_chunking_invariance_staged(chain):
    w = synth.make("c2", n=(2 << 20) + 999, n_patterns=300)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_STAGED, chain_bytes=chain), oracle_keys(o, w.text))


def test_in_kernel_offsets_more_ctas_than_sms():
    # 16-byte chains over 8 MiB: 512 staged CTAs (> 148 SMs, not all
    # co-resident) chain their totals through the in-kernel look-back; a
    # ragged tail of 13 bytes goes to the side-stream kernel
    w = synth.make("c1", n=(8 << 20) + 13)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_STAGED, variant=4, chain_bytes=16), oracle_keys(o, w.text))


@pytest.mark.parametrize("chain", [1, 7, 16, 64, 1000, 1 << 20])
def test_chunking_invariance_global(chain):
    w = synth.make("c1", n=(1 << 18) + 3)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    assert_same(gpu_keys(stt, w.text, kernel=ac.KERNEL_GLOBAL, chain_bytes=chain), oracle_keys(o, w.text))


# --------------------------------------------------------------- edge cases
def test_empty_and_short_texts():
    pats = [b"abc", b"b", b"abcdefgh"]
    o = Oracle(pats)
    stt = ac.build(pats)
    for t in [b"", b"a", b"b", b"ab", b"abc", b"abcdefg", b"abcdefgh"]:
        arr = np.frombuffer(t, np.uint8)
        for k in KERNELS:
            assert_same(gpu_keys(stt, arr, kernel=k), oracle_keys(o, arr))


def test_boundary_straddling_everywhere():
    rng = np.random.default_rng(11)
    pats = [b"0123456789abcdefghijklmnopqrstuvwxyz"[:L] for L in (2, 5, 17, 31, 36)] + [b"Z"]
    text = rng.integers(ord("A"), ord("Y"), size=(1 << 20) + 333, dtype=np.uint8)
    p = np.frombuffer(pats[4], np.uint8)
    for chain in (256, 1024):
        for boundary in range(chain, text.size - 64, chain * 7):
            j = int(rng.integers(0, p.size))
            text[boundary - j: boundary - j + p.size] = p
    text[:p.size] = p
    text[-p.size:] = p
    o = Oracle(pats)
    want = oracle_keys(o, text)
    stt = ac.build(pats)
    for chain in (256, 1024):
        assert_same(gpu_keys(stt, text, kernel=ac.KERNEL_STAGED, chain_bytes=chain), want)
        assert_same(gpu_keys(stt, text, kernel=ac.KERNEL_GLOBAL, chain_bytes=chain // 4), want)


def test_all_byte_values_and_nul():
    rng = np.random.default_rng(3)
    text = rng.integers(0, 256, size=(1 << 19) + 1, dtype=np.uint8)
    text[1000:1010] = 0
    pats = [bytes([b]) for b in range(0, 256, 5)] + [b"\x00\x00\x00", text[5000:5009].tobytes(), b"\xff\x00"]
    o = Oracle(pats)
    want = oracle_keys(o, text)
    stt = ac.build(pats)
    assert stt.maxlen == 9
    for k in KERNELS:
        assert_same(gpu_keys(stt, text, kernel=k), want)


def test_single_byte_patterns_no_halo():
    text = np.frombuffer(b"abracadabra" * 20000, np.uint8)
    pats = [b"a", b"r", b"a"]
    o = Oracle(pats)
    stt = ac.build(pats)
    assert stt.maxlen == 1
    for k in KERNELS:
        assert_same(gpu_keys(stt, text, kernel=k), oracle_keys(o, text))


def test_no_pattern_bytes():
    stt = ac.build([b"xyz", b"q"])
    t = torch.full((1 << 20,), ord("a"), dtype=torch.uint8, device="cuda")
    assert ac.count(stt, t) == 0
    c, recs = ac.match(stt, t)
    assert c == 0 and recs.numel() == 0


def test_duplicates_and_nested():
    pats = [b"ab", b"ab", b"b", b"abab", b"bab", b"ababababab"]
    text = np.frombuffer(b"xababab" * 30000 + b"ab", np.uint8)
    o = Oracle(pats)
    stt = ac.build(pats)
    for k in KERNELS:
        assert_same(gpu_keys(stt, text, kernel=k), oracle_keys(o, text))


@pytest.mark.parametrize("n", [31, 1 << 16, (1 << 20) + 17])
def test_adversarial_runs_closed_form(n):
    K = 32
    pats = [b"a" * k for k in range(1, K + 1)]
    stt = ac.build(pats)
    t = torch.full((n,), ord("a"), dtype=torch.uint8, device="cuda")
    want_count = K * n - K * (K - 1) // 2 if n >= K else n * (n + 1) // 2
    for k in KERNELS:
        assert ac.count(stt, t, kernel=k) == want_count
        c, recs = ac.match(stt, t, kernel=k)
        assert c == want_count
        r = recs.cpu().numpy()
        s = r >> 24
        p = r & 0xFFFFFF
        # start-major, pattern ids ascending, pattern p (length p+1) fits
        exp_s = np.repeat(np.arange(n), np.minimum(K, n - np.arange(n)))
        assert np.array_equal(s, exp_s)
        first = np.concatenate([[True], s[1:] != s[:-1]])
        exp_p = np.arange(r.size) - np.maximum.accumulate(np.where(first, np.arange(r.size), 0))
        assert np.array_equal(p, exp_p)


@pytest.mark.parametrize("off", [1, 3, 7, 8, 13, 15])
def test_misaligned_text_pointer(off):
    w = synth.make("c2", n=(1 << 20) + 100, n_patterns=200)
    o = Oracle(w.patterns)
    big = torch.from_numpy(w.text).cuda()
    sub = big[off:]
    assert sub.data_ptr() % 16 == off % 16
    c, recs = ac.match(ac.build(w.patterns), sub, kernel=ac.KERNEL_STAGED)
    assert_same(recs.cpu().numpy(), oracle_keys(o, w.text[off:]))


def test_capacity_error_and_count_only():
    w = synth.make("c1", n=1 << 18)
    stt = ac.build(w.patterns)
    t = torch.from_numpy(w.text).cuda()
    need = ac.count(stt, t)
    assert need > 10
    out = torch.empty(need - 1, dtype=torch.int64, device="cuda")
    with pytest.raises(ac.CapacityError) as e:
        ac.match(stt, t, out)
    assert e.value.count == need
    out = torch.empty(need, dtype=torch.int64, device="cuda")
    c, _ = ac.match(stt, t, out)
    assert c == need


@pytest.mark.parametrize("which", ["c2", "english5k-events"])
def test_shard_api_concatenation(which):
    if which == "c2":
        w = synth.make("c2", n=(3 << 20) + 11, n_patterns=400)
        text, pats, kw = w.text, w.patterns, {}
    else:  # dense outputs: shards through the EVENTS single pass (base offsets in the events)
        voc = synth.english_vocabulary(5002)
        text = synth.text_english((1 << 20) + 11, 5000, voc)
        pats, kw = synth.patterns_substrings(text, 5000, 4, 32, 5001), {"two_pass": 4}
    o = Oracle(pats)
    want = oracle_keys(o, text)
    stt = ac.build(pats)
    t = torch.from_numpy(text).cuda()
    n = t.numel()
    rng = np.random.default_rng(1)
    for G in (2, 3, 8):
        cuts = np.sort(rng.integers(0, n, size=G - 1)).tolist()
        bounds = [0] + cuts + [n]
        parts = []
        for lo, hi in zip(bounds[:-1], bounds[1:]):
            halo = min(stt.maxlen - 1, n - hi)
            c, recs = ac.match(stt, t[lo:hi + halo], n_halo=halo, base=lo, **kw)
            parts.append(recs.cpu().numpy())
        assert_same(np.concatenate(parts), want)


def test_match_sharded_nccl_world1():
    import os
    import socket
    import torch.distributed as dist
    from paper_conf_ipps_tranlhc13_b200.dist import match_sharded, plan_shards
    w = synth.make("c2", n=(1 << 20) + 3, n_patterns=200)
    o = Oracle(w.patterns)
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        stt = ac.build(w.patterns)
        (sh,) = plan_shards(w.text.size, 1, stt.maxlen)
        t = torch.from_numpy(w.text[sh.lo:sh.read_hi]).cuda()
        total, recs = match_sharded(stt, t, sh, gather=True)
        want = oracle_keys(o, w.text)
        assert total == want.size
        assert_same(recs.cpu().numpy(), want)
    finally:
        dist.destroy_process_group()


def test_host_entry_point():
    w = synth.make("c1", n=(1 << 18) + 5)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    host = torch.from_numpy(w.text).pin_memory()
    want = oracle_keys(o, w.text)
    out = torch.empty(want.size + 10, dtype=torch.int64).pin_memory()
    c = ac.match_host(stt, host, out)
    assert c == want.size
    assert_same(out[:c].numpy(), want)
    assert ac.match_host(stt, host, None) == want.size


def test_host_entry_point_pipelined_chunks():
    # > 32 MiB: several pipelined chunks (shards with halos) through ac_match_host
    w = synth.make("c1", n=(70 << 20) + 5)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    want = oracle_keys(o, w.text)
    host = torch.from_numpy(w.text).pin_memory()
    out = torch.empty(want.size, dtype=torch.int64).pin_memory()
    assert ac.match_host(stt, host, out) == want.size
    assert_same(out.numpy(), want)
    small = torch.empty(want.size // 2, dtype=torch.int64).pin_memory()
    with pytest.raises(ac.CapacityError) as e:
        ac.match_host(stt, host, small)
    assert e.value.count == want.size


@pytest.mark.parametrize("name", ["c3", "c2"])
def test_packet_segments(name):
    """NEXT-2 packet batches: every segment scanned on its own."""
    w = synth.make(name, n=(1 << 20) + 13)
    o = Oracle(w.patterns)
    stt = ac.build(w.patterns)
    rng = np.random.default_rng(5)
    cuts = np.unique(np.concatenate([[0, w.text.size], rng.integers(0, w.text.size, size=900),
                                     rng.integers(0, 64, size=5)]))  # includes empty-ish and tiny segments
    parts = []
    for lo, hi in zip(cuts[:-1].tolist(), cuts[1:].tolist()):
        parts.append(oracle_keys(o, w.text[lo:hi]) + (lo << 24))
    want = np.concatenate(parts)
    t = torch.from_numpy(w.text).cuda()
    seg = torch.from_numpy(cuts.astype(np.int64)).cuda()
    c, recs = ac.match_segments(stt, t, seg)
    assert c == want.size
    assert_same(recs.cpu().numpy(), want)
    # segments == [0, n) is the plain scan
    c1, r1 = ac.match_segments(stt, t, torch.tensor([0, t.numel()], dtype=torch.int64, device="cuda"))
    assert_same(r1.cpu().numpy(), oracle_keys(o, w.text))


def test_determinism():
    w = synth.make("c2", n=(2 << 20) + 1, n_patterns=500)
    stt = ac.build(w.patterns)
    t = torch.from_numpy(w.text).cuda()
    a = ac.match(stt, t)[1].cpu().numpy()
    b = ac.match(stt, t)[1].cpu().numpy()
    assert np.array_equal(a, b)


# ------------------------------------------------- full BASELINE.json sizes
# Every config at its full size, compared with the oracle over the WHOLE text
# (the oracle runs as start-owned windows on every host core, P:163-164 one
# level up): the complete canonical list where the oracle can hold it (C2,
# C3), else the full count plus the order-free multiset digest (count, sum,
# xor of splitmix64(start << 24 | pid)) computed independently on each side
# (SURVEY 8(c) "GPU parity").  The list comes from the launch configuration
# bench.py times (auto tier, auto kernel, single emitting pass).
_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def _np_mix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 over a uint64 array (wrapping arithmetic), test-side copy."""
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def digest_keys(keys: np.ndarray):
    """(count, sum mod 2^64, xor) of splitmix64 over the records (uint64 view)."""
    k = keys.view(np.uint64)
    c, sm, x = int(k.size), 0, 0
    for lo in range(0, k.size, 1 << 26):
        h = _np_mix64(k[lo:lo + (1 << 26)])
        with np.errstate(over="ignore"):
            sm = (sm + int(h.sum(dtype=np.uint64))) & ((1 << 64) - 1)
        x ^= int(np.bitwise_xor.reduce(h)) if h.size else 0
    return c, sm, x


def _s64(c: int) -> int:
    return c - (1 << 64) if c >= 1 << 63 else c


def _torch_mix64(z: torch.Tensor) -> torch.Tensor:
    """splitmix64 over an int64 tensor (two's-complement wrapping = uint64
    arithmetic; logical shifts by masking the arithmetic ones)."""
    def shr(v, k):
        return (v >> k) & ((1 << (64 - k)) - 1)
    z = z + _s64(0x9E3779B97F4A7C15)
    z = (z ^ shr(z, 30)) * _s64(0xBF58476D1CE4E5B9)
    z = (z ^ shr(z, 27)) * _s64(0x94D049BB133111EB)
    return z ^ shr(z, 31)


def digest_keys_torch(keys: torch.Tensor, chunk: int = 1 << 27):
    """digest_keys on the device (test side, for lists too large to copy to
    the host): the same (count, sum mod 2^64, xor) of splitmix64."""
    k = keys.reshape(-1)
    sm, x = 0, 0
    for lo in range(0, k.numel(), chunk):
        h = _torch_mix64(k[lo:lo + chunk])
        sm = (sm + int(h.sum()) % (1 << 64)) % (1 << 64)
        while h.numel() > 1:
            if h.numel() & 1:  # fold the odd element into the first
                h = torch.cat([h[:1] ^ h[-1:], h[1:-1]])
            half = h.numel() // 2
            h = h[:half] ^ h[half:]
        x ^= int(h[0]) % (1 << 64) if h.numel() else 0
    return int(k.numel()), sm, x


def test_torch_digest_matches_numpy():
    rng = np.random.default_rng(3)
    for n in (0, 1, 7, 1000, (1 << 20) + 3):
        a = rng.integers(0, 1 << 62, size=n, dtype=np.int64) << 1
        assert digest_keys_torch(torch.from_numpy(a).cuda(), chunk=1 << 18) == digest_keys(a)


def test_np_mix64_known_values():
    assert int(_np_mix64(np.array([0], np.uint64))[0]) == 0xE220A8397B1DCDAF


def _full_list(name):
    w = synth.make(name)
    stt = ac.build(w.patterns)
    t = torch.from_numpy(w.text).cuda()
    c, recs = ac.match(stt, t)
    assert ac.count(stt, t) == c
    r = recs.cpu().numpy()
    del t, recs
    torch.cuda.empty_cache()
    return w, stt, c, r


@pytest.mark.slow
@pytest.mark.parametrize("name", ["c2", "c3"])
def test_full_size_whole_list(name):
    w, stt, c, r = _full_list(name)
    o = Oracle(w.patterns)
    ends, pids = o.match_parallel(w.text)
    starts = ends.astype(np.int64) - o.lens[pids].astype(np.int64) + 1
    assert_same(r, (starts << 24) | pids.astype(np.int64))


@pytest.mark.slow
@pytest.mark.parametrize("name", ["c4", "c5-english-5000-30", "c5-snort-10000-30"])
def test_full_size_count_and_digest(name):
    w, stt, c, r = _full_list(name)
    assert c == r.size and (c == 0 or np.all(r[1:] > r[:-1]))  # canonical, duplicate free
    o = Oracle(w.patterns)
    assert digest_keys(r) == o.digest_parallel(w.text)


@pytest.mark.slow
def test_full_size_adversarial_runs_4gib():
    # C5 adversarial a^n with {a^1..a^32} at n = 2^32: count = K n - K(K-1)/2
    # (closed form P4-i); the 1.1 TB list cannot be held, so count mode over
    # the whole text plus the list of sampled sub-texts via the shard API
    K, n = 32, 1 << 32
    stt = ac.build([b"a" * k for k in range(1, K + 1)])
    t = torch.full((n,), ord("a"), dtype=torch.uint8, device="cuda")
    assert ac.count(stt, t) == K * n - K * (K - 1) // 2
    for lo in (0, (1 << 31) + 7, n - 4096):
        hi = min(n, lo + 4096)
        halo = min(K - 1, n - hi)
        c, recs = ac.match(stt, t[lo:hi + halo], n_halo=halo, base=lo)
        r = recs.cpu().numpy()
        per = np.minimum(K, n - np.arange(lo, hi))
        assert c == int(per.sum())
        assert np.array_equal(r >> 24, np.repeat(np.arange(lo, hi), per))
    del t


@pytest.mark.slow
def test_full_size_closed_form_kmers():
    # all 4^6 6-mers over ACGT, ids lexicographic: one match per start, pid =
    # base-4 value of text[i:i+6] (closed form P4-ii, exact at any size)
    A = b"ACGT"
    import itertools
    pats = [bytes(t) for t in itertools.product(A, repeat=6)]
    n = 1 << 30
    digits = synth.rng_for(424242).integers(0, 4, size=n, dtype=np.uint8)
    text = np.frombuffer(A, np.uint8)[digits]
    stt = ac.build(pats)
    c, recs = ac.match(stt, torch.from_numpy(text).cuda())
    assert c == n - 5
    r = recs.cpu().numpy()
    assert np.array_equal(r >> 24, np.arange(n - 5))
    d = digits.astype(np.int64)
    val = d[:-5] * 1024 + d[1:-4] * 256 + d[2:-3] * 64 + d[3:-2] * 16 + d[4:-1] * 4 + d[5:]
    assert np.array_equal(r & 0xFFFFFF, val)


def test_cache_policy_knobs():
    # the L2 knobs change where bytes live, never the result: text policy
    # (normal / evict-first / per-sector pair), TMA L2 promotion, and the
    # persisting access-policy window over the global table
    w = synth.make("c3", n=(2 << 20) + 77)
    o = Oracle(w.patterns)
    want = oracle_keys(o, w.text)
    stt = ac.build(w.patterns)
    t = torch.from_numpy(w.text).cuda()
    for knobs in (dict(text_policy=1), dict(text_policy=2), dict(text_policy=3), dict(text_promotion=1),
                  dict(text_promotion=3), dict(l2_window_mib=16), dict(l2_window_mib=64, text_policy=1)):
        c, recs = ac.match(stt, t, kernel=ac.KERNEL_STAGED, **knobs)
        assert_same(recs.cpu().numpy(), want)
    res = torch.zeros(2, dtype=torch.int64, device="cuda")
    for bad in (dict(text_policy=4), dict(text_promotion=5)):
        with pytest.raises(ac.AcError):
            ac.match_async(stt, t, None, res, **bad)
