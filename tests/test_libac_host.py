"""CPU tests of libac: the library loads and exports every symbol of
include/ac.h, the host builder (phase 1) equals the oracle's
goto/failure/output definitions state by state, and the device entry points
fail loudly without a GPU (no CPU fallback)."""
from __future__ import annotations

import ctypes
import random
import re
from pathlib import Path

import numpy as np
import pytest
import torch

import paper_conf_ipps_tranlhc13_b200 as ac
from oracle import Oracle

ROOT = Path(__file__).resolve().parents[1]


@pytest.fixture(scope="session", autouse=True)
def _built():
    ac.build_library()


def test_exports_every_declared_symbol():
    header = (ROOT / "include" / "ac.h").read_text()
    declared = set(re.findall(r"^\s*(?:const\s+)?[\w\s\*]+?\b(ac_\w+)\s*\(", header, re.M))
    declared = {d for d in declared if not d.startswith("ac_match_t")}
    assert {"ac_build", "ac_match", "ac_match_shard", "ac_free", "ac_compile"} <= declared
    L = ac.lib()
    for name in sorted(declared):
        assert hasattr(L, name), name
    assert set(ac.EXPORTED) == declared
    assert "sm_100a" in ac.version()


def test_status_strings():
    L = ac.lib()
    for s in range(8):
        assert L.ac_status_string(s).decode().startswith("AC_")


def _map_states(o: Oracle, t: ac.HostTable, forward: bool, pats):
    """oracle state -> builder state, by walking each oracle state's string."""
    C = t.info["n_classes"]
    stride = t.info["row_stride"]
    eb = t.info["entry_bytes"]
    mask = 0x7FFF if eb == 2 else 0x7FFFFFFF
    stt = t.stt.astype(np.int64)
    strs = {0: b""}
    frontier = [0]
    while frontier:
        nxt = []
        for s in frontier:
            for a in range(256):
                u = o.goto(s, a)
                if u is None or (s == 0 and u == 0):
                    continue
                strs[u] = strs[s] + bytes([a])
                nxt.append(u)
        frontier = nxt
    mp = {}
    for s, w in strs.items():
        b = 0
        for a in w:
            b = int(stt[b, t.class_map[a]] & mask)
        mp[s] = b
    assert stride >= C
    return mp, stt, mask


def _check_builder(pats, forward: bool):
    opats = pats if forward else [p[::-1] for p in pats]
    o = Oracle(opats)
    t = ac.compile_table(pats, forward=forward)
    assert t.info["n_states"] == o.num_states
    assert t.info["maxlen"] == max(len(p) for p in pats)
    mp, stt, mask = _map_states(o, t, forward, pats)
    assert sorted(mp.values()) == list(range(o.num_states))  # a bijection
    flag = 0x8000 if t.info["entry_bytes"] == 2 else 0x80000000
    # BFS numbering: depth is non-decreasing with the builder's state id
    depth_by_b = {mp[s]: o.depth(s) for s in mp}
    d = [depth_by_b[i] for i in range(o.num_states)]
    assert d == sorted(d)
    ic = t.info["info_col"]
    eb = t.info["entry_bytes"]
    assert ic >= t.info["n_classes"] and (eb == 4 or ic % 2 == 0)
    raw = t.stt.view(np.uint8).reshape(o.num_states, -1)
    for s, b in mp.items():
        outs = o.output(s)
        assert t.out_ids[t.out_off[b]:t.out_off[b + 1]].tolist() == outs
        # output summary in the row padding: payload u32, then the count
        payload = int(raw[b, ic * eb: ic * eb + 4].view(np.uint32)[0])
        cnt = int(stt[b, ic + (2 if eb == 2 else 1)])
        assert cnt == min(len(outs), 0xFFFF if eb == 2 else 1 << 32)
        assert payload == (outs[0] if len(outs) == 1 else int(t.out_off[b]))
        row = stt[b]
        for a in range(256):
            u = o.delta(s, a)
            e = int(row[t.class_map[a]])
            assert e & mask == mp[u], (s, a)
            assert bool(e & flag) == bool(o.output(u)), (s, a)


def test_builder_worked_example_forward():
    pats = [b"he", b"she", b"his", b"hers"]
    _check_builder(pats, forward=True)
    # P:66-68 through the builder, in creation-order names via the oracle map
    o = Oracle(pats)
    t = ac.compile_table(pats, forward=True)
    mp, stt, mask = _map_states(o, t, True, pats)
    inv = {v: k for k, v in mp.items()}
    walk = []
    s = 0
    for ch in b"ushers":
        s = int(stt[s, t.class_map[ch]] & mask)
        walk.append(inv[s])
    assert walk == [0, 3, 4, 5, 8, 9]


@pytest.mark.parametrize("forward", [True, False])
@pytest.mark.parametrize("seed", range(25))
def test_builder_random_tiny(seed, forward):
    rng = random.Random(seed)
    A = rng.randint(1, 5)
    alphabet = list(range(97, 97 + A)) if seed % 3 else [0, 255, 7, 128, 64][:A]
    pats = [bytes(rng.choice(alphabet) for _ in range(rng.randint(1, 7))) for _ in range(rng.randint(1, 12))]
    _check_builder(pats, forward)


@pytest.mark.parametrize("forward", [True, False])
def test_builder_c1_dictionary(forward):
    import synth
    _check_builder(synth.make("c1", n=1 << 12).patterns, forward)


def test_builder_snort_like_entry4():
    import synth
    pats = synth.patterns_snort(150, 77)
    t = ac.compile_table(pats, entry_bytes=4)
    assert t.info["entry_bytes"] == 4 and t.info["row_stride"] % 2 == 1
    _check_builder(pats, False)


def _decode_compact(t):
    """The COMPACT lookup rule of include/ac.h, vectorised: returns the entry
    table E[x, c] (compact ids, bit 15 = output flag) and the output table."""
    d = t.info
    S, C = d["n_states"], d["n_classes"]
    nd, ds = d["compact_dense"], d["compact_dstride"]
    blob = t.compact
    dense = blob[:nd * ds * 2].view(np.uint16).reshape(nd, ds)[:, :C].astype(np.int64)
    rec = blob[d["compact_sparse_off"]:d["compact_sparse_off"] + (S - nd) * 8].view(np.uint32).reshape(-1, 2)
    fd = rec[:, 0] >> 16
    c1, c2 = rec[:, 0] & 0xFF, (rec[:, 0] >> 8) & 0xFF
    assert ((c1 == 0xFF) | (c1 % 2 == 0)).all() and ((c2 == 0xFF) | (c2 % 2 == 0)).all()
    c1, c2 = np.where(c1 == 0xFF, 0xFF, c1 // 2), np.where(c2 == 0xFF, 0xFF, c2 // 2)  # doubled classes
    t1, t2 = rec[:, 1] & 0xFFFF, rec[:, 1] >> 16
    cls = np.arange(C)[None, :]
    sparse = np.where(cls == c1[:, None], t1[:, None],
                      np.where(cls == c2[:, None], t2[:, None], dense[fd]))
    E = np.concatenate([dense, sparse.astype(np.int64)])
    E = (E >> 1) | ((E & 1) << 15)  # entries are 2 x + flag -> x | flag << 15
    nout = d["compact_od"] + d["compact_os"]
    ot = blob[d["compact_out_off"]:d["compact_out_off"] + nout * 8].view(np.uint32).reshape(-1, 2)
    return E, ot


@pytest.mark.parametrize("which", ["c2", "c1", "tiny"])
def test_compact_encoding_equals_dense(which):
    import synth
    if which == "tiny":
        pats = [b"he", b"she", b"his", b"hers", b"h", b"hershey"]
    else:
        pats = synth.make(which, n=1 << 16).patterns if which == "c1" else synth.make("c2", n=1 << 22).patterns
    t = ac.compile_table(pats, compact=True)
    d = t.info
    S, C = d["n_states"], d["n_classes"]
    perm = t.perm.astype(np.int64)
    assert perm[0] == 0 and sorted(perm.tolist()) == list(range(S))
    inv = np.empty(S, np.int64)
    inv[perm] = np.arange(S)
    E, ot = _decode_compact(t)
    dense_bfs = t.stt[:, :C].astype(np.int64)
    want = inv[dense_bfs[perm] & 0x7FFF] | (dense_bfs[perm] & 0x8000)
    assert np.array_equal(E, want)
    # output-state numbering and the output table
    nd, od, os_ = d["compact_dense"], d["compact_od"], d["compact_os"]
    has_out = np.diff(t.out_off.astype(np.int64))[perm] > 0
    # output states are exactly the contiguous ids [nd - od, nd + os)
    assert has_out[nd - od:nd + os_].all() and not has_out[:nd - od].any() and not has_out[nd + os_:].any()
    for x in range(nd - od, nd + os_):
        s = perm[x]
        outs = t.out_ids[t.out_off[s]:t.out_off[s + 1]].tolist()
        oidx = x - (nd - od)
        payload, count = ot[oidx].tolist()
        assert count == len(outs) and payload == (outs[0] if count == 1 else int(t.out_off[s]))
    # fits next to the lean staged variant's ring (32 warps x 2 slots x 512 B, unswizzled:
    # no alignment pad), its mbarriers, the class map and 128 B of slack
    assert d["compact_bytes"] <= 232448 - (32 * 2 * 512 + 512 + 16 + 256) - 128
    if which == "c2":
        assert S > 15000 and d["stt_bytes"] > 1_000_000  # the dense table would not fit


@pytest.mark.parametrize("which", ["dna", "tiny"])
def test_stride2_table_is_delta_composed(which):
    """NEXT-4 table: T2(s, c1 c2) = delta(delta(s,c1),c2) with both flags."""
    import synth
    if which == "dna":
        w = synth.make("c4", n=1 << 16, n_patterns=300)
        pats = w.patterns
    else:
        pats = [b"AC", b"CA", b"A", b"GTT", b"TTTT"]
    t = ac.compile_table(pats, entry_bytes=4, stride=2)
    d = t.info
    C, S = d["n_classes"], d["n_states"]
    assert d["stride"] == 2 and d["stride2_cols"] >= C * C and d["stride2_cols"] % 2 == 1
    T1 = t.stt[:, :C].astype(np.int64)
    nxt, flag = T1 & 0x7FFFFFFF, (T1 >> 31) & 1
    T2 = t.stt2[:, :C * C].astype(np.int64).reshape(S, C, C)
    mid = nxt  # [s, c1]
    want_state = nxt[mid]  # [s, c1, c2]
    assert np.array_equal(T2 & ((1 << 30) - 1), want_state)
    assert np.array_equal((T2 >> 31) & 1, flag[mid])
    assert np.array_equal((T2 >> 30) & 1, np.broadcast_to(flag[:, :, None], (S, C, C)))


def test_classes_and_stride():
    t = ac.compile_table([b"abc", b"zz"])
    assert t.info["n_classes"] == 5  # a, b, c, z + class 0
    assert t.class_map[ord("a")] == 1 and t.class_map[ord("z")] == 4 and t.class_map[0] == 0
    words = t.info["row_stride"] * t.info["entry_bytes"] // 4
    assert words % 2 == 1  # odd number of 4-byte words per row
    all_bytes = [bytes([b]) for b in range(256)]
    t2 = ac.compile_table(all_bytes)
    assert t2.info["n_classes"] == 256 and list(t2.class_map) == list(range(256))


def test_builder_errors():
    with pytest.raises(ac.AcError) as e:
        ac.compile_table([b"ok", b""])
    assert e.value.status == ac.AC_ERR_EMPTY_PATTERN
    rng = random.Random(3)
    many = [bytes(rng.randrange(97, 123) for _ in range(8)) for _ in range(8000)]  # > 32768 states
    with pytest.raises(ac.AcError) as e:
        ac.compile_table(many, entry_bytes=2)
    assert e.value.status == ac.AC_ERR_TOO_LARGE
    with pytest.raises(ac.AcError):
        ac.compile_table([b"a"], entry_bytes=3)


def test_empty_dictionary_compiles():
    t = ac.compile_table([])
    assert t.info["n_states"] == 1 and t.info["out_entries"] == 0


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU failure mode")
def test_no_device_fails_loudly():
    with pytest.raises(ac.AcError) as e:
        ac.build([b"he"], device=0)
    assert e.value.status in (ac.AC_ERR_NO_DEVICE, ac.AC_ERR_CUDA)


def test_compact_rejects_wide_alphabets():
    """COMPACT stores doubled classes in bytes: at most 127 classes."""
    ok = [bytes([b]) + bytes([b + 1]) for b in range(0, 120, 2)]  # 121 classes
    t = ac.compile_table(ok, compact=True)
    assert t.info["n_classes"] <= 127 and t.info["compact_bytes"] > 0
    wide = [bytes([b, (b * 7) % 256]) for b in range(200)]
    with pytest.raises(ac.AcError):
        ac.compile_table(wide, compact=True)


def _decode_split(t):
    """The SPLIT lookup rule of include/ac.h, vectorised over the hot states:
    E[s, c] = 32-bit entry (BFS id | flag << 31) where the shared-memory part
    answers, -1 where the global table must (cold record or escaped entry)."""
    d = t.info
    C = d["n_classes"]
    D, H, ds = d["split_dense"], d["split_records"], d["split_dstride"]
    blob = t.split
    rows = blob[:(D + 1) * ds * 2].view(np.uint16).reshape(D + 1, ds)[:, :C].astype(np.int64)
    assert (rows[D] == 0xFFFF).all()  # the escape row
    assert blob.size == (D + 1) * ds * 2 + (H - D) * 8
    rec = blob[(D + 1) * ds * 2:].view(np.uint32).reshape(-1, 2).astype(np.int64)
    cls4 = np.stack([(rec[:, 0] >> (8 * i)) & 0xFF for i in range(4)], axis=1)      # children's classes
    fd = rec[:, 1] & 0xFFF
    flags = (rec[:, 1] >> 12) & 0xF
    f2 = rec[:, 1] >> 16  # 2 first - 1
    assert (fd <= D).all() and (f2 % 2 == 1).all()
    c = np.arange(C)[None, :]
    # first matching class byte k (lowest index) -> child first + k (16-bit form 2 x + flag)
    k = np.full((H - D, C), -1, np.int64)
    for i in range(3, -1, -1):
        k = np.where(cls4[:, i:i + 1] == c, i, k)
    child = (f2[:, None] + 1 + 2 * np.maximum(k, 0)) | ((flags[:, None] >> np.maximum(k, 0)) & 1)
    e16_sparse = np.where(k >= 0, child, rows[fd])
    e16 = np.concatenate([rows[:D], e16_sparse])
    E = (e16 >> 1) | ((e16 & 1) << 31)
    cold = (fd == D) & (f2 == 0xFFFD)
    return np.where(e16 > 0xFFFD, -1, E), int(cold.sum())


@pytest.mark.parametrize("which", ["c3", "english5k", "tiny"])
def test_split_encoding_equals_dense(which):
    """Every transition the SPLIT shared-memory part answers equals the dense
    table's delta; the rest are marked for the global table."""
    import synth
    if which == "tiny":
        pats = [b"he", b"she", b"his", b"hers", b"h", b"hershey"]
    elif which == "c3":
        pats = synth.patterns_snort(10000, 3001)
    else:
        pats = synth.make("c5-english-5000-22").patterns
    t = ac.compile_table(pats, split=True)
    d = t.info
    assert d["entry_bytes"] == 4 and d["split_bytes"] > 0
    C, D, H = d["n_classes"], d["split_dense"], d["split_records"]
    E, n_cold = _decode_split(t)
    assert n_cold == d["split_cold_records"]
    want = t.stt[:H, :C].astype(np.int64)
    ok = E >= 0
    assert np.array_equal(E[ok], want[ok])
    # escapes only where the next id does not fit 15 bits, or cold records
    esc_dense = ~ok[:D]
    assert ((want[:D][esc_dense] & 0x7FFFFFFF) >= 32767).all()
    assert D >= 1
    # fits next to the SPLIT staged variant's ring (32 warps x 1 slot x 1 KB, 1 KB swizzle alignment)
    assert d["split_bytes"] <= 232448 - (1024 + 32 * 1024 + 256 + 16 + 256) - 128
    if which == "c3":
        # depth <= 1 dense (root + one state per used last byte), every depth-2 state a children
        # record, cold only with more than four children
        assert D == 1 + len({p[-1] for p in pats})
        assert H - D >= 7000 and d["split_cold_records"] < (H - D) // 50


@pytest.mark.parametrize("which", ["dna", "snort"])
def test_parallel_build_is_identical(which):
    """NEXT-3 faster build: phase 1 on 1, 3 and 8 host threads gives the same
    table byte for byte (levels here exceed the 2,048-state grain, so the
    threaded passes really split).  The 1-thread build is the one the
    oracle pins above."""
    import synth
    if which == "dna":
        rng = random.Random(11)
        pats = [bytes(rng.choice(b"ACGT") for _ in range(rng.randint(6, 14))) for _ in range(6000)]
    else:
        pats = synth.patterns_snort(3000, 91)
    tabs = [ac.compile_table(pats, threads=t, split=(which == "snort")) for t in (1, 3, 8)]
    a = tabs[0]
    assert a.info["n_states"] > 8000
    for b in tabs[1:]:
        assert a.info == b.info
        for f in ("class_map", "stt", "out_off", "out_ids", "split"):
            x, y = getattr(a, f), getattr(b, f)
            assert (x is None and y is None) or np.array_equal(x, y), f
