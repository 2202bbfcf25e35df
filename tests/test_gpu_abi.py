"""The synchronous C-ABI calls ac_match and ac_match_shard (include/ac.h),
called directly through ctypes with device buffers -- their status and count
mapping (finish_sync) and argument checks, against the oracle.

ac_match (phase 2): every occurrence of the dictionary in d_text[0, n),
canonical (start, pattern) order (readings R2/R3), *count always set on
AC_OK and AC_ERR_CAPACITY.  ac_match_shard: the chunk + overlap rule of
P:163-164 one level up, start ownership (R9).
"""
from __future__ import annotations

import ctypes

import numpy as np
import pytest
import torch

import paper_conf_ipps_tranlhc13_b200 as ac
import synth
from oracle import Oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def case():
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    w = synth.make("c2", n=(1 << 20) + 4321, n_patterns=300)
    o = Oracle(w.patterns)
    ends, pids = o.match(w.text)
    starts = ends.astype(np.int64) - o.lens[pids].astype(np.int64) + 1
    want = (starts << 24) | pids.astype(np.int64)
    stt = ac.build(w.patterns)
    big = torch.zeros(w.text.size + 32, dtype=torch.uint8, device="cuda")
    return w, o, want, stt, big


def _call_match(stt, text: torch.Tensor, n, out: torch.Tensor | None, cap):
    L = ac.lib()
    cnt = ctypes.c_uint64(0xDEADBEEF)
    rc = L.ac_match(stt.handle, text.data_ptr() if n else None, n, out.data_ptr() if out is not None else None,
                    cap, ctypes.byref(cnt), ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    return rc, cnt.value


def _call_shard(stt, text: torch.Tensor, n_owned, n_halo, base, out, cap):
    L = ac.lib()
    cnt = ctypes.c_uint64(0xDEADBEEF)
    rc = L.ac_match_shard(stt.handle, text.data_ptr(), n_owned, n_halo, base,
                          out.data_ptr() if out is not None else None, cap, ctypes.byref(cnt),
                          ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    return rc, cnt.value


def test_ac_match_count_only(case):
    w, o, want, stt, _ = case
    t = torch.from_numpy(w.text).cuda()
    rc, c = _call_match(stt, t, t.numel(), None, 0)
    assert rc == ac.AC_OK and c == want.size


def test_ac_match_list(case):
    w, o, want, stt, _ = case
    t = torch.from_numpy(w.text).cuda()
    out = torch.full((want.size + 5,), -1, dtype=torch.int64, device="cuda")
    rc, c = _call_match(stt, t, t.numel(), out, out.numel())
    assert rc == ac.AC_OK and c == want.size
    assert np.array_equal(out[:c].cpu().numpy(), want)


def test_ac_match_capacity_short_by_one(case):
    w, o, want, stt, _ = case
    t = torch.from_numpy(w.text).cuda()
    out = torch.empty(want.size - 1, dtype=torch.int64, device="cuda")
    rc, c = _call_match(stt, t, t.numel(), out, out.numel())
    assert rc == ac.AC_ERR_CAPACITY and c == want.size
    assert b"cap" in ac.lib().ac_last_error()
    # the exact size succeeds afterwards (the failed call left no state behind)
    out = torch.empty(want.size, dtype=torch.int64, device="cuda")
    rc, c = _call_match(stt, t, t.numel(), out, out.numel())
    assert rc == ac.AC_OK and c == want.size


def test_ac_match_empty_text(case):
    _, _, _, stt, big = case
    out = torch.empty(4, dtype=torch.int64, device="cuda")
    rc, c = _call_match(stt, big, 0, out, 4)
    assert rc == ac.AC_OK and c == 0
    rc, c = _call_match(stt, big, 0, None, 0)
    assert rc == ac.AC_OK and c == 0


@pytest.mark.parametrize("off", [1, 5, 11])
def test_ac_match_misaligned(case, off):
    w, o, _, stt, big = case
    big[off:off + w.text.size].copy_(torch.from_numpy(w.text))
    sub = big[off:off + w.text.size]
    assert sub.data_ptr() % 16 != 0
    ends, pids = o.match(w.text)
    starts = ends.astype(np.int64) - o.lens[pids].astype(np.int64) + 1
    want = (starts << 24) | pids.astype(np.int64)
    out = torch.empty(want.size, dtype=torch.int64, device="cuda")
    rc, c = _call_match(stt, sub, w.text.size, out, out.numel())
    assert rc == ac.AC_OK and c == want.size
    assert np.array_equal(out.cpu().numpy(), want)


def test_ac_match_null_stt():
    L = ac.lib()
    cnt = ctypes.c_uint64(0)
    assert L.ac_match(None, None, 0, None, 0, ctypes.byref(cnt), None) == ac.AC_ERR_INVALID_ARG


def test_ac_match_shard_pieces(case):
    w, o, want, stt, _ = case
    t = torch.from_numpy(w.text).cuda()
    n = t.numel()
    H = stt.maxlen - 1
    cuts = [0, 1, 4096 + 3, n // 2, n - 7, n]
    parts = []
    for lo, hi in zip(cuts[:-1], cuts[1:]):
        halo = min(H, n - hi)
        out = torch.empty(max(1, want.size), dtype=torch.int64, device="cuda")
        rc, c = _call_shard(stt, t[lo:], hi - lo, halo, lo, out, out.numel())
        assert rc == ac.AC_OK
        rcc, cc = _call_shard(stt, t[lo:], hi - lo, halo, lo, None, 0)
        assert rcc == ac.AC_OK and cc == c
        parts.append(out[:c].cpu().numpy())
    assert np.array_equal(np.concatenate(parts), want)


def test_ac_match_shard_capacity(case):
    w, o, want, stt, _ = case
    t = torch.from_numpy(w.text).cuda()
    n = t.numel()
    lo, hi = 1000, n // 3
    s = want >> 24
    need = int(((s >= lo) & (s < hi)).sum())
    out = torch.empty(need - 1, dtype=torch.int64, device="cuda")
    rc, c = _call_shard(stt, t[lo:], hi - lo, stt.maxlen - 1, lo, out, out.numel())
    assert rc == ac.AC_ERR_CAPACITY and c == need


def test_ac_match_shard_rejects_wide_halo(case):
    w, o, want, stt, _ = case
    t = torch.from_numpy(w.text).cuda()
    out = torch.empty(16, dtype=torch.int64, device="cuda")
    rc, c = _call_shard(stt, t, 1000, stt.maxlen, 0, out, 16)  # n_halo > maxlen - 1
    assert rc == ac.AC_ERR_INVALID_ARG
    assert b"n_halo" in ac.lib().ac_last_error()
