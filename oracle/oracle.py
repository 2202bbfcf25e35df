"""ctypes wrapper of the CPU oracle (oracle/ac_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / ``--impl reference`` legs -- never by the product
package.  Nothing here shares code with paper_conf_ipps_tranlhc13_b200/.

Every function returns occurrences as ``(end, pid)`` pairs (end = 0-based
inclusive index of the last byte, "at the end of position"; DESIGN.md
reading R2).  ``canonical`` order is start = end - len + 1 ascending, then
pattern id ascending (reading R3).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from concurrent.futures import ThreadPoolExecutor
from pathlib import Path

import numpy as np

_HERE = Path(__file__).resolve().parent
_SRC = _HERE / "ac_oracle.c"
_LIB = _HERE / "liboracle.so"

_u8p = ctypes.POINTER(ctypes.c_uint8)
_u32p = ctypes.POINTER(ctypes.c_uint32)
_u64p = ctypes.POINTER(ctypes.c_uint64)


def build_oracle(force: bool = False) -> Path:
    """Compile ac_oracle.c with gcc (plain -O2; the oracle is not tuned)."""
    if force or not _LIB.exists() or _LIB.stat().st_mtime < _SRC.stat().st_mtime:
        tmp = _LIB.with_suffix(f".so.tmp{os.getpid()}")
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", str(tmp), str(_SRC)])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(str(build_oracle()))
        lib.oracle_build.restype = ctypes.c_void_p
        lib.oracle_build.argtypes = [ctypes.POINTER(_u8p), _u32p, ctypes.c_uint32]
        lib.oracle_free.argtypes = [ctypes.c_void_p]
        lib.oracle_free.restype = None
        for name in ("oracle_num_states", "oracle_maxlen"):
            getattr(lib, name).restype = ctypes.c_uint32
            getattr(lib, name).argtypes = [ctypes.c_void_p]
        for name in ("oracle_fail", "oracle_depth"):
            getattr(lib, name).restype = ctypes.c_uint32
            getattr(lib, name).argtypes = [ctypes.c_void_p, ctypes.c_uint32]
        lib.oracle_goto.restype = ctypes.c_int64
        lib.oracle_goto.argtypes = [ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint8]
        lib.oracle_delta.restype = ctypes.c_uint32
        lib.oracle_delta.argtypes = [ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint8]
        lib.oracle_output.restype = ctypes.c_uint32
        lib.oracle_output.argtypes = [ctypes.c_void_p, ctypes.c_uint32, _u32p, ctypes.c_uint32]
        lib.oracle_match.restype = ctypes.c_uint64
        lib.oracle_match.argtypes = [ctypes.c_void_p, _u8p, ctypes.c_uint64, ctypes.c_uint64,
                                     _u64p, _u32p, ctypes.c_uint64]
        lib.oracle_match_window.restype = ctypes.c_uint64
        lib.oracle_match_window.argtypes = [ctypes.c_void_p, _u8p, ctypes.c_uint64, ctypes.c_uint64,
                                            ctypes.c_uint64, ctypes.c_uint64, _u64p, _u32p,
                                            ctypes.c_uint64]
        lib.oracle_match_chunked.restype = ctypes.c_uint64
        lib.oracle_match_chunked.argtypes = [ctypes.c_void_p, _u8p, ctypes.c_uint64, ctypes.c_uint64,
                                             ctypes.c_uint64, _u64p, _u32p, ctypes.c_uint64]
        lib.oracle_digest_window.restype = None
        lib.oracle_digest_window.argtypes = [ctypes.c_void_p, _u8p, ctypes.c_uint64, ctypes.c_uint64,
                                             ctypes.c_uint64, ctypes.c_uint64, _u64p]
        lib.oracle_transitions.restype = None
        lib.oracle_transitions.argtypes = [ctypes.c_void_p, _u8p, ctypes.c_uint64, _u64p]
        lib.oracle_canonical_sort.restype = ctypes.c_int
        lib.oracle_canonical_sort.argtypes = [ctypes.c_void_p, _u64p, _u32p, ctypes.c_uint64]
        _lib = lib
    return _lib


def _as_u8(text) -> np.ndarray:
    if isinstance(text, (bytes, bytearray, memoryview)):
        return np.frombuffer(bytes(text), dtype=np.uint8)
    a = np.ascontiguousarray(text)
    if a.dtype != np.uint8:
        raise TypeError("text must be bytes or a uint8 array")
    return a


def _ptr(a: np.ndarray, t):
    return a.ctypes.data_as(t) if a.size else ctypes.cast(ctypes.c_void_p(0), t)


class Oracle:
    """The textbook goto/failure/output machine of P:47-58 (AC'75 Alg. 1-3)."""

    def __init__(self, patterns):
        lib = _load()
        pats = [bytes(p) for p in patterns]
        self.patterns = pats
        self._bufs = [np.frombuffer(p, dtype=np.uint8).copy() if p else np.zeros(1, np.uint8) for p in pats]
        arr = (_u8p * max(1, len(pats)))(*[b.ctypes.data_as(_u8p) for b in self._bufs])
        self.lens = np.array([len(p) for p in pats], dtype=np.uint32)
        h = lib.oracle_build(arr, _ptr(self.lens, _u32p), len(pats))
        if not h:
            raise ValueError("oracle_build failed (empty pattern?)")
        self._h = ctypes.c_void_p(h)
        self._lib = lib

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and self._lib is not None:
            self._lib.oracle_free(h)
            self._h = None

    # --- the three functions of Fig. 1 and the DFA next-move of P:62 -------
    @property
    def num_states(self) -> int:
        return int(self._lib.oracle_num_states(self._h))

    @property
    def maxlen(self) -> int:
        return int(self._lib.oracle_maxlen(self._h))

    def goto(self, s: int, a: int):
        """g(s, a); None stands for the paper's ``fail``."""
        t = self._lib.oracle_goto(self._h, s, a)
        return None if t < 0 else int(t)

    def fail(self, s: int) -> int:
        return int(self._lib.oracle_fail(self._h, s))

    def depth(self, s: int) -> int:
        return int(self._lib.oracle_depth(self._h, s))

    def output(self, s: int) -> list[int]:
        k = self._lib.oracle_output(self._h, s, None, 0)
        buf = np.zeros(max(1, k), dtype=np.uint32)
        self._lib.oracle_output(self._h, s, _ptr(buf, _u32p), k)
        return [int(x) for x in buf[:k]]

    def delta(self, s: int, a: int) -> int:
        return int(self._lib.oracle_delta(self._h, s, a))

    # --- Phase 2 -------------------------------------------------------------
    def _collect(self, fn, *args):
        n = fn(self._h, *args, None, None, 0)
        ends = np.zeros(max(1, n), dtype=np.uint64)
        pids = np.zeros(max(1, n), dtype=np.uint32)
        n2 = fn(self._h, *args, _ptr(ends, _u64p), _ptr(pids, _u32p), n)
        assert n2 == n
        return ends[:n], pids[:n]

    def count(self, text, base: int = 0) -> int:
        t = _as_u8(text)
        return int(self._lib.oracle_match(self._h, _ptr(t, _u8p), t.size, base, None, None, 0))

    def match(self, text, base: int = 0, canonical: bool = True):
        """All (end, pid) occurrences; canonical order unless canonical=False (walk order)."""
        t = _as_u8(text)
        ends, pids = self._collect(self._lib.oracle_match, _ptr(t, _u8p), t.size, base)
        if canonical:
            self.sort(ends, pids)
        return ends, pids

    def match_window(self, text, lo: int, own_hi: int, base: int = 0, canonical: bool = True):
        """Occurrences whose start lies in [lo, own_hi); ends reported as base + index."""
        t = _as_u8(text)
        ends, pids = self._collect(self._lib.oracle_match_window, _ptr(t, _u8p), t.size, lo, own_hi, base)
        if canonical:
            self.sort(ends, pids)
        return ends, pids

    def match_chunked(self, text, chunk: int, base: int = 0, canonical: bool = True):
        t = _as_u8(text)
        ends, pids = self._collect(self._lib.oracle_match_chunked, _ptr(t, _u8p), t.size, base, chunk)
        if canonical:
            self.sort(ends, pids)
        return ends, pids

    def transitions(self, text):
        """(goto transitions, failure transitions) of the walk over the text (P6)."""
        t = _as_u8(text)
        out = np.zeros(2, dtype=np.uint64)
        self._lib.oracle_transitions(self._h, _ptr(t, _u8p), t.size, _ptr(out, _u64p))
        return int(out[0]), int(out[1])

    def sort(self, ends: np.ndarray, pids: np.ndarray) -> None:
        """In-place canonical sort (start asc, pid asc) done by the C oracle."""
        assert ends.dtype == np.uint64 and pids.dtype == np.uint32
        if ends.size:
            rc = self._lib.oracle_canonical_sort(self._h, _ptr(ends, _u64p), _ptr(pids, _u32p), ends.size)
            if rc != 0:
                raise MemoryError("oracle_canonical_sort")

    # --- whole texts on every host core --------------------------------------
    # The chunked mode of P:163-164 one level up: window [lo, hi) is walked
    # from state 0 over [lo, min(hi + maxlen - 1, n)) and keeps the
    # occurrences whose start it owns (reading R9), one window per thread.
    # ctypes releases the GIL for the duration of each C call, so the windows
    # run concurrently.  Concatenating the windows' canonical lists in window
    # order is the canonical list of the whole text (start-major order).
    def _windows(self, n: int, threads: int | None, min_window: int = 1 << 20):
        threads = threads or os.cpu_count() or 1
        k = max(1, min(4 * threads, (n + min_window - 1) // min_window))
        cuts = [n * i // k for i in range(k + 1)]
        return threads, [(cuts[i], cuts[i + 1]) for i in range(k) if cuts[i] < cuts[i + 1]]

    def match_parallel(self, text, threads: int | None = None, base: int = 0):
        """(ends, pids) of the whole text in canonical order, windows on `threads` cores."""
        t = _as_u8(text)
        threads, wins = self._windows(t.size, threads)

        def one(w):
            return self.match_window(t, w[0], w[1], base=base, canonical=True)

        with ThreadPoolExecutor(threads) as ex:
            parts = list(ex.map(one, wins))
        if not parts:
            return np.zeros(0, np.uint64), np.zeros(0, np.uint32)
        return np.concatenate([p[0] for p in parts]), np.concatenate([p[1] for p in parts])

    def digest_window(self, text, lo: int, own_hi: int, base: int = 0):
        """(count, sum, xor) of splitmix64(start << 24 | pid) over the window's owned occurrences."""
        t = _as_u8(text)
        out = np.zeros(3, dtype=np.uint64)
        self._lib.oracle_digest_window(self._h, _ptr(t, _u8p), t.size, lo, own_hi, base, _ptr(out, _u64p))
        return int(out[0]), int(out[1]), int(out[2])

    def digest_parallel(self, text, threads: int | None = None, base: int = 0):
        """Multiset digest of the whole text: (count, sum mod 2^64, xor)."""
        t = _as_u8(text)
        threads, wins = self._windows(t.size, threads)
        with ThreadPoolExecutor(threads) as ex:
            parts = list(ex.map(lambda w: self.digest_window(t, w[0], w[1], base=base), wins))
        c, sm, x = 0, 0, 0
        for pc, ps, px in parts:
            c += pc
            sm = (sm + ps) & ((1 << 64) - 1)
            x ^= px
        return c, sm, x
