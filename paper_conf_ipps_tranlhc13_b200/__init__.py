"""Python binding of libac -- the B200-native Aho-Corasick matching scan.

Argument marshalling only: every step of phase 2 runs in libac's sm_100a
kernels (paper_conf_ipps_tranlhc13_b200/csrc/).  PyTorch supplies device
memory, streams and process groups.  There is no CPU fallback: if libac.so
is missing or no sm_100 device is present, calls raise.

    stt = build([b"he", b"she", b"his", b"hers"], device=0)
    count, recs = match(stt, text_u8_cuda)          # canonical list
    starts(recs), pattern_ids(recs), ends(recs, stt.lens)

Paper: Tran, Lee, Hong, Choi, IPDPS-W 2013 (P:31 two phases; P:118 STT;
P:137 built once on the host; P:222 build/copies untimed).
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass
from pathlib import Path

import torch

from . import _build

_PKG = Path(__file__).resolve().parent
LIB_PATH = _PKG / "libac.so"

AC_OK, AC_ERR_INVALID_ARG, AC_ERR_EMPTY_PATTERN, AC_ERR_TOO_LARGE = 0, 1, 2, 3
AC_ERR_CAPACITY, AC_ERR_NO_MEMORY, AC_ERR_CUDA, AC_ERR_NO_DEVICE = 4, 5, 6, 7
TIER_AUTO, TIER_SMEM, TIER_HYBRID, TIER_GLOBAL, TIER_COMPACT, TIER_SPLIT = 0, 1, 2, 3, 4, 5
KERNEL_AUTO, KERNEL_STAGED, KERNEL_GLOBAL = 0, 1, 2
TIER_NAMES = {1: "smem", 2: "hybrid", 3: "global", 4: "compact", 5: "split"}

EXPORTED = [
    "ac_build", "ac_free", "ac_stt_query", "ac_stt_pattern_lengths", "ac_match", "ac_match_shard",
    "ac_match_async", "ac_match_segments", "ac_last_launch_count", "ac_last_launch_name", "ac_last_launch_text_bytes", "ac_last_scratch_record_bytes", "ac_match_host", "ac_compile", "ac_table_query",
    "ac_table_export", "ac_table_export_compact", "ac_table_export_stride2", "ac_table_export_split", "ac_table_free", "ac_status_string", "ac_last_error", "ac_version",
]


class AcError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{_status_name(status)}: {detail}")
        self.status = status


class CapacityError(AcError):
    def __init__(self, status: int, detail: str, count: int):
        super().__init__(status, detail)
        self.count = count


class ac_build_opts(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_uint32), ("entry_bytes", ctypes.c_uint32), ("tier", ctypes.c_uint32),
                ("hot_rows", ctypes.c_uint32), ("forward", ctypes.c_uint32), ("stride", ctypes.c_uint32),
                ("threads", ctypes.c_uint32)]


class ac_stt_info(ctypes.Structure):
    _fields_ = [("n_patterns", ctypes.c_uint32), ("n_states", ctypes.c_uint32), ("n_classes", ctypes.c_uint32),
                ("row_stride", ctypes.c_uint32), ("entry_bytes", ctypes.c_uint32), ("tier", ctypes.c_uint32),
                ("hot_rows", ctypes.c_uint32), ("maxlen", ctypes.c_uint32), ("forward", ctypes.c_uint32),
                ("info_col", ctypes.c_uint32), ("stt_bytes", ctypes.c_uint64), ("out_entries", ctypes.c_uint64),
                ("compact_dense", ctypes.c_uint32), ("compact_od", ctypes.c_uint32), ("compact_os", ctypes.c_uint32),
                ("compact_dstride", ctypes.c_uint32), ("compact_sparse_off", ctypes.c_uint32),
                ("compact_out_off", ctypes.c_uint32), ("compact_bytes", ctypes.c_uint64),
                ("stride", ctypes.c_uint32), ("stride2_cols", ctypes.c_uint32), ("stt2_bytes", ctypes.c_uint64),
                ("split_dense", ctypes.c_uint32), ("split_records", ctypes.c_uint32),
                ("split_dstride", ctypes.c_uint32), ("split_cold_records", ctypes.c_uint32),
                ("split_bytes", ctypes.c_uint64)]


class ac_match_opts(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_uint32), ("kernel", ctypes.c_uint32), ("chain_bytes", ctypes.c_uint32),
                ("variant", ctypes.c_uint32), ("scratch_slots", ctypes.c_uint32), ("two_pass", ctypes.c_uint32),
                ("stride", ctypes.c_uint32),
                ("n_events", ctypes.c_uint32),
                ("events", ctypes.POINTER(ctypes.c_void_p)),
                ("text_policy", ctypes.c_uint32), ("text_promotion", ctypes.c_uint32),
                ("l2_window_mib", ctypes.c_uint32)]


_lib = None
_vp, _u64, _u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32
_u64p = ctypes.POINTER(ctypes.c_uint64)


def lib():
    """Load libac.so (it must have been built: __graft_entry__.build())."""
    global _lib
    if _lib is None:
        if not LIB_PATH.exists():
            raise RuntimeError(f"{LIB_PATH} is missing -- run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = ctypes.CDLL(str(LIB_PATH))
        L.ac_build.argtypes = [_vp, _vp, _u32, ctypes.c_int, ctypes.POINTER(ac_build_opts), ctypes.POINTER(_vp)]
        L.ac_compile.argtypes = [_vp, _vp, _u32, ctypes.POINTER(ac_build_opts), ctypes.POINTER(_vp)]
        L.ac_free.argtypes = [_vp]
        L.ac_free.restype = None
        L.ac_table_free.argtypes = [_vp]
        L.ac_table_free.restype = None
        L.ac_stt_query.argtypes = [_vp, ctypes.POINTER(ac_stt_info)]
        L.ac_table_query.argtypes = [_vp, ctypes.POINTER(ac_stt_info)]
        L.ac_table_export.argtypes = [_vp, _vp, _vp, _vp, _vp]
        L.ac_table_export_compact.argtypes = [_vp, _vp, _vp]
        L.ac_table_export_stride2.argtypes = [_vp, _vp]
        L.ac_table_export_split.argtypes = [_vp, _vp]
        L.ac_stt_pattern_lengths.argtypes = [_vp, _vp]
        L.ac_match.argtypes = [_vp, _vp, _u64, _vp, _u64, _u64p, _vp]
        L.ac_match_shard.argtypes = [_vp, _vp, _u64, _u64, _u64, _vp, _u64, _u64p, _vp]
        L.ac_match_async.argtypes = [_vp, _vp, _u64, _u64, _u64, _vp, _u64, _vp, _vp, ctypes.POINTER(ac_match_opts)]
        L.ac_match_host.argtypes = [_vp, _vp, _u64, _vp, _u64, _u64p, _vp]
        L.ac_match_segments.argtypes = [_vp, _vp, _vp, _u64, _vp, _u64, _vp, _vp]
        L.ac_last_launch_count.restype = _u32
        L.ac_last_launch_count.argtypes = []
        L.ac_last_launch_name.restype = ctypes.c_char_p
        L.ac_last_launch_name.argtypes = [_u32]
        L.ac_last_launch_text_bytes.restype = _u64
        L.ac_last_launch_text_bytes.argtypes = [_u32]
        L.ac_last_scratch_record_bytes.restype = _u32
        L.ac_last_scratch_record_bytes.argtypes = []
        L.ac_status_string.restype = ctypes.c_char_p
        L.ac_status_string.argtypes = [ctypes.c_int]
        L.ac_last_error.restype = ctypes.c_char_p
        L.ac_last_error.argtypes = []
        L.ac_version.restype = ctypes.c_char_p
        L.ac_version.argtypes = []
        _lib = L
    return _lib


def build_library(force: bool = False) -> Path:
    return _build.build(force=force)


def _status_name(s: int) -> str:
    try:
        return lib().ac_status_string(s).decode()
    except Exception:  # pragma: no cover
        return f"status {s}"


def _check(status: int):
    if status != AC_OK:
        raise AcError(status, lib().ac_last_error().decode())


def _pattern_arrays(patterns):
    pats = [bytes(p) for p in patterns]
    bufs = [ctypes.create_string_buffer(p, max(1, len(p))) for p in pats]
    ptrs = (ctypes.c_void_p * max(1, len(pats)))(*[ctypes.cast(b, ctypes.c_void_p) for b in bufs])
    lens = (ctypes.c_uint32 * max(1, len(pats)))(*[len(p) for p in pats])
    return pats, bufs, ptrs, lens


def _opts(entry_bytes=0, tier=TIER_AUTO, hot_rows=0, forward=False, stride=0, threads=0):
    return ac_build_opts(ctypes.sizeof(ac_build_opts), entry_bytes, tier, hot_rows, 1 if forward else 0, stride,
                         threads)


def _info_dict(info: ac_stt_info) -> dict:
    return {f: getattr(info, f) for f, _ in info._fields_ if f != "reserved"}


class Stt:
    """A device STT (phase-1 result), immutable, freed with the object."""

    def __init__(self, patterns, device: int = 0, entry_bytes: int = 0, tier: int = TIER_AUTO, hot_rows: int = 0,
                 stride: int = 0, threads: int = 0):
        L = lib()
        self.patterns, bufs, ptrs, lens = _pattern_arrays(patterns)
        h = ctypes.c_void_p()
        o = _opts(entry_bytes, tier, hot_rows, stride=stride, threads=threads)
        _check(L.ac_build(ptrs, lens, len(self.patterns), int(device), ctypes.byref(o), ctypes.byref(h)))
        self._h = h
        self.device = int(device)
        info = ac_stt_info()
        _check(L.ac_stt_query(h, ctypes.byref(info)))
        self.info = _info_dict(info)
        self.maxlen = self.info["maxlen"]
        self.lens = torch.tensor([len(p) for p in self.patterns], dtype=torch.int64)

    @property
    def handle(self):
        return self._h

    @property
    def tier_name(self) -> str:
        return TIER_NAMES.get(self.info["tier"], "?")

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and _lib is not None:
            _lib.ac_free(h)
            self._h = None


def build(patterns, device: int = 0, **kw) -> Stt:
    """Phase 1: dictionary -> device STT."""
    return Stt(patterns, device=device, **kw)


def _stream_ptr(stream) -> int:
    s = stream if stream is not None else torch.cuda.current_stream()
    return int(s.cuda_stream)


def _check_text(text: torch.Tensor):
    if not isinstance(text, torch.Tensor) or text.dtype != torch.uint8 or not text.is_cuda:
        raise TypeError("text must be a torch.uint8 CUDA tensor")
    if text.dim() != 1 or not text.is_contiguous():
        raise ValueError("text must be 1-D and contiguous")


def _mopts(kernel: int = KERNEL_AUTO, chain_bytes: int = 0, variant: int = 0, scratch_slots: int = 0,
           two_pass: int = 0, events=None, stride: int = 0, text_policy: int = 0, text_promotion: int = 0,
           l2_window_mib: int = 0):
    o = ac_match_opts(ctypes.sizeof(ac_match_opts), kernel, chain_bytes, variant, scratch_slots,
                      int(two_pass), stride, 0, None, text_policy, text_promotion, l2_window_mib)
    if events:
        arr = (ctypes.c_void_p * (2 * len(events)))(*[e.cuda_event for pair in events for e in pair])
        o.n_events = len(events)
        o.events = ctypes.cast(arr, ctypes.POINTER(ctypes.c_void_p))
        o._keep = arr
    return o


def match_async(stt: Stt, text: torch.Tensor, out: torch.Tensor | None, result: torch.Tensor, *,
                n_halo: int = 0, base: int = 0, stream=None, kernel: int = KERNEL_AUTO, chain_bytes: int = 0,
                variant: int = 0, scratch_slots: int = 0, two_pass: int = 0, stride: int = 0,
                events=None, text_policy: int = 0, text_promotion: int = 0, l2_window_mib: int = 0) -> int:
    """Enqueue the scan; result (int64[2] CUDA) receives (count, status).
    ``text`` holds n_owned + n_halo bytes.  ``kernel``/``chain_bytes``/
    ``variant``/``scratch_slots``/``two_pass`` select the scan (ac_match_opts; ``two_pass``: 0 auto,
    1 two passes, 2/3 single-pass ablations, 4 the EVENTS single pass).  ``events``: optional list
    of (start, end) torch.cuda.Event pairs (already created, i.e. recorded
    once) recorded around each kernel launch.  Returns the number of kernel
    launches issued."""
    _check_text(text)
    n_total = text.numel()
    if n_halo > n_total:
        raise ValueError("n_halo > len(text)")
    if result.dtype != torch.int64 or result.numel() < 2 or not result.is_cuda:
        raise TypeError("result must be an int64 CUDA tensor with 2 elements")
    cap = 0
    optr = None
    if out is not None:
        if out.dtype != torch.int64 or not out.is_cuda or not out.is_contiguous():
            raise TypeError("out must be a contiguous int64 CUDA tensor")
        cap = out.numel()
        # non-NULL selects list mode; with cap == 0 the status gates every write
        optr = out.data_ptr() if cap else result.data_ptr()
    o = _mopts(kernel, chain_bytes, variant, scratch_slots, two_pass, events, stride, text_policy, text_promotion,
               l2_window_mib)
    L = lib()
    _check(L.ac_match_async(stt.handle, text.data_ptr() if n_total else None, n_total - n_halo, n_halo, base,
                            optr, cap, result.data_ptr(), _stream_ptr(stream), ctypes.byref(o)))
    return int(L.ac_last_launch_count())


def count(stt: Stt, text: torch.Tensor, *, n_halo: int = 0, stream=None, **knobs) -> int:
    """Number of occurrences (count-only scan); knobs as in match_async."""
    res = torch.zeros(2, dtype=torch.int64, device=text.device)
    match_async(stt, text, None, res, n_halo=n_halo, stream=stream, **knobs)
    return int(res[0].item())


def match(stt: Stt, text: torch.Tensor, out: torch.Tensor | None = None, *, n_halo: int = 0, base: int = 0,
          stream=None, **knobs):
    """Phase 2: (count, records) with records = out[:count] in canonical
    (start, pattern) order.  Without ``out`` a count pass sizes the buffer."""
    res = torch.zeros(2, dtype=torch.int64, device=text.device)
    if out is None:
        match_async(stt, text, None, res, n_halo=n_halo, base=base, stream=stream, **knobs)
        need = int(res[0].item())
        out = torch.empty(max(1, need), dtype=torch.int64, device=text.device)
        res.zero_()
    match_async(stt, text, out, res, n_halo=n_halo, base=base, stream=stream, **knobs)
    c, st = (int(x) for x in res.tolist())
    if st == AC_ERR_CAPACITY:
        raise CapacityError(st, f"{c} records do not fit in {out.numel()}", c)
    _check(st)
    return c, out[:c]


def match_segments(stt: Stt, text: torch.Tensor, seg_off: torch.Tensor, out: torch.Tensor | None = None, *,
                   stream=None):
    """Packet batch (NEXT-2): segment i = text[seg_off[i]:seg_off[i+1]] is
    scanned on its own (no match crosses a boundary).  seg_off: int64 CUDA
    tensor of n_seg + 1 ascending offsets.  Returns (count, records) with
    starts relative to ``text``; without ``out`` a count pass sizes it."""
    _check_text(text)
    if seg_off.dtype != torch.int64 or not seg_off.is_cuda or seg_off.dim() != 1 or seg_off.numel() < 1:
        raise TypeError("seg_off must be a 1-D int64 CUDA tensor of n_seg + 1 offsets")
    n_seg = seg_off.numel() - 1
    L = lib()
    res = torch.zeros(2, dtype=torch.int64, device=text.device)
    s = _stream_ptr(stream)
    tp = text.data_ptr() if text.numel() else None
    if out is None:
        _check(L.ac_match_segments(stt.handle, tp, seg_off.data_ptr(), n_seg, None, 0, res.data_ptr(), s))
        out = torch.empty(max(1, int(res[0].item())), dtype=torch.int64, device=text.device)
    _check(L.ac_match_segments(stt.handle, tp, seg_off.data_ptr(), n_seg, out.data_ptr(), out.numel(),
                               res.data_ptr(), s))
    c, st = (int(x) for x in res.tolist())
    if st == AC_ERR_CAPACITY:
        raise CapacityError(st, f"{c} records do not fit in {out.numel()}", c)
    _check(st)
    return c, out[:c]


def match_host(stt: Stt, text_host: torch.Tensor, out_host: torch.Tensor | None, *, stream=None) -> int:
    """End-to-end call with HOST buffers (H2D of the text, scan, D2H of the
    count and list inside libac).  Returns the count."""
    if text_host.dtype != torch.uint8 or text_host.is_cuda or not text_host.is_contiguous():
        raise TypeError("text_host must be a contiguous CPU uint8 tensor")
    cap = 0 if out_host is None else out_host.numel()
    c = ctypes.c_uint64(0)
    optr = None if out_host is None else out_host.data_ptr()
    st = lib().ac_match_host(stt.handle, text_host.data_ptr() if text_host.numel() else None, text_host.numel(),
                             optr, cap, ctypes.byref(c), _stream_ptr(stream))
    if st == AC_ERR_CAPACITY:
        raise CapacityError(st, lib().ac_last_error().decode(), int(c.value))
    _check(st)
    return int(c.value)


def last_launch_count() -> int:
    return int(lib().ac_last_launch_count())


def last_launch_names() -> list[str]:
    L = lib()
    return [L.ac_last_launch_name(i).decode() for i in range(L.ac_last_launch_count())]


def last_launch_text_bytes() -> list[int]:
    """Owned text bytes each launch of the last match_async walked (0 = not a scan)."""
    L = lib()
    return [int(L.ac_last_launch_text_bytes(i)) for i in range(min(16, int(L.ac_last_launch_count())))]


def last_scratch_record_bytes() -> int:
    """4 (narrow), 8 or 0: scratch bytes per record of the last list-mode call."""
    return int(lib().ac_last_scratch_record_bytes())


def version() -> str:
    return lib().ac_version().decode()


# ----------------------------------------------------------- record decoding
def starts(recs: torch.Tensor) -> torch.Tensor:
    return recs >> 24


def pattern_ids(recs: torch.Tensor) -> torch.Tensor:
    return recs & 0xFFFFFF


def ends(recs: torch.Tensor, lens: torch.Tensor) -> torch.Tensor:
    """The paper's "end of position": start + len(pattern) - 1."""
    return (recs >> 24) + lens.to(recs.device)[recs & 0xFFFFFF] - 1


# ------------------------------------------------------- host-only builder
@dataclass
class HostTable:
    info: dict
    class_map: "object"
    stt: "object"
    out_off: "object"
    out_ids: "object"
    compact: "object" = None   # COMPACT blob (uint8) if requested
    stt2: "object" = None      # two-byte table (uint32, S x stride2_cols) if requested
    perm: "object" = None      # compact id -> dense BFS id
    split: "object" = None     # SPLIT shared-memory part (uint8) if requested


def compile_table(patterns, forward: bool = False, entry_bytes: int = 0, compact: bool = False,
                  stride: int = 0, split: bool = False, threads: int = 0) -> HostTable:
    """Phase 1 on the host only (no device) -- for builder tests."""
    import numpy as np
    L = lib()
    pats, bufs, ptrs, lens = _pattern_arrays(patterns)
    h = ctypes.c_void_p()
    tier = TIER_COMPACT if compact else TIER_SPLIT if split else TIER_AUTO
    o = _opts(entry_bytes=entry_bytes, forward=forward, tier=tier, stride=stride, threads=threads)
    _check(L.ac_compile(ptrs, lens, len(pats), ctypes.byref(o), ctypes.byref(h)))
    try:
        info = ac_stt_info()
        _check(L.ac_table_query(h, ctypes.byref(info)))
        d = _info_dict(info)
        cm = np.zeros(256, dtype=np.uint8)
        dt = np.uint16 if d["entry_bytes"] == 2 else np.uint32
        stt = np.zeros(d["n_states"] * d["row_stride"], dtype=dt)
        off = np.zeros(d["n_states"] + 1, dtype=np.uint32)
        ids = np.zeros(max(1, d["out_entries"]), dtype=np.uint32)
        _check(L.ac_table_export(h, cm.ctypes.data, stt.ctypes.data, off.ctypes.data, ids.ctypes.data))
        blob = perm = None
        if compact:
            blob = np.zeros(d["compact_bytes"], dtype=np.uint8)
            perm = np.zeros(d["n_states"], dtype=np.uint32)
            _check(L.ac_table_export_compact(h, blob.ctypes.data, perm.ctypes.data))
        t2 = None
        if d["stride"] == 2:
            t2 = np.zeros(d["n_states"] * d["stride2_cols"], dtype=np.uint32)
            _check(L.ac_table_export_stride2(h, t2.ctypes.data))
            t2 = t2.reshape(d["n_states"], d["stride2_cols"])
        sp = None
        if split:
            sp = np.zeros(d["split_bytes"], dtype=np.uint8)
            _check(L.ac_table_export_split(h, sp.ctypes.data))
        return HostTable(d, cm, stt.reshape(d["n_states"], d["row_stride"]), off, ids[:d["out_entries"]],
                         compact=blob, stt2=t2, perm=perm, split=sp)
    finally:
        L.ac_table_free(h)
