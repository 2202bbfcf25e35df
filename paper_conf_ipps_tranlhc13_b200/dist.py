"""Multi-GPU matching: contiguous text shards with halos, one process per GPU.

SURVEY 8(e).  The scan has no exchange inside it (every shard is scanned
independently, exactly like the paper's per-thread chunks, one
level up): rank g owns the match STARTS in [lo_g, hi_g) and reads
[lo_g, hi_g + halo_g) with halo_g = min(maxlen - 1, n - hi_g).  Because the
canonical order is start-major and ownership is by start, the rank-order
concatenation of the per-rank canonical lists IS the global canonical list --
no merge.  The only real exchange steps are the combine:

  * all_reduce(SUM) of the per-rank counts (the global match count), and
  * an allgatherv of the match lists when every rank wants the whole list
    (NCCL has no allgatherv: all_gather the counts, pad to the max, one
    all_gather_into_tensor, trim).

`torch.distributed` supplies the process group (NCCL over NVLink/NVSwitch on
a B200 box; gloo on CPU for the host-logic tests).  The per-shard scan is
libac's ac_match_shard (binding: ``match(..., n_halo=, base=)``).
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as dist


@dataclass(frozen=True)
class Shard:
    rank: int
    lo: int      # first owned start
    hi: int      # one past the last owned start
    halo: int    # bytes read past hi (<= maxlen - 1)

    @property
    def owned(self) -> int:
        return self.hi - self.lo

    @property
    def read_hi(self) -> int:
        return self.hi + self.halo


def plan_shards(n: int, world: int, maxlen: int, align: int = 16) -> list[Shard]:
    """Contiguous shards: lo_g = floor(g*n/G) rounded down to `align` bytes
    (so every shard starts on a TMA-friendly address when the text does), the
    last shard takes the remainder; halo_g = min(maxlen - 1, n - hi_g)."""
    if world < 1:
        raise ValueError("world must be >= 1")
    H = max(0, maxlen - 1)
    bounds = [0]
    for g in range(1, world):
        b = (g * n // world) // align * align
        bounds.append(max(b, bounds[-1]))
    bounds.append(n)
    return [Shard(g, bounds[g], bounds[g + 1], min(H, n - bounds[g + 1])) for g in range(world)]


def _comm_device(t: torch.Tensor, group=None):
    """gloo moves host tensors (CPU tests, or GPU ranks without NCCL); NCCL
    moves device tensors over NVLink/NVSwitch."""
    return torch.device("cpu") if dist.get_backend(group) == "gloo" else t.device


def allreduce_count(count, device, group=None) -> int:
    """Global match count: all_reduce(SUM) of the per-rank counts (an int or a
    1-element int64 tensor)."""
    t = count.reshape(1).to(torch.int64) if isinstance(count, torch.Tensor) else \
        torch.tensor([count], dtype=torch.int64, device=device)
    t = t.to(_comm_device(t, group)).clone()
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return int(t.item())


def allgatherv(records: torch.Tensor, group=None) -> torch.Tensor:
    """Concatenate every rank's 1-D int64 tensor in rank order (on all ranks)."""
    world = dist.get_world_size(group)
    home = records.device
    dev = _comm_device(records, group)
    records = records.to(dev)
    n = torch.tensor([records.numel()], dtype=torch.int64, device=dev)
    counts = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in range(world)]
    dist.all_gather(counts, n, group=group)
    counts = [int(c.item()) for c in counts]
    m = max(counts) if counts else 0
    if m == 0:
        return records.new_empty(0).to(home)
    padded = torch.full((m,), -1, dtype=torch.int64, device=dev)
    padded[:records.numel()] = records
    out = torch.empty(world * m, dtype=torch.int64, device=dev)
    dist.all_gather_into_tensor(out, padded, group=group)
    return torch.cat([out[g * m:g * m + c] for g, c in enumerate(counts)]).to(home)


def default_capacity(owned: int) -> int:
    """Count-free output capacity: one record per 8 owned bytes (an output
    buffer the size of the text).  Enough for the BASELINE configs (<= 0.07
    matches per byte); a denser shard reports its exact need and is re-run."""
    return owned // 8 + 64


def match_sharded(stt, shard_text: torch.Tensor, shard: Shard, *, out: torch.Tensor | None = None,
                  gather: bool = True, group=None, stream=None, **knobs):
    """Scan this rank's shard (device tensor holding text[shard.lo : shard.read_hi])
    in ONE emitting pass and combine.  Returns (global_count, records): the
    global canonical list when gather=True, else this rank's slice of it
    (rank-order concatenation of the slices is the global list).  ``out``:
    optional int64 device buffer (default: default_capacity)."""
    from . import AC_ERR_CAPACITY, _check, match_async  # the CUDA path; no fallback
    if shard_text.numel() != shard.read_hi - shard.lo:
        raise ValueError("shard_text must hold text[lo:hi + halo]")
    dev = shard_text.device
    if out is None:
        out = torch.empty(default_capacity(shard.owned), dtype=torch.int64, device=dev)
    res = torch.zeros(2, dtype=torch.int64, device=dev)
    match_async(stt, shard_text, out, res, n_halo=shard.halo, base=shard.lo, stream=stream, **knobs)
    c, st = (int(x) for x in res.tolist())
    if st == AC_ERR_CAPACITY:  # denser than the default bound: exact size, scan again
        out = torch.empty(max(1, c), dtype=torch.int64, device=dev)
        match_async(stt, shard_text, out, res, n_halo=shard.halo, base=shard.lo, stream=stream, **knobs)
        c, st = (int(x) for x in res.tolist())
    _check(st)
    recs = out[:c]
    total = allreduce_count(res[:1], dev, group)
    if gather:
        recs = allgatherv(recs.contiguous(), group)
    return total, recs
