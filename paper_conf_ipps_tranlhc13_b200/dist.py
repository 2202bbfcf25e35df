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


def allreduce_count(count: int, device, group=None) -> int:
    t = torch.tensor([count], dtype=torch.int64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return int(t.item())


def allgatherv(records: torch.Tensor, group=None) -> torch.Tensor:
    """Concatenate every rank's 1-D int64 tensor in rank order (on all ranks)."""
    world = dist.get_world_size(group)
    dev = records.device
    n = torch.tensor([records.numel()], dtype=torch.int64, device=dev)
    counts = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in range(world)]
    dist.all_gather(counts, n, group=group)
    counts = [int(c.item()) for c in counts]
    m = max(counts) if counts else 0
    if m == 0:
        return records.new_empty(0)
    padded = torch.full((m,), -1, dtype=torch.int64, device=dev)
    padded[:records.numel()] = records
    out = torch.empty(world * m, dtype=torch.int64, device=dev)
    dist.all_gather_into_tensor(out, padded, group=group)
    return torch.cat([out[g * m:g * m + c] for g, c in enumerate(counts)])


def match_sharded(stt, shard_text: torch.Tensor, shard: Shard, *, gather: bool = True, group=None,
                  stream=None, **knobs):
    """Scan this rank's shard (device tensor holding text[shard.lo : shard.read_hi])
    and combine.  Returns (global_count, records): the global canonical list
    when gather=True, else this rank's slice of it (rank-order concatenation
    of the slices is the global list)."""
    from . import match  # the CUDA path; no fallback
    if shard_text.numel() != shard.read_hi - shard.lo:
        raise ValueError("shard_text must hold text[lo:hi + halo]")
    c, recs = match(stt, shard_text, n_halo=shard.halo, base=shard.lo, stream=stream, **knobs)
    total = allreduce_count(c, shard_text.device, group)
    if gather:
        recs = allgatherv(recs.contiguous(), group)
    return total, recs
