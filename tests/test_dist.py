"""Multi-process host logic of the sharded scan on CPU: gloo,
world_size 2 and 3.  The per-shard scan is played by the oracle's window
mode (tests may call oracle/); the product path calls libac instead
(dist.match_sharded, covered by the GPU tests)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_tranlhc13_b200.dist import Shard, allgatherv, allreduce_count, plan_shards


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("n,world,maxlen", [(0, 2, 5), (10, 3, 4), (1000, 8, 32), (1 << 20, 7, 64), (17, 8, 1)])
def test_plan_shards(n, world, maxlen):
    sh = plan_shards(n, world, maxlen)
    assert len(sh) == world and sh[0].lo == 0 and sh[-1].hi == n
    for a, b in zip(sh[:-1], sh[1:]):
        assert a.hi == b.lo
    for s in sh:
        assert s.lo <= s.hi and s.halo == min(maxlen - 1, n - s.hi)
        assert s.lo % 16 == 0 or s.lo == n


def _keys(o, text, lo, hi):
    ends, pids = o.match_window(text, lo, hi)
    starts = ends.astype(np.int64) - o.lens[pids].astype(np.int64) + 1
    return torch.from_numpy(np.ascontiguousarray((starts << 24) | pids.astype(np.int64)))


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        from oracle import Oracle
        w = synth.make("c2", n=(1 << 18) + 37, n_patterns=150)
        o = Oracle(w.patterns)
        shards = plan_shards(w.text.size, world, o.maxlen)
        me = shards[rank]
        local_text = w.text[me.lo:me.read_hi]           # what this rank holds
        local = _keys(o, local_text, 0, me.owned)       # its shard scan (starts local)
        local = local + (me.lo << 24)                   # base = lo
        total = allreduce_count(local.numel(), "cpu")
        full = allgatherv(local)
        want = _keys(o, w.text, 0, w.text.size)
        ok = total == want.numel() and torch.equal(full, want)
        # only rank 0 contributes: every rank must receive exactly rank 0's
        # slice (each rank recomputes it from the oracle to compare)
        r0 = _keys(o, w.text[:shards[0].read_hi], 0, shards[0].owned)
        got0 = allgatherv(torch.empty(0, dtype=torch.int64) if rank else local)
        ok = ok and torch.equal(got0, r0)
        # and nobody contributes
        ok = ok and allgatherv(torch.empty(0, dtype=torch.int64)).numel() == 0
        q.put((rank, bool(ok), total, want.numel()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_combine_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(ok for _, ok, _, _ in res), res
