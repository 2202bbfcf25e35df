"""The sharded scan with libac on every rank: world size 2 and
3, every rank on cuda:0 (one GPU in this pool), gloo carrying the combine
(all_reduce of the counts, allgatherv of the lists) through host memory.
Checked against the oracle over the whole text: the rank-order concatenation
of start-owned shards is the canonical list (P:163-164 one level up)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_tranlhc13_b200 as ac
        import synth
        from oracle import Oracle
        from paper_conf_ipps_tranlhc13_b200.dist import match_sharded, plan_shards
        w = synth.make("c2", n=(3 << 20) + 37, n_patterns=300)
        stt = ac.build(w.patterns, device=0)
        me = plan_shards(w.text.size, world, stt.maxlen)[rank]
        t = torch.from_numpy(np.ascontiguousarray(w.text[me.lo:me.read_hi])).cuda()
        total, recs = match_sharded(stt, t, me, gather=True)
        # rank-local slice only, tiny capacity: exercises the capacity re-run
        tot2, mine = match_sharded(stt, t, me, gather=False,
                                   out=torch.empty(3, dtype=torch.int64, device="cuda"))
        o = Oracle(w.patterns)
        ends, pids = o.match(w.text)
        starts = ends.astype(np.int64) - o.lens[pids].astype(np.int64) + 1
        want = (starts << 24) | pids.astype(np.int64)
        s = want >> 24
        mine_want = want[(s >= me.lo) & (s < me.hi)]
        ok = (total == want.size and tot2 == want.size and np.array_equal(recs.cpu().numpy(), want)
              and np.array_equal(mine.cpu().numpy(), mine_want))
        q.put((rank, bool(ok), int(total), int(want.size)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_match_sharded_libac_gloo(world):
    assert torch.cuda.is_available()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert all(ok for _, ok, _, _ in res), res
