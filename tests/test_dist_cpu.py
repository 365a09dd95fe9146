"""World-size-2 CPU (gloo) tests of the multi-GPU host logic (no GPU needed).

Replicated mode: rank r serves samples [r*B, (r+1)*B) of each global batch with its own
cache over ONE node-shared host tier (/dev/shm); no data-path collective.  Timing is the
max over ranks.  Here each rank runs the oracle replica on its shard (the CUDA path is
covered by tests/test_gpu_*.py); the union of the ranks' outputs must be the plain
definition for the global batch, and the shared host tier must be identical on both.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import oracle as O
from workload import configs, shm


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, name, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        w = configs.get("cfg0").with_(batch_size=64)
        def ago(x):
            out = [None] * world
            dist.all_gather_object(out, x)
            return out
        node = 0  # CPU test: both ranks on node 0 -> one copy, created by the lowest rank
        creator = shm.creator_ranks(rank, node, ago)
        assert creator == (rank == 0)
        buf, tabs, cleanup = shm.shared_tables(name, w.cards, w.dims, 0, rank, dist.barrier, node=node,
                                               creator=creator)
        orc = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes)
        outs = []
        for b in range(4):
            bt = w.batch(b, rank=rank)
            outs.append(orc.query(bt.ids))
        # host-tier identity across ranks: checksum of the shared pages
        cs = torch.tensor([float(np.float64(buf[::997].astype(np.float64).sum()))], dtype=torch.float64)
        allcs = [torch.zeros_like(cs) for _ in range(world)]
        dist.all_gather(allcs, cs)
        # max over ranks (the bench's timing reduction)
        t = torch.tensor([float(rank + 1)])
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        gathered = [None] * world
        dist.all_gather_object(gathered, [o.tolist() for o in outs])
        dist.barrier()
        cleanup()
        if rank == 0:
            q.put((gathered, [float(x) for x in allcs], float(t)))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_replicated_two_ranks_cover_the_global_batch():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    name = f"fleche_test_{os.getpid()}_{port}"
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in procs:
        p.start()
    gathered, cs, tmax = q.get(timeout=240)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    assert cs[0] == cs[1] and tmax == 2.0
    # the global batch (2B samples) looked up directly
    w = configs.get("cfg0").with_(batch_size=64)
    wg = w.with_(batch_size=128)
    _, tabs = w.make_tables()
    for b in range(4):
        g = wg.batch(b)
        for r in range(world):
            got = np.array(gathered[r][b], np.float32)
            off = 0
            for t, ids in enumerate(g.ids):
                d = w.dims[t]
                mine = ids[r * 64:(r + 1) * 64]
                ref = np.zeros((64, d), np.float32)
                ok = (mine >= 0) & (mine < w.cards[t])
                ref[ok] = tabs[t][mine[ok]]
                assert np.array_equal(got[off:off + 64 * d].reshape(64, d), ref)
                off += 64 * d
    assert not os.path.exists(os.path.join("/dev/shm", name))


# ------------------------------------------------------------------ key-sharded plumbing
def _sharded_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_eurosys_xiellwgrs22_b200.sharded import ShardedCache
        from tests.shard_double import ShardDouble
        w = configs.get("cfg0").with_(batch_size=40, invalid_ppm=20000)
        _, tabs = w.make_tables()
        dbl = ShardDouble(w.cards, w.dims, tabs, max_lookups=w.batch_size * w.n * world)
        sc = ShardedCache(dbl, row_floats=w.dims[0], device=torch.device("cpu"))
        res = []
        for b in range(3):
            bt = w.batch(b, rank=rank)
            out = torch.zeros(sum(x.size * d for x, d in zip(bt.ids, w.dims)))
            ex = sc.query([torch.from_numpy(x) for x in bt.ids], out)
            res.append((out.numpy().tolist(), ex))
        gathered = [None] * world
        dist.all_gather_object(gathered, res)
        if rank == 0:
            q.put(gathered)
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_sharded_plumbing_two_ranks():
    # ranks exchange keys and rows with all-to-alls (gloo here, NCCL on GPUs); every
    # rank's output must be the plain definition for its own shard of the batch, and the
    # keys each rank sends must equal the keys the owners receive
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sharded_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    gathered = q.get(timeout=240)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    w = configs.get("cfg0").with_(batch_size=40, invalid_ppm=20000)
    _, tabs = w.make_tables()
    for b in range(3):
        sent = sum(gathered[r][b][1]["sent_keys"] for r in range(world))
        recv = sum(gathered[r][b][1]["recv_keys"] for r in range(world))
        assert sent == recv > 0
        for r in range(world):
            got = np.array(gathered[r][b][0], np.float32)
            bt = w.batch(b, rank=r)
            off = 0
            for t, ids in enumerate(bt.ids):
                d = w.dims[t]
                ref = np.zeros((ids.size, d), np.float32)
                ok = (ids >= 0) & (ids < w.cards[t])
                ref[ok] = tabs[t][ids[ok]]
                assert np.array_equal(got[off:off + ids.size * d].reshape(ids.size, d), ref)
                off += ids.size * d
