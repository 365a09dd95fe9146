"""Key-sharded mode on one B200: the routing kernel's owner grouping, and a one-rank NCCL
group running the full route -> all-to-all -> owner query -> all-to-all -> restore path
(needs a GPU; multi-rank plumbing is covered on CPU by tests/test_dist_cpu.py)."""
import socket

import numpy as np
import pytest

from oracle import oracle as O
from tests import harness as H
from tests.shard_double import owner_of
from workload import configs

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _tables(w):
    return [np.ascontiguousarray(t) for t in w.make_tables()[1]]


@pytest.mark.parametrize("world", [1, 3, 8])
def test_route_groups_unique_keys_by_owner(world):
    import paper_conf_eurosys_xiellwgrs22_b200 as fl
    w = configs.get("cfg0").with_(invalid_ppm=5000)
    tabs = _tables(w)
    gpu = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n, 0, 1.0, 0, H.HASH_SEED)
    _, base, _ = O.encode(w.cards)
    seed = 0x2545F491
    for b in range(3):
        bt = w.batch(b)
        ids = [torch.from_numpy(x).cuda() for x in bt.ids]
        sk = torch.empty(w.batch_size * w.n, dtype=torch.int32, device="cuda")
        sc = torch.empty(world, dtype=torch.int64, device="cuda")
        gpu.route(ids, world, seed, sk, sc)
        torch.cuda.synchronize()
        counts = sc.cpu().numpy()
        keys = sk[:counts.sum()].cpu().numpy().view(np.uint32).astype(np.int64)
        ref = set()
        for t, x in enumerate(bt.ids):
            ok = (x >= 0) & (x < w.cards[t])
            ref |= set((int(base[t]) + x[ok]).tolist())
        assert len(keys) == len(set(keys.tolist())) == len(ref) and set(keys.tolist()) == ref
        off = 0
        for o, c in enumerate(counts):
            assert (owner_of(keys[off:off + c], seed, world) == o).all()
            off += c


def test_sharded_one_rank_nccl_bit_exact_and_exact_hits():
    import torch.distributed as dist

    import paper_conf_eurosys_xiellwgrs22_b200 as fl
    from paper_conf_eurosys_xiellwgrs22_b200.sharded import ShardedCache
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    try:
        w = configs.get("cfg0").with_(cache_frac=0.25, invalid_ppm=3000)
        tabs = _tables(w)
        gpu = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n, 0, 1.0, 0, H.HASH_SEED)
        sc = ShardedCache(gpu, row_floats=w.dims[0])
        orc = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_SETASSOC, hash_seed=H.HASH_SEED)
        for b in range(20):
            bt = w.batch(b)
            ids = [torch.from_numpy(x).cuda() for x in bt.ids]
            out = torch.full((gpu.out_floats([x.size for x in bt.ids]),), float("nan"), device="cuda")
            sc.query(ids, out)
            torch.cuda.synchronize()
            ref = orc.query(bt.ids)
            assert H.bits_equal(out.cpu().numpy(), ref), b
        so, ss, sg = orc.stats(), gpu.shard_stats(), gpu.stats()
        # one rank owns every key: per-lookup hits, unique keys, inserts equal the oracle's
        assert ss["hits"] == so["hits"] and ss["invalid"] == so["invalid"] and ss["lookups"] == so["lookups"]
        assert ss["unique_routed"] == so["unique_keys"] == sg["lookups"]
        for k in ("unique_hits", "unique_misses", "inserted", "evicted"):
            assert sg[k] == so[k], k
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("ha", [False, True])
def test_sharded_p2p_one_rank_nccl_sync_free(monkeypatch, ha):
    """The fused exchange on a real NCCL group (one rank): counts all-gathered into device
    memory and read there by the owner query (grid-strided over the device-side total) and
    the restore, no host read per batch (fleche_query_keys_seg_dev / fleche_restore_p2p_dev);
    out bit-exact and per-lookup hits equal to the set oracle's every batch."""
    import torch.distributed as dist

    import paper_conf_eurosys_xiellwgrs22_b200 as fl
    from paper_conf_eurosys_xiellwgrs22_b200.sharded import ShardedCache
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    try:
        w = configs.get("cfg0").with_(cache_frac=0.25, invalid_ppm=3000)
        tabs = _tables(w)
        monkeypatch.setenv("FLECHE_HA_MIN_ROWS", "0")  # cfg0's few misses per batch: assist every batch
        gpu = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n, 0, 1.0, 0, H.HASH_SEED,
                           fl.binding.FLAG_HOST_ASSIST if ha else 0)
        sc = ShardedCache(gpu, row_floats=w.dims[0], p2p=True)
        orc = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_SETASSOC, hash_seed=H.HASH_SEED)
        for b in range(20):
            bt = w.batch(b)
            ids = [torch.from_numpy(x).cuda() for x in bt.ids]
            out = torch.full((gpu.out_floats([x.size for x in bt.ids]),), float("nan"), device="cuda")
            h0 = gpu.shard_stats()["hits"]
            o0 = orc.stats()["hits"]
            sc.query(ids, out)
            torch.cuda.synchronize()
            assert H.bits_equal(out.cpu().numpy(), orc.query(bt.ids)), b
            assert gpu.shard_stats()["hits"] - h0 == orc.stats()["hits"] - o0, b
        st = gpu.stats()
        if ha:  # the owner's misses went through the host threads, none timed out
            assert st["assisted_rows"] > 0 and st["assist_timeouts"] == 0, st
        sc.close()
    finally:
        dist.destroy_process_group()


def test_p2p_two_processes_one_gpu(tmp_path):
    """The fused exchange (fleche_restore_p2p: every requester reads its rows in place from
    the owners' answer buffers through CUDA IPC mappings) with two ranks sharing cuda:0
    (gloo for the small collectives): `out` bit-exact on both ranks; the requesters saw
    hits, and never more than their valid lookups."""
    import json
    import subprocess
    import sys
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    procs = [subprocess.Popen([sys.executable, "tests/p2p_worker.py", str(r), "2", str(tmp_path / f"r{r}.json"),
                               str(port)]) for r in range(2)]
    for p in procs:
        assert p.wait(timeout=300) == 0
    res = [json.load(open(tmp_path / f"r{r}.json")) for r in range(2)]
    assert all(r["ok"] for r in res), res
    for r in res:
        assert 0 < r["req_hits"] <= r["req_lookups"] - r["invalid"], r
        assert r["owner_hits"] > 0
    # hit ratio vs an oracle of G shard caches (SURVEY 8(e) tests): shard g is one cache
    # of the per-GPU budget that sees, batch by batch, every valid lookup of every rank
    # whose key it owns (same owner() as the route kernel, tests/shard_double.py); the
    # requesters' per-lookup hits must match its hits within 1 pp (concurrent insert order)
    from paper_conf_eurosys_xiellwgrs22_b200.sharded import DEFAULT_OWNER_SEED
    G = 2
    w = configs.get("cfg0").with_(invalid_ppm=3000, cache_frac=0.1)  # as in tests/p2p_worker.py
    tabs = _tables(w)
    _, base, _ = O.encode(w.cards)
    orcs = [O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_GLOBAL) for _ in range(G)]
    for b in range(12):
        bts = [w.batch(b, rank=r) for r in range(G)]
        for g in range(G):
            ids_g = []
            for t in range(w.n):
                parts = []
                for r in range(G):
                    x = bts[r].ids[t]
                    ok = (x >= 0) & (x < w.cards[t])
                    own = owner_of(int(base[t]) + np.where(ok, x, 0), DEFAULT_OWNER_SEED, G) == g
                    parts.append(x[ok & own])
                ids_g.append(np.concatenate(parts))
            orcs[g].query(ids_g)
    o_hits = sum(o.stats()["hits"] for o in orcs)
    o_valid = sum(o.stats()["lookups"] for o in orcs)
    req_hits = sum(r["req_hits"] for r in res)
    req_valid = sum(r["req_lookups"] - r["invalid"] for r in res)
    assert req_valid == o_valid, (req_valid, o_valid)
    assert abs(req_hits - o_hits) <= 0.01 * o_valid, (req_hits, o_hits, o_valid)
