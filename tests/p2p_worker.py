"""Worker for test_gpu_sharded.test_p2p_two_processes_one_gpu: one rank of a 2-rank gloo
group on cuda:0 running the fused key-sharded exchange (CUDA IPC peer reads), checked
bit-exact against the oracle's values.  Writes a JSON result line to argv[3]."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402


def main():
    rank, world, outp, port = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3], sys.argv[4]
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    import paper_conf_eurosys_xiellwgrs22_b200 as fl
    from paper_conf_eurosys_xiellwgrs22_b200.sharded import ShardedCache
    from oracle import oracle as O
    from tests import harness as H
    from workload import configs
    w = configs.get("cfg0").with_(invalid_ppm=3000, cache_frac=0.1)
    tabs = [np.ascontiguousarray(t) for t in w.make_tables()[1]]
    cache = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n * world, 0, 1.0, 0, H.HASH_SEED)
    sh = ShardedCache(cache, row_floats=w.dims[0], p2p=True)
    ref = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_GLOBAL)  # values only
    ok, owner_hits = True, 0
    for b in range(12):
        bt = w.batch(b, rank=rank)
        ids = [torch.from_numpy(x).cuda() for x in bt.ids]
        out = torch.full((cache.out_floats([x.size for x in bt.ids]),), float("nan"), device="cuda")
        sh.query(ids, out)
        torch.cuda.synchronize()
        if not H.bits_equal(out.cpu().numpy(), ref.query(bt.ids)):
            ok = False
    torch.cuda.synchronize()
    ss = cache.shard_stats()
    lk, hits, inv = ss["lookups"], ss["hits"], ss["invalid"]
    st = cache.stats()
    sh.close()
    with open(outp, "w") as f:
        f.write(json.dumps({"rank": rank, "ok": ok, "owner_hits": st["hits"], "owner_lookups": st["lookups"],
                            "req_hits": int(hits), "req_lookups": int(lk), "invalid": int(inv)}))
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
