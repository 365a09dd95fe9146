"""Small workload for compute-sanitizer runs (memcheck / racecheck / synccheck):
one-hot uniform, mixed widths, pooled, static, key-sharded route, each a few batches,
checked bit-exact against the oracle."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_eurosys_xiellwgrs22_b200 as fl  # noqa: E402
from oracle import oracle as O  # noqa: E402
from tests import harness as H  # noqa: E402
from workload import configs  # noqa: E402

nb = int(os.environ.get("NB", "3"))
for name, kw, flags in [("uniform", dict(cache_frac=0.02, invalid_ppm=3000), 0),
                        ("mixed", dict(cache_frac=0.05, dims=[8, 16, 32, 64, 128, 8, 256]), 0),
                        ("static", dict(cache_frac=0.05), 2)]:
    w = configs.get("cfg0").with_(batch_size=100, **kw)
    tabs = [np.ascontiguousarray(t) for t in w.make_tables()[1]]
    g = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n, 0, 1.0, 0, H.HASH_SEED, flags)
    o = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_GLOBAL)
    for b in range(nb):
        bt = w.batch(b)
        got = H.run_batch_gpu(g, bt.ids, torch)
        assert H.bits_equal(got, o.query(bt.ids)), (name, b)
    print(name, "ok", g.stats()["hits"])
w = configs.get("cfg4").with_(cards=[max(3, c // 1000) for c in configs.get("cfg4").cards], batch_size=16)
tabs = [np.ascontiguousarray(t) for t in w.make_tables()[1]]
g = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, 8192, 0, 1.0, 0, H.HASH_SEED)
o = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_GLOBAL)
for b in range(nb):
    bt = w.batch(b)
    ids = [torch.from_numpy(x).cuda() for x in bt.ids]
    offs = [torch.from_numpy(x).cuda() for x in bt.offsets]
    out = torch.empty(g.pooled_floats([x.size - 1 for x in bt.offsets]), device="cuda")
    g.query_pooled(ids, offs, out)
    torch.cuda.synchronize()
    assert H.bits_equal(out.cpu().numpy(), o.query_pooled(bt.ids, bt.offsets)), ("pooled", b)
print("pooled ok")
w = configs.get("cfg0").with_(batch_size=100)
tabs = [np.ascontiguousarray(t) for t in w.make_tables()[1]]
g = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n, 0, 1.0, 0, H.HASH_SEED)
ids = [torch.from_numpy(x).cuda() for x in w.batch(0).ids]
sk = torch.empty(w.batch_size * w.n, dtype=torch.int32, device="cuda")
sc = torch.empty(4, dtype=torch.int64, device="cuda")
g.route(ids, 4, 7, sk, sc)
torch.cuda.synchronize()
print("route ok", sc.cpu().tolist())
