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
                        ("static", dict(cache_frac=0.05), 2),
                        # host-assisted (forced, every batch): request forwarding and early-fetch side CTAs of KQ
                        ("assisted", dict(cache_frac=0.02, invalid_ppm=3000), 8)]:
    if name == "assisted":
        os.environ.update(FLECHE_HA_MIN_ROWS="0", FLECHE_HA_EARLY_MIN="0", FLECHE_HA_FRAC="0.5")
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

# later round-1 paths: watermark scan (uniform + bytes layout), short flat keys, prefill,
# decoupled hit copy, host-assisted split.  (Not the early fetch: KF spins on KQ's
# progress, and the sanitizer serialises kernels.)
for name, kw, flags, extra in [("watermark", dict(cache_frac=0.25), 0, "wm"),
                               ("watermark_mixed", dict(cache_frac=0.2, dims=[8, 16, 32, 64, 128, 8, 256]), 0, "wm"),
                               ("short_keys", dict(cache_frac=0.1), 0, "kb"),
                               ("prefill", dict(cache_frac=0.1), 0, "pf"),
                               ("decoupled", dict(cache_frac=0.05), 0, "dc"),
                               ("ha_split", dict(cache_frac=0.05), 8, "ha")]:
    if extra == "dc":
        os.environ["FLECHE_DECOUPLE_MIN"] = "0"
    if extra == "ha":
        os.environ["FLECHE_HA_FRAC"] = "0.5"
    w = configs.get("cfg0").with_(batch_size=100, **kw)
    tabs = [np.ascontiguousarray(t) for t in w.make_tables()[1]]
    g = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n, 0, 1.0, 0, H.HASH_SEED, flags,
                     12 if extra == "kb" else 0)
    o = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_GLOBAL)
    if extra == "kb":
        o.set_key_bits(12)
    if extra == "wm":
        g.set_watermarks(0.5, 0.3)
    if extra == "pf":
        g.prefill([torch.from_numpy(x).cuda() for x in w.batch(50).ids])
        o.query(w.batch(50).ids)
    for b in range(nb):
        bt = w.batch(b)
        got = H.run_batch_gpu(g, bt.ids, torch)
        assert H.bits_equal(got, o.query(bt.ids)), (name, b)
    print(name, "ok", g.stats()["hits"], g.stats()["scans"])
    os.environ.pop("FLECHE_DECOUPLE_MIN", None)
    os.environ.pop("FLECHE_HA_FRAC", None)
