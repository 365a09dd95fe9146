"""Debug helper: structural check of the static per-table layout after a few batches."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_eurosys_xiellwgrs22_b200 as fl  # noqa: E402
from oracle import oracle as O  # noqa: E402
from tests import harness as H  # noqa: E402
from workload import configs  # noqa: E402

w = configs.get("cfg2").with_(cards=[max(3, c // 20) for c in configs.KAGGLE], batch_size=1024)
tabs = [np.ascontiguousarray(t) for t in w.make_tables()[1]]
gpu = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n, 0, 1.0, 0, H.HASH_SEED, 0x2)
tot = w.table_bytes
rows = [(w.cache_bytes * c) // tot for c in w.cards]
sets = [(r + 31) // 32 for r in rows]
off = np.concatenate([[0], np.cumsum(sets)])
orcs = [O.Oracle([c], [d], [tabs[t]], rows[t] * 4 * d, O.MODE_SETASSOC, hash_seed=H.HASH_SEED)
        for t, (c, d) in enumerate(zip(w.cards, w.dims))]
for b in range(30):
    bt = w.batch(b)
    s0 = gpu.stats()
    o0 = [o.stats() for o in orcs]
    H.run_batch_gpu(gpu, bt.ids, torch)
    for o, x in zip(orcs, bt.ids):
        o.query([x])
    dg = H.delta(s0, gpu.stats())
    do = [H.delta(a, o.stats()) for a, o in zip(o0, orcs)]
    print(b, "gpu hits", dg["hits"], "ins", dg["inserted"], "ev", dg["evicted"], "byp", dg["bypassed"], "| orc hits",
          sum(x["hits"] for x in do), "ins", sum(x["inserted"] for x in do), "ev", sum(x["evicted"] for x in do),
          "byp", sum(x["bypassed"] for x in do))
keys, ts, _ = gpu.snapshot()
_, base, fb = gpu.encoding()
span = 1 << fb.astype(np.int64)
bad = 0
per_t = np.zeros(w.n, int)
for way in np.nonzero(keys != 0xFFFFFFFF)[0]:
    k = int(keys[way])
    t = int(np.nonzero((base <= k) & (k < base + span))[0][0])
    s = way // 32
    per_t[t] += 1
    if not (off[t] <= s < off[t + 1]):
        bad += 1
print("keys outside their partition:", bad)
print("live per table:", per_t.tolist())
print("rows per table:", rows)
print("gpu stats", gpu.stats())
