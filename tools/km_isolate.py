"""Miss-kernel isolation on cfg2 (dev tool): per-kernel device times of the batch's
kernels next to plain random-row bursts (fleche_probe_host_read) over the SAME host tier
in the same process, so the miss kernel's time can be compared with what the link gives
a burst of the same number of rows.

  python tools/km_isolate.py [cfg] [batches]
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_eurosys_xiellwgrs22_b200 as fl  # noqa: E402
from workload import configs  # noqa: E402
from workload import gen as _gen  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg2"
NB = int(sys.argv[2]) if len(sys.argv) > 2 else 40
w = configs.get(cfg)
# FLECHE_TIER: how the host tier is allocated -- "numpy" (malloc, first touch by the
# generator's threads), "pinned" (cudaHostAlloc via torch), "touch1" (malloc, first touched
# by one thread in address order before the generator runs)
tier = os.environ.get("FLECHE_TIER", "numpy")
if tier == "pinned":
    pin = torch.empty(w.table_bytes // 4, dtype=torch.float32, pin_memory=True)
    hostbuf, tabs = w.make_tables(buf=pin.numpy())
elif tier == "touch1":
    raw = np.empty(w.table_bytes // 4, dtype=np.float32)
    raw.fill(0.0)
    hostbuf, tabs = w.make_tables(buf=raw)
else:
    hostbuf, tabs = w.make_tables()
N = w.batch(0).lookups
cache = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, N, 0, 1.0, _gen.seeds()["admit"], 0x9E3779B9, 0)
dev = torch.device("cuda", 0)
out = torch.empty(cache.out_floats([w.batch_size] * w.n), device=dev)


def dev_batch(b):
    ids = torch.from_numpy(np.concatenate(w.batch(b).ids)).to(dev)
    return list(torch.split(ids, [w.batch_size] * w.n))


P = 300 if cfg == "cfg2" else 60
for b in range(P):
    cache.query(dev_batch(b), out)
torch.cuda.synchronize()
pre = [dev_batch(P + i) for i in range(NB)]
torch.cuda.synchronize()
res = {"cfg": cfg, "km2": os.environ.get("FLECHE_KM2", "default"), "tier": tier}
s0 = cache.stats()
cache.set_profiling(True)
for i in range(NB):
    cache.query(pre[i], out)
torch.cuda.synchronize()
kms, nq = cache.kernel_times_ex()
cache.set_profiling(False)
s1 = cache.stats()
um = (s1["unique_misses"] - s0["unique_misses"]) / NB
res.update({k + "_us": v / nq * 1e3 for k, v in kms.items()})
res["unique_misses_per_batch"] = um
# bursts of the same row count over the same host tier
hp, nb = int(hostbuf.ctypes.data), int(hostbuf.nbytes)
row = 4 * w.dims[0]
for rows in (int(um), 2048, 32768):
    g = fl.binding.probe_host_read(hp, nb, row, rows, 11)
    res[f"burst_{rows}_us"] = rows * row / (g * 1e9) * 1e6
# back to back: batch, burst, batch, burst ... (does a burst right after a batch slow down?)
t = []
for i in range(10):
    cache.query(pre[i], out)
    g = fl.binding.probe_host_read(hp, nb, row, int(um), (i + 1) * 0x9E3779B97F4A7C15 % (1 << 63))
    t.append(int(um) * row / (g * 1e9) * 1e6)
res["burst_after_batch_us"] = sorted(t)[len(t) // 2]
print(json.dumps(res))
