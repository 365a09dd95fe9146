"""Per-batch early-fetch dynamics (experiment build): KQ lookups vs the last fetch warp's exit
for the last 60 batches of a bench-like run (fresh batches back to back, 4 rotating outputs).
usage: python tools/kf_batches.py [cfg2] [batches]
"""
import ctypes
import os
import sys

os.environ["FLECHE_LIB"] = "libfleche_exp.so"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_eurosys_xiellwgrs22_b200 as fl  # noqa: E402
from workload import configs  # noqa: E402

w = configs.get(sys.argv[1] if len(sys.argv) > 1 else "cfg2")
nb = int(sys.argv[2]) if len(sys.argv) > 2 else 300
_, tabs = w.make_tables()
N = w.batch_size * w.n
c = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, N, 0, 1.0, 0, 0x9E3779B9)
lib = fl.binding._lib
lib.fleche_exp_timeline.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]
outs = [torch.empty(sum(w.batch_size * d for d in w.dims), device="cuda") for _ in range(4)]
pre = [[torch.from_numpy(x).cuda() for x in w.batch(b).ids] for b in range(nb)]
torch.cuda.synchronize()
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
for b in range(nb - 100):  # prefill to steady state
    c.query(pre[b], outs[b % 4])
ev[0].record()
for b in range(nb - 100, nb):
    c.query(pre[b], outs[b % 4])
ev[1].record()
torch.cuda.synchronize()
print(f"last 100 of {nb} batches: {ev[0].elapsed_time(ev[1]) * 1000 / 100:.1f} us per batch")
buf = np.zeros(592 * 16 + 8 + 512, np.uint64)
lib.fleche_exp_timeline(c.h, buf.ctypes.data, buf.size)
ring = buf[592 * 16 + 264: 592 * 16 + 264 + 256].astype(np.int64).reshape(64, 4)
st = c.stats()
print("unique misses/batch %.0f, assisted rows/batch %.0f, timeouts %d" % (
    st["unique_misses"] / st["batches"], st["assisted_rows"] / st["batches"], st["assist_timeouts"]))
print("ui_share_ppm", st["ui_share_ppm"])
rows = []
for e in range(nb - 59, nb + 1):
    r = ring[e % 64]
    if r[0] and r[1]:
        rows.append(((r[1] - r[0]) / 1e3, (r[2] - r[0]) / 1e3 if r[2] else float("nan")))
a = np.array(rows)
print("KQ lookups us: p50 %.1f p90 %.1f max %.1f | last fetch exit us: p50 %.1f p90 %.1f max %.1f" % (
    np.median(a[:, 0]), np.percentile(a[:, 0], 90), a[:, 0].max(), np.nanmedian(a[:, 1]),
    np.nanpercentile(a[:, 1], 90), np.nanmax(a[:, 1])))
print("per batch (lookups, fetch exit):", " ".join("%.0f/%.0f" % tuple(x) for x in rows[-20:]))
