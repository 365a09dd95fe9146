"""Host-assisted miss fetch timeline on cfg2 (experiment build, libfleche_exp.so).

Per batch: KQ's doorbell (GPU globaltimer), when each host thread saw it and finished
its blocks (CLOCK_REALTIME; the box's globaltimer tracks it closely enough to read
tens of microseconds), KM warps' start / first rows landed / end.
usage: python tools/ha_timeline.py [cfg2] [threads]
"""
import ctypes
import os
import sys

os.environ["FLECHE_LIB"] = "libfleche_exp.so"
if len(sys.argv) > 2:
    os.environ["FLECHE_HA_THREADS"] = sys.argv[2]
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_eurosys_xiellwgrs22_b200 as fl  # noqa: E402
from workload import configs  # noqa: E402

w = configs.get(sys.argv[1] if len(sys.argv) > 1 else "cfg2")
_, tabs = w.make_tables()
N = w.batch_size * w.n
c = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, N, 0, 1.0, 0, 0x9E3779B9, fl.binding.FLAG_HOST_ASSIST)
tl = fl.binding._lib.fleche_exp_timeline
tl.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]
ht = fl.binding._lib.fleche_exp_ha_times
ht.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]
nth = int(os.environ.get("FLECHE_HA_THREADS", "12"))
out = torch.empty(N * w.dims[0], device="cuda")
pre = [[torch.from_numpy(x).cuda() for x in w.batch(b).ids] for b in range(330)]
for b in range(330):
    c.query(pre[b], out)
    if b >= 320:
        torch.cuda.synchronize()
        buf = np.zeros(c.max_lookups * 16 // 256 * 16 + 100000, np.uint64)
        tl(c.h, buf.ctypes.data, buf.size)
        hbuf = np.zeros(64 * 128, np.uint64)
        ht(c.h, hbuf.ctypes.data, hbuf.size)
        e = b + 1  # epochs are 1-based
        seen = hbuf[(e % 64) * 128: (e % 64) * 128 + nth].astype(np.int64)
        done = hbuf[(e % 64) * 128 + 64: (e % 64) * 128 + 64 + nth].astype(np.int64)
        slots = int(np.nonzero(buf)[0].max()) if buf.any() else 0
        t = buf[: (buf.size // 4) * 4].reshape(-1, 4).astype(np.int64)
        bell = int(buf[slots]) if slots else 0
        t0 = seen.min()
        print(f"batch {b}: host threads saw the doorbell within {np.ptp(seen) / 1e3:.1f} us, finished "
              f"{np.min(done - t0) / 1e3:.1f}..{np.max(done - t0) / 1e3:.1f} us after it "
              f"(gather {np.median(done - seen) / 1e3:.1f} us/thread)")

# per-block view of the last batch: CPU publish vs GPU flag seen / rows landed / done,
# all relative to the doorbell (CPU clock aligned by the first thread's doorbell sighting)
hb = fl.binding._lib.fleche_exp_ha_blocks
hb.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]
nb = (int(c.stats()["unique_misses"]) and 4096)
blk = np.zeros(nb * 5, np.uint64)
hb(c.h, blk.ctypes.data, nb)
blk = blk.reshape(-1, 5).astype(np.int64)
e = 330
seen = hbuf[(e % 64) * 128: (e % 64) * 128 + nth].astype(np.int64)
off = seen.min() - bell  # CPU clock - GPU clock (+ the doorbell's link latency)
use = blk[(blk[:, 3] >= bell) & (blk[:, 3] > 0)]
rel = lambda x: (x - bell) / 1e3  # noqa: E731
print(f"{len(use)} blocks of the last batch (us after the doorbell):")
for q in (0, 10, 50, 90, 100):
    print(f"  p{q:3d}: GPU wait start {np.percentile(rel(use[:, 0]), q):7.1f}  CPU published "
          f"{np.percentile(rel(use[:, 4] - off), q):7.1f}  GPU saw flag {np.percentile(rel(use[:, 1]), q):7.1f}  "
          f"rows landed {np.percentile(rel(use[:, 2]), q):7.1f}  block done {np.percentile(rel(use[:, 3]), q):7.1f}")
lag = (use[:, 1] - (use[:, 4] - off)) / 1e3
print(f"  flag lag (GPU saw - CPU published): p50 {np.median(lag):.1f} p90 {np.percentile(lag, 90):.1f} us; "
      f"load {np.median((use[:, 2] - use[:, 1]) / 1e3):.1f} us, place {np.median((use[:, 3] - use[:, 2]) / 1e3):.1f} us")
