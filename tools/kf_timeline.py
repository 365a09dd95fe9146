"""Early-fetch timeline (experiment build, libfleche_exp.so): for one steady-state batch,
when KQ started and its lookups ended (GPU globaltimer), when the host threads saw the start
word and finished (CLOCK_REALTIME, aligned to KQ's start by the first thread's sighting), and
per staging block: CPU published / early-fetch mirrored / copied to HBM / KM done.
usage: python tools/kf_timeline.py [cfg2] [batches]
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
nbatch = int(sys.argv[2]) if len(sys.argv) > 2 else 200
_, tabs = w.make_tables()
N = w.batch_size * w.n
c = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, N, 0, 1.0, 0, 0x9E3779B9)
lib = fl.binding._lib
for f in (lib.fleche_exp_timeline, lib.fleche_exp_ha_times, lib.fleche_exp_ha_blocks):
    f.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]
nth = int(os.environ.get("FLECHE_HA_THREADS", "12"))
outs = [torch.empty(sum(w.batch_size * d for d in w.dims), device="cuda") for _ in range(4)]
pre = [[torch.from_numpy(x).cuda() for x in w.batch(b).ids] for b in range(nbatch)]
for b in range(nbatch):  # like bench.py: fresh batches back to back, rotating output buffers
    c.query(pre[b], outs[b % 4])
torch.cuda.synchronize()
buf = np.zeros(c.max_lookups * 16 // 256 * 16 + 200000, np.uint64)
lib.fleche_exp_timeline(c.h, buf.ctypes.data, buf.size)
hbuf = np.zeros(64 * 128, np.uint64)
lib.fleche_exp_ha_times(c.h, hbuf.ctypes.data, hbuf.size)
nb = 8192
blk = np.zeros(nb * 7, np.uint64)
lib.fleche_exp_ha_blocks(c.h, blk.ctypes.data, nb)
blk = blk.reshape(-1, 7).astype(np.int64)
e = nbatch
nz = np.nonzero(buf)[0]
# KQ's stamps: exp_slots + 1: start, + 2: lookups end; exp_slots + 8 + w: fetch warp w's exit
exp_slots = int(os.environ.get("KM_BLOCKS", "592")) * 16
kq0, kqend = int(buf[exp_slots + 1]), int(buf[exp_slots + 2])
kf_exit = buf[exp_slots + 8: exp_slots + 8 + 256].astype(np.int64)
kf_exit = kf_exit[kf_exit > 0]
if len(kf_exit):
    print("early-fetch warps exit: p0 %.1f p50 %.1f p100 %.1f us after KQ start (lookups end %.1f)" % (
        (kf_exit.min() - kq0) / 1e3, (np.median(kf_exit) - kq0) / 1e3, (kf_exit.max() - kq0) / 1e3, (kqend - kq0) / 1e3))
seen = hbuf[(e % 64) * 128: (e % 64) * 128 + nth].astype(np.int64)
done = hbuf[(e % 64) * 128 + 64: (e % 64) * 128 + 64 + nth].astype(np.int64)
tail = buf[-200000:]
print("host threads: saw start within %.1f us; finished %.1f .. %.1f us after the first sighting" % (
    np.ptp(seen) / 1e3, np.min(done - seen.min()) / 1e3, np.max(done - seen.min()) / 1e3))
st = c.stats()
print("stats:", {k: st[k] for k in ("unique_misses", "ha_rows", "ha_timeouts") if k in st})
use = blk[(blk[:, 5] > 0) | (blk[:, 3] > 0)]
cur = use[use[:, 3] >= use[:, 3].max() - 5_000_000] if len(use) else use  # the last batch's blocks
# GPU anchor: earliest early-fetch mirror of the last batch; CPU anchor: first thread sighting
g0 = cur[cur[:, 4] > 0, 4].min() if (cur[:, 4] > 0).any() else cur[:, 0].min()
c0 = seen.min()
rg = lambda x: (x - g0) / 1e3  # noqa: E731
rc = lambda x: (x - c0) / 1e3  # noqa: E731
print(f"KQ lookups: {(kqend - kq0) / 1e3:.1f} us (start = GPU anchor)")
g0 = kq0
print(f"{len(cur)} blocks of the last batch; GPU times rel. to KQ start, CPU rel. to the first start sighting")
for q in (0, 10, 50, 90, 100):
    f = lambda col, fn=rg: np.percentile(fn(cur[cur[:, col] > 0, col]), q) if (cur[:, col] > 0).any() else float("nan")  # noqa: E731
    print(f"  p{q:3d}: CPU published {f(6, rc):7.1f}  KF mirrored {f(4):7.1f}  KF copied {f(5):7.1f}  "
          f"KM wait {f(0):7.1f}  KM ready {f(1):7.1f}  KM landed {f(2):7.1f}  KM done {f(3):7.1f}")
ok = cur[(cur[:, 1] > 0) & (cur[:, 6] > 0) & (cur[:, 2] > 0) & (cur[:, 3] > 0)]
if len(ok):
    lag_seen = (ok[:, 1] - g0) / 1e3 - (ok[:, 6] - c0) / 1e3
    print("  per block: published->KM saw ready p50 %.1f p90 %.1f | ready->landed p50 %.1f p90 %.1f | landed->done p50 %.1f p90 %.1f us" % (
        np.median(lag_seen), np.percentile(lag_seen, 90), np.median((ok[:, 2] - ok[:, 1]) / 1e3),
        np.percentile((ok[:, 2] - ok[:, 1]) / 1e3, 90), np.median((ok[:, 3] - ok[:, 2]) / 1e3),
        np.percentile((ok[:, 3] - ok[:, 2]) / 1e3, 90)))
m = cur[(cur[:, 4] > 0) & (cur[:, 5] > 0)]
if len(m):
    print(f"  copy after mirror: p50 {np.median((m[:, 5] - m[:, 4]) / 1e3):.1f} us, p90 {np.percentile((m[:, 5] - m[:, 4]) / 1e3, 90):.1f}")
