"""KM per-warp timeline on cfg2 (experiment build): when do host rows land?"""
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
_, tabs = w.make_tables()
N = w.batch_size * w.n
c = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, N, 0, 1.0, 0, 0x9E3779B9)
f = fl.binding._lib.fleche_exp_timeline
f.restype = ctypes.c_int
f.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t]
out = torch.empty(N * w.dims[0], device="cuda")
for b in range(320):
    ids = [torch.from_numpy(x).cuda() for x in w.batch(b).ids]
    c.query(ids, out)
    if b >= 316:
        torch.cuda.synchronize()
        buf = np.zeros(c.max_lookups * 16 // 256 * 16 + 100000, np.uint64)
        f(c.h, buf.ctypes.data, buf.size)
        t = buf[: (buf.size // 4) * 4].reshape(-1, 4).astype(np.int64)
        act = t[(t[:, 1] > 0) & (t[:, 0] > 0)]
        t0 = t[t[:, 0] > 0][:, 0].min()
        start = (act[:, 0] - t0) / 1e3
        land = (act[:, 1] - t0) / 1e3
        end = (act[:, 2] - t0) / 1e3
        allend = (t[t[:, 0] > 0][:, 2].max() - t0) / 1e3
        lat = land - start
        print(f"batch {b}: {len(act)} busy warps; start p50 {np.median(start):.1f} max {start.max():.1f} us; "
              f"rows landed p10 {np.percentile(land,10):.1f} p50 {np.median(land):.1f} p90 {np.percentile(land,90):.1f} "
              f"max {land.max():.1f}; fetch latency p50 {np.median(lat):.1f} max {lat.max():.1f}; "
              f"busy end max {end.max():.1f}; kernel end {allend:.1f} us")
