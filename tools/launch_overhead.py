"""Host-side cost of one fleche_query call (dev tool): calls enqueued back to back without
a sync (launch-bound when the batch is tiny), and call + stream sync, on a tiny workload."""
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

w = configs.get("cfg0").with_(batch_size=64)
_, tabs = w.make_tables()
c = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n, 0, 1.0, 0, 0x9E3779B9)
s = torch.cuda.Stream()
torch.cuda.set_stream(s)
ids = [torch.from_numpy(x).cuda() for x in w.batch(0).ids]
out = torch.empty(c.out_floats([x.numel() for x in ids]), device="cuda")
prep = c.prepare(ids)
sh = int(s.cuda_stream)
ip, lp, _ = prep
res = {"km_coop": os.environ.get("FLECHE_KM_COOP", "1"), "pdl": os.environ.get("FLECHE_NO_PDL", "on")}
for name, fn in [("query_prepared", lambda: c.query_prepared(prep, out, stream=sh)),
                 ("raw_ctypes", lambda: fl.binding.fleche_query(c.h, ip, lp, out.data_ptr(), sh))]:
    for _ in range(50):
        fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(500):
        fn()
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    res[name + "_call_us"] = (t1 - t0) / 500 * 1e6
    lat = []
    for _ in range(200):
        t0 = time.perf_counter()
        fn()
        s.synchronize()
        lat.append((time.perf_counter() - t0) * 1e6)
    lat.sort()
    res[name + "_p50_sync_us"] = lat[100]
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(200):
    c.query_prepared(prep, out, stream=sh)
e1.record()
torch.cuda.synchronize()
res["device_us_per_query_back_to_back"] = e0.elapsed_time(e1) / 200 * 1e3
print(json.dumps(res))
