import os, sys
sys.path.insert(0, '/root/repo')
os.environ.setdefault("FLECHE_HA_FRAC", "0.5")
import torch, numpy as np
import paper_conf_eurosys_xiellwgrs22_b200 as fl
from workload import configs
w = configs.get("cfg5")
_, tabs = w.make_tables()
N = w.batch_size * w.n
c = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, N, 0, 1.0, 0, 0x9E3779B9, fl.binding.FLAG_HOST_ASSIST)
out = torch.empty(N * w.dims[0], device="cuda")
prev = c.stats()
for b in range(12):
    ids = [torch.from_numpy(x).cuda() for x in w.batch(b).ids]
    c.query(ids, out); torch.cuda.synchronize()
    s = c.stats()
    print(b, "umiss", s["unique_misses"] - prev["unique_misses"], "assisted", s["assisted_rows"] - prev["assisted_rows"],
          "timeouts", s["assist_timeouts"] - prev["assist_timeouts"], "ui_ppm", s["ui_share_ppm"])
    prev = s
