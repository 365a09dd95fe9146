"""Kernel-maintenance sweep (paper Exp #6 / Fig 14, Exp #11 / Fig 19, Issue 2 / Fig 4:
P:L479-497): a fixed number of query keys per batch (10K
or 100K) spread equally over n tables; batch latency of

  flat      one flat cache, one self-identified query launch (Fleche, the default)
  flat_pt   the same flat cache, one query launch per table (fusion off)
  static_pt one static cache per table + one launch per table (HugeCTR-like)

Tables follow the paper's synthetic default: 0.25M features each, d 32,
power law alpha = -1.2 (Zipf a = 1.2); cache 5 % of the table bytes.  Latency = host
clock around fleche_query + stream sync (includes launch and sync: the paper's
"maintenance"), and device time from CUDA events; median over the measured batches.

python tools/maintenance_sweep.py [--keys 10000,100000] [--tables 1,5,10,20,40,60,100] > out.jsonl
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from workload import configs, gen  # noqa: E402

MODES = {"flat": 0, "flat_pt": 0x4, "static_pt": 0x2 | 0x4}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--keys", default="10000,100000")
    ap.add_argument("--tables", default="1,5,10,20,40,60,100")
    ap.add_argument("--warm", type=int, default=150)
    ap.add_argument("--measure", type=int, default=200)
    a = ap.parse_args()
    import torch
    import paper_conf_eurosys_xiellwgrs22_b200 as fl
    torch.cuda.set_device(0)
    stream = torch.cuda.Stream()
    nmax = max(int(x) for x in a.tables.split(","))
    for K in [int(x) for x in a.keys.split(",")]:
        for n in [int(x) for x in a.tables.split(",")]:
            w = configs.Workload("syn", 6, [250_000] * n, [32] * n, [1.2] * n, K // n, 0.05)
            _, tabs = w.make_tables()
            batches = []
            for b in range(a.warm + a.measure):
                bt = w.batch(b)
                batches.append([torch.from_numpy(x).cuda() for x in bt.ids])
            out = torch.empty(w.batch_size * n * 32, device="cuda")
            for mode, flags in MODES.items():
                cache = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * n, 0, 1.0, 0, 0x9E3779B9,
                                     flags)
                with torch.cuda.stream(stream):
                    for b in range(a.warm):
                        cache.query(batches[b], out, stream=stream)
                stream.synchronize()
                s0 = cache.stats()
                lat, dev = [], []
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                for b in range(a.warm, a.warm + a.measure):
                    t0 = time.perf_counter()
                    e0.record(stream)
                    cache.query(batches[b], out, stream=stream)
                    e1.record(stream)
                    stream.synchronize()
                    lat.append((time.perf_counter() - t0) * 1e6)
                    dev.append(e0.elapsed_time(e1) * 1e3)
                s1 = cache.stats()
                d = {k: s1[k] - s0[k] for k in ("hits", "misses", "kernels_launched", "lookups")}
                print(json.dumps({"keys": K, "tables": n, "mode": mode, "p50_latency_us": float(np.median(lat)),
                                  "p50_device_us": float(np.median(dev)),
                                  "maintenance_us": float(np.median(lat)) - float(np.median(dev)),
                                  "hit_ratio": d["hits"] / max(1, d["hits"] + d["misses"]),
                                  "kernels_per_batch": d["kernels_launched"] / a.measure}), flush=True)
                cache.close()
            del tabs, batches


if __name__ == "__main__":
    main()
