"""Host-link micro-benchmark (SURVEY §7 P0 / hard part H1).

Random-row zero-copy read bandwidth from pinned, mapped host memory with the KQ
miss-fetch access pattern (fleche_probe_host_read), versus
  * row size (128 / 256 / 512 B),
  * span of the host buffer (TLB / IOMMU reach),
  * how the host memory was obtained: malloc + cudaHostRegister (4 KiB pages),
    THP-backed mmap (madvise(MADV_HUGEPAGE)) + cudaHostRegister, cudaHostAlloc (torch pinned),
plus the copy-engine H2D bandwidth for context.  Prints one JSON object.
"""
import json
import mmap
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_xiellwgrs22_b200 import binding as B  # noqa: E402

def thp_array(nbytes):
    m = mmap.mmap(-1, nbytes, flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
    try:
        m.madvise(mmap.MADV_HUGEPAGE)
    except Exception:
        pass
    a = np.frombuffer(m, dtype=np.float32)
    a[:: 1024] = 1.0  # touch every 4 KiB page
    return a, m


def probe(ptr, nbytes, row, rows=1 << 21):
    return B.probe_host_read(ptr, nbytes, row, rows, 11)


def main():
    torch.cuda.init()
    res = {"thp": open("/sys/kernel/mm/transparent_hugepage/enabled").read().strip()}
    spans = [int(x) for x in os.environ.get("SPANS", str(1 << 30) + "," + str(8 << 30)).split(",")]
    for kind in ["malloc", "thp", "cudaHostAlloc"]:
        for span in spans:
            t0 = time.time()
            keep = None
            if kind == "malloc":
                a = np.ones(span // 4, dtype=np.float32)
            elif kind == "thp":
                a, keep = thp_array(span)
            else:
                a = torch.ones(span // 4, dtype=torch.float32).pin_memory().numpy()
            alloc_s = time.time() - t0
            # register via a throwaway ctx (1 table covering the buffer, 64 B rows)
            t1 = time.time()
            try:
                ctx = B.FlatCache([span // 64], [16], [a], 0, 32)
            except Exception as e:
                res[f"{kind}_{span >> 20}MiB_error"] = repr(e)
                print(kind, span, repr(e), file=sys.stderr, flush=True)
                continue
            reg_s = time.time() - t1
            for row in (128, 256, 512):
                g = probe(int(a.ctypes.data), span, row)
                res[f"{kind}_{span >> 20}MiB_{row}B_gbs"] = round(g, 2)
            res[f"{kind}_{span >> 20}MiB_alloc_s"] = round(alloc_s, 2)
            res[f"{kind}_{span >> 20}MiB_register_s"] = round(reg_s, 2)
            ctx.close()
            del a, keep
    # copy-engine bandwidth (sequential DMA) for context
    h = torch.empty(1 << 28, dtype=torch.uint8).pin_memory()
    d = torch.empty(1 << 28, dtype=torch.uint8, device="cuda")
    d.copy_(h)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(5):
        d.copy_(h, non_blocking=True)
    e1.record()
    torch.cuda.synchronize()
    res["h2d_copy_gbs"] = round(5 * (1 << 28) / (e0.elapsed_time(e1) * 1e-3) / 1e9, 2)
    e0.record()
    for _ in range(5):
        h.copy_(d, non_blocking=True)
    e1.record()
    torch.cuda.synchronize()
    res["d2h_copy_gbs"] = round(5 * (1 << 28) / (e0.elapsed_time(e1) * 1e-3) / 1e9, 2)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
