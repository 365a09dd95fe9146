"""Random-row zero-copy read rate vs burst size at a fixed span (dev helper)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_xiellwgrs22_b200 import binding as B  # noqa: E402

span = int(os.environ.get("SPAN", str(8 << 30)))
a = np.ones(span // 4, dtype=np.float32)
torch.cuda.init()
ctx = B.FlatCache([span // 64], [16], [a], 0, 32)
res = {}
for rows in (1024, 4096, 8192, 16384, 65536, 1 << 20):
    for row in (128, 256):
        g = B.probe_host_read(int(a.ctypes.data), span, row, rows, 5)
        res[f"rows{rows}_{row}B"] = {"gbs": round(g, 2), "us": round(rows * row / g / 1e3, 1)}
print(json.dumps(res))
