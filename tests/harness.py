"""Shared test plumbing: run the same seeded batches through the CUDA path (via the
C ABI) and the CPU oracle, and compare element by element."""
from __future__ import annotations

import numpy as np

from oracle import oracle as O

HASH_SEED = 0x9E3779B9


def make_pair(w, tabs, mode=O.MODE_SETASSOC, max_lookups=None, admit_p=1.0, admit_seed=0, hash_seed=HASH_SEED,
              cache_bytes=None, flags=0):
    import paper_conf_eurosys_xiellwgrs22_b200 as fl
    cb = w.cache_bytes if cache_bytes is None else cache_bytes
    if max_lookups is None:
        max_lookups = w.batch_size * w.n
    gpu = fl.FlatCache(w.cards, w.dims, tabs, cb, max_lookups, 0, admit_p, admit_seed, hash_seed, flags)
    orc = O.Oracle(w.cards, w.dims, tabs, cb, mode, admit_p, admit_seed, hash_seed)
    return gpu, orc


def run_batch_gpu(gpu, ids_np, torch):
    ids = [torch.from_numpy(x).cuda() for x in ids_np]
    n_out = gpu.out_floats([x.size for x in ids_np])
    out = torch.full((max(n_out, 1),), float("nan"), device="cuda", dtype=torch.float32)
    gpu.query(ids, out)
    torch.cuda.synchronize()
    return out[:n_out].cpu().numpy()


def bits_equal(a: np.ndarray, b: np.ndarray) -> bool:
    return a.shape == b.shape and np.array_equal(a.view(np.uint32), b.view(np.uint32))


def first_mismatch(a, b, dims, lens):
    """(table, position) of the first differing output row, for error messages."""
    off = 0
    for t, (d, L) in enumerate(zip(dims, lens)):
        x = a[off: off + d * L].reshape(L, d).view(np.uint32)
        y = b[off: off + d * L].reshape(L, d).view(np.uint32)
        bad = np.nonzero((x != y).any(axis=1))[0]
        if bad.size:
            return t, int(bad[0])
        off += d * L
    return None


STAT_KEYS_EXACT = ["lookups", "hits", "misses", "invalid", "unique_keys", "unique_hits", "unique_misses",
                   "inserted", "evicted", "bypassed", "occupancy_bytes"]


def delta(a: dict, b: dict) -> dict:
    return {k: b[k] - a[k] for k in b if isinstance(b[k], int) and not isinstance(b[k], bool)}
