"""Test double of the key-sharded C-ABI building blocks (route / query_keys / restore),
in numpy, for CPU (gloo) tests of sharded.ShardedCache's collective plumbing.  It
follows the contract in include/fleche.h; it is NOT used by the product path."""
from __future__ import annotations

import numpy as np
import torch

from oracle import oracle as O


def fmix32(h: np.ndarray) -> np.ndarray:
    h = h.astype(np.uint64) & 0xFFFFFFFF
    h ^= h >> 16
    h = (h * 0x85EBCA6B) & 0xFFFFFFFF
    h ^= h >> 13
    h = (h * 0xC2B2AE35) & 0xFFFFFFFF
    h ^= h >> 16
    return h


def owner_of(fk: np.ndarray, seed: int, world: int) -> np.ndarray:
    h = fmix32((fk.astype(np.uint64) ^ seed ^ 0x85EBCA77) & 0xFFFFFFFF)
    return ((h * world) >> 32).astype(np.int64)


class ShardDouble:
    def __init__(self, cards, dims, tables, max_lookups):
        self.cards, self.dims, self.tables = list(cards), list(dims), tables
        self.max_lookups = max_lookups
        _, self.base, _ = O.encode(cards)
        self.base = self.base.astype(np.int64)
        self.order = np.argsort(self.base)

    def route(self, ids, world, seed, send_keys, send_counts, lengths=None):
        ids = [x.numpy() if hasattr(x, "numpy") else x for x in ids]
        fks, self.valid = [], []
        for t, x in enumerate(ids):
            ok = (x >= 0) & (x < self.cards[t])
            self.valid.append(ok)
            fks.append(np.where(ok, self.base[t] + x, -1))
        allk = np.concatenate(fks)
        uniq, first = np.unique(allk[allk >= 0], return_index=True)
        uniq = allk[allk >= 0][np.sort(first)]  # first-occurrence order
        own = owner_of(uniq, seed, world)
        order = np.argsort(own, kind="stable")
        grouped = uniq[order]
        counts = np.bincount(own, minlength=world)
        send_keys[:grouped.size] = torch.from_numpy(grouped.astype(np.int64).astype(np.uint32).view(np.int32))
        send_counts.copy_(torch.from_numpy(counts.astype(np.int64)))
        self.pos_of = {int(k): i for i, k in enumerate(grouped)}
        self.fks = fks

    def query_keys(self, keys, count, rows, flags=None):
        k = keys[:count].numpy().view(np.uint32).astype(np.int64)
        t = self.order[np.searchsorted(self.base[self.order], k, side="right") - 1]
        for i in range(count):
            rows[i] = torch.from_numpy(self.tables[t[i]][k[i] - self.base[t[i]]])
        if flags is not None:
            flags[:count] = 0

    def restore(self, rows_back, flags_back, out):
        off = 0
        for t, fk in enumerate(self.fks):
            d = self.dims[t]
            for j, k in enumerate(fk):
                o = out[off + j * d: off + (j + 1) * d]
                o[:] = rows_back[self.pos_of[int(k)]] if k >= 0 else 0.0
            off += fk.size * d
