"""The five BASELINE.json configurations as concrete synthetic workloads.

Shapes only; no method arithmetic.  ``Workload.batch(b)`` regenerates batch ``b``
for either side (oracle or CUDA path) from the counter-based streams in
``workload.gen``.

Cardinalities for the Criteo shapes are the public DLRM per-feature counts; they
are NOT in the paper, whose Table 2 gives only totals ("34M",
"0.9B") that these sums (33,762,577 and 882,774,559) reproduce.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import gen

KAGGLE = [1460, 583, 10131227, 2202608, 305, 24, 12517, 633, 3, 93145, 5683, 8351593, 3194, 27, 14992,
          5461306, 10, 5652, 2173, 4, 7046547, 18, 15, 286181, 105, 142572]
TERABYTE = [227605432, 39060, 17295, 7424, 20265, 3, 7122, 1543, 63, 130229467, 3067956, 405282, 10, 2209,
            11938, 155, 4, 976, 14, 292775614, 40790948, 187188510, 590152, 12973, 108, 36]


@dataclass
class Batch:
    """One batch: per-table int64 IDs (+ CSR bag offsets when pooled)."""
    ids: list  # [n] np.int64
    offsets: list | None = None  # [n] np.int64 (bags+1), pooled only

    @property
    def lookups(self) -> int:
        return int(sum(x.size for x in self.ids))


@dataclass
class Workload:
    name: str
    index: int  # selects the ID seed S_id(index)
    cards: list
    dims: list
    skews: list
    batch_size: int  # samples (one-hot) or bags per table (pooled)
    cache_frac: float
    hotness: list | None = None  # mean bag length m_t (pooled); None = one-hot
    invalid_ppm: int = 0
    value_mode: int = 0  # 0 = exact grid, 1 = arbitrary bits
    meta: dict = field(default_factory=dict)

    @property
    def n(self) -> int:
        return len(self.cards)

    @property
    def pooled(self) -> bool:
        return self.hotness is not None

    @property
    def table_bytes(self) -> int:
        return int(sum(int(c) * int(d) * 4 for c, d in zip(self.cards, self.dims)))

    @property
    def cache_bytes(self) -> int:
        return int(self.cache_frac * self.table_bytes)

    @property
    def out_floats(self) -> int:
        return int(sum(self.batch_size * d for d in self.dims)) if self.pooled else None

    def with_(self, **kw) -> "Workload":
        d = dict(self.__dict__)
        d.update(kw)
        return Workload(**d)

    def make_tables(self, nthreads: int = 0, buf=None):
        return gen.make_tables(self.cards, self.dims, self.value_mode, nthreads, buf)

    def batch(self, b: int, rank: int = 0, nthreads: int = 0) -> Batch:
        """Batch b; rank r takes samples [r*B, (r+1)*B) of the global batch (SURVEY d-2 cfg5)."""
        s_id = gen.id_seed(self.index)
        B = self.batch_size
        ids, offs = [], []
        for t in range(self.n):
            if not self.pooled:
                ids.append(gen.gen_ids(s_id, b, t, self.cards[t], self.skews[t], B, j0=rank * B,
                                       invalid_ppm=self.invalid_ppm, nthreads=nthreads))
            else:
                off = gen.gen_bag_offsets(b, t, self.hotness[t], B, bag0=rank * B)
                x = np.empty(int(off[-1]), dtype=np.int64)
                gen.lib().flg_gen_bag_ids(s_id, gen.seeds()["perm"], b, t, self.cards[t], self.skews[t],
                                          rank * B, B, off.ctypes.data, self.invalid_ppm, x.ctypes.data,
                                          nthreads)
                ids.append(x)
                offs.append(off)
        return Batch(ids, offs if self.pooled else None)


def _cfg4_tables():
    u = gen.u01
    cards = [int(round(10 ** (3 + 4 * u(4 * 1000003 + 2 * t)))) for t in range(100)]
    dims = [[8, 16, 32, 64, 128][t % 5] for t in range(100)]
    skews = [0.8 + 0.4 * u(4 * 1000003 + 2 * t + 1) for t in range(100)]
    hot = [[1, 1, 2, 4, 8][(t // 5) % 5] for t in range(100)]
    return cards, dims, skews, hot


def get(name: str) -> Workload:
    """cfg0 (tiny, seconds), cfg1..cfg5 as in BASELINE.json ``configs``."""
    if name == "cfg0":  # tiny: several tiles + ragged tail, oracle in milliseconds
        return Workload("cfg0", 0, [5000, 3, 1000, 20000, 77, 4096, 10], [32] * 7, [1.05] * 7, 300, 0.05)
    if name == "cfg1":
        return Workload("cfg1", 1, [100_000] * 26, [32] * 26, [1.05] * 26, 1024, 0.10)
    if name == "cfg2":
        return Workload("cfg2", 2, list(KAGGLE), [64] * 26, [1.05] * 26, 8192, 0.05)
    if name == "cfg3":
        return Workload("cfg3", 3, list(TERABYTE), [64] * 26, [1.05] * 26, 32768, 0.01)
    if name == "cfg3h":  # cfg3 at d = 32 (113 GB host tier): the GPU box has 196 GB of RAM
        return Workload("cfg3h", 3, list(TERABYTE), [32] * 26, [1.05] * 26, 32768, 0.01)
    if name == "cfg4":
        c, d, s, h = _cfg4_tables()
        return Workload("cfg4", 4, c, d, s, 16384, 0.05, hotness=h)
    if name == "cfg5":
        return Workload("cfg5", 5, list(KAGGLE), [64] * 26, [1.05] * 26, 65536, 0.05)
    raise KeyError(name)
