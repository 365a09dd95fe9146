"""Mixed row widths (bytes layout) and sum-pooled bags, CUDA path vs CPU oracle (needs a B200).

Bar: pooled and one-hot outputs bit-exact every batch (the GPU accumulates each bag in
bag order, as the oracle does); per-lookup hit ratio within 1 pp of the oracle's
global byte-LRU policy; structural invariants of the byte-budgeted sets.
"""
import numpy as np
import pytest

from oracle import oracle as O
from tests import harness as H
from workload import configs

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _tables(w):
    return [np.ascontiguousarray(t) for t in w.make_tables()[1]]


MIXED = dict(dims=[8, 16, 32, 64, 128, 8, 256])


def _check_bytes_layout(gpu, w, tabs):
    """Every live way's row (via its location) equals its host row; rows of a set do not
    overlap and fit its region; occupancy equals the sum of live row bytes."""
    keys, ts, slab = gpu.snapshot()
    loc = gpu.locations()
    _, base, fb = gpu.encoding()
    span = 1 << fb.astype(np.int64)
    sets = slab.shape[0]
    region_units = slab.shape[1] // 8
    total = 0
    for s in range(sets):
        used = np.zeros(region_units, np.int32)
        for w_ in range(32):
            k = int(keys[s * 32 + w_])
            if k == 0xFFFFFFFF:
                continue
            l = int(loc[s * 32 + w_])
            off, sz = l & 0xFF, l >> 8
            used[off:off + sz] += 1
            t = int(np.nonzero((base <= k) & (k < base + span))[0][0])
            d = w.dims[t]
            assert sz * 8 == d
            row = slab[s, off * 8: off * 8 + d]
            assert H.bits_equal(row, tabs[t][k - int(base[t])]), (s, w_, t)
            total += 4 * d
        assert used.max(initial=0) <= 1, f"overlapping rows in set {s}"
    st = gpu.stats()
    assert st["occupancy_bytes"] == total <= st["capacity_bytes"]


@pytest.mark.parametrize("value_mode", [0, 1])
def test_mixed_widths_one_hot_bit_exact(value_mode):
    w = configs.get("cfg0").with_(value_mode=value_mode, invalid_ppm=3000, cache_frac=0.05, **MIXED)
    tabs = _tables(w)
    gpu, glob = H.make_pair(w, tabs, O.MODE_GLOBAL)
    for b in range(25):
        bt = w.batch(b)
        got = H.run_batch_gpu(gpu, bt.ids, torch)
        ref = glob.query(bt.ids)
        assert H.bits_equal(got, ref), (b, H.first_mismatch(got, ref, w.dims, [x.size for x in bt.ids]))
    _check_bytes_layout(gpu, w, tabs)


def test_mixed_widths_churn_and_compaction():
    # tiny budget (8 sets) + low skew: constant eviction, fragmentation and compaction
    w = configs.get("cfg0").with_(skews=[0.6] * 7, batch_size=200, **MIXED)
    tabs = _tables(w)
    gpu, glob = H.make_pair(w, tabs, O.MODE_GLOBAL, cache_bytes=8 * 4096)
    for b in range(40):
        bt = w.batch(b)
        got = H.run_batch_gpu(gpu, bt.ids, torch)
        assert H.bits_equal(got, glob.query(bt.ids)), b
        if b % 10 == 9:
            _check_bytes_layout(gpu, w, tabs)
    st = gpu.stats()
    assert st["evicted"] > 0 and st["inserted"] - st["evicted"] > 0


def _pooled_batch_gpu(gpu, bt):
    ids = [torch.from_numpy(x).cuda() for x in bt.ids]
    offs = [torch.from_numpy(o).cuda() for o in bt.offsets]
    n_out = gpu.pooled_floats([o.size - 1 for o in bt.offsets])
    out = torch.full((max(n_out, 1),), float("nan"), device="cuda")
    gpu.query_pooled(ids, offs, out)
    torch.cuda.synchronize()
    return out[:n_out].cpu().numpy()


@pytest.mark.parametrize("value_mode", [0, 1])
def test_pooled_bit_exact_cfg4_shape(value_mode):
    # cfg4's structure (100 tables, widths 8..128, skew 0.8..1.2, mean bag 1..8), scaled
    # down 64x so the oracle runs in seconds; arbitrary-bit values too, since the GPU sums
    # each bag sequentially in bag order exactly like the oracle
    w = configs.get("cfg4")
    w = w.with_(cards=[max(3, c // 64) for c in w.cards], batch_size=128, value_mode=value_mode, invalid_ppm=2000)
    tabs = _tables(w)
    gpu, glob = H.make_pair(w, tabs, O.MODE_GLOBAL, max_lookups=sum(w.batch(0).lookups for _ in [0]) * 2)
    for b in range(12):
        bt = w.batch(b)
        got = _pooled_batch_gpu(gpu, bt)
        ref = glob.query_pooled(bt.ids, bt.offsets)
        assert H.bits_equal(got, ref), b


def test_pooled_empty_bags_and_invalid():
    w = configs.get("cfg0").with_(**MIXED)
    tabs = _tables(w)
    gpu, glob = H.make_pair(w, tabs, O.MODE_GLOBAL, max_lookups=4096)
    rng = np.random.default_rng(3)
    for b in range(6):
        ids, offs = [], []
        for t, c in enumerate(w.cards):
            L = rng.integers(0, 4, size=int(rng.integers(0, 40)))  # includes empty bags / tables
            off = np.concatenate([[0], np.cumsum(L)]).astype(np.int64)
            ids.append(rng.integers(-2, c + 2, size=int(off[-1])).astype(np.int64))
            offs.append(off)
        bt = configs.Batch(ids, offs)
        got = _pooled_batch_gpu(gpu, bt)
        assert H.bits_equal(got, glob.query_pooled(ids, offs)), b


def test_cfg4_quarter_hit_ratio_within_1pp():
    # cfg4 at 1/4 of its cardinalities and batch: per-lookup hit ratio of the byte-budgeted
    # set-associative GPU cache vs the oracle's global byte-LRU over a measured window
    w = configs.get("cfg4")
    w = w.with_(cards=[max(3, c // 4) for c in w.cards], batch_size=4096)
    tabs = _tables(w)
    n0 = w.batch(0).lookups
    gpu, glob = H.make_pair(w, tabs, O.MODE_GLOBAL, max_lookups=int(n0 * 1.2))
    warm, meas = 60, 20
    for b in range(warm + meas):
        if b == warm:
            g0, o0 = gpu.stats(), glob.stats()
        bt = w.batch(b)
        got = _pooled_batch_gpu(gpu, bt)
        ref = glob.query_pooled(bt.ids, bt.offsets)
        if b % 10 == 0 or b >= warm + meas - 3:
            assert H.bits_equal(got, ref), b
    dg, do = H.delta(g0, gpu.stats()), H.delta(o0, glob.stats())
    hg = dg["hits"] / (dg["hits"] + dg["misses"])
    ho = do["hits"] / (do["hits"] + do["misses"])
    assert abs(hg - ho) < 0.01, (hg, ho)
