"""Watermark (full-scan) eviction on the GPU (fleche_set_watermarks, reading
R23) vs the CPU oracle (needs a B200).

The scan evicts whole age classes, so its result does not depend on thread order: with
no set overflowing within a batch, every counter must equal the set-associative oracle
run with the same watermarks (byte thresholds = floor(fraction x the GPU's capacity)),
and `out` stays bit-exact whatever the policy does.
"""
import numpy as np
import pytest

from oracle import oracle as O
from tests import harness as H
from workload import configs

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

import paper_conf_eurosys_xiellwgrs22_b200 as fl  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _tables(w):
    return [np.ascontiguousarray(t) for t in w.make_tables()[1]]


def _pair(w, tabs, hi, lo, mode=O.MODE_SETASSOC, **kw):
    gpu, orc = H.make_pair(w, tabs, mode, **kw)
    gpu.set_watermarks(hi, lo)
    cap = gpu.stats()["capacity_bytes"]
    orc.set_watermarks(int(hi * cap), int(lo * cap))
    return gpu, orc


@pytest.mark.parametrize("hi,lo", [(0.6, 0.4), (0.9, 0.85), (0.3, 0.05)])
def test_watermark_exact_vs_setassoc_oracle(hi, lo):
    w = configs.get("cfg0").with_(cache_frac=0.25, invalid_ppm=1000)
    tabs = _tables(w)
    gpu, orc = _pair(w, tabs, hi, lo)
    for b in range(40):
        bt = w.batch(b)
        g0, o0 = gpu.stats(), orc.stats()
        got = H.run_batch_gpu(gpu, bt.ids, torch)
        ref = orc.query(bt.ids)
        assert H.bits_equal(got, ref), b
        dg, do = H.delta(g0, gpu.stats()), H.delta(o0, orc.stats())
        assert do["bypassed"] == 0  # no set overflow: the exact regime
        for k in H.STAT_KEYS_EXACT:
            assert dg[k] == do[k], (b, k, dg[k], do[k])
    st = gpu.stats()
    assert st["scans"] == orc.scans() > 0
    assert st["occupancy_bytes"] <= int(hi * st["capacity_bytes"])


def test_watermark_cached_keys_match_oracle_after_churn():
    """After many scans the GPU's cached key set equals the oracle's (same eviction set)."""
    w = configs.get("cfg0").with_(cache_frac=0.25, skews=[0.9] * 7)
    tabs = _tables(w)
    gpu, orc = _pair(w, tabs, 0.5, 0.3)
    for b in range(60):
        bt = w.batch(b)
        H.run_batch_gpu(gpu, bt.ids, torch)
        orc.query(bt.ids)
    keys, _, _ = gpu.snapshot()
    _, base, _ = gpu.encoding()
    got = set(keys[keys != 0xFFFFFFFF].tolist())
    want = {int(base[t]) + i for t, i in orc.cached_keys()}
    assert got == want
    assert gpu.stats()["scans"] == orc.scans() > 5


def test_watermark_mixed_widths_bytes_layout():
    """Bytes layout (mixed widths): scan evictions are by whole age classes too; compare
    with the byte-budgeted set oracle (exact while no set overflows) and check the
    layout invariants."""
    w = configs.get("cfg0").with_(cache_frac=0.2, dims=[8, 16, 32, 64, 128, 8, 256])
    tabs = _tables(w)
    gpu, orc = H.make_pair(w, tabs, O.MODE_GLOBAL)
    S, _, rf = gpu.geometry()
    sob = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_SETBYTES, hash_seed=H.HASH_SEED, ways=32,
                   set_bytes=-rf * 4)
    gpu.set_watermarks(0.5, 0.3)
    cap = gpu.stats()["capacity_bytes"]
    sob.set_watermarks(int(0.5 * cap), int(0.3 * cap))
    for b in range(30):
        bt = w.batch(b)
        got = H.run_batch_gpu(gpu, bt.ids, torch)
        assert H.bits_equal(got, orc.query(bt.ids)), b
        sob.query(bt.ids)
    sg, so = gpu.stats(), sob.stats()
    assert so["bypassed"] == 0
    for k in ("hits", "inserted", "evicted", "occupancy_bytes"):
        assert sg[k] == so[k], (k, sg[k], so[k])
    assert sg["scans"] == sob.scans() > 0


def test_watermark_off_and_invalid_args():
    w = configs.get("cfg0").with_(cache_frac=0.25)
    tabs = _tables(w)
    gpu, orc = H.make_pair(w, tabs, O.MODE_SETASSOC)
    with pytest.raises(fl.binding.FlecheError):
        gpu.set_watermarks(0.3, 0.5)
    with pytest.raises(fl.binding.FlecheError):
        gpu.set_watermarks(0.0, 0.0)
    gpu.set_watermarks(1.0, 0.5)  # hi >= 1: the canonical policy, no extra launches
    k0 = gpu.stats()["kernels_launched"]
    for b in range(10):
        bt = w.batch(b)
        assert H.bits_equal(H.run_batch_gpu(gpu, bt.ids, torch), orc.query(bt.ids))
    sg, so = gpu.stats(), orc.stats()
    assert sg["scans"] == 0
    for k in H.STAT_KEYS_EXACT:
        assert sg[k] == so[k], k
    assert sg["kernels_launched"] - k0 <= 4 * 10
