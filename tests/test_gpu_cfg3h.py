"""cfg3 (Criteo-Terabyte shape) on one B200, as cfg3h: the 26 Terabyte cardinalities
(882,774,559 rows, a 31-bit size-aware flat-key code) at d = 32 (a 113 GB host tier; the
GPU box has 196 GB of RAM, so d = 64's 226 GB cannot be built: DESIGN.md §8), batch
32,768 samples per table (851,968 lookups), cache 1 % of the table bytes.

Both miss paths run side by side on the same host tier, in lockstep with the CPU oracle
(global policy): zero-copy only, and the host-assisted split that is the default above
32 GiB of host tier.  Warm-up: 2x the Che fill time (177 batches at 1 %, SURVEY c-6),
through fleche_prefill on the GPU side.  Then every measured batch: `out` bit-exact vs the
oracle (which reads the same host tier: the plain definition), sampled rows also checked
against the generator's closed form E_t[r][c] (SURVEY c-1, d-5), and the per-lookup hit
ratio over the window within 1 pp of the oracle's.
"""
import os

import numpy as np
import pytest

from oracle import oracle as O
from tests import harness as H
from workload import configs, gen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

import paper_conf_eurosys_xiellwgrs22_b200 as fl  # noqa: E402


def _host_ram_bytes() -> int:
    return os.sysconf("SC_PAGE_SIZE") * os.sysconf("SC_PHYS_PAGES")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def test_cfg3h_terabyte_shape_both_miss_paths(monkeypatch):
    w = configs.get("cfg3h")
    if _host_ram_bytes() < w.table_bytes + (40 << 30):
        pytest.skip(f"needs {w.table_bytes / 2**30:.0f} GiB of host tier + headroom")
    kb, _, _, _ = fl.binding.encode(w.cards)
    assert kb == 31  # the Terabyte cardinalities need 31-bit flat keys
    hostbuf, tabs = w.make_tables()
    N = w.batch(0).lookups
    zc = ha = None
    try:
        zc = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, N, 0, 1.0, 0, H.HASH_SEED,
                          fl.binding.FLAG_NO_HOST_ASSIST)  # registers the tier
        monkeypatch.delenv("FLECHE_HA_FRAC", raising=False)  # the default share (0.85 above 32 GiB)
        ha = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, N, 0, 1.0, 0, H.HASH_SEED, fl.binding.FLAG_HOST_ASSIST)
        assert zc.encoding()[0] == 31
        glob = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_GLOBAL)
        warm, meas = 354, 12
        rng = np.random.default_rng(3)
        for b in range(warm + meas):
            if b == warm:
                g0 = [zc.stats(), ha.stats()]
                o0 = glob.stats()
            bt = w.batch(b)
            if b < warm:
                ids = [torch.from_numpy(x).cuda() for x in bt.ids]
                zc.prefill(ids)
                ha.prefill(ids)
                glob.query(bt.ids)
                if b % 32 == 31:
                    torch.cuda.synchronize()
                continue
            ref = glob.query(bt.ids)
            for gpu in (zc, ha):
                got = H.run_batch_gpu(gpu, bt.ids, torch)
                assert H.bits_equal(got, ref), (b, H.first_mismatch(got, ref, w.dims, [x.size for x in bt.ids]))
            # sampled rows against the generator's closed form (no second copy of the tier)
            d = w.dims[0]
            for _ in range(64):
                t = int(rng.integers(w.n))
                j = int(rng.integers(bt.ids[t].size))
                r = int(bt.ids[t][j])
                row = ref[(t * w.batch_size + j) * d:(t * w.batch_size + j + 1) * d]
                exp = np.array([gen.value(t, r, c, w.value_mode) for c in range(d)], np.float32)
                assert H.bits_equal(row, exp), (t, r)
        do = H.delta(o0, glob.stats())
        ho = do["hits"] / (do["hits"] + do["misses"])
        for gpu, s0 in zip((zc, ha), g0):
            dg = H.delta(s0, gpu.stats())
            hg = dg["hits"] / (dg["hits"] + dg["misses"])
            assert abs(hg - ho) < 0.01, (hg, ho)
            st = gpu.stats()
            assert st["occupancy_bytes"] <= st["capacity_bytes"]
        dha = H.delta(g0[1], ha.stats())
        assert dha["assisted_rows"] > 0, dha  # the host threads staged part of the misses
    finally:
        if ha is not None:
            ha.close()  # first: it did not register the tier
        if zc is not None:
            zc.close()
