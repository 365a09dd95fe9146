"""BASELINE configs at FULL size in the launch configuration bench.py times (needs a B200):
cfg5 (65,536 samples per table per GPU, 1.7M lookups per batch; also with the
host-assisted split) and cfg4 (100 mixed-width tables, 5.2M pooled lookups per batch).
`out` is compared with the CPU oracle element by element on every checked batch; the
hit ratio over a measured window within 1 pp of the oracle's global policy."""
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


@pytest.fixture(scope="module")
def cfg5_tables():
    w = configs.get("cfg5")
    return [np.ascontiguousarray(t) for t in w.make_tables()[1]]


@pytest.mark.parametrize("ha", ["off", "split", "default"])
def test_cfg5_full_size(monkeypatch, cfg5_tables, ha):
    flags = fl.binding.FLAG_NO_HOST_ASSIST if ha == "off" else 0
    if ha == "split":
        monkeypatch.setenv("FLECHE_HA_FRAC", "0.5")
        flags = fl.binding.FLAG_HOST_ASSIST
    w = configs.get("cfg5")
    gpu, glob = H.make_pair(w, cfg5_tables, O.MODE_GLOBAL, flags=flags)
    warm, meas = 30, 8
    for b in range(warm + meas):
        if b == warm:
            g0, o0 = gpu.stats(), glob.stats()
        bt = w.batch(b)
        got = H.run_batch_gpu(gpu, bt.ids, torch)
        ref = glob.query(bt.ids)
        if b % 6 == 0 or b >= warm:
            assert H.bits_equal(got, ref), b
    dg, do = H.delta(g0, gpu.stats()), H.delta(o0, glob.stats())
    hg = dg["hits"] / (dg["hits"] + dg["misses"])
    ho = do["hits"] / (do["hits"] + do["misses"])
    assert abs(hg - ho) < 0.01, (hg, ho)
    st = gpu.stats()
    assert st["occupancy_bytes"] <= st["capacity_bytes"]
    if ha != "off":
        # the host threads idle (50 us polls) while the oracle runs between batches here, so
        # some staging blocks time out and are fetched zero-copy: allowed (values are checked
        # above), as long as the host threads still stage most of their share
        assert 0 < dg["assisted_rows"] <= dg["unique_misses"], dg
        if ha == "split":  # a fixed share of 0.5 leaves half the blocks to the GPU's zero-copy reads;
            # the tuned default may settle at any share, all-host (ui 0) included (DESIGN R25)
            assert dg["assisted_rows"] < dg["unique_misses"], dg
        blocks = dg["unique_misses"] / 64
        assert dg["assist_timeouts"] < 0.25 * blocks, dg


def test_cfg4_full_size_pooled():
    w = configs.get("cfg4")
    tabs = [np.ascontiguousarray(t) for t in w.make_tables()[1]]
    n0 = w.batch(0).lookups
    gpu, glob = H.make_pair(w, tabs, O.MODE_GLOBAL, max_lookups=int(n0 * 1.25))
    warm, meas = 14, 4
    for b in range(warm + meas):
        if b == warm:
            g0, o0 = gpu.stats(), glob.stats()
        bt = w.batch(b)
        ids = [torch.from_numpy(x).cuda() for x in bt.ids]
        offs = [torch.from_numpy(o).cuda() for o in bt.offsets]
        n_out = gpu.pooled_floats([o.size - 1 for o in bt.offsets])
        out = torch.full((n_out,), float("nan"), device="cuda")
        gpu.query_pooled(ids, offs, out)
        torch.cuda.synchronize()
        ref = glob.query_pooled(bt.ids, bt.offsets)
        if b % 5 == 0 or b >= warm:
            assert H.bits_equal(out.cpu().numpy(), ref), b
    dg, do = H.delta(g0, gpu.stats()), H.delta(o0, glob.stats())
    hg = dg["hits"] / (dg["hits"] + dg["misses"])
    ho = do["hits"] / (do["hits"] + do["misses"])
    assert abs(hg - ho) < 0.01, (hg, ho)
