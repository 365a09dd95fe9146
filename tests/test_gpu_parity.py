"""CUDA path vs CPU oracle, element by element, through the C ABI (needs a B200).

Bar (BASELINE north_star): lookups bit-exact every batch; stats exact vs the
set-associative oracle mode when no set overflows within a batch; per-lookup hit
ratio within 1 pp of the paper-level global policy.
"""
import numpy as np
import pytest

from oracle import oracle as O
from tests import harness as H
from workload import configs, gen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

import paper_conf_eurosys_xiellwgrs22_b200 as fl  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _tables(w):
    return [np.ascontiguousarray(t) for t in w.make_tables()[1]]


def _run(w, tabs, batches, mode=O.MODE_SETASSOC, exact_stats=True, b0=0, require_sync=False, **kw):
    """Bit-exact `out` every batch, and stats exactly equal to the set-associative oracle's
    every batch -- also when sets overflow: the GPU keeps each set's earliest-occurring
    misses (first-occurrence priority), which is the oracle's insert order (reading R7)."""
    gpu, orc = H.make_pair(w, tabs, mode, **kw)
    overflowed = False
    for b in range(b0, b0 + batches):
        bt = w.batch(b)
        g0, o0 = gpu.stats(), orc.stats()
        got = H.run_batch_gpu(gpu, bt.ids, torch)
        ref = orc.query(bt.ids)
        assert H.bits_equal(got, ref), (b, H.first_mismatch(got, ref, w.dims, [x.size for x in bt.ids]))
        if exact_stats:
            dg, do = H.delta(g0, gpu.stats()), H.delta(o0, orc.stats())
            for k in H.STAT_KEYS_EXACT:
                assert dg[k] == do[k], (b, k, dg[k], do[k])
            overflowed |= do["bypass_full"] > 0
    if require_sync:
        assert not overflowed, "expected a configuration without set overflow"
    return gpu, orc


def test_encoding_matches_oracle():
    for name in ["cfg0", "cfg1"]:
        w = configs.get(name)
        tabs = _tables(w)
        gpu, _ = H.make_pair(w, tabs)
        kb, base, fb = gpu.encoding()
        ob, obase, ofb = O.encode(w.cards)
        assert kb == ob and np.array_equal(base, obase) and np.array_equal(fb, ofb)


@pytest.mark.parametrize("value_mode", [0, 1])
def test_cfg0_bit_exact_and_exact_stats(value_mode):
    # 25 % cache: no set overflows, so the cached sets must stay identical to the
    # set-associative oracle's for every batch
    w = configs.get("cfg0").with_(value_mode=value_mode, invalid_ppm=5000, cache_frac=0.25)
    _run(w, _tables(w), 30, require_sync=True)


def test_cfg0_tiny_cache_churn_no_stale_rows():
    # low skew + 0.2 % cache: thousands of evictions; every cached slab row must equal
    # its host row (no stale rows), no key twice, occupancy == rows x row bytes
    w = configs.get("cfg0").with_(skews=[0.5] * 7, cache_frac=0.002, batch_size=500)
    tabs = _tables(w)
    gpu, orc = _run(w, tabs, 60)
    keys, ts, slab = gpu.snapshot()
    _, base, fb = gpu.encoding()
    live = keys != 0xFFFFFFFF
    assert len(set(keys[live].tolist())) == int(live.sum())
    st = gpu.stats()
    assert st["occupancy_bytes"] == int(live.sum()) * 4 * w.dims[0] <= st["capacity_bytes"]
    for way in np.nonzero(live)[0]:
        k = int(keys[way])
        t = int(np.nonzero((base <= k) & (k < base + (1 << fb.astype(np.int64))))[0][0])
        assert H.bits_equal(slab[way], tabs[t][k - int(base[t])])
    # every batch overflows the sets: the GPU's first-occurrence priority must still leave
    # exactly the oracle's keys cached
    so = orc.stats()
    assert so["bypass_full"] > 0 and st["bypassed"] == so["bypassed"]
    ok = {(t, i) for t, i in orc.cached_keys()}
    gk = set()
    for way in np.nonzero(live)[0]:
        k = int(keys[way])
        t = int(np.nonzero((base <= k) & (k < base + (1 << fb.astype(np.int64))))[0][0])
        gk.add((t, k - int(base[t])))
    assert gk == ok


def test_partial_last_set_and_forced_collisions():
    # 40 rows = one full set + one 8-way set: heavy same-set contention
    w = configs.get("cfg0").with_(cache_frac=0.0)
    tabs = _tables(w)
    _run(w, tabs, 25, cache_bytes=40 * 4 * 32, exact_stats=True)


def test_zero_capacity_and_empty_and_ragged():
    w = configs.get("cfg0")
    tabs = _tables(w)
    gpu, orc = H.make_pair(w, tabs, cache_bytes=0)
    rng = np.random.default_rng(0)
    for b in range(6):
        lens = [0 if (b + t) % 3 == 0 else int(rng.integers(1, 70)) for t in range(w.n)]
        if b == 2:
            lens = [0] * w.n  # an entirely empty batch
        ids = [rng.integers(-1, c + 1, size=L).astype(np.int64) for c, L in zip(w.cards, lens)]
        got = H.run_batch_gpu(gpu, ids, torch)
        ref = orc.query(ids)
        assert H.bits_equal(got, ref)
    sg, so = gpu.stats(), orc.stats()
    assert sg["hits"] == 0 and sg["inserted"] == 0 and sg["invalid_seen"]
    for k in H.STAT_KEYS_EXACT:
        assert sg[k] == so[k], k


@pytest.mark.parametrize("mode", ["decoupled", "fused", "fused_flag"])
def test_decoupled_hit_copy_exact(monkeypatch, mode):
    # the hit copy on a side stream (KG, concurrent with the miss kernel) relies on epoch
    # protection: this batch's hit ways are never victims, so their slab rows stay valid
    monkeypatch.setenv("FLECHE_DECOUPLE_MIN", "0")
    if mode == "fused":
        monkeypatch.setenv("FLECHE_FUSED_GATHER", "1")
    w = configs.get("cfg0").with_(cache_frac=0.01, invalid_ppm=3000, skews=[0.6] * 7, batch_size=400)
    gpu, _ = _run(w, _tables(w), 30, flags=fl.binding.FLAG_FUSED_HIT_COPY if mode == "fused_flag" else 0)
    per_batch = gpu.stats()["kernels_launched"] / 30
    assert per_batch == (3 if mode == "decoupled" else 2)  # KQ + KM (+ KG): at most 2 on the batch's stream


def test_admission_probability_exact():
    w = configs.get("cfg0").with_(cache_frac=0.25)
    _run(w, _tables(w), 20, admit_p=0.3, admit_seed=gen.seeds()["admit"])


def test_host_buffer_entry_point_matches_device_path():
    w = configs.get("cfg0")
    tabs = _tables(w)
    gpu, orc = H.make_pair(w, tabs)
    for b in range(5):
        bt = w.batch(b)
        flat = np.concatenate(bt.ids)
        lens = [x.size for x in bt.ids]
        views, o = [], 0
        for L in lens:
            views.append(flat[o:o + L])
            o += L
        out = np.empty(gpu.out_floats(lens), np.float32)
        gpu.query_host(views, out)
        torch.cuda.synchronize()
        assert H.bits_equal(out, orc.query(bt.ids))


def test_cuda_graph_replay_advances_epoch():
    # the epoch lives on the device, so a captured query replays with fresh semantics
    w = configs.get("cfg0")
    tabs = _tables(w)
    gpu, orc = H.make_pair(w, tabs)
    lens = [w.batch_size] * w.n
    ids_dev = [torch.zeros(L, dtype=torch.int64, device="cuda") for L in lens]
    out = torch.zeros(gpu.out_floats(lens), device="cuda")
    s = torch.cuda.Stream()
    g = torch.cuda.CUDAGraph()
    bt = w.batch(0)
    for d, x in zip(ids_dev, bt.ids):
        d.copy_(torch.from_numpy(x))
    torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=s):
        gpu.query(ids_dev, out, stream=s)
    # capture does not execute: replay batch 0 .. 9
    for b in range(10):
        bt = w.batch(b)
        for d, x in zip(ids_dev, bt.ids):
            d.copy_(torch.from_numpy(x))
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        ref = orc.query(bt.ids)
        assert H.bits_equal(out.cpu().numpy(), ref), b
    so = orc.stats()
    keys, _, _ = gpu.snapshot()
    assert int((keys != 0xFFFFFFFF).sum()) * 4 * w.dims[0] == so["occupancy_bytes"]


def test_cfg1_parity_and_hit_ratio():
    # cfg1 in full: bit-exact every batch vs the global-policy oracle; per-lookup hit
    # ratio within 1 pp of it; exact stats vs the set-associative oracle
    w = configs.get("cfg1")
    tabs = _tables(w)
    gpu, glob = H.make_pair(w, tabs, O.MODE_GLOBAL)
    seta = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_SETASSOC, hash_seed=H.HASH_SEED)
    warm, meas = 60, 60
    for b in range(warm + meas):
        if b == warm:
            g0, o0 = gpu.stats(), glob.stats()
        bt = w.batch(b)
        s0, q0 = gpu.stats(), seta.stats()
        got = H.run_batch_gpu(gpu, bt.ids, torch)
        ref = glob.query(bt.ids)
        seta.query(bt.ids)
        assert H.bits_equal(got, ref), b
        dg, ds = H.delta(s0, gpu.stats()), H.delta(q0, seta.stats())
        if ds["bypassed"] == 0:
            for k in H.STAT_KEYS_EXACT:
                assert dg[k] == ds[k], (b, k)
    dg, do = H.delta(g0, gpu.stats()), H.delta(o0, glob.stats())
    hg = dg["hits"] / (dg["hits"] + dg["misses"])
    ho = do["hits"] / (do["hits"] + do["misses"])
    assert abs(hg - ho) < 0.01, (hg, ho)
    assert dg["host_bytes_fetched"] == dg["unique_misses"] * 128


@pytest.mark.parametrize("miss_path", ["default", "zero_copy"])
def test_cfg2_full_size_parity(miss_path):
    # BASELINE configs[1] at full size in the bench's launch configuration: 8.64 GB host
    # tier, 1,688,128-row cache, 212,992 lookups per batch; out bit-exact each batch,
    # hit ratio within 1 pp of the oracle's global policy over the window.  default: the
    # host-assisted split (on by default for a >= 1 GiB host tier); zero_copy: unified
    # index only (FLAG_NO_HOST_ASSIST)
    w = configs.get("cfg2")
    tabs = _tables(w)
    gpu, glob = H.make_pair(w, tabs, O.MODE_GLOBAL,
                            flags=fl.binding.FLAG_NO_HOST_ASSIST if miss_path == "zero_copy" else 0)
    warm, meas = 150, 30
    for b in range(warm + meas):
        if b == warm:
            g0, o0 = gpu.stats(), glob.stats()
        bt = w.batch(b)
        got = H.run_batch_gpu(gpu, bt.ids, torch)
        ref = glob.query(bt.ids)
        if b % 10 == 0 or b >= warm:
            assert H.bits_equal(got, ref), b
    dg, do = H.delta(g0, gpu.stats()), H.delta(o0, glob.stats())
    hg = dg["hits"] / (dg["hits"] + dg["misses"])
    ho = do["hits"] / (do["hits"] + do["misses"])
    assert abs(hg - ho) < 0.01, (hg, ho)
    st = gpu.stats()
    assert st["occupancy_bytes"] <= st["capacity_bytes"]
    if miss_path == "default":
        assert dg["assisted_rows"] > 0.5 * dg["unique_misses"], dg  # the host threads staged most rows
    else:
        assert st["assisted_rows"] == 0


@pytest.mark.parametrize("ordered", ["0", "1"])
def test_address_ordered_scratch_exact(monkeypatch, ordered):
    # the address-ordered miss scratch (KM hands each warp a contiguous host-address
    # window) must leave results and stats unchanged: force it on / off for a small tier
    if ordered == "1":
        monkeypatch.setenv("FLECHE_ORDER_MIN_SPAN", "0")
    else:
        monkeypatch.setenv("FLECHE_NO_ORDER", "1")
    w = configs.get("cfg0").with_(cache_frac=0.02, invalid_ppm=3000, skews=[0.7] * 7)
    gpu, orc = _run(w, _tables(w), 25)
    keys, _, slab = gpu.snapshot()
    _, base, fb = gpu.encoding()
    tabs = _tables(w)
    live = np.nonzero(keys != 0xFFFFFFFF)[0]
    assert {(int(np.nonzero((base <= k) & (k < base + (1 << fb.astype(np.int64))))[0][0]), 0) for k in keys[live]}
    for way in live:
        k = int(keys[way])
        t = int(np.nonzero((base <= k) & (k < base + (1 << fb.astype(np.int64))))[0][0])
        assert H.bits_equal(slab[way], tabs[t][k - int(base[t])])


def test_prefill_is_a_batch_without_output():
    """fleche_prefill = one batch of the policy whose rows are discarded:
    after it, queries match an oracle that ran the same batch as a query."""
    w = configs.get("cfg0").with_(cache_frac=0.25)
    tabs = _tables(w)
    gpu, orc = H.make_pair(w, tabs)
    for b in (100, 101):  # warm with two batches the queries below never saw
        bt = w.batch(b)
        gpu.prefill([torch.from_numpy(x).cuda() for x in bt.ids])
        orc.query(bt.ids)
    torch.cuda.synchronize()
    sg, so = gpu.stats(), orc.stats()
    for k in H.STAT_KEYS_EXACT:
        assert sg[k] == so[k], k
    for b in range(6):
        bt = w.batch(b)
        assert H.bits_equal(H.run_batch_gpu(gpu, bt.ids, torch), orc.query(bt.ids)), b
    sg, so = gpu.stats(), orc.stats()
    for k in H.STAT_KEYS_EXACT:
        assert sg[k] == so[k], k


@pytest.mark.parametrize("B", [10, 12, 14, 15])
def test_short_keys_encoding_matches_oracle(B):
    """key_bits < B_min (R24): the library's code (fleche_get_encoding) equals the
    oracle's lossy size-aware code."""
    w = configs.get("cfg0")
    tabs = _tables(w)
    gpu = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n, 0, 1.0, 0, H.HASH_SEED, 0, B)
    kb, base, bits = gpu.encoding()
    lossy, obase, obits, oex = O.encode_short(w.cards, B)
    assert kb == B and lossy > 0
    assert base.tolist() == obase.tolist() and bits.tolist() == obits.tolist()


@pytest.mark.parametrize("B", [12, 14])
def test_short_keys_parity(B):
    """Short flat keys: out = E_t[h_t(id)] bit for bit, stats exactly the set-associative
    oracle's with the same code (colliding IDs share one entry)."""
    w = configs.get("cfg0").with_(cache_frac=0.1, invalid_ppm=2000)
    tabs = _tables(w)
    gpu = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, w.batch_size * w.n, 0, 1.0, 0, H.HASH_SEED, 0, B)
    orc = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_SETASSOC, hash_seed=H.HASH_SEED)
    assert orc.set_key_bits(B) > 0
    for b in range(25):
        bt = w.batch(b)
        g0, o0 = gpu.stats(), orc.stats()
        got = H.run_batch_gpu(gpu, bt.ids, torch)
        ref = orc.query(bt.ids)
        assert H.bits_equal(got, ref), b
        dg, do = H.delta(g0, gpu.stats()), H.delta(o0, orc.stats())
        if do["bypassed"] == 0:
            for k in H.STAT_KEYS_EXACT:
                assert dg[k] == do[k], (b, k, dg[k], do[k])
    with pytest.raises(fl.binding.FlecheError):  # the key-sharded mode needs exact codes
        gpu.route([torch.zeros(1, dtype=torch.int64, device="cuda")] * w.n, 2, 1,
                  torch.empty(8, dtype=torch.int32, device="cuda"), torch.empty(2, dtype=torch.int64, device="cuda"))


def test_host_buffer_calls_pipelined_back_to_back():
    """fleche_query_host overlaps call k's output copy with call k+1's lookups (two staging
    buffers): six calls enqueued without a sync, then a device-buffer query, must all equal
    the oracle run in call order."""
    w = configs.get("cfg0").with_(cache_frac=0.05, invalid_ppm=2000)
    tabs = _tables(w)
    gpu, orc = H.make_pair(w, tabs)
    s = torch.cuda.Stream()
    outs, refs = [], []
    for b in range(6):
        bt = w.batch(b)
        lens = [x.size for x in bt.ids]
        ids = [torch.from_numpy(x).pin_memory().numpy() for x in bt.ids]
        out = torch.empty(gpu.out_floats(lens), dtype=torch.float32).pin_memory()
        gpu.query_host(ids, out.numpy(), stream=s)
        outs.append((out, ids))
        refs.append(orc.query(bt.ids))
    bt = w.batch(6)
    dev_ids = [torch.from_numpy(x).cuda() for x in bt.ids]
    dout = torch.empty(gpu.out_floats([x.size for x in bt.ids]), device="cuda")
    gpu.query(dev_ids, dout)  # another stream: ordered after the host calls by the ctx
    s.synchronize()
    torch.cuda.synchronize()
    for (out, _), ref in zip(outs, refs):
        assert H.bits_equal(out.numpy(), ref)
    assert H.bits_equal(dout.cpu().numpy(), orc.query(bt.ids))
    so, sg = orc.stats(), gpu.stats()
    for k in H.STAT_KEYS_EXACT:
        assert sg[k] == so[k], k


def test_query_host_output_copy_orders_after_stream():
    """fleche_query_host's lookups do not wait for `stream` (call k+1's lookups overlap call
    k's output copy), but its output copy does: a read of `out` the caller enqueued on
    `stream` between two calls into the same host buffer sees the first call's rows."""
    w = configs.get("cfg0").with_(cache_frac=0.05)
    tabs = _tables(w)
    gpu, orc = H.make_pair(w, tabs)
    s = torch.cuda.Stream()
    bt0, bt1 = w.batch(0), w.batch(1)
    lens = [x.size for x in bt0.ids]
    ids0 = [torch.from_numpy(x).pin_memory().numpy() for x in bt0.ids]
    ids1 = [torch.from_numpy(x).pin_memory().numpy() for x in bt1.ids]
    out = torch.empty(gpu.out_floats(lens), dtype=torch.float32).pin_memory()
    snap = torch.empty(out.numel(), device="cuda")
    gpu.query_host(ids0, out.numpy(), stream=s)
    with torch.cuda.stream(s):
        snap.copy_(out, non_blocking=True)  # reads out on `stream`, before call 2 overwrites it
    gpu.query_host(ids1, out.numpy(), stream=s)
    s.synchronize()
    assert H.bits_equal(snap.cpu().numpy(), orc.query(bt0.ids))
    assert H.bits_equal(out.numpy(), orc.query(bt1.ids))


@pytest.mark.parametrize("n,d", [(300, 8), (513 - 1, 16), (5, 256), (9, 8)])
def test_table_count_and_width_extremes(n, d):
    """The 512-table kernel instantiation (n > 128), and the narrowest / widest uniform rows
    (d = 8, 256): bit-exact and exact stats vs the set oracle, with ragged and empty tables."""
    rng = np.random.default_rng(n * 1000 + d)
    cards = [int(x) for x in rng.integers(1, 3000, n)]
    w = configs.Workload("edge", 9, cards, [d] * n, [1.0] * n, 40, 0.05, invalid_ppm=5000)
    tabs = _tables(w)
    gpu, orc = H.make_pair(w, tabs)
    for b in range(6):
        bt = w.batch(b)
        ids = [x[: int(rng.integers(0, x.size + 1))] for x in bt.ids]  # ragged, some empty
        g0, o0 = gpu.stats(), orc.stats()
        got = H.run_batch_gpu(gpu, ids, torch)
        assert H.bits_equal(got, orc.query(ids)), b
        dg, do = H.delta(g0, gpu.stats()), H.delta(o0, orc.stats())
        if do["bypassed"] == 0:
            for k in H.STAT_KEYS_EXACT:
                assert dg[k] == do[k], (b, k)
