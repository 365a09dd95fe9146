#!/usr/bin/env python
"""bench.py — keys/s of the flat-cache lookup path on BASELINE configs[1] (cfg2).

One step = one batch of the whole hot path: KQ (fused
self-identified probe + hit gather + miss dedup + zero-copy host fetch) and KI
(dup fill + admission + per-set LRU insert), through the C ABI (libfleche.so).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config cfg2] [--impl fleche|reference]

N > 1 runs under torchrun: every rank serves its own shard of each global batch
with its own replicated cache (no data-path collective; "scaling": "weak").
`--impl reference` times the CPU oracle (oracle/) on the same workload, rank 0 only.
"""
from __future__ import annotations

import argparse
import faulthandler
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from workload import configs  # noqa: E402

PREFILL = {"cfg0": 20, "cfg1": 150, "cfg2": 300, "cfg4": 30, "cfg5": 60}  # >= 2x the Che fill time
# cfg3 (TB shape, batch 32768): Che fill time 177 / 437 / 1,492 / 3,898 batches at 1 / 2 / 5 / 10 %
PREFILL_CFG3 = {0.01: 360, 0.02: 880, 0.05: 3000, 0.10: 7800}
HASH_SEED = 0x9E3779B9


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=1000)
    p.add_argument("--warmup", type=int, default=20)
    p.add_argument("--config", default="cfg2")
    p.add_argument("--impl", default="fleche", choices=["fleche", "reference"])
    p.add_argument("--prefill", type=int, default=None, help="untimed batches to reach steady state")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--cpu-seconds", type=float, default=15.0, help="oracle sample budget")
    p.add_argument("--flags", type=int, default=0, help="fleche_config.flags (ablations)")
    p.add_argument("--host-assist", action="store_true",
                   help="FLECHE_FLAG_HOST_ASSIST: host threads stage the missed rows (paper Fig 8b CPU-DRAM layer)")
    p.add_argument("--cache-frac", type=float, default=None, help="override the config's cache fraction (sweeps)")
    p.add_argument("--dim", type=int, default=None, help="override every table's row width (sensitivity sweeps)")
    p.add_argument("--batch", type=int, default=None, help="override the samples per table per batch (sweeps)")
    p.add_argument("--p2p", action="store_true",
                   help="--mode sharded: fused exchange (owners' rows read in place over peer memory)")
    p.add_argument("--watermarks", default=None,
                   help="hi,lo: full-scan eviction between these fractions of capacity (P:L660-662, reading R23)")
    p.add_argument("--ha-frac", type=float, default=None,
                   help="--host-assist: share of the miss blocks the host threads stage (rest: zero-copy)")
    p.add_argument("--admit-prob", type=float, default=1.0, help="admission probability p (P:L655-659); 1 = canonical")
    p.add_argument("--mode", default="replicated", choices=["replicated", "sharded"],
                   help="multi-GPU partitioning: per-GPU replicated caches, or one key-sharded cache (NCCL all-to-all)")
    return p.parse_args()


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {"hbm_gbs": 6650.0, "_fallback": True}


class ClockSampler:
    """Samples SM clock and throttle reasons via NVML during the timed region."""

    def __init__(self, device_index: int):
        self.samples, self.ok = [], False
        try:
            import pynvml
            import torch
            pynvml.nvmlInit()
            uuid = "GPU-" + str(torch.cuda.get_device_properties(device_index).uuid)
            self.h = pynvml.nvmlDeviceGetHandleByUUID(uuid.encode())
            self.nv = pynvml
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = repr(e)
        self._stop = threading.Event()
        self.window = None

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                mhz = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                self.samples.append((time.perf_counter(), mhz, r))
            except Exception:
                pass
            time.sleep(0.01)

    def start(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()

    def mark(self, t0, t1):
        self.window = (t0, t1)

    def stop(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"]}
        self._stop.set()
        self.t.join()
        nv = self.nv
        t0, t1 = self.window or (0, 1e30)
        pad = max(0.05, 0.0)
        sel = [s for s in self.samples if t0 - pad <= s[0] <= t1 + pad] or self.samples
        names = {
            "gpu_idle": getattr(nv, "nvmlClocksEventReasonGpuIdle", 0x1),
            "sw_power_cap": getattr(nv, "nvmlClocksEventReasonSwPowerCap", 0x4),
            "hw_slowdown": getattr(nv, "nvmlClocksEventReasonHwSlowdown", 0x8),
            "sw_thermal_slowdown": getattr(nv, "nvmlClocksEventReasonSwThermalSlowdown", 0x20),
            "hw_thermal_slowdown": getattr(nv, "nvmlClocksEventReasonHwThermalSlowdown", 0x40),
            "hw_power_brake_slowdown": getattr(nv, "nvmlClocksEventReasonHwPowerBrakeSlowdown", 0x80),
        }
        seen = set()
        for _, _, r in sel:
            for k, bit in names.items():
                if r & bit and k != "gpu_idle":
                    seen.add(k)
        return {"sm_mhz": statistics.median([s[1] for s in sel]), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(seen), "samples": len(sel)}


def algorithmic_bytes(st: dict, n_queries: int, row: float, row_miss: float, pooled_out: float = 0) -> dict:
    """Per-launch algorithmic bytes of KQ and KM.

    row: lookup-weighted mean row bytes; row_miss: mean row bytes of unique misses
    (= host bytes / unique misses, from the run's own counters); pooled_out: bytes of
    pooled output rows per batch (0 for one-hot)."""
    q = max(n_queries, 1)
    N = st["lookups"] / q
    U = st["unique_keys"] / q
    Uh = st["unique_hits"] / q
    Um = st["unique_misses"] / q
    Ui = st["inserted"] / q
    Nd = (st["misses"] - st["unique_misses"]) / q  # duplicate misses (restored in KM)
    Nm = st["misses"] / q  # missed lookups (owners + duplicates)
    # KQ: IDs in, one 128 B set line per unique key, hit rows read + ts sector touched,
    #     out rows written for every non-missed lookup, 8 B dedup tag + 24 B record per unique miss
    kq_hbm = N * 8 + U * 128 + Uh * (row + 32) + (N - Nm) * row + Um * (8 + 24) + Nd * 24
    # KM: miss record in, host row in (host link), owner + duplicate out rows written,
    #     per insert: the set's key+ts lines (256 B) read, the row and key/ts written
    km_host = Um * row_miss
    km_hbm = Um * 24 + Um * row_miss + Ui * (256 + row_miss + 8)
    # KD: duplicate record + owner row read, duplicate row written
    kd_hbm = Nd * (16 + 8 + 2 * row)
    # KP (pooled only): staged rows read once, pooled rows written
    kp_hbm = (N * row + pooled_out) if pooled_out else 0
    return {"N": N, "U": U, "U_hit": Uh, "U_miss": Um, "U_ins": Ui, "kq_hbm": kq_hbm, "km_host": km_host,
            "km_hbm": km_hbm, "kd_hbm": kd_hbm, "kp_hbm": kp_hbm}


def run_reference(args, w, P, W, K):
    """CPU oracle on the same workload (the reference arm for this tier), rank 0 only."""
    from oracle import oracle as O
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    t_gen = time.time()
    _, tabs = w.make_tables()
    t_gen = time.time() - t_gen
    orc = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_GLOBAL)
    for b in range(P + W):
        orc.query(w.batch(b).ids)
    batches = [w.batch(P + W + k).ids for k in range(K)]
    s0 = orc.stats()
    t0 = time.perf_counter()
    for ids in batches:
        orc.query(ids)
    dt = time.perf_counter() - t0
    s1 = orc.stats()
    lk = s1["lookups"] - s0["lookups"]
    v = lk / dt / 1e6
    hits = s1["hits"] - s0["hits"]
    print(json.dumps({
        "impl": "reference", "metric": "embedding lookups/s", "value": v, "unit": "Mkeys/s", "n_gpus": args.gpus,
        "steps": K, "warmup": W, "ms_per_step": dt / K * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": w.name, "tables": w.n, "dim": w.dims[0], "batch": w.batch_size,
                   "lookups_per_step": w.batch_size * w.n, "cache_frac": w.cache_frac, "prefill_batches": P},
        "hit_ratio": hits / max(1, hits + s1["misses"] - s0["misses"]),
        "cpu_baseline": {"value": v, "unit": "Mkeys/s", "cores": 1, "kind": "oracle",
                         "sample": f"{K} full batches of {w.name} after {P + W} untimed batches; single-threaded "
                                   f"C++ oracle (global byte-LRU policy); host tables generated in {t_gen:.0f}s"},
        "e2e": {"value": v, "unit": "Mkeys/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def cpu_baseline(w, tabs, budget_s):
    """Oracle timed on a bounded sample of the same workload (cold start, batches 0..B-1)."""
    from oracle import oracle as O
    orc = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_GLOBAL)
    t0 = time.perf_counter()
    nb, lk = 0, 0
    gen_t = 0.0
    while time.perf_counter() - t0 - gen_t < budget_s:
        tg = time.perf_counter()
        ids = w.batch(nb).ids
        gen_t += time.perf_counter() - tg
        orc.query(ids)
        nb += 1
        lk += sum(x.size for x in ids)
    dt = time.perf_counter() - t0 - gen_t
    return {"value": lk / dt / 1e6, "unit": "Mkeys/s", "cores": 1, "kind": "oracle",
            "sample": f"batches 0..{nb - 1} of {w.name} from a cold cache ({lk} lookups, {dt:.1f}s CPU), "
                      f"single-threaded C++ oracle, 1 of {os.cpu_count()} host cores"}


def log(*a):
    print(f"[bench {time.strftime('%H:%M:%S')}]", *a, file=sys.stderr, flush=True)


def main():
    # NCCL's version banner goes to stdout, which must carry exactly one JSON line
    os.environ["NCCL_DEBUG"] = os.environ.get("BENCH_NCCL_DEBUG", "WARN")
    faulthandler.enable()
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    w = configs.get(args.config)
    if args.cache_frac is not None:
        w = w.with_(cache_frac=args.cache_frac)
    if args.dim is not None:
        w = w.with_(dims=[args.dim] * w.n)
    if args.batch is not None:
        w = w.with_(batch_size=args.batch)
    P = PREFILL.get(args.config, 300) if args.prefill is None else args.prefill
    if args.prefill is None and args.config.startswith("cfg3"):
        P = PREFILL_CFG3.get(round(w.cache_frac, 2), 360)
    W, K = max(args.warmup, 0), max(args.steps, 1)
    if args.host_assist:
        args.flags |= 0x8
        if args.ha_frac is not None:
            os.environ["FLECHE_HA_FRAC"] = str(args.ha_frac)
    if args.impl == "reference":
        return run_reference(args, w, P, W, K)

    import torch
    import paper_conf_eurosys_xiellwgrs22_b200 as fl
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    b0 = w.batch(0, rank=rank)
    N = int(b0.lookups * (1.25 if w.pooled else 1))  # max_lookups (bag lengths vary per batch)
    d = w.dims[0]
    uniform = len(set(w.dims)) == 1

    # host tier: every table in one buffer, page-locked + mapped by fleche_create
    log("host tier")
    t_gen = time.time()
    shm_cleanup = None
    if dist:  # one copy per node in /dev/shm, mapped by every local rank
        from workload import shm
        hostbuf, tabs, shm_cleanup = shm.shared_tables(
            f"fleche_{w.name}_{os.environ.get('MASTER_PORT', '0')}", w.cards, w.dims, w.value_mode, local,
            dist.barrier)
    else:
        hostbuf, tabs = w.make_tables()
    t_gen = time.time() - t_gen
    log("create")
    sharded = args.mode == "sharded"
    if sharded and (w.pooled or not uniform):
        raise SystemExit("--mode sharded supports one-hot, uniform-width configs (cfg1, cfg2, cfg5)")
    from workload import gen as _gen
    cache = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, N * (world if sharded else 1), local,
                         args.admit_prob, _gen.seeds()["admit"], HASH_SEED, args.flags)
    wm = None
    if args.watermarks:
        wm = [float(x) for x in args.watermarks.split(",")]
        cache.set_watermarks(wm[0], wm[1])
    shard = None
    if sharded:
        if dist is None:
            import torch.distributed as dist
            dist.init_process_group("nccl", init_method="tcp://127.0.0.1:%d" % (29600 + os.getpid() % 300),
                                    rank=0, world_size=1, device_id=torch.device("cuda", local))
        from paper_conf_eurosys_xiellwgrs22_b200.sharded import ShardedCache
        shard = ShardedCache(cache, row_floats=d, p2p=args.p2p)
    stream = torch.cuda.current_stream()

    def gen_batch(b):
        return w.batch(b, rank=rank)

    class DevBatch:
        """One batch resident in HBM: flat IDs (+ flat CSR offsets when pooled)."""

        def __init__(self, bt):
            self.lens = [int(x.size) for x in bt.ids]
            self.ids = torch.from_numpy(np.concatenate(bt.ids)).to(dev)
            self.idv, o = [], 0
            for L in self.lens:
                self.idv.append(self.ids[o:o + L])
                o += L
            self.bags = None
            if bt.offsets is not None:
                self.bags = [int(x.size) - 1 for x in bt.offsets]
                self.offs = torch.from_numpy(np.concatenate(bt.offsets)).to(dev)
                self.offv, o = [], 0
                for x in bt.offsets:
                    self.offv.append(self.offs[o:o + x.size])
                    o += x.size

        def out_floats(self):
            return cache.pooled_floats(self.bags) if self.bags is not None else cache.out_floats(self.lens)

        def run(self, out):
            if self.bags is not None:
                cache.query_pooled(self.idv, self.offv, out, bags=self.bags, nnz=self.lens)
            elif shard is not None:
                shard.query(self.idv, out, lengths=self.lens)
            else:
                cache.query(self.idv, out, lengths=self.lens)

    out_max = int(DevBatch(b0).out_floats() * 1.25)
    outs = [torch.empty(out_max, dtype=torch.float32, device=dev) for _ in range(4)]  # 4 x out > L2 when large

    # steady state: untimed prefill batches
    log("prefill")
    for b in range(P):
        DevBatch(gen_batch(b)).run(outs[b % 4])
        if b % 16 == 15:
            torch.cuda.synchronize()
    torch.cuda.synchronize()

    # pre-generated device-resident batches for warm-up, timed and profiled passes (at most
    # ~8 GB of them; beyond that the timed steps cycle through the pre-generated batches)
    log("pregen")
    KP = min(K, 300)
    per_step = b0.lookups * 8 * (1.1 if w.pooled else 1.0)
    R = int(min(W + K + KP, max(8, 8e9 // per_step)))
    pre = [DevBatch(gen_batch(P + i)) for i in range(R)]
    torch.cuda.synchronize()

    def step(i, out):
        pre[i % R].run(out)

    log("timed")
    clock = ClockSampler(local)
    clock.start()
    for i in range(W):
        step(i, outs[i % 4])
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    s0 = cache.stats()
    r0 = cache.shard_stats() if sharded else None
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    tw0 = time.perf_counter()
    e0.record(stream)
    for k in range(K):
        step(W + k, outs[k % 4])
    e1.record(stream)
    torch.cuda.synchronize()
    tw1 = time.perf_counter()
    clock.mark(tw0, tw1)
    if dist:
        dist.barrier()
    ms = e0.elapsed_time(e1)
    s1 = cache.stats()
    clk = clock.stop()
    ms_max = ms
    if dist:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_max = float(t.item())
    dst = {k: s1[k] - s0[k] for k in fl.STAT_FIELDS}
    keys_total = dst["lookups"] * world
    hit = dst["hits"] / max(1, dst["hits"] + dst["misses"])
    uhit = dst["unique_hits"] / max(1, dst["unique_keys"])
    if sharded:  # requester side: this rank's batch lookups and how many hit at their owner
        r1 = cache.shard_stats()
        dr = {k: r1[k] - r0[k] for k in r1}
        keys_total = dr["lookups"] * world
        hit = dr["hits"] / max(1, dr["lookups"] - dr["invalid"])
        uhit = dst["unique_hits"] / max(1, dst["unique_keys"])  # at this rank as an owner
        dst["unique_misses_owner"] = dst["unique_misses"]
    value = keys_total / (ms_max * 1e-3) / 1e6

    # per-kernel device time (profiled pass: CUDA events on the launching stream)
    log("profiled pass")
    cache.set_profiling(True)
    sp0 = cache.stats()
    for k in range(KP):
        step(W + K + k, outs[k % 4])
    torch.cuda.synchronize()
    kms, nq = cache.kernel_times_ex()
    sp1 = cache.stats()
    cache.set_profiling(False)
    dsp = {k: sp1[k] - sp0[k] for k in fl.STAT_FIELDS}
    kavg = {k: v / max(nq, 1) for k, v in kms.items()}
    kq_avg, ki_avg = kavg["kq"], kavg["km"] + kavg["kd"] + kavg["kp"]
    # lookup-weighted and miss-weighted mean row bytes (uniform configs: both 4d)
    row_lk = sum(L * 4 * dd for L, dd in zip(pre[0].lens, w.dims)) / max(1, sum(pre[0].lens))
    row_ms = dsp["host_bytes_fetched"] / max(1, dsp["unique_misses"])
    ab = algorithmic_bytes(dsp, nq, row_lk, row_ms, pooled_out=(
        sum(b * 4 * dd for b, dd in zip(pre[0].bags, w.dims)) if w.pooled else 0))

    # host-link peaks, both measured in-run with KM's access pattern (16 B vector loads,
    # one row per lane) over rows of 4d bytes: (a) uniformly random rows over the WHOLE host
    # tier = the ceiling for this workload's misses (large spans are limited by address
    # translation, ~80-90 M rows/s on this platform: profiles/hostlink_r01.json);
    # (b) random rows inside a 1 GiB window = the link's bandwidth
    log("host probe")
    hp = int(hostbuf.ctypes.data)
    prow = min((128, 256, 512, 1024), key=lambda r: abs(r - row_ms))
    host_rand = fl.binding.probe_host_read(hp, int(hostbuf.nbytes), prow, 1 << 21, 7)
    host_link = fl.binding.probe_host_read(hp, min(1 << 30, int(hostbuf.nbytes)), prow, 1 << 21, 9)
    # (c) host-assisted mode: KM reads a contiguous pinned staging buffer (cudaHostAlloc),
    # so its ceiling is the link rate over a small pinned window
    ha = bool(args.flags & 0x8)
    host_stage = None
    if ha:
        pin = torch.empty(64 << 20, dtype=torch.uint8).pin_memory()
        host_stage = fl.binding.probe_host_read(int(pin.data_ptr()), int(pin.numel()), prow, 1 << 21, 11)
        del pin
    if prow != round(row_ms):  # mixed widths: the large-span ceiling is a row rate; scale to the mean miss row
        host_rand *= row_ms / prow
        host_link *= row_ms / prow
        if host_stage:
            host_stage *= row_ms / prow
    hbm_peak = float(peaks().get("hbm_gbs", 6650.0))
    kern = {
        "kq_kernel": {"ms": kq_avg, "bound": "hbm", "bytes": ab["kq_hbm"], "peak": hbm_peak,
                      "peak_source": "MEASURED_PEAKS.json hbm_gbs (of measured)"},
        "km_kernel": {"ms": kavg["km"], "bound": "host_link", "bytes": ab["km_host"],
                      "peak": host_stage if ha else host_rand,
                      "peak_source": (f"measured in-run: {prow} B-row zero-copy reads inside a 64 MiB pinned buffer "
                                      "(the host-assisted staging pattern)") if ha else
                                     f"measured in-run: random {prow} B-row zero-copy read over the whole host tier",
                      "hbm_bytes": ab["km_hbm"]},
        "kd_kernel": {"ms": kavg["kd"], "bound": "hbm", "bytes": ab["kd_hbm"], "peak": hbm_peak,
                      "peak_source": "MEASURED_PEAKS.json hbm_gbs (of measured)"},
    }
    if w.pooled:
        kern["kp_kernel"] = {"ms": kavg["kp"], "bound": "hbm", "bytes": ab["kp_hbm"], "peak": hbm_peak,
                             "peak_source": "MEASURED_PEAKS.json hbm_gbs (of measured)"}
    for kd in kern.values():
        kd["achieved"] = kd["bytes"] / (kd["ms"] * 1e-3) / 1e9
        kd["frac"] = kd["achieved"] / kd["peak"]
    km = kern["km_kernel"]
    if not ha and km["achieved"] > km["peak"]:
        # the misses have page locality (e.g. cfg4: most misses fall in a few hot tables), so
        # the uniform-random ceiling understates what the link gives them: take the next
        # measured ceiling, the link's rate inside a 1 GiB window
        km["peak"] = host_link
        km["peak_source"] = ("measured in-run: random-row zero-copy read inside a 1 GiB window (the misses beat "
                             "the whole-tier random-row rate %.1f GB/s: they have page locality)" % host_rand)
        km["frac"] = km["achieved"] / km["peak"]
    dom = max(kern, key=lambda k: kern[k]["ms"])
    kd = kern[dom]
    traffic, traffic_src = None, None
    try:  # committed ncu --set full summary of this config's kernels (profiles/ncu_traffic_r01.json)
        tr = json.load(open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles",
                                         "ncu_traffic_r01.json")))[args.config][dom]
        if not (args.flags or args.watermarks or args.dim or args.batch or args.cache_frac or args.mode != "replicated"
                or args.admit_prob != 1.0):  # only the exact captured configuration
            traffic, traffic_src = tr["dram_bytes"], tr["source"]
    except (OSError, KeyError, ValueError):
        pass
    roof = {"bound": kd["bound"], "achieved": kd["achieved"], "peak": kd["peak"], "unit": "GB/s", "frac": kd["frac"],
            "traffic": traffic, "traffic_source": traffic_src, "kernel": dom, "kernel_ms": kd["ms"], "share_of_step": kd["ms"] / (kq_avg + ki_avg),
            "peak_source": kd["peak_source"], "host_link_1GiB_gbs": host_link,
            "frac_of_link_bw": kern["km_kernel"]["achieved"] / host_link, "kernels": kern,
            "algorithmic_bytes_per_step": {"hbm": ab["kq_hbm"] + ab["km_hbm"] + ab["kd_hbm"] + ab["kp_hbm"], "host": ab["km_host"]}}
    t_roof_step = max((ab["kq_hbm"] + ab["km_hbm"] + ab["kd_hbm"] + ab["kp_hbm"]) / (hbm_peak * 1e9),
                      ab["km_host"] / (kern["km_kernel"]["peak"] * 1e9))
    roof["step_roofline_us"] = t_roof_step * 1e6
    roof["step_frac"] = t_roof_step / (ms / K * 1e-3)

    # latency mode: host clock around query + stream sync (includes launch overhead)
    log("latency")
    lat = []
    nlat = min(200, K)
    fresh = [DevBatch(gen_batch(P + W + K + KP + 1000 + i)) for i in range(nlat)]  # never seen by the cache
    torch.cuda.synchronize()
    for k in range(nlat):
        t0 = time.perf_counter()
        fresh[k].run(outs[k % 4])
        stream.synchronize()
        lat.append((time.perf_counter() - t0) * 1e6)
    lat.sort()
    del fresh

    # end to end through the host-buffer entry point: H2D ids + query + D2H out per step
    log("e2e")
    e2e = None
    if not args.no_e2e and not w.pooled and not sharded:
        KE = min(K, 100)
        lens = [w.batch_size] * w.n
        hids = [torch.from_numpy(np.concatenate(gen_batch(P + W + K + KP + i).ids)).pin_memory() for i in range(KE)]
        hout = torch.empty(cache.out_floats(lens), dtype=torch.float32).pin_memory()
        hv = [[h.numpy()[i * w.batch_size:(i + 1) * w.batch_size] for i in range(w.n)] for h in hids]
        torch.cuda.synchronize()
        if dist:
            dist.barrier()
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        for i in range(KE):
            cache.query_host(hv[i], hout, lengths=lens)
        f1.record(stream)
        torch.cuda.synchronize()
        ems = f0.elapsed_time(f1)
        if dist:
            t = torch.tensor([ems], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        NL = sum(lens)
        e2e = {"value": KE * NL * world / (ems * 1e-3) / 1e6, "unit": "Mkeys/s", "h2d_bytes_per_step": NL * 8,
               "d2h_bytes_per_step": cache.out_floats(lens) * 4, "steps": KE,
               "note": "fleche_query_host: pinned host IDs -> HBM, query, full output -> pinned host"}

    log("cpu baseline")
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(w, tabs, args.cpu_seconds)

    if rank == 0:
        print(json.dumps({
            "metric": "embedding lookups/s", "value": value, "unit": "Mkeys/s", "n_gpus": world, "steps": K,
            "warmup": W, "ms_per_step": ms_max / K, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f32", "data": "synthetic",
            "config": {"workload": f"{w.name}: {w.n} tables, dim {d if uniform else 'mixed 8-128'}, "
                                   f"{'bags' if w.pooled else 'batch'} {w.batch_size} per table per GPU"
                                   f"{' (multi-hot, sum-pooled)' if w.pooled else ''}, cache "
                                   f"{w.cache_frac:.0%} of table bytes, Zipf a={min(w.skews):.2f}-{max(w.skews):.2f}",
                       "tables": w.n, "dim": d if uniform else sorted(set(w.dims)), "batch": w.batch_size,
                       "lookups_per_step": dst["lookups"] / K,
                       "cache_bytes": w.cache_bytes, "host_table_bytes": w.table_bytes,
                       "parallelism": (f"key-sharded x{world} (" + ("keys and rows over peer memory, fused in the route and restore kernels"
                                                                     if args.p2p else "NCCL all-to-all") + ")"
                                       if sharded else
                                       (f"replicated x{world}" if world > 1 else "single GPU")),
                       "prefill_batches": P, "distinct_timed_batches": min(R, K), "admit_prob": args.admit_prob,
                       "miss_fetch": ("host-assisted: %s host threads stage the missed rows (FLECHE_FLAG_HOST_ASSIST)"
                                      % os.environ.get("FLECHE_HA_THREADS", "12")
                                      + ", share %s of the blocks" % os.environ.get("FLECHE_HA_FRAC", "0.5")) if ha else
                                     "unified index: zero-copy reads of the host rows",
                       "flags": args.flags,
                       "eviction": (f"full-scan between watermarks hi={wm[0]} lo={wm[1]} (reading R23)" if wm else
                                    "on demand (canonical, reading R2)"),
                       "l2": "inputs larger than L2: fresh ID batch per step, 4 rotating output buffers "
                             f"({4 * out_max * 4 / 1e6:.0f} MB), {w.cache_bytes / 1e6:.0f} MB slab"},
            "hit_ratio": hit, "hit_ratio_unique": uhit,
            "unique_misses_per_step": dst["unique_misses"] / K,
            "p50_batch_latency_us": lat[len(lat) // 2], "p99_batch_latency_us": lat[int(len(lat) * 0.99) - 1],
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e,
            "assisted_rows_per_step": dst["assisted_rows"] / K, "assist_timeouts": dst["assist_timeouts"],
            "gpu_launches": int(dst["kernels_launched"]), "clocks": clk, "scans_per_step": dst["scans"] / K,
            "host_tier_gen_s": t_gen,
        }), flush=True)
    if dist:
        dist.barrier()
        if shm_cleanup:
            shm_cleanup()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
