#!/usr/bin/env python
"""bench.py — keys/s of the flat-cache lookup path on BASELINE configs[1] (cfg2).

One step = one batch of the whole hot path through the C ABI
(libfleche.so): KQ (fused self-identified probe + hit gather + miss dedup) and KM (the
unified-index miss fetch over the host link + admission + per-set LRU insert + the
restore of duplicate misses), two kernel launches per batch.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config cfg2] [--impl fleche|reference]

The timed region (K steps) is repeated 3 times and the median reported (the paper
averages 3 runs).  A cfg4 sub-measurement (mixed widths, pooled bags) is
appended to the same JSON line (`also`), unless --no-also.
N > 1 runs under torchrun: every rank serves its own shard of each global batch
with its own replicated cache (no data-path collective; "scaling": "weak").
`--impl reference` times the CPU oracle (oracle/) on the same workload, rank 0 only.
"""
from __future__ import annotations

import argparse
import faulthandler
import json
import os

# the workload generator's OpenMP threads must not spin-wait after their parallel regions:
# they would compete for cores with the ctx's host-assist threads (must be set before libgomp loads)
os.environ.setdefault("OMP_WAIT_POLICY", "PASSIVE")
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
                   help="FLECHE_FLAG_HOST_ASSIST: force the host-assisted miss fetch (paper Fig 8b CPU-DRAM layer); "
                        "it is on by default for host tiers >= 1 GiB")
    p.add_argument("--no-host-assist", action="store_true",
                   help="FLECHE_FLAG_NO_HOST_ASSIST: unified-index zero-copy reads only")
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
    p.add_argument("--reps", type=int, default=3, help="repetitions of the timed region (median reported)")
    p.add_argument("--no-also", action="store_true", help="skip the appended cfg4 sub-measurement")
    p.add_argument("--no-graph", action="store_true", help="skip the CUDA-graph replay measurement")
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


DATASHEET_HBM_GBS = 8000.0       # B200 HBM3e (DGX figure; 7.7 TB/s HGX)
DATASHEET_LINK_GBS = 63.0        # PCIe Gen5 x16 per direction after 128b/130b


def algorithmic_bytes(st: dict, n_queries: int, row: float, row_miss: float, pooled_out: float = 0) -> dict:
    """Per-batch algorithmic bytes, from the run's own counters.

    row: lookup-weighted mean row bytes; row_miss: mean row bytes of unique misses (= host
    bytes / unique misses); pooled_out: bytes of pooled output rows per batch (0: one-hot).
    Step formulas (§8(d-3)): HBM = 8N + row*N + 128U + (U_hit + U_ins)(row + 32),
    host = row_miss * U_miss.  Per kernel: KQ (probe + hit gather), KM (miss fetch + insert
    + restore), KP (pooling)."""
    q = max(n_queries, 1)
    N = st["lookups"] / q
    U = st["unique_keys"] / q
    Uh = st["unique_hits"] / q
    Um = st["unique_misses"] / q
    Ui = st["inserted"] / q
    Nd = (st["misses"] - st["unique_misses"]) / q  # duplicate misses (restored in KM)
    Nm = st["misses"] / q  # missed lookups (owners + duplicates)
    step_hbm = 8 * N + row * N + 128 * U + (Uh + Ui) * (row + 32) + (N * row + pooled_out if pooled_out else 0)
    step_host = Um * row_miss
    # KQ: IDs in, one 128 B set line per unique key, hit rows read + ts sector touched,
    #     out rows written for every non-missed lookup, 8 B dedup tag + 24 B record per unique miss
    kq_hbm = N * 8 + U * 128 + Uh * (row + 32) + (N - Nm) * row + Um * (8 + 24) + Nd * 24
    # KM: miss record in, host row in (host link), owner row written, per insert the set's
    #     key+ts lines (256 B) read and the row + key/ts written; restore: record + owner row
    #     read, duplicate row written
    km_host = Um * row_miss
    km_hbm = Um * 24 + Um * row_miss + Ui * (256 + row_miss + 8) + Nd * (16 + 8 + 2 * row)
    # KP (pooled only): staged rows read once, pooled rows written
    kp_hbm = (N * row + pooled_out) if pooled_out else 0
    return {"N": N, "U": U, "U_hit": Uh, "U_miss": Um, "U_ins": Ui, "N_dup": Nd, "kq_hbm": kq_hbm,
            "km_host": km_host, "km_hbm": km_hbm, "kp_hbm": kp_hbm, "step_hbm": step_hbm, "step_host": step_host}


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


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown CPU"


def cpu_baseline(w, tabs, budget_s):
    """Oracle timed on a bounded sample of the same workload (cold start, batches 0..B-1),
    single-threaded and pinned to one core (sched_setaffinity)."""
    from oracle import oracle as O
    orc = O.Oracle(w.cards, w.dims, tabs, w.cache_bytes, O.MODE_GLOBAL)
    old = os.sched_getaffinity(0)
    core = max(old)
    os.sched_setaffinity(0, {core})
    try:
        t0 = time.perf_counter()
        nb, lk = 0, 0
        gen_t = 0.0
        while time.perf_counter() - t0 - gen_t < budget_s:
            tg = time.perf_counter()
            ids = w.batch(nb, nthreads=1).ids
            gen_t += time.perf_counter() - tg
            orc.query(ids)
            nb += 1
            lk += sum(x.size for x in ids)
        dt = time.perf_counter() - t0 - gen_t
    finally:
        os.sched_setaffinity(0, old)
    return {"value": lk / dt / 1e6, "unit": "Mkeys/s", "cores": 1, "kind": "oracle",
            "sample": f"batches 0..{nb - 1} of {w.name} from a cold cache ({lk} lookups, {dt:.1f}s CPU), "
                      f"single-threaded C++ oracle pinned to core {core}: 1 of {os.cpu_count()} host cores, "
                      f"{cpu_model()}"}


def log(*a):
    print(f"[bench {time.strftime('%H:%M:%S')}]", *a, file=sys.stderr, flush=True)


def host_link_peaks(fl, hostbuf, row_bytes):
    """Host-link rates measured in-run (GB/s): the copy engine's H2D rate over a 1 GiB pinned
    buffer (the link's peak), random rows of the miss size inside a 64 MiB pinned region
    (zero-copy reads with every translation cached), and random rows over the whole host
    tier (the address-translation ceiling of scattered reads on this platform; diagnostic)."""
    import torch
    prow = min((128, 256, 512, 1024), key=lambda r: abs(r - row_bytes))
    pin = torch.empty(1 << 30, dtype=torch.uint8).pin_memory()
    dst = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
    dst.copy_(pin, non_blocking=True)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    best = 0.0
    for _ in range(3):
        e0.record()
        dst.copy_(pin, non_blocking=True)
        e1.record()
        torch.cuda.synchronize()
        best = max(best, (1 << 30) / (e0.elapsed_time(e1) * 1e-3) / 1e9)
    rand64 = fl.binding.probe_host_read(int(pin.data_ptr()), 64 << 20, prow, 1 << 20, 11)
    tier = fl.binding.probe_host_read(int(hostbuf.ctypes.data), int(hostbuf.nbytes), prow, 1 << 20, 7)
    del pin, dst
    scale = row_bytes / prow  # mixed widths: the random-row rates are row rates; scale to the mean miss row
    return {"ce_h2d_gbs": best, "random_64MiB_gbs": rand64 * scale, "translation_ceiling_gbs": tier * scale,
            "probe_row_bytes": prow}


def run_config(args, w, P, W, K, world, rank, local, dist, primary: bool, extra_note: str = ""):
    """Build the host tier and a ctx for workload w, prefill, time K steps (args.reps times),
    profile per kernel, measure latency / graph replay / end to end.  Returns a dict of
    the JSON line's fields (rank 0) or None."""
    import numpy as np
    import torch
    import paper_conf_eurosys_xiellwgrs22_b200 as fl
    from workload import gen as _gen
    dev = torch.device("cuda", local)
    b0 = w.batch(0, rank=rank)
    N = int(b0.lookups * (1.25 if w.pooled else 1))  # max_lookups (bag lengths vary per batch)
    d = w.dims[0]
    uniform = len(set(w.dims)) == 1

    # host tier: every table in one buffer, page-locked + mapped by fleche_create
    log(w.name, "host tier")
    t_gen = time.time()
    shm_cleanup = None
    numa = None
    if dist:  # one copy per NUMA node in /dev/shm, mapped by every local rank on that node
        from workload import shm
        node = shm.gpu_numa_node(local)

        def all_gather_object(x):
            out = [None] * world
            dist.all_gather_object(out, x)
            return out

        creator = shm.creator_ranks(local, node, all_gather_object)
        hostbuf, tabs, shm_cleanup = shm.shared_tables(
            f"fleche_{w.name}_{os.environ.get('MASTER_PORT', '0')}", w.cards, w.dims, w.value_mode, local,
            dist.barrier, node=node, creator=creator)
        numa = {"node": node, "nodes": shm.numa_nodes(), "copy_creator": creator}
    else:
        hostbuf, tabs = w.make_tables()
    t_gen = time.time() - t_gen
    log(w.name, "create")
    sharded = args.mode == "sharded" and primary
    if sharded and (w.pooled or not uniform):
        raise SystemExit("--mode sharded supports one-hot, uniform-width configs (cfg1, cfg2, cfg5)")
    flags = args.flags if primary else 0
    cache = fl.FlatCache(w.cards, w.dims, tabs, w.cache_bytes, N * (world if sharded else 1), local,
                         args.admit_prob if primary else 1.0, _gen.seeds()["admit"], HASH_SEED, flags)
    wm = None
    if args.watermarks and primary:
        wm = [float(x) for x in args.watermarks.split(",")]
        cache.set_watermarks(wm[0], wm[1])
    shard = None
    if sharded:
        if dist is None:
            import torch.distributed as tdist
            tdist.init_process_group("nccl", init_method="tcp://127.0.0.1:%d" % (29600 + os.getpid() % 300),
                                     rank=0, world_size=1, device_id=torch.device("cuda", local))
            dist = tdist
        from paper_conf_eurosys_xiellwgrs22_b200.sharded import ShardedCache
        shard = ShardedCache(cache, row_floats=d, p2p=args.p2p)
    # every query of this run goes to one dedicated stream, so the CUDA-graph capture below
    # records on the stream the ctx was last used on (no cross-stream ordering in the capture)
    prev_stream = torch.cuda.current_stream()
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)

    def gen_batch(b):
        return w.batch(b, rank=rank)

    class DevBatch:
        """One batch resident in HBM: flat IDs (+ flat CSR offsets when pooled)."""

        def __init__(self, bt):
            self.lens = [int(x.size) for x in bt.ids]
            self.ids = torch.from_numpy(np.concatenate(bt.ids)).to(dev)
            self.idv = list(torch.split(self.ids, self.lens))
            self.bags = None
            if bt.offsets is not None:
                self.bags = [int(x.size) - 1 for x in bt.offsets]
                self.offs = torch.from_numpy(np.concatenate(bt.offsets)).to(dev)
                self.offv = list(torch.split(self.offs, [x.size for x in bt.offsets]))
            else:
                self.prep = cache.prepare(self.idv, self.lens)  # validated + marshalled once

        def out_floats(self):
            return cache.pooled_floats(self.bags) if self.bags is not None else cache.out_floats(self.lens)

        def run(self, out, s=None):
            if self.bags is not None:
                cache.query_pooled(self.idv, self.offv, out, stream=s, bags=self.bags, nnz=self.lens)
            elif shard is not None:
                shard.query(self.idv, out, lengths=self.lens)
            else:
                cache.query_prepared(self.prep, out, stream=s)

    out_max = int(DevBatch(b0).out_floats() * 1.25)
    outs = [torch.empty(out_max, dtype=torch.float32, device=dev) for _ in range(4)]  # 4 x out > L2 when large

    log(w.name, "prefill")
    for b in range(P):
        DevBatch(gen_batch(b)).run(outs[b % 4])
        if b % 16 == 15:
            torch.cuda.synchronize()
    torch.cuda.synchronize()

    # pre-generated device-resident batches for warm-up, timed and profiled passes (at most
    # ~8 GB of them; beyond that the timed steps cycle through them; a multiple of 4 so a
    # batch always pairs with the same output buffer)
    log(w.name, "pregen")
    KP = min(K, 300)
    per_step = b0.lookups * 8 * (1.1 if w.pooled else 1.0)
    R = int(min(W + max(1, args.reps) * K + KP + 4, max(8, 8e9 // per_step)))  # every step a fresh batch
    R = max(4, R - R % 4)
    pre = [DevBatch(gen_batch(P + i)) for i in range(R)]
    torch.cuda.synchronize()

    def step(i, out):
        pre[i % R].run(out)

    log(w.name, "timed")
    clock = ClockSampler(local) if primary else None
    if clock:
        clock.start()
    for i in range(W):
        step(i, outs[i % 4])
    torch.cuda.synchronize()
    reps, stats, submit_us = [], [], []
    r0 = cache.shard_stats() if sharded else None
    s0 = cache.stats()
    tw0 = time.perf_counter()
    for rep in range(max(1, args.reps)):
        if dist:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        ts0 = time.perf_counter()
        for k in range(K):
            step(W + rep * K + k, outs[k % 4])
        submit_us.append((time.perf_counter() - ts0) * 1e6 / K)
        e1.record(stream)
        torch.cuda.synchronize()
        if dist:
            dist.barrier()
        ms = e0.elapsed_time(e1)
        if dist:
            t = torch.tensor([ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        reps.append(ms)
    tw1 = time.perf_counter()
    s1 = cache.stats()
    clk = None
    if clock:
        clock.mark(tw0, tw1)
        clk = clock.stop()
    nrep = len(reps)
    ms_med = statistics.median(reps)
    dst = {k: s1[k] - s0[k] for k in fl.STAT_FIELDS}
    steps_timed = K * nrep
    keys_total = dst["lookups"] / nrep * world
    hit = dst["hits"] / max(1, dst["hits"] + dst["misses"])
    uhit = dst["unique_hits"] / max(1, dst["unique_keys"])
    if sharded:  # requester side: this rank's batch lookups and how many hit at their owner
        r1 = cache.shard_stats()
        dr = {k: r1[k] - r0[k] for k in r1}
        keys_total = dr["lookups"] / nrep * world
        hit = dr["hits"] / max(1, dr["lookups"] - dr["invalid"])
    value = keys_total / (ms_med * 1e-3) / 1e6

    # per-kernel device time (profiled pass: CUDA events on the launching stream)
    log(w.name, "profiled pass")
    cache.set_profiling(True)
    sp0 = cache.stats()
    for k in range(KP):
        step(W + nrep * K + k, outs[k % 4])
    torch.cuda.synchronize()
    kms, nq = cache.kernel_times_ex()
    sp1 = cache.stats()
    cache.set_profiling(False)
    dsp = {k: sp1[k] - sp0[k] for k in fl.STAT_FIELDS}
    kavg = {k: v / max(nq, 1) for k, v in kms.items()}
    row_lk = sum(L * 4 * dd for L, dd in zip(pre[0].lens, w.dims)) / max(1, sum(pre[0].lens))
    row_ms = dsp["host_bytes_fetched"] / max(1, dsp["unique_misses"])
    ab = algorithmic_bytes(dsp, nq, row_lk, row_ms, pooled_out=(
        sum(b * 4 * dd for b, dd in zip(pre[0].bags, w.dims)) if w.pooled else 0))

    log(w.name, "host-link peaks")
    hl = host_link_peaks(fl, hostbuf, row_ms)
    log(w.name, "host link", json.dumps(hl), "row_ms", row_ms, "row_lk", row_lk)
    hbm_peak = float(peaks().get("hbm_gbs", 6650.0))
    kern = {
        "kq_kernel": {"ms": kavg["kq"], "bound": "hbm", "bytes": ab["kq_hbm"], "peak": hbm_peak,
                      "peak_source": "MEASURED_PEAKS.json hbm_gbs (of measured)"},
        "km_kernel": {"ms": kavg["km"] + kavg["kd"], "bound": "hbm+host_link", "bytes": ab["km_host"],
                      "peak": hl["ce_h2d_gbs"], "hbm_bytes": ab["km_hbm"],
                      "peak_source": "measured in-run: copy-engine H2D rate over a 1 GiB pinned buffer"},
    }
    kern["km_kernel"]["bound"] = "host_link"
    if w.pooled:
        kern["kp_kernel"] = {"ms": kavg["kp"], "bound": "hbm", "bytes": ab["kp_hbm"], "peak": hbm_peak,
                             "peak_source": "MEASURED_PEAKS.json hbm_gbs (of measured)"}
    for kd_ in kern.values():
        kd_["achieved"] = kd_["bytes"] / (kd_["ms"] * 1e-3) / 1e9
        kd_["frac"] = kd_["achieved"] / kd_["peak"]
    km = kern["km_kernel"]
    km["frac_of_datasheet_link"] = km["achieved"] / DATASHEET_LINK_GBS
    km["frac_of_translation_ceiling"] = km["achieved"] / max(hl["translation_ceiling_gbs"], 1e-9)
    step_sum = sum(v["ms"] for v in kern.values())
    dom = max(kern, key=lambda k: kern[k]["ms"])
    kd_ = kern[dom]
    traffic, traffic_src = None, None
    try:  # committed ncu --set full summary of this config's kernels
        tr = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic_r02.json")))[w.name][dom]
        if not (args.flags or args.watermarks or args.dim or args.batch or args.cache_frac or args.mode != "replicated"
                or args.admit_prob != 1.0):  # only the exact captured configuration
            traffic, traffic_src = tr["dram_bytes"], tr["source"]
    except (OSError, KeyError, ValueError):
        pass
    ms_step = ms_med / K
    t_meas = {"hbm": hbm_peak, "link": hl["ce_h2d_gbs"]}
    t_data = {"hbm": DATASHEET_HBM_GBS, "link": DATASHEET_LINK_GBS}

    def t_roof(bw):
        return max(ab["step_hbm"] / (bw["hbm"] * 1e9), ab["step_host"] / (bw["link"] * 1e9))

    roof = {"bound": kd_["bound"], "achieved": kd_["achieved"], "peak": kd_["peak"], "unit": "GB/s",
            "frac": kd_["frac"], "traffic": traffic, "traffic_source": traffic_src, "kernel": dom,
            "kernel_ms": kd_["ms"], "share_of_step": kd_["ms"] / step_sum, "peak_source": kd_["peak_source"],
            "host_link": hl, "kernels": kern,
            "algorithmic_bytes_per_step": {"hbm": ab["step_hbm"], "host": ab["step_host"],
                                           "formula": "hbm = 8N + row*N + 128U + (U_hit + U_ins)(row + 32); "
                                                      "host = row * U_miss (SURVEY 8(d-3))",
                                           "N": ab["N"], "U": ab["U"], "U_hit": ab["U_hit"], "U_miss": ab["U_miss"],
                                           "U_ins": ab["U_ins"], "row": row_lk},
            "step_roofline_us": t_roof(t_meas) * 1e6, "step_frac": t_roof(t_meas) / (ms_step * 1e-3),
            "step_roofline_us_datasheet": t_roof(t_data) * 1e6,
            "step_frac_datasheet": t_roof(t_data) / (ms_step * 1e-3),
            "step_frac_note": "T_roof = max(HBM bytes / HBM BW, host bytes / link BW) over the measured step; "
                              "measured: MEASURED_PEAKS hbm_gbs + in-run copy-engine H2D; datasheet: 8 TB/s + 63 GB/s"}
    res = {"value": value, "ms_per_step": ms_step, "repetitions_ms_per_step": [r / K for r in reps],
           # host time to submit one step (a step is host-bound when this reaches the device time)
           "submit_us_per_step": sorted(submit_us)[len(submit_us) // 2],
           "hit_ratio": hit, "hit_ratio_unique": uhit, "unique_misses_per_step": dst["unique_misses"] / steps_timed,
           "roofline": roof, "gpu_launches_per_step": dst["kernels_launched"] / steps_timed,
           "gpu_launches": int(dst["kernels_launched"] / nrep), "clocks": clk,
           "host_tier_gen_s": t_gen, "steps": K, "config_fields": {
               "workload": f"{w.name}: {w.n} tables, dim {d if uniform else 'mixed ' + str(min(w.dims)) + '-' + str(max(w.dims))}, "
                           f"{'bags' if w.pooled else 'batch'} {w.batch_size} per table per GPU"
                           f"{' (multi-hot, sum-pooled)' if w.pooled else ''}, cache "
                           f"{w.cache_frac:.0%} of table bytes, Zipf a={min(w.skews):.2f}-{max(w.skews):.2f}{extra_note}",
               "tables": w.n, "dim": d if uniform else sorted(set(w.dims)), "batch": w.batch_size,
               "lookups_per_step": dst["lookups"] / steps_timed, "cache_bytes": w.cache_bytes,
               "host_table_bytes": w.table_bytes, "prefill_batches": P, "distinct_timed_batches": min(R, K * nrep),
               "l2": "inputs larger than L2: fresh ID batch per step, 4 rotating output buffers "
                     f"({4 * out_max * 4 / 1e6:.0f} MB), {w.cache_bytes / 1e6:.0f} MB slab"},
           "scans_per_step": dst["scans"] / steps_timed, "assisted_rows_per_step": dst["assisted_rows"] / steps_timed,
           "assist_timeouts": dst["assist_timeouts"], "sharded": sharded, "wm": wm,
           "ui_share": s1["ui_share_ppm"] / 1e6, "numa": numa}
    if not primary:
        del outs, pre
        cache.close()
        torch.cuda.set_stream(prev_stream)
        return res

    # latency mode: host clock around query + stream sync (includes launch overhead), on
    # batches the cache has never seen; then the same with each query replayed from a CUDA graph
    log(w.name, "latency")
    nlat = min(200, K)
    fresh = [DevBatch(gen_batch(P + W + nrep * K + KP + 1000 + i)) for i in range(2 * nlat)]
    torch.cuda.synchronize()
    lat = []
    for k in range(nlat):
        t0 = time.perf_counter()
        fresh[k].run(outs[k % 4])
        stream.synchronize()
        lat.append((time.perf_counter() - t0) * 1e6)
    lat.sort()
    res["p50_batch_latency_us"] = lat[len(lat) // 2]
    res["p99_batch_latency_us"] = lat[int(len(lat) * 0.99) - 1]
    res["graph"] = None
    if not args.no_graph and not sharded and not w.pooled:
        log(w.name, "graph")
        graphs = []
        for k in range(nlat):  # capture only: nothing runs until replay
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=stream):
                fresh[nlat + k].run(outs[k % 4], s=stream)
            graphs.append(g)
        torch.cuda.synchronize()
        glat = []
        for k in range(nlat // 2):  # latency: replay + sync
            t0 = time.perf_counter()
            graphs[k].replay()
            stream.synchronize()
            glat.append((time.perf_counter() - t0) * 1e6)
        glat.sort()
        torch.cuda.synchronize()
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        f0.record()
        for k in range(nlat // 2, nlat):  # throughput: replays back to back
            graphs[k].replay()
        f1.record()
        torch.cuda.synchronize()
        gms = f0.elapsed_time(f1) / (nlat - nlat // 2)
        res["graph"] = {"value": sum(fresh[0].lens) * world / (gms * 1e-3) / 1e6, "unit": "Mkeys/s",
                        "ms_per_step": gms, "p50_batch_latency_us": glat[len(glat) // 2],
                        "steps": nlat - nlat // 2,
                        "note": "each query captured once into a CUDA graph (2 kernel nodes), replayed on "
                                "batches the cache had not seen"}
        del graphs
    del fresh
    res["launch_overhead_us"] = res["p50_batch_latency_us"] - ms_step * 1e3

    # end to end through the host-buffer entry point: H2D ids + query + D2H out per step
    e2e = None
    if not args.no_e2e and not w.pooled and not sharded:
        log(w.name, "e2e")
        KE = min(K, 100)
        lens = [w.batch_size] * w.n
        hids = [torch.from_numpy(np.concatenate(gen_batch(P + W + nrep * K + KP + i).ids)).pin_memory()
                for i in range(KE)]
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
    res["e2e"] = e2e

    res["cpu_baseline"] = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        log(w.name, "cpu baseline")
        res["cpu_baseline"] = cpu_baseline(w, tabs, args.cpu_seconds)
    res["_cleanup"] = shm_cleanup
    del outs, pre
    cache.close()
    torch.cuda.set_stream(prev_stream)
    return res


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
    if args.no_host_assist:
        args.flags |= 0x20
    if args.host_assist:
        args.flags |= 0x8
        if args.ha_frac is not None:
            os.environ["FLECHE_HA_FRAC"] = str(args.ha_frac)
    if args.impl == "reference":
        return run_reference(args, w, P, W, K)

    import torch
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    r = run_config(args, w, P, W, K, world, rank, local, dist, primary=True)

    also = None
    if not args.no_also and args.config != "cfg4" and world == 1 and rank == 0:
        # cfg4 (mixed widths 8-128, multi-hot sum-pooled bags): the largest single-GPU BASELINE
        # config, measured in the same run (fewer steps; its host tier is 21 GB)
        try:
            w4 = configs.get("cfg4")
            a = run_config(args, w4, PREFILL["cfg4"], 3, max(5, min(K, 20)), 1, 0, local, None, primary=False)
            also = {"cfg4": {"metric": "embedding lookups/s", "value": a["value"], "unit": "Mkeys/s",
                             "ms_per_step": a["ms_per_step"], "repetitions_ms_per_step": a["repetitions_ms_per_step"],
                             "hit_ratio": a["hit_ratio"], "hit_ratio_unique": a["hit_ratio_unique"],
                             "gpu_launches_per_step": a["gpu_launches_per_step"],
                             "roofline": {k: a["roofline"][k] for k in ("kernel", "kernel_ms", "share_of_step", "frac",
                                                                        "achieved", "peak", "step_frac",
                                                                        "step_roofline_us", "step_frac_datasheet")},
                             "kernels": {k: {"ms": v["ms"], "achieved": v["achieved"], "frac": v["frac"]}
                                         for k, v in a["roofline"]["kernels"].items()},
                             "config": a["config_fields"], "steps": a["steps"]}}
        except Exception as e:  # the primary line must still print
            also = {"cfg4": {"error": repr(e)}}

    if rank == 0:
        cf = r["config_fields"]
        cf["parallelism"] = (f"key-sharded x{world} (" + ("keys and rows over peer memory, fused in the route and "
                                                          "restore kernels" if args.p2p else "NCCL all-to-all") + ")"
                             if r["sharded"] else (f"replicated x{world}" if world > 1 else "single GPU"))
        cf["admit_prob"] = args.admit_prob
        cf["miss_fetch"] = (("host-assisted split: host threads stage a share of each batch's unique misses "
                             "(%.0f of %.0f per step, share FLECHE_HA_FRAC=%s), the miss kernel reads the rest "
                             "zero-copy (unified index; its share of the blocks %.2f, %s)") % (
                                r["assisted_rows_per_step"], r["unique_misses_per_step"],
                                os.environ.get("FLECHE_HA_FRAC", "tuned"), r["ui_share"],
                                "fixed by FLECHE_HA_FRAC" if os.environ.get("FLECHE_HA_FRAC") else
                                "tuned online by the paper's loop, P:L861-872")
                            if r["assisted_rows_per_step"] > 0 else
                            "unified index: zero-copy reads of the host rows, address-ordered")
        cf["flags"] = args.flags
        cf["eviction"] = (f"full-scan between watermarks hi={r['wm'][0]} lo={r['wm'][1]} (reading R23)" if r["wm"]
                          else "on demand (canonical, reading R2)")
        cf["timing"] = f"median of {args.reps} timed regions of {K} steps (CUDA events on the launching stream)"
        if r["numa"]:
            cf["host_tier"] = ("one /dev/shm copy per NUMA node (%d nodes), pages bound to the node of the GPUs "
                               "that map it; rank 0's GPU on node %d" % (r["numa"]["nodes"], r["numa"]["node"]))
        line = {
            "metric": "embedding lookups/s", "value": r["value"], "unit": "Mkeys/s", "n_gpus": world, "steps": K,
            "warmup": W, "ms_per_step": r["ms_per_step"], "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic", "config": cf,
            "repetitions_ms_per_step": r["repetitions_ms_per_step"], "submit_us_per_step": r["submit_us_per_step"],
            "hit_ratio": r["hit_ratio"], "hit_ratio_unique": r["hit_ratio_unique"],
            "unique_misses_per_step": r["unique_misses_per_step"],
            "p50_batch_latency_us": r["p50_batch_latency_us"], "p99_batch_latency_us": r["p99_batch_latency_us"],
            "launch_overhead_us": r["launch_overhead_us"], "graph": r["graph"],
            "roofline": r["roofline"], "cpu_baseline": r["cpu_baseline"], "e2e": r["e2e"],
            "assisted_rows_per_step": r["assisted_rows_per_step"], "assist_timeouts": r["assist_timeouts"],
            "gpu_launches": r["gpu_launches"], "gpu_launches_per_step": r["gpu_launches_per_step"],
            "clocks": r["clocks"], "scans_per_step": r["scans_per_step"], "host_tier_gen_s": r["host_tier_gen_s"],
            "also": also,
        }
        print(json.dumps(line), flush=True)
    if dist:
        dist.barrier()
        if r.get("_cleanup"):
            r["_cleanup"]()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
