"""Thin ctypes binding of libfleche.so (include/fleche.h).  Argument marshalling only:
every step of the lookup path runs in the library's CUDA kernels.  There is no CPU
fallback: if the shared library is missing this module raises at import time.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, os.environ.get("FLECHE_LIB", "libfleche.so"))  # FLECHE_LIB: experiment builds

if not os.path.exists(LIB_PATH):
    raise ImportError(f"libfleche.so not built at {LIB_PATH}: run `make` (or __graft_entry__.build()) first; "
                      "the flat cache has no CPU fallback")

_lib = ctypes.CDLL(LIB_PATH)

OK, EINVAL, ENOMEM, ECUDA, ENCCL, ERANGE, ESTATE = 0, -1, -2, -3, -4, -5, -6
FLAG_STATIC_PER_TABLE, FLAG_PER_TABLE_LAUNCH, FLAG_HOST_ASSIST, FLAG_FUSED_HIT_COPY = 0x2, 0x4, 0x8, 0x10
FLAG_NO_HOST_ASSIST = 0x20
MAX_TABLES = 512

_vp, _i64, _i32, _u64, _u32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, ctypes.c_uint32


class fleche_config(ctypes.Structure):
    _fields_ = [("num_tables", _i32), ("cardinalities", _vp), ("dims", _vp), ("cache_bytes", _u64),
                ("host_tables", _vp), ("max_lookups", _i64), ("device", _i32), ("admit_prob", ctypes.c_double),
                ("admit_seed", _u64), ("hash_seed", _u32), ("flags", _u32), ("key_bits", _i32), ("reserved", _i32)]


STAT_FIELDS = ["batches", "lookups", "hits", "misses", "invalid", "unique_keys", "unique_hits", "unique_misses",
               "inserted", "evicted", "bypassed", "occupancy_bytes", "capacity_bytes", "index_bytes",
               "host_bytes_fetched", "kernels_launched", "assisted_rows", "assist_timeouts", "scans", "ui_share_ppm"]


class fleche_stats_t(ctypes.Structure):
    _fields_ = [(f, _u64) for f in STAT_FIELDS]


def _sig(name, res, args):
    f = getattr(_lib, name)
    f.restype = res
    f.argtypes = args
    return f


fleche_create = _sig("fleche_create", ctypes.c_int, [ctypes.POINTER(fleche_config), ctypes.POINTER(_vp)])
fleche_query = _sig("fleche_query", ctypes.c_int, [_vp, _vp, _vp, _vp, _vp])
fleche_prefill = _sig("fleche_prefill", ctypes.c_int, [_vp, _vp, _vp, _vp])
fleche_query_host = _sig("fleche_query_host", ctypes.c_int, [_vp, _vp, _vp, _vp, _vp])
fleche_stats = _sig("fleche_stats", ctypes.c_int, [_vp, ctypes.POINTER(fleche_stats_t)])
fleche_reset_stats = _sig("fleche_reset_stats", ctypes.c_int, [_vp])
fleche_destroy = _sig("fleche_destroy", ctypes.c_int, [_vp])
fleche_strerror = _sig("fleche_strerror", ctypes.c_char_p, [ctypes.c_int])
fleche_get_encoding = _sig("fleche_get_encoding", ctypes.c_int, [_vp, _vp, _vp, ctypes.POINTER(_i32)])
fleche_encode = _sig("fleche_encode", ctypes.c_int, [_i32, _vp, _i32, _vp, _vp, _vp, ctypes.POINTER(_i32)])
fleche_get_geometry = _sig("fleche_get_geometry", ctypes.c_int,
                           [_vp, ctypes.POINTER(_i64), ctypes.POINTER(_i64), ctypes.POINTER(_i32)])
fleche_debug_snapshot = _sig("fleche_debug_snapshot", ctypes.c_int, [_vp, _vp, _vp, ctypes.c_size_t, _vp,
                                                                     ctypes.c_size_t])

fleche_set_profiling = _sig("fleche_set_profiling", ctypes.c_int, [_vp, ctypes.c_int])
fleche_kernel_times = _sig("fleche_kernel_times", ctypes.c_int, [_vp, ctypes.POINTER(ctypes.c_double),
                                                                 ctypes.POINTER(ctypes.c_double),
                                                                 ctypes.POINTER(_u64)])
fleche_kernel_times_ex = _sig("fleche_kernel_times_ex", ctypes.c_int, [_vp, _vp, ctypes.POINTER(_u64)])
fleche_probe_host_read = _sig("fleche_probe_host_read", ctypes.c_int, [_vp, _u64, _i32, _i64, _u64, _vp,
                                                                       ctypes.POINTER(ctypes.c_double)])

fleche_query_pooled = _sig("fleche_query_pooled", ctypes.c_int, [_vp, _vp, _vp, _vp, _vp, _vp, _vp])
fleche_route = _sig("fleche_route", ctypes.c_int, [_vp, _vp, _vp, _i32, _u32, _vp, _vp, _vp])
fleche_query_keys = _sig("fleche_query_keys", ctypes.c_int, [_vp, _vp, _i64, _vp, _vp, _vp])
fleche_restore = _sig("fleche_restore", ctypes.c_int, [_vp, _vp, _vp, _vp, _vp])
fleche_shard_stats = _sig("fleche_shard_stats", ctypes.c_int, [_vp, ctypes.POINTER(_u64), ctypes.POINTER(_u64),
                                                               ctypes.POINTER(_u64), ctypes.POINTER(_u64)])
fleche_debug_ctl = _sig("fleche_debug_ctl", ctypes.c_int, [_vp, _vp, ctypes.c_size_t])
fleche_set_watermarks = _sig("fleche_set_watermarks", ctypes.c_int, [_vp, ctypes.c_double, ctypes.c_double])
fleche_route_p2p = _sig("fleche_route_p2p", ctypes.c_int, [_vp, _vp, _vp, _i32, _u32, _vp, _vp, _vp])
fleche_query_keys_seg = _sig("fleche_query_keys_seg", ctypes.c_int, [_vp, _vp, _vp, _i32, _vp, _vp, _vp])
fleche_restore_p2p = _sig("fleche_restore_p2p", ctypes.c_int, [_vp, _i32, _vp, _vp, _vp, _vp, _vp])
fleche_query_keys_seg_dev = _sig("fleche_query_keys_seg_dev", ctypes.c_int, [_vp, _vp, _vp, _i32, _i32, _vp, _vp, _vp])
fleche_restore_p2p_dev = _sig("fleche_restore_p2p_dev", ctypes.c_int, [_vp, _i32, _vp, _vp, _vp, _i32, _vp, _vp])
fleche_ipc_alloc = _sig("fleche_ipc_alloc", ctypes.c_int, [ctypes.c_size_t, ctypes.POINTER(_vp)])
fleche_ipc_free = _sig("fleche_ipc_free", ctypes.c_int, [_vp])
fleche_ipc_handle = _sig("fleche_ipc_handle", ctypes.c_int, [_vp, _vp])
fleche_ipc_open = _sig("fleche_ipc_open", ctypes.c_int, [_vp, ctypes.POINTER(_vp)])
fleche_ipc_close = _sig("fleche_ipc_close", ctypes.c_int, [_vp])
fleche_debug_locations = _sig("fleche_debug_locations", ctypes.c_int, [_vp, _vp, ctypes.c_size_t])

EXPORTED = ["fleche_create", "fleche_query", "fleche_query_pooled", "fleche_query_host", "fleche_stats",
            "fleche_reset_stats", "fleche_destroy", "fleche_strerror", "fleche_get_encoding", "fleche_get_geometry",
            "fleche_debug_snapshot", "fleche_debug_locations", "fleche_set_profiling", "fleche_kernel_times",
            "fleche_probe_host_read", "fleche_route", "fleche_query_keys", "fleche_restore", "fleche_shard_stats",
            "fleche_kernel_times_ex", "fleche_set_watermarks", "fleche_prefill", "fleche_debug_ctl",
            "fleche_restore_p2p", "fleche_ipc_handle", "fleche_ipc_open", "fleche_ipc_close", "fleche_ipc_alloc",
            "fleche_ipc_free", "fleche_route_p2p", "fleche_query_keys_seg", "fleche_encode",
            "fleche_query_keys_seg_dev", "fleche_restore_p2p_dev"]


def encode(cards, key_bits: int = 0):
    """The flat-key code fleche_create builds (host-only, no GPU): (key_bits, base[n], fbits[n], hashed[n])."""
    c = np.ascontiguousarray(cards, dtype=np.int64)
    n = len(c)
    base = np.zeros(n, dtype=np.uint64)
    fb = np.zeros(n, dtype=np.int32)
    h = np.zeros(n, dtype=np.int32)
    kb = _i32()
    _check(fleche_encode(n, c.ctypes.data, int(key_bits), base.ctypes.data, fb.ctypes.data, h.ctypes.data,
                         ctypes.byref(kb)), "fleche_encode")
    return int(kb.value), base, fb, h


def ipc_alloc(nbytes: int) -> int:
    p = _vp()
    _check(fleche_ipc_alloc(int(nbytes), ctypes.byref(p)), "fleche_ipc_alloc")
    return int(p.value)


def ipc_free(ptr: int):
    _check(fleche_ipc_free(ptr), "fleche_ipc_free")


def ipc_handle(ptr: int) -> bytes:
    """64-byte CUDA IPC handle of a device allocation (its base pointer)."""
    h = (ctypes.c_uint8 * 64)()
    _check(fleche_ipc_handle(ptr, h), "fleche_ipc_handle")
    return bytes(h)


def ipc_open(handle: bytes) -> int:
    h = (ctypes.c_uint8 * 64).from_buffer_copy(handle)
    p = _vp()
    _check(fleche_ipc_open(h, ctypes.byref(p)), "fleche_ipc_open")
    return int(p.value)


def ipc_close(ptr: int):
    _check(fleche_ipc_close(ptr), "fleche_ipc_close")


def probe_host_read(host_ptr: int, nbytes: int, row_bytes: int, rows: int, seed: int = 1, stream=None) -> float:
    """Random-row zero-copy read bandwidth (GB/s) of an already-registered host buffer."""
    g = ctypes.c_double()
    _check(fleche_probe_host_read(host_ptr, nbytes, row_bytes, rows, seed, _stream_handle(stream), ctypes.byref(g)),
           "fleche_probe_host_read")
    return float(g.value)


class FlecheError(RuntimeError):
    def __init__(self, status: int, what: str):
        super().__init__(f"{what}: {fleche_strerror(status).decode()} ({status})")
        self.status = status


def _check(status: int, what: str, allow=(OK,)):
    if status not in allow:
        raise FlecheError(status, what)
    return status


def _ptr(x) -> int:
    """Raw address of a torch tensor / numpy array / int."""
    if x is None:
        return 0
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return int(x.data_ptr())
    if isinstance(x, np.ndarray):
        return int(x.ctypes.data)
    raise TypeError(type(x))


def _stream_handle(stream) -> int:
    if stream is None:
        import torch
        return int(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return stream
    return int(stream.cuda_stream)


def _check_ids(ids, n: int, device, what: str):
    """int64, contiguous, on `device` (None: host memory) -- for tensors and numpy arrays;
    raw pointers (ints) are passed through unchecked."""
    if len(ids) != n:
        raise ValueError(f"{what}: {len(ids)} ID arrays for {n} tables")
    for t, x in enumerate(ids):
        if isinstance(x, int) or x is None:
            continue
        if isinstance(x, np.ndarray):
            if device is not None:
                raise ValueError(f"{what}: table {t} IDs are a host array, a device tensor is needed")
            if x.dtype != np.int64 or not x.flags.c_contiguous:
                raise ValueError(f"{what}: table {t} IDs must be contiguous int64")
            continue
        if str(x.dtype) != "torch.int64" or not x.is_contiguous():
            raise ValueError(f"{what}: table {t} IDs must be contiguous int64 (got {x.dtype})")
        dev = x.device.index if x.is_cuda else None
        if (device is None) != (not x.is_cuda) or (device is not None and dev != device):
            raise ValueError(f"{what}: table {t} IDs on {x.device}, expected "
                             f"{'host memory' if device is None else f'cuda:{device}'}")


def _check_out(out, floats: int, device, what: str):
    """fp32, contiguous, >= floats elements, on `device` (None: host memory)."""
    if isinstance(out, int) or out is None:
        return
    if isinstance(out, np.ndarray):
        ok = device is None and out.dtype == np.float32 and out.flags.c_contiguous and out.size >= floats
    else:
        ok = (str(out.dtype) == "torch.float32" and out.is_contiguous() and out.numel() >= floats and
              (out.device.index == device if device is not None else not out.is_cuda) and
              (device is None or out.is_cuda))
    if not ok:
        raise ValueError(f"{what}: out must be a contiguous float32 buffer of >= {floats} elements in "
                         f"{'host memory' if device is None else f'cuda:{device}'}")


class FlatCache:
    """One flat GPU cache over the given host tables (fleche_create / fleche_query / fleche_stats)."""

    def __init__(self, cards, dims, host_tables, cache_bytes: int, max_lookups: int, device: int = 0,
                 admit_prob: float = 1.0, admit_seed: int = 0, hash_seed: int = 0, flags: int = 0,
                 key_bits: int = 0):
        self.n = len(cards)
        self.cards = np.ascontiguousarray(cards, dtype=np.int64)
        self.dims = np.ascontiguousarray(dims, dtype=np.int32)
        self._tables = list(host_tables)  # keep the host tier alive for the ctx's lifetime
        self._tp = (_vp * self.n)(*[_ptr(t) for t in self._tables])
        cfg = fleche_config(self.n, self.cards.ctypes.data, self.dims.ctypes.data, int(cache_bytes),
                            ctypes.cast(self._tp, _vp), int(max_lookups), int(device), float(admit_prob),
                            int(admit_seed), int(hash_seed), int(flags), int(key_bits), 0)
        h = _vp()
        _check(fleche_create(ctypes.byref(cfg), ctypes.byref(h)), "fleche_create")
        self.h = h.value
        self.device = device
        self.max_lookups = int(max_lookups)

    def close(self):
        if getattr(self, "h", None):
            fleche_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_watermarks(self, hi: float, lo: float):
        """Full-scan eviction between the watermarks hi/lo (fractions of capacity_bytes),
        P:L660-662, reading R23; hi >= 1 turns it off."""
        _check(fleche_set_watermarks(self.h, float(hi), float(lo)), "fleche_set_watermarks")

    def out_floats(self, lengths) -> int:
        return int(sum(int(l) * int(d) for l, d in zip(lengths, self.dims)))

    def query(self, ids, out, stream=None, lengths=None):
        """ids: list of n device int64 tensors (or pointers with `lengths`); out: device fp32 buffer."""
        _check_ids(ids, self.n, self.device, "query")
        if lengths is None:
            lengths = [int(x.numel()) for x in ids]
        _check_out(out, self.out_floats(lengths), self.device, "query")
        lp = (_i64 * self.n)(*lengths)
        ip = (_vp * self.n)(*[_ptr(x) for x in ids])
        _check(fleche_query(self.h, ip, lp, _ptr(out), _stream_handle(stream)), "fleche_query")

    def prepare(self, ids, lengths=None):
        """Validate and marshal a batch's ID arrays once (the caller keeps them alive and
        unchanged); `query_prepared` then only checks `out`."""
        _check_ids(ids, self.n, self.device, "prepare")
        if lengths is None:
            lengths = [int(x.numel()) for x in ids]
        return ((_vp * self.n)(*[_ptr(x) for x in ids]), (_i64 * self.n)(*lengths), self.out_floats(lengths))

    def query_prepared(self, prep, out, stream=None):
        ip, lp, floats = prep
        _check_out(out, floats, self.device, "query")
        _check(fleche_query(self.h, ip, lp, _ptr(out), _stream_handle(stream)), "fleche_query")

    def prefill(self, ids, stream=None, lengths=None):
        """Warm start: one batch of lookups through the cache, rows discarded."""
        _check_ids(ids, self.n, self.device, "prefill")
        if lengths is None:
            lengths = [int(x.numel()) for x in ids]
        lp = (_i64 * self.n)(*lengths)
        ip = (_vp * self.n)(*[_ptr(x) for x in ids])
        _check(fleche_prefill(self.h, ip, lp, _stream_handle(stream)), "fleche_prefill")

    def pooled_floats(self, bags) -> int:
        return int(sum(int(b) * int(d) for b, d in zip(bags, self.dims)))

    def query_pooled(self, ids, offsets, out, stream=None, bags=None, nnz=None):
        """ids/offsets: lists of n device int64 tensors (CSR per table); out: device fp32 buffer."""
        _check_ids(ids, self.n, self.device, "query_pooled")
        _check_ids(offsets, self.n, self.device, "query_pooled offsets")
        if bags is None:
            bags = [int(o.numel()) - 1 for o in offsets]
        if nnz is None:
            nnz = [int(x.numel()) for x in ids]
        _check_out(out, self.pooled_floats(bags), self.device, "query_pooled")
        bp = (_i64 * self.n)(*bags)
        npp = (_i64 * self.n)(*nnz)
        ip = (_vp * self.n)(*[_ptr(x) for x in ids])
        op = (_vp * self.n)(*[_ptr(o) for o in offsets])
        _check(fleche_query_pooled(self.h, ip, op, bp, npp, _ptr(out), _stream_handle(stream)), "fleche_query_pooled")

    # ---- key-sharded building blocks (see include/fleche.h and sharded.py)
    def route(self, ids, world, owner_seed, send_keys, send_counts, stream=None, lengths=None):
        if lengths is None:
            lengths = [int(x.numel()) for x in ids]
        lp = (_i64 * self.n)(*lengths)
        ip = (_vp * self.n)(*[_ptr(x) for x in ids])
        _check(fleche_route(self.h, ip, lp, int(world), int(owner_seed), _ptr(send_keys), _ptr(send_counts),
                            _stream_handle(stream)), "fleche_route")

    def query_keys(self, keys, count, rows, hit_flags=None, stream=None):
        _check(fleche_query_keys(self.h, _ptr(keys), int(count), _ptr(rows), _ptr(hit_flags), _stream_handle(stream)),
               "fleche_query_keys")

    def route_p2p(self, ids, world, owner_seed, peer_slots, send_counts, stream=None, lengths=None):
        if lengths is None:
            lengths = [int(x.numel()) for x in ids]
        lp = (_i64 * self.n)(*lengths)
        ip = (_vp * self.n)(*[_ptr(x) for x in ids])
        sp = (_vp * world)(*[int(p) for p in peer_slots])
        _check(fleche_route_p2p(self.h, ip, lp, int(world), int(owner_seed), sp, _ptr(send_counts),
                                _stream_handle(stream)), "fleche_route_p2p")

    def query_keys_seg(self, segs, counts, rows, hit_flags=None, stream=None):
        G = len(segs)
        sp = (_vp * G)(*[int(p) for p in segs])
        cp = (_i64 * G)(*[int(x) for x in counts])
        _check(fleche_query_keys_seg(self.h, sp, cp, G, _ptr(rows), _ptr(hit_flags), _stream_handle(stream)),
               "fleche_query_keys_seg")

    def query_keys_seg_dev(self, segs, counts_dev, me, rows, hit_flags=None, stream=None):
        """Sync-free owner query: counts_dev = the G x G routed-count matrix (device int64)."""
        G = len(segs)
        sp = (_vp * G)(*[int(p) for p in segs])
        _check(fleche_query_keys_seg_dev(self.h, sp, _ptr(counts_dev), G, int(me), _ptr(rows), _ptr(hit_flags),
                                         _stream_handle(stream)), "fleche_query_keys_seg_dev")

    def restore_p2p_dev(self, peer_rows, peer_flags, counts_dev, me, out, stream=None):
        """Sync-free fused restore: offsets into the owners' answers from the device count matrix."""
        W = len(peer_rows)
        rp = (_vp * W)(*[int(p) for p in peer_rows])
        fp = (_vp * W)(*[int(p) for p in peer_flags]) if peer_flags is not None else None
        _check(fleche_restore_p2p_dev(self.h, W, rp, fp, _ptr(counts_dev), int(me), _ptr(out), _stream_handle(stream)),
               "fleche_restore_p2p_dev")

    def restore_p2p(self, peer_rows, peer_flags, peer_off, out, stream=None):
        """Fused exchange: restore from every owner's rows in place (peer pointers, ints)."""
        W = len(peer_rows)
        rp = (_vp * W)(*[int(p) for p in peer_rows])
        fp = (_vp * W)(*[int(p) for p in peer_flags]) if peer_flags is not None else None
        op = (_i64 * W)(*[int(x) for x in peer_off])
        _check(fleche_restore_p2p(self.h, W, rp, fp, op, _ptr(out), _stream_handle(stream)), "fleche_restore_p2p")

    def restore(self, rows, hit_flags, out, stream=None):
        _check(fleche_restore(self.h, _ptr(rows), _ptr(hit_flags), _ptr(out), _stream_handle(stream)),
               "fleche_restore")

    def shard_stats(self) -> dict:
        v = [_u64() for _ in range(4)]
        _check(fleche_shard_stats(self.h, *[ctypes.byref(x) for x in v]), "fleche_shard_stats")
        return dict(zip(["lookups", "hits", "invalid", "unique_routed"], [int(x.value) for x in v]))

    def locations(self):
        sets, _, _ = self.geometry()
        loc = np.empty(sets * 32, np.uint16)
        _check(fleche_debug_locations(self.h, loc.ctypes.data, loc.size), "fleche_debug_locations")
        return loc

    def query_host(self, ids, out, stream=None, lengths=None):
        """ids: list of n host int64 arrays (ideally pinned); out: host fp32 buffer."""
        _check_ids(ids, self.n, None, "query_host")
        if lengths is None:
            lengths = [int(x.size if isinstance(x, np.ndarray) else x.numel()) for x in ids]
        _check_out(out, self.out_floats(lengths), None, "query_host")
        lp = (_i64 * self.n)(*lengths)
        ip = (_vp * self.n)(*[_ptr(x) for x in ids])
        _check(fleche_query_host(self.h, ip, lp, _ptr(out), _stream_handle(stream)), "fleche_query_host")

    def stats(self, allow_invalid: bool = True) -> dict:
        s = fleche_stats_t()
        st = fleche_stats(self.h, ctypes.byref(s))
        _check(st, "fleche_stats", (OK, ERANGE) if allow_invalid else (OK,))
        d = {f: int(getattr(s, f)) for f in STAT_FIELDS}
        d["invalid_seen"] = st == ERANGE
        return d

    def reset_stats(self):
        _check(fleche_reset_stats(self.h), "fleche_reset_stats")

    def set_profiling(self, on: bool):
        _check(fleche_set_profiling(self.h, 1 if on else 0), "fleche_set_profiling")

    def kernel_times_ex(self):
        """({'kq','km','kd','kp'} ms totals, profiled queries) since the last call."""
        ms = (ctypes.c_double * 4)()
        q = _u64()
        _check(fleche_kernel_times_ex(self.h, ms, ctypes.byref(q)), "fleche_kernel_times_ex")
        return dict(zip(["kq", "km", "kd", "kp"], [float(x) for x in ms])), int(q.value)

    def kernel_times(self):
        """(KQ ms total, KI ms total, profiled queries) since the last call."""
        a, b, q = ctypes.c_double(), ctypes.c_double(), _u64()
        _check(fleche_kernel_times(self.h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(q)), "fleche_kernel_times")
        return float(a.value), float(b.value), int(q.value)

    def encoding(self):
        base = np.zeros(self.n, dtype=np.uint64)
        fb = np.zeros(self.n, dtype=np.int32)
        kb = _i32()
        _check(fleche_get_encoding(self.h, base.ctypes.data, fb.ctypes.data, ctypes.byref(kb)), "fleche_get_encoding")
        return int(kb.value), base, fb

    def geometry(self):
        s, r, d = _i64(), _i64(), _i32()
        _check(fleche_get_geometry(self.h, ctypes.byref(s), ctypes.byref(r), ctypes.byref(d)), "fleche_get_geometry")
        return int(s.value), int(r.value), int(d.value)

    def snapshot(self):
        """keys, ts and the slab: uniform layout -> [S*32, d] rows; bytes layout -> [S, region floats]."""
        sets, rows, d = self.geometry()
        keys = np.empty(sets * 32, np.uint32)
        ts = np.empty(sets * 32, np.uint32)
        if d == 0:  # static per-table partitions: flat slab (rows of each table's width)
            _check(fleche_debug_snapshot(self.h, keys.ctypes.data, ts.ctypes.data, keys.size, 0, 0),
                   "fleche_debug_snapshot")
            return keys, ts, None
        per = d if d > 0 else -d
        nrow = sets * 32 if d > 0 else sets
        slab = np.empty(nrow * per, np.float32)
        _check(fleche_debug_snapshot(self.h, keys.ctypes.data, ts.ctypes.data, keys.size, slab.ctypes.data, slab.size),
               "fleche_debug_snapshot")
        return keys, ts, slab.reshape(nrow, per)
