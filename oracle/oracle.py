"""ctypes wrapper of the CPU oracle (oracle/oracle.cpp).

TEST INFRASTRUCTURE ONLY: imported by tests/, ``__graft_entry__.smoke()`` and
bench.py's ``cpu_baseline`` / ``--impl reference`` legs.  The product package never
imports this module.  See oracle.cpp's header for what is computed and which paper
passages each part follows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libfleche_oracle.so")
_lib = None

MODE_GLOBAL = 0
MODE_SETASSOC = 1
MODE_SETBYTES = 2

STAT_FIELDS = ["batches", "lookups", "hits", "misses", "invalid", "unique_keys", "unique_hits", "unique_misses",
               "inserted", "evicted", "bypassed", "occupancy_bytes", "capacity_bytes", "bypass_full"]


class _Stats(ctypes.Structure):
    _fields_ = [(f, ctypes.c_uint64) for f in STAT_FIELDS]


def lib():
    global _lib
    if _lib is None:
        src = os.path.join(_HERE, "oracle.cpp")
        if not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
            subprocess.check_call(["make", "-s", "-C", os.path.dirname(_HERE), "oracle/libfleche_oracle.so"])
        L = ctypes.CDLL(_LIB_PATH)
        vp, i64, i32, u64, u32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, ctypes.c_uint32
        L.or_encode.restype = ctypes.c_int
        L.or_encode.argtypes = [ctypes.c_int, vp, ctypes.c_int, vp, vp]
        L.or_self_identify.restype = None
        L.or_self_identify.argtypes = [ctypes.c_int, vp, i64, ctypes.POINTER(i32), ctypes.POINTER(i64)]
        L.or_set_hash.restype = u32
        L.or_set_hash.argtypes = [u32, u32]
        L.or_create.restype = vp
        L.or_create.argtypes = [ctypes.c_int, vp, vp, vp, u64, ctypes.c_int, ctypes.c_double, u64, u32]
        L.or_create_setbytes.restype = vp
        L.or_create_setbytes.argtypes = [ctypes.c_int, vp, vp, vp, u64, ctypes.c_int, u64, ctypes.c_double, u64, u32]
        L.or_destroy.restype = None
        L.or_destroy.argtypes = [vp]
        L.or_query.restype = ctypes.c_int
        L.or_query.argtypes = [vp, vp, vp, vp]
        L.or_query_pooled.restype = ctypes.c_int
        L.or_query_pooled.argtypes = [vp, vp, vp, vp, vp]
        L.or_stats.restype = None
        L.or_stats.argtypes = [vp, ctypes.POINTER(_Stats)]
        L.or_encode_short.restype = ctypes.c_int
        L.or_encode_short.argtypes = [ctypes.c_int, vp, ctypes.c_int, vp, vp, vp]
        L.or_encode_fixed.restype = ctypes.c_int
        L.or_encode_fixed.argtypes = [ctypes.c_int, vp, ctypes.c_int, vp, vp, vp]
        L.or_short_id.restype = i64
        L.or_short_id.argtypes = [i32, i64, i32, i32]
        L.or_set_key_bits.restype = ctypes.c_int
        L.or_set_key_bits.argtypes = [vp, ctypes.c_int]
        L.or_set_watermarks.restype = ctypes.c_int
        L.or_set_watermarks.argtypes = [vp, u64, u64]
        L.or_scans.restype = u64
        L.or_scans.argtypes = [vp]
        L.or_cached_keys.restype = i64
        L.or_cached_keys.argtypes = [vp, vp, vp, i64]
        _lib = L
    return _lib


def encode(cards, key_bits: int = 32):
    """Size-aware flat-key coding. Returns (B_min, base[n], fbits[n]) or None."""
    n = len(cards)
    c = np.ascontiguousarray(cards, dtype=np.int64)
    base = np.zeros(n, dtype=np.uint64)
    fb = np.zeros(n, dtype=np.int32)
    bmin = lib().or_encode(n, c.ctypes.data, key_bits, base.ctypes.data, fb.ctypes.data)
    if bmin < 0:
        return None
    return bmin, base, fb


def encode_short(cards, key_bits: int, fixed: bool = False):
    """Short flat keys (reading R24; fixed=True: the fixed-length comparison coder).
    Returns (lossy tables, base[n], bits[n], exact[n])."""
    c = np.ascontiguousarray(cards, dtype=np.int64)
    n = len(c)
    base = np.zeros(n, dtype=np.uint64)
    bits = np.zeros(n, dtype=np.int32)
    ex = np.zeros(n, dtype=np.int32)
    f = lib().or_encode_fixed if fixed else lib().or_encode_short
    lossy = f(n, c.ctypes.data, key_bits, base.ctypes.data, bits.ctypes.data, ex.ctypes.data)
    return lossy, base, bits, ex


def short_id(t: int, i: int, bits: int, exact: int) -> int:
    return int(lib().or_short_id(t, i, bits, exact))


def self_identify(scan, tid: int):
    """(phi, local) for fused-kernel thread tid."""
    s = np.ascontiguousarray(scan, dtype=np.int64)
    phi = ctypes.c_int32()
    loc = ctypes.c_int64()
    lib().or_self_identify(len(s) - 1, s.ctypes.data, tid, ctypes.byref(phi), ctypes.byref(loc))
    return phi.value, loc.value


def set_hash(fk: int, seed: int) -> int:
    return int(lib().or_set_hash(fk, seed))


def _ptr_array(arrs):
    return (ctypes.c_void_p * len(arrs))(*[a.ctypes.data for a in arrs])


class Oracle:
    """CPU reference cache.  ``tables`` are float32 [c_t, d_t] arrays (kept alive here)."""

    def __init__(self, cards, dims, tables, cache_bytes: int, mode: int = MODE_GLOBAL, admit_p: float = 1.0,
                 admit_seed: int = 0, hash_seed: int = 0, ways: int = 32, set_bytes: int = 8192):
        self.n = len(cards)
        self.cards = np.ascontiguousarray(cards, dtype=np.int64)
        self.dims = np.ascontiguousarray(dims, dtype=np.int32)
        self.tables = [np.ascontiguousarray(t, dtype=np.float32) for t in tables]
        for t, (c, d) in zip(self.tables, zip(cards, dims)):
            assert t.shape == (c, d)
        self._tp = _ptr_array(self.tables)
        if mode == MODE_SETBYTES:
            self.h = lib().or_create_setbytes(self.n, self.cards.ctypes.data, self.dims.ctypes.data, self._tp,
                                              cache_bytes, ways, set_bytes, admit_p, admit_seed, hash_seed)
        else:
            self.h = lib().or_create(self.n, self.cards.ctypes.data, self.dims.ctypes.data, self._tp, cache_bytes,
                                     mode, admit_p, admit_seed, hash_seed)
        if not self.h:
            raise ValueError("or_create rejected the configuration")

    def __del__(self):
        try:
            if getattr(self, "h", None) and _lib is not None:
                _lib.or_destroy(self.h)
                self.h = None
        except Exception:  # interpreter shutdown
            pass

    def out_size(self, lens) -> int:
        return int(sum(int(l) * int(d) for l, d in zip(lens, self.dims)))

    def query(self, ids, out: np.ndarray | None = None) -> np.ndarray:
        ids = [np.ascontiguousarray(x, dtype=np.int64) for x in ids]
        lens = np.array([x.size for x in ids], dtype=np.int64)
        if out is None:
            out = np.empty(self.out_size(lens), dtype=np.float32)
        lib().or_query(self.h, _ptr_array(ids), lens.ctypes.data, out.ctypes.data)
        return out

    def query_pooled(self, ids, offsets, out: np.ndarray | None = None) -> np.ndarray:
        ids = [np.ascontiguousarray(x, dtype=np.int64) for x in ids]
        offsets = [np.ascontiguousarray(x, dtype=np.int64) for x in offsets]
        bags = np.array([o.size - 1 for o in offsets], dtype=np.int64)
        if out is None:
            out = np.empty(self.out_size(bags), dtype=np.float32)
        lib().or_query_pooled(self.h, _ptr_array(ids), _ptr_array(offsets), bags.ctypes.data, out.ctypes.data)
        return out

    def set_key_bits(self, key_bits: int) -> int:
        """Short flat keys (reading R24), before the first query; returns the lossy table count."""
        r = lib().or_set_key_bits(self.h, int(key_bits))
        if r < 0:
            raise ValueError("or_set_key_bits rejected the key width")
        return r

    def set_watermarks(self, hi_bytes: int, lo_bytes: int):
        """Full-scan eviction after each batch (reading R23): if cached row
        bytes > hi_bytes, evict whole age classes of untouched entries, oldest first,
        until <= lo_bytes."""
        if lib().or_set_watermarks(self.h, int(hi_bytes), int(lo_bytes)) != 0:
            raise ValueError("lo_bytes > hi_bytes")

    def scans(self) -> int:
        return int(lib().or_scans(self.h))

    def stats(self) -> dict:
        s = _Stats()
        lib().or_stats(self.h, ctypes.byref(s))
        return {f: int(getattr(s, f)) for f in STAT_FIELDS}

    def cached_keys(self):
        cap = 1 << 16
        while True:
            t = np.empty(cap, dtype=np.int32)
            i = np.empty(cap, dtype=np.int64)
            k = lib().or_cached_keys(self.h, t.ctypes.data, i.ctypes.data, cap)
            if k <= cap:
                return list(zip(t[:k].tolist(), i[:k].tolist()))
            cap = int(k)
