"""Seeded synthetic inputs shared by the oracle and the CUDA path.

Thin ctypes wrapper over ``workload/libflgen.so`` (built from ``workload/gen.c``).
Holds none of the method's arithmetic: only table values, power-law IDs and
bag lengths.  Seeds follow SURVEY §8(d-1):

* ``S_base = 0xF1EC4E2022``; ``S_val = sm64(S_base ^ 1)``; ``S_perm = sm64(S_base ^ 3)``;
  ``S_admit = sm64(S_base ^ 5)``; ``S_bag = sm64(S_base ^ 7)``; ``S_id(k) = sm64(S_base ^ (0x10 + k))``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libflgen.so")
_lib = None

S_BASE = 0xF1EC4E2022


def _build():
    subprocess.check_call(["make", "-s", "-C", os.path.dirname(_HERE), "workload/libflgen.so"])


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(
            os.path.join(_HERE, "gen.c")
        ):
            _build()
        L = ctypes.CDLL(_LIB_PATH)
        u64, i64, i32, f64 = ctypes.c_uint64, ctypes.c_int64, ctypes.c_int32, ctypes.c_double
        vp = ctypes.c_void_p
        L.flg_splitmix64.restype = u64
        L.flg_splitmix64.argtypes = [u64]
        L.flg_u01.restype = f64
        L.flg_u01.argtypes = [u64]
        L.flg_value.restype = ctypes.c_float
        L.flg_value.argtypes = [u64, i64, i64, i64, ctypes.c_int]
        L.flg_fill_table.restype = None
        L.flg_fill_table.argtypes = [u64, i64, i64, i64, i32, i64, ctypes.c_int, vp, ctypes.c_int]
        L.flg_zipf_rank.restype = i64
        L.flg_zipf_rank.argtypes = [f64, i64, u64]
        L.flg_perm.restype = i64
        L.flg_perm.argtypes = [u64, i64, i64, i64]
        L.flg_gen_ids.restype = None
        L.flg_gen_ids.argtypes = [u64, u64, i64, i64, i64, f64, i64, i64, i32, vp, ctypes.c_int]
        L.flg_gen_bag_offsets.restype = i64
        L.flg_gen_bag_offsets.argtypes = [u64, i64, i64, i32, i64, i64, vp]
        L.flg_gen_bag_ids.restype = None
        L.flg_gen_bag_ids.argtypes = [u64, u64, i64, i64, i64, f64, i64, i64, vp, i32, vp, ctypes.c_int]
        _lib = L
    return _lib


def splitmix64(x: int) -> int:
    return int(lib().flg_splitmix64(x & 0xFFFFFFFFFFFFFFFF))


def u01(x: int) -> float:
    return float(lib().flg_u01(x & 0xFFFFFFFFFFFFFFFF))


def seeds():
    b = S_BASE
    return {
        "val": splitmix64(b ^ 1),
        "perm": splitmix64(b ^ 3),
        "admit": splitmix64(b ^ 5),
        "bag": splitmix64(b ^ 7),
    }


def id_seed(cfg_index: int) -> int:
    return splitmix64(S_BASE ^ (0x10 + cfg_index))


def value(t: int, row: int, col: int, mode: int = 0) -> float:
    return float(lib().flg_value(seeds()["val"], t, row, col, mode))


def fill_table(dst: np.ndarray, t: int, mode: int = 0, row0: int = 0, nthreads: int = 0):
    """Fill a C-contiguous float32 [rows, d] view with E_t[row0 + r][c]."""
    assert dst.dtype == np.float32 and dst.ndim == 2 and dst.flags["C_CONTIGUOUS"]
    rows, d = dst.shape
    lib().flg_fill_table(seeds()["val"], t, row0, rows, d, d, mode, dst.ctypes.data, nthreads)


def alloc_host_f32(n: int) -> np.ndarray:
    """A float32 host buffer of n elements backed by transparent huge pages where the kernel
    allows it (anonymous mmap + MADV_HUGEPAGE; THP "madvise" mode).  A host tier of several
    GiB in 4 KiB pages makes every scattered row read of the host-assist threads a TLB miss
    and page walk; 2 MiB pages keep their gather near the memory system's rate."""
    import mmap

    nbytes = max(4, 4 * int(n))
    if nbytes < (64 << 20) or os.environ.get("FLECHE_TIER_NO_THP"):  # (A/B: 4 KiB pages)
        return np.empty(int(n), dtype=np.float32)
    mm = mmap.mmap(-1, nbytes, flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS,
                   prot=mmap.PROT_READ | mmap.PROT_WRITE)
    if hasattr(mm, "madvise") and hasattr(mmap, "MADV_HUGEPAGE"):
        try:
            mm.madvise(mmap.MADV_HUGEPAGE)
        except OSError:
            pass
    return np.frombuffer(mm, dtype=np.float32, count=int(n))


def make_tables(cards, dims, mode: int = 0, nthreads: int = 0, buf: np.ndarray | None = None):
    """One contiguous float32 buffer holding every table row-major; returns (buf, [views]).
    `buf` (optional): a caller-provided float32 buffer of at least sum(c_t * d_t) elements
    (e.g. driver-allocated pinned memory) to generate into."""
    sizes = [int(c) * int(d) for c, d in zip(cards, dims)]
    total = sum(sizes)
    if buf is None:
        buf = alloc_host_f32(total)
    assert buf.dtype == np.float32 and buf.flags["C_CONTIGUOUS"] and buf.size >= total
    buf = buf[:total]
    views = []
    off = 0
    for t, (c, d) in enumerate(zip(cards, dims)):
        v = buf[off : off + int(c) * int(d)].reshape(int(c), int(d))
        fill_table(v, t, mode, 0, nthreads)
        views.append(v)
        off += int(c) * int(d)
    return buf, views


def zipf_rank(a: float, n: int, q: int) -> int:
    return int(lib().flg_zipf_rank(a, n, q & 0xFFFFFFFFFFFFFFFF))


def perm(t: int, c: int, rank0: int) -> int:
    return int(lib().flg_perm(seeds()["perm"], t, c, rank0))


def gen_ids(s_id: int, b: int, t: int, c: int, a: float, n: int, j0: int = 0, invalid_ppm: int = 0,
            out: np.ndarray | None = None, nthreads: int = 0) -> np.ndarray:
    if out is None:
        out = np.empty(n, dtype=np.int64)
    assert out.dtype == np.int64 and out.flags["C_CONTIGUOUS"] and out.size >= n
    lib().flg_gen_ids(s_id, seeds()["perm"], b, t, c, a, j0, n, invalid_ppm, out.ctypes.data, nthreads)
    return out


def gen_bag_offsets(b: int, t: int, m: int, bags: int, bag0: int = 0) -> np.ndarray:
    off = np.empty(bags + 1, dtype=np.int64)
    lib().flg_gen_bag_offsets(seeds()["bag"], b, t, m, bag0, bags, off.ctypes.data)
    return off
