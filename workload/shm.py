"""Host tier shared by the processes of one node (replicated multi-GPU runs).

One copy of the tables per NUMA node: the first local rank whose GPU
sits on a node creates and fills a file in /dev/shm with its pages bound to that node
(mbind), and the other local ranks of that node map the same pages after a barrier.  So
every GPU reads its missed rows from the DRAM of its own socket (no cross-socket traffic
for the zero-copy reads and the host-assist gathers), and an 8-GPU two-socket node holds
two copies of the tables instead of eight.  Each process still page-locks and maps the
pages for its own GPU in fleche_create.  Plumbing only: the values come from
``workload.gen``.
"""
from __future__ import annotations

import ctypes
import mmap
import os

import numpy as np

from . import gen

_MPOL_BIND = 2
_SYS_MBIND = 237  # x86_64


def _views(buf, cards, dims):
    views, off = [], 0
    for c, d in zip(cards, dims):
        n = int(c) * int(d)
        views.append(buf[off:off + n].reshape(int(c), int(d)))
        off += n
    return views


def gpu_numa_node(device_index: int) -> int:
    """NUMA node of a CUDA device's PCI function (sysfs), 0 when unknown or not NUMA."""
    try:
        import torch
        p = torch.cuda.get_device_properties(device_index)
        bus = "%04x:%02x:%02x.0" % (int(getattr(p, "pci_domain_id", 0)), int(p.pci_bus_id), int(p.pci_device_id))
        with open(f"/sys/bus/pci/devices/{bus}/numa_node") as f:
            return max(0, int(f.read().strip()))
    except Exception:
        return 0


def numa_nodes() -> int:
    try:
        return len([d for d in os.listdir("/sys/devices/system/node") if d.startswith("node") and d[4:].isdigit()])
    except OSError:
        return 1


def bind_to_node(addr: int, nbytes: int, node: int) -> bool:
    """mbind(MPOL_BIND) a mapping to one NUMA node before its pages are first touched;
    False when the kernel refuses (no NUMA support, container policy)."""
    if numa_nodes() <= 1:
        return False
    mask = (ctypes.c_ulong * 16)()
    mask[node // 64] = 1 << (node % 64)
    libc = ctypes.CDLL(None, use_errno=True)
    r = libc.syscall(_SYS_MBIND, ctypes.c_void_p(addr), ctypes.c_ulong(nbytes), _MPOL_BIND, mask,
                     ctypes.c_ulong(16 * 64), 0)
    return r == 0


def creator_ranks(local_rank: int, node: int, all_gather_object) -> bool:
    """True for the lowest local rank of each NUMA node (it creates that node's copy)."""
    nodes = all_gather_object((local_rank, node))
    return min(r for r, n in nodes if n == node) == local_rank


def shared_tables(name: str, cards, dims, mode: int, local_rank: int, barrier, nthreads: int = 0,
                  node: int = 0, creator: bool | None = None):
    """(buffer, per-table views, cleanup) of the tables in /dev/shm/<name>_n<node>.

    creator: this rank creates and fills the node's copy (default: local rank 0, i.e. one
    copy per host); every rank calls ``barrier`` exactly once."""
    path = os.path.join("/dev/shm", f"{name}_n{node}")
    total = sum(int(c) * int(d) for c, d in zip(cards, dims))
    nbytes = total * 4
    if creator is None:
        creator = local_rank == 0
    if creator:
        fd = os.open(path, os.O_CREAT | os.O_RDWR | os.O_TRUNC, 0o600)
        os.ftruncate(fd, nbytes)
        mm = mmap.mmap(fd, nbytes, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
        os.close(fd)
        buf = np.frombuffer(mm, dtype=np.float32, count=total)
        bind_to_node(buf.ctypes.data, nbytes, node)  # before the first touch: pages on this socket
        for t, v in enumerate(_views(buf, cards, dims)):
            gen.fill_table(v, t, mode, 0, nthreads)
        barrier()
    else:
        barrier()
        fd = os.open(path, os.O_RDWR)
        mm = mmap.mmap(fd, nbytes, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
        os.close(fd)
        buf = np.frombuffer(mm, dtype=np.float32, count=total)

    def cleanup():
        if creator:
            try:
                os.unlink(path)
            except FileNotFoundError:
                pass

    return buf, _views(buf, cards, dims), cleanup
