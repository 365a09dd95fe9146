"""Host tier shared by the processes of one node (replicated multi-GPU runs).

Local rank 0 creates and fills a file in /dev/shm; the other local ranks map the same
pages after a barrier, so an 8-GPU node holds one copy of the tables instead of eight
(each process still page-locks and maps the pages for its own GPU in fleche_create).
Plumbing only: the values come from ``workload.gen``.
"""
from __future__ import annotations

import mmap
import os

import numpy as np

from . import gen


def _views(buf, cards, dims):
    views, off = [], 0
    for c, d in zip(cards, dims):
        n = int(c) * int(d)
        views.append(buf[off:off + n].reshape(int(c), int(d)))
        off += n
    return views


def shared_tables(name: str, cards, dims, mode: int, local_rank: int, barrier, nthreads: int = 0):
    """(buffer, per-table views, cleanup) of the tables in /dev/shm/<name>."""
    path = os.path.join("/dev/shm", name)
    total = sum(int(c) * int(d) for c, d in zip(cards, dims))
    nbytes = total * 4
    if local_rank == 0:
        fd = os.open(path, os.O_CREAT | os.O_RDWR | os.O_TRUNC, 0o600)
        os.ftruncate(fd, nbytes)
        mm = mmap.mmap(fd, nbytes, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
        os.close(fd)
        buf = np.frombuffer(mm, dtype=np.float32, count=total)
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
        if local_rank == 0:
            try:
                os.unlink(path)
            except FileNotFoundError:
                pass

    return buf, _views(buf, cards, dims), cleanup
