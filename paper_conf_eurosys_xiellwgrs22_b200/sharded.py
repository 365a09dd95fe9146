"""Key-sharded flat cache across the ranks of a torch.distributed group.

Every step of the lookup path runs in libfleche.so (route, owner query, restore); this
module is the collective plumbing between them: three all-to-alls per batch over NCCL
(NVLink 5 / NVSwitch on an HGX B200 node) — per-owner key counts, the keys, and the rows
(+ per-key hit flags) back — plus one 2 x G x 8-byte device->host read of the counts to
size the variable all-to-alls.

Owner of a flat key: (fmix32(fk ^ seed ^ 0x85EBCA77) * G) >> 32 (include/fleche.h), so
rank r caches only its share of the key space and the per-GPU cache budgets aggregate.

p2p=True (the fused exchange): neither keys nor rows travel in a
collective.  Every rank maps every owner's receive and answer buffers (CUDA IPC, peer
access over NVLink).  The route's pack kernel stores each unique key straight into its
owner's slot for this rank (fleche_route_p2p); a G x G counts all-gather (stream-ordered
behind every rank's route, so it is also the "keys are in place" barrier) sizes the
owner query over its per-source segments (fleche_query_keys_seg_dev, reading the G x G
counts matrix in device memory with a grid-strided launch) and gives each rank its
offset in every owner's answer order, computed by the restore kernel on the device;
after a one-element all-reduce (a stream-ordered barrier: every owner's answers are
written; answers are double-buffered by batch parity) each requester's restore kernel
(fleche_restore_p2p_dev) reads its rows in place from the owners' HBM.  With NCCL no step
reads anything back to the host; with the gloo backend (CPU / one-GPU tests) the small
collectives go through host copies.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

DEFAULT_OWNER_SEED = 0x2545F491


class ShardedCache:
    """Wraps a FlatCache (this rank's shard) for key-sharded queries.

    ``cache`` must expose route / query_keys / restore with the C-ABI contract; the
    device buffers are sized once from ``cache.max_lookups`` (no allocation per batch),
    which bounds both this rank's batch and the keys it may receive as an owner: create
    the FlatCache with max_lookups >= world x the per-rank batch."""

    def __init__(self, cache, row_floats: int, group=None, owner_seed: int = DEFAULT_OWNER_SEED, device=None,
                 p2p: bool = False):
        self.cache = cache
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.seed = owner_seed
        self.d = int(row_floats)
        dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        n = int(cache.max_lookups)
        W = self.world
        self.send_keys = torch.empty(n, dtype=torch.int32, device=dev)
        self.recv_keys = torch.empty(n, dtype=torch.int32, device=dev)
        self.send_counts = torch.zeros(W, dtype=torch.int64, device=dev)
        self.recv_counts = torch.zeros(W, dtype=torch.int64, device=dev)
        self.rows = torch.empty((n, self.d), dtype=torch.float32, device=dev)
        self.flags = torch.empty(n, dtype=torch.uint8, device=dev)
        self.rows_back = torch.empty((n, self.d), dtype=torch.float32, device=dev)
        self.flags_back = torch.empty(n, dtype=torch.uint8, device=dev)
        self.last_exchange = None
        self.p2p = bool(p2p)
        self.batch = 0
        self.cpu_coll = dist.get_backend(group) == "gloo"
        if self.p2p:
            self._setup_p2p(n)

    def _setup_p2p(self, n):
        from . import binding as B
        W, me = self.world, self.rank
        # [parity] owner answer buffers, exported to every rank
        self.own_rows = [B.ipc_alloc(n * self.d * 4) for _ in range(2)]
        self.own_flags = [B.ipc_alloc(max(n, 16)) for _ in range(2)]
        self.own_recv = B.ipc_alloc(W * n * 4)  # [source][n] keys routed to this owner
        mine = [B.ipc_handle(p) for p in self.own_rows + self.own_flags + [self.own_recv]]
        allh = [None] * W
        dist.all_gather_object(allh, mine, group=self.group)
        self.peer_rows, self.peer_flags, self._opened = [[], []], [[], []], []
        for o in range(W):
            for par in range(2):
                if o == me:
                    r, f = self.own_rows[par], self.own_flags[par]
                else:
                    r, f = B.ipc_open(allh[o][par]), B.ipc_open(allh[o][2 + par])
                    self._opened += [r, f]
                self.peer_rows[par].append(r)
                self.peer_flags[par].append(f)
        # this rank's slot in every owner's receive buffer, and this owner's per-source segments
        self.peer_slots = []
        for o in range(W):
            base = self.own_recv if o == me else B.ipc_open(allh[o][4])
            if o != me:
                self._opened.append(base)
            self.peer_slots.append(base + me * n * 4)
        self.own_segs = [self.own_recv + src * n * 4 for src in range(W)]
        self.bar = torch.zeros(1, dtype=torch.int32, device="cpu" if self.cpu_coll else self.send_counts.device)
        self.dC = torch.zeros(W * W, dtype=torch.int64, device=self.send_counts.device)  # routed counts [src][owner]

    def close(self):
        if getattr(self, "p2p", False) and getattr(self, "own_rows", None):
            from . import binding as B
            torch.cuda.synchronize()
            dist.barrier(group=self.group)  # no peer reads our buffers any more
            for p in self._opened:
                B.ipc_close(p)
            for p in self.own_rows + self.own_flags + [self.own_recv]:
                B.ipc_free(p)
            self.own_rows = None

    def _all_gather_counts(self):
        if self.cpu_coll:
            torch.cuda.synchronize()
            mine = self.send_counts.cpu()
            allc = [torch.zeros_like(mine) for _ in range(self.world)]
            dist.all_gather(allc, mine, group=self.group)
            return torch.stack(allc)
        allc = [torch.zeros_like(self.send_counts) for _ in range(self.world)]
        dist.all_gather(allc, self.send_counts, group=self.group)
        return torch.stack(allc).cpu()

    def _keys_all_to_all(self, nr, ns, R, S):
        if self.cpu_coll:
            torch.cuda.synchronize()
            rk = torch.empty(nr, dtype=torch.int32)
            dist.all_to_all_single(rk, self.send_keys[:ns].cpu(), R, S, group=self.group)
            self.recv_keys[:nr].copy_(rk)
        else:
            dist.all_to_all_single(self.recv_keys[:nr], self.send_keys[:ns], R, S, group=self.group)

    def _barrier(self):
        if self.cpu_coll:
            torch.cuda.synchronize()
        dist.all_reduce(self.bar, group=self.group)

    def query_p2p(self, ids, out, lengths=None):
        """One batch through the fused exchange (see the module docstring).  With NCCL the
        host never waits: the counts matrix is all-gathered into device memory and read there
        by the owner query and the restore (fleche_*_dev); gloo (CPU tests) gathers through
        host memory."""
        c, W, me = self.cache, self.world, self.rank
        par = self.batch & 1
        self.batch += 1
        # keys: the route's pack kernel stores them straight into the owners' slots (peer HBM)
        c.route_p2p(ids, W, self.seed, self.peer_slots, self.send_counts, lengths=lengths)
        # counts: all-gather (stream-ordered behind every rank's route: the keys are in place)
        if self.cpu_coll:
            self.dC.copy_(self._all_gather_counts().reshape(-1))
        else:
            dist.all_gather_into_tensor(self.dC, self.send_counts, group=self.group)  # C[src][owner], device
        c.query_keys_seg_dev(self.own_segs, self.dC, me, self.own_rows[par], self.own_flags[par])
        self._barrier()  # every owner's answers of this batch are in place
        # rows: each requester reads its answers in place from the owners' HBM
        c.restore_p2p_dev(self.peer_rows[par], self.peer_flags[par], self.dC, me, out)
        self.last_exchange = None  # the per-batch byte counts stay on the device (no host read)
        return self.last_exchange

    def query(self, ids, out, lengths=None):
        """One batch: this rank's per-table ID lists -> `out` (layout of fleche_query)."""
        if self.p2p:
            return self.query_p2p(ids, out, lengths=lengths)
        c = self.cache
        c.route(ids, self.world, self.seed, self.send_keys, self.send_counts, lengths=lengths)
        dist.all_to_all_single(self.recv_counts, self.send_counts, group=self.group)
        cnt = torch.stack([self.send_counts, self.recv_counts]).cpu()  # sizes the variable all-to-alls
        S = [int(x) for x in cnt[0]]
        R = [int(x) for x in cnt[1]]
        ns, nr = sum(S), sum(R)
        dist.all_to_all_single(self.recv_keys[:nr], self.send_keys[:ns], R, S, group=self.group)
        c.query_keys(self.recv_keys, nr, self.rows, self.flags)
        dist.all_to_all_single(self.rows_back[:ns], self.rows[:nr], S, R, group=self.group)
        dist.all_to_all_single(self.flags_back[:ns], self.flags[:nr], S, R, group=self.group)
        c.restore(self.rows_back, self.flags_back, out)
        self.last_exchange = {"sent_keys": ns, "recv_keys": nr, "nvlink_bytes_out": ns * 4 + nr * (4 * self.d + 1)}
        return self.last_exchange
