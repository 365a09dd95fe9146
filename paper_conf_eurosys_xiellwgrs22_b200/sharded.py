"""Key-sharded flat cache across the ranks of a torch.distributed group.

Every step of the lookup path runs in libfleche.so (route, owner query, restore); this
module is the collective plumbing between them: three all-to-alls per batch over NCCL
(NVLink 5 / NVSwitch on an HGX B200 node) — per-owner key counts, the keys, and the rows
(+ per-key hit flags) back — plus one 2 x G x 8-byte device->host read of the counts to
size the variable all-to-alls.

Owner of a flat key: (fmix32(fk ^ seed ^ 0x85EBCA77) * G) >> 32 (include/fleche.h), so
rank r caches only its share of the key space and the per-GPU cache budgets aggregate.
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

    def __init__(self, cache, row_floats: int, group=None, owner_seed: int = DEFAULT_OWNER_SEED, device=None):
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

    def query(self, ids, out, lengths=None):
        """One batch: this rank's per-table ID lists -> `out` (layout of fleche_query)."""
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
