"""One process per GPU: query-sharded MEM extraction with a gather to rank 0.

Partition: rank g owns the MEMs whose query start q lies in
[a_g, b_g) = [g*|Q|//G, (g+1)*|Q|//G). Every rank packs R and Q itself and builds
the (deterministic) index of R locally -- recomputing it is cheaper than
broadcasting the 4^ls-entry table -- then runs gpumem_find_mems on its own range
(the library scans query positions up to b_g + step - 2 and keeps only starts in
[a_g, b_g), so the shards are disjoint and their union is the whole MEM set).
The only exchange is the final gather: an all_gather of the per-rank counts and
point-to-point sends of each rank's sorted triples to rank 0 (NCCL over NVLink on
the GPU box; gloo in the CPU tests), followed by rank 0's merge kernel
(gpumem_merge_sorted). No collective touches the data path before that.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_range(n_q: int, rank: int, world: int):
    """Contiguous equal split of the query start positions."""
    return (n_q * rank) // world, (n_q * (rank + 1)) // world


def gather_to_root(local: torch.Tensor, group=None):
    """Gather variable-length (N_g, 3) int32 tensors to rank 0.

    Returns the list of per-rank tensors on rank 0 (rank order) and None elsewhere.
    Works with any backend that has all_gather/send/recv (NCCL, gloo)."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    if local.is_cuda and dist.get_backend(group) == "gloo":  # gloo moves host tensors only
        runs = gather_to_root(local.cpu(), group)
        return None if runs is None else [r.to(local.device) for r in runs]
    dev = local.device
    cnt = torch.tensor([local.shape[0]], dtype=torch.int64, device=dev)
    counts = [torch.zeros_like(cnt) for _ in range(world)]
    dist.all_gather(counts, cnt, group=group)
    counts = [int(c.item()) for c in counts]
    if rank == 0:
        runs = [local]
        for g in range(1, world):
            buf = torch.empty((counts[g], 3), dtype=local.dtype, device=dev)
            if counts[g]:
                dist.recv(buf, src=g, group=group)
            runs.append(buf)
        return runs
    if counts[rank]:
        dist.send(local.contiguous(), dst=0, group=group)
    return None


def find_mems_sharded(R_dev: torch.Tensor, Q_dev: torch.Tensor, min_len: int, seed_len: int, group=None):
    """Whole multi-GPU step on this rank: pack, index, find own shard, gather,
    merge on rank 0. Returns the merged gpumem.Mems on rank 0, None elsewhere.
    Also returns the local (unmerged) Mems so callers can keep it alive."""
    from . import gpumem as gm
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    R = gm.pack(R_dev)
    Q = gm.pack(Q_dev)
    idx = gm.index_build(R, seed_len, min_len)
    a, b = shard_range(Q_dev.numel(), rank, world)
    local = gm.find_mems(idx, Q, (a, b))
    if world == 1:
        return local, local
    runs = gather_to_root(local.view_u32().view(torch.int32), group)
    if rank == 0:
        return gm.merge_sorted(runs), local
    return None, local


class ShardedPipeline:
    """This rank's share of the whole step as a CUDA-graph pipeline (gpumem_pipeline_*):
    pack, index, find over the rank's MEM-start range [a_g, b_g) and the output sort in
    one graph launch; `finish` checks the result and, for world > 1, gathers the sorted
    runs to rank 0 and merges them there (the only exchange, as in find_mems_sharded)."""

    def __init__(self, n_r: int, n_q: int, min_len: int, seed_len: int, group=None):
        from . import gpumem as gm
        self.gm = gm
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.q_range = shard_range(n_q, self.rank, self.world)
        self.pl = gm.Pipeline(n_r, n_q, seed_len, min_len, self.q_range)
        self.merged = None

    def run(self, R_dev: torch.Tensor, Q_dev: torch.Tensor):
        """Async: one graph launch on the current stream's pipeline."""
        if self.merged is not None:
            self.merged.free()
            self.merged = None
        self.pl.run(R_dev, Q_dev)

    def finish(self):
        """Synchronise, check (alphabet, capacity fallback), gather + merge for world > 1.
        Returns the number of MEMs on rank 0 (this rank's count when world == 1), None
        on other ranks."""
        n = self.pl.result()
        if self.world == 1:
            return n
        runs = gather_to_root(self.pl.view_u32().view(torch.int32), self.group)
        if self.rank == 0:
            self.merged = self.gm.merge_sorted(runs)
            return len(self.merged)
        return None

    def free(self):
        if self.merged is not None:
            self.merged.free()
        self.pl.free()
