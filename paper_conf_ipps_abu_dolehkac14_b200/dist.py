"""One process per GPU: query-sharded MEM extraction with a gather + merge on rank 0.

Partition: rank g owns the MEMs whose query start q lies in
[a_g, b_g) = [g*|Q|//G, (g+1)*|Q|//G). Every rank packs R and Q itself and builds
the (deterministic) index of R locally -- recomputing it is cheaper than
broadcasting the index -- then finds the MEMs of its own range (the library scans
query positions up to b_g + step - 2 and keeps only starts in [a_g, b_g), so the
shards are disjoint and their union is the whole MEM set). The only exchange is the
final gather to rank 0 and its merge (K9, gpumem_merge_sorted), which replaces the
paper's host merge-sort of out-tile triplets (§III-C2).

Two gathers:
 * ShardedPipeline (what bench.py times): every rank's result stays in its own HBM,
   in an IPC-exportable pipeline arena. Rank 0 maps the peers' arenas once
   (cudaIpcOpenMemHandle over NVLink/NVSwitch) and its merge kernel reads the peers'
   sorted runs directly -- gather and merge are one kernel, each triple crossing
   NVLink once. Per step the process group carries only 24 bytes per rank (count,
   "result is in the exported buffer", capture generation) and one barrier that
   keeps the peers from overwriting their results before rank 0 has merged them.
   A rank whose graph overflowed (result recomputed elsewhere) sends its triples
   point-to-point instead.
 * gather_to_root (direct calls, find_mems_sharded): count all_gather + point-to-point
   sends of each rank's triples to rank 0 (NCCL send/recv on the GPU box).
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_range(n_q: int, rank: int, world: int):
    """Contiguous equal split of the query start positions."""
    return (n_q * rank) // world, (n_q * (rank + 1)) // world


def _ctrl_device(group=None):
    """Device of the small control tensors: the process group's (NCCL moves device
    tensors, gloo -- the CPU tests -- host tensors)."""
    return torch.device("cuda", torch.cuda.current_device()) if dist.get_backend(group) == "nccl" \
        else torch.device("cpu")


def gather_to_root(local: torch.Tensor, group=None):
    """Gather variable-length (N_g, 3) int32 tensors to rank 0 (all_gather of the counts,
    then point-to-point sends). Returns the list of per-rank tensors on rank 0 (rank
    order) and None elsewhere. `local` lives where the group's backend moves data
    (CUDA tensors for NCCL)."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
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


def find_mems_sharded(R_dev: torch.Tensor, Q_dev: torch.Tensor, min_len: int, seed_len: int, group=None,
                      gather=gather_to_root):
    """Whole multi-GPU step on this rank with direct calls: pack, index, find own shard,
    gather, merge on rank 0. Returns (merged Mems on rank 0 / None elsewhere, the
    local Mems, kept alive by the caller)."""
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
    runs = gather(local.view_u32().view(torch.int32), group)
    if rank == 0:
        return gm.merge_sorted(runs), local
    return None, local


class ShardedPipeline:
    """This rank's share of the whole step as a CUDA-graph pipeline (gpumem_pipeline_*):
    pack, index, find over the rank's MEM-start range [a_g, b_g) and the output sort in
    one graph launch; `finish` checks the result and, for world > 1, runs the fused
    gather + merge on rank 0 (module docstring)."""

    def __init__(self, n_r: int, n_q: int, min_len: int, seed_len: int, group=None):
        from . import gpumem as gm
        self.gm = gm
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.q_range = shard_range(n_q, self.rank, self.world)
        self.pl = gm.Pipeline(n_r, n_q, seed_len, min_len, self.q_range)
        if self.world > 1:
            self.pl.set_exportable(True)
        self.merged = None
        self.peer_gen = [None] * self.world   # capture generation of each peer's mapping
        self.peer_ptr = [None] * self.world   # rank 0: device address of each peer's result
        self.peer_base = [None] * self.world
        self.p2p_ranks = 0                    # ranks that sent point-to-point in the last step

    def run(self, R_dev: torch.Tensor, Q_dev: torch.Tensor):
        """Async: one graph launch on the current stream's pipeline."""
        if self.merged is not None:
            self.merged.free()
            self.merged = None
        self.pl.run(R_dev, Q_dev)

    def run_host(self, R_host, Q_host):
        """The same from (pinned) host memory: the copies overlap the R half of the graph."""
        if self.merged is not None:
            self.merged.free()
            self.merged = None
        self.pl.run_host(R_host, Q_host)

    def _remap(self):
        """(Re)exchange the IPC handles of every rank whose capture generation changed
        (first step, or a recapture on new input pointers)."""
        handle, off, gen = self.pl.export()
        objs = [None] * self.world
        dist.all_gather_object(objs, (handle, off, gen), group=self.group)
        for g in range(1, self.world):
            if self.rank == 0 and self.peer_base[g] is not None:
                self.gm.ipc_close(self.peer_base[g])
                self.peer_base[g] = self.peer_ptr[g] = None
            h, o, gg = objs[g]
            if self.rank == 0:
                self.peer_base[g] = self.gm.ipc_open(h)
                self.peer_ptr[g] = self.peer_base[g] + o
            self.peer_gen[g] = gg
        self.peer_gen[0] = gen

    def finish(self):
        """Synchronise, check (alphabet, capacity fallback); for world > 1 gather + merge
        on rank 0. Returns the number of MEMs on rank 0 (this rank's count when
        world == 1), None on other ranks."""
        n = self.pl.result()
        if self.world == 1:
            return n
        exported = self.pl.stats()["attempts"] == 1  # the result is the graph's, in the arena
        gen = self.pl.export(handle=False)[2]
        dev = _ctrl_device(self.group)
        meta = torch.tensor([n, int(exported), gen], dtype=torch.int64, device=dev)
        metas = [torch.empty_like(meta) for _ in range(self.world)]
        dist.all_gather(metas, meta, group=self.group)
        metas = torch.stack(metas).tolist()
        if any(metas[g][2] != self.peer_gen[g] for g in range(self.world)):
            self._remap()
        p2p = [g for g in range(1, self.world) if not metas[g][1] and metas[g][0]]
        self.p2p_ranks = len(p2p)
        out = None
        if self.rank == 0:
            ptrs, counts, keep = [], [], []
            ptrs.append(self.pl._ptr)
            counts.append(n)
            for g in range(1, self.world):
                cnt = metas[g][0]
                if g in p2p:  # overflow fallback on that rank: its triples come point-to-point
                    buf = torch.empty((cnt, 3), dtype=torch.int32, device="cuda")
                    dist.recv(buf, src=g, group=self.group)
                    keep.append(buf)
                    ptrs.append(buf.data_ptr())
                else:
                    ptrs.append(self.peer_ptr[g])
                counts.append(cnt)
            self.merged = self.gm.merge_runs(ptrs, counts)
            torch.cuda.current_stream().synchronize()  # the peers' runs have been read
            out = len(self.merged)
        elif self.rank in p2p:
            dist.send(self.pl.view_u32().view(torch.int32).contiguous(), dst=0, group=self.group)
        # peers keep their results untouched until rank 0 has merged them
        dist.barrier(group=self.group)
        return out

    def free(self):
        if self.merged is not None:
            self.merged.free()
            self.merged = None
        for g in range(1, self.world):
            if self.peer_base[g] is not None:
                self.gm.ipc_close(self.peer_base[g])
                self.peer_base[g] = None
        if self.world > 1 and dist.is_initialized():
            dist.barrier(group=self.group)  # no rank frees an arena a peer still maps
        self.pl.free()
