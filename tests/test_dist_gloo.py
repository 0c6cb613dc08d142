"""Host-side logic of the multi-GPU path on CPU: world_size 2 with the gloo backend.

The GPU engine is stood in for by the oracle restricted to each rank's query
range (the same contract gpumem_find_mems has: MEMs whose start q is in
[a_g, b_g)); the sharding rule, the count all_gather, the point-to-point gather
to rank 0 and the merge are the product's (paper_conf_ipps_abu_dolehkac14_b200.dist)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_abu_dolehkac14_b200 import synth
from paper_conf_ipps_abu_dolehkac14_b200.dist import gather_to_root, shard_range


def test_shard_range_partitions():
    for n in (0, 1, 7, 1000, 150_000_001):
        for world in (1, 2, 3, 8):
            cuts = [shard_range(n, g, world) for g in range(world)]
            assert cuts[0][0] == 0 and cuts[-1][1] == n
            assert all(cuts[i][1] == cuts[i + 1][0] for i in range(world - 1))
            assert all(b - a in ((n // world), (n // world) + 1) for a, b in cuts)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        P = synth.make_pair("c1", scale=0.5)
        a, b = shard_range(len(P.Q), rank, world)
        local = oracle.mems(P.R, P.Q, P.L, P.ls, 0, a, b).astype(np.int32)
        runs = gather_to_root(torch.from_numpy(local))
        if rank == 0:
            cat = np.concatenate([r.numpy() for r in runs]).astype(np.uint32)
            cat = cat[np.lexsort((cat[:, 1], cat[:, 0]))]
            whole = oracle.mems(P.R, P.Q, P.L, P.ls)
            q.put(("ok", bool(np.array_equal(cat, whole)), len(whole), [len(r) for r in runs]))
        else:
            assert runs is None
    except Exception as e:  # pragma: no cover
        q.put(("err", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gather_merge_equals_whole(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    res = q.get(timeout=5)
    assert res[0] == "ok" and res[1], res
    assert res[2] > 100 and sum(res[3]) == res[2]
