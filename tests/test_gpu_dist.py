"""Multi-process path on the GPU: two ranks share cuda:0 (NCCL refuses two ranks on
one device, so the exchange runs over gloo with host staging); each rank packs,
indexes and finds its query shard with the CUDA path, rank 0 merges the gathered
runs with gpumem_merge_sorted. The merged set must equal the oracle's."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, cfg, scale, q, mode="direct"):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        from paper_conf_ipps_abu_dolehkac14_b200 import synth
        from paper_conf_ipps_abu_dolehkac14_b200.dist import find_mems_sharded
        P = synth.make_pair(cfg, scale=scale)
        Rt, Qt = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
        if mode == "pipeline":  # the launch configuration bench.py times at N > 1
            from paper_conf_ipps_abu_dolehkac14_b200.dist import ShardedPipeline
            sp = ShardedPipeline(len(P.R), len(P.Q), P.L, P.ls)
            for _ in range(2):
                sp.run(Rt, Qt)
                n = sp.finish()
            merged, n_local = sp.merged, len(sp.pl)
        else:
            merged, local = find_mems_sharded(Rt, Qt, P.L, P.ls)
            n_local = len(local)
        if rank == 0:
            import oracle
            got = merged.numpy()
            want = oracle.mems(P.R, P.Q, P.L, P.ls)
            if mode == "pipeline":
                assert n == len(want)
            q.put(("ok", bool(np.array_equal(got, want)), len(want), n_local))
    except Exception as e:  # pragma: no cover
        q.put(("err", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["direct", "pipeline"])
@pytest.mark.parametrize("world,cfg,scale", [(2, "c1", 1.0), (3, "c2", 0.2)])
def test_sharded_find_gather_merge(world, cfg, scale, mode):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cfg, scale, q, mode)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(300)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    res = q.get(timeout=10)
    assert res[0] == "ok" and res[1], res
    assert 0 < res[3] < res[2]  # rank 0 found only its shard
