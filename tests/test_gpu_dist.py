"""Multi-process path on the GPU. Two or three ranks share cuda:0 (NCCL refuses two
ranks on one device, so the control plane runs over gloo here): each rank packs,
indexes and finds its query shard with the CUDA path, rank 0 merges. In the
pipeline mode (what bench.py times) rank 0's merge kernel reads the other ranks'
results through CUDA IPC mappings of their pipeline arenas -- the fused gather +
merge of dist.ShardedPipeline, exercised between processes exactly as across GPUs.
The direct mode gathers with host staging (test-only: gloo moves host tensors).
With two or more GPUs, the NCCL test runs one rank per GPU. The merged set must
equal the oracle's."""
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


def _staged_gather(local, group=None):
    """gather_to_root over gloo: host copies in, device copies out (test-only)."""
    from paper_conf_ipps_abu_dolehkac14_b200.dist import gather_to_root
    runs = gather_to_root(local.cpu(), group)
    return None if runs is None else [r.to(local.device) for r in runs]


def _worker(rank, world, port, cfg, scale, q, mode="direct", backend="gloo"):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dev = rank if backend == "nccl" else 0
    torch.cuda.set_device(dev)
    if backend == "nccl":
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", dev))
    else:
        dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_abu_dolehkac14_b200 import synth
        from paper_conf_ipps_abu_dolehkac14_b200.dist import find_mems_sharded
        P = synth.make_pair(cfg, scale=scale)
        Rt, Qt = torch.from_numpy(P.R).cuda(), torch.from_numpy(P.Q).cuda()
        if mode == "pipeline":  # the launch configuration bench.py times at N > 1
            from paper_conf_ipps_abu_dolehkac14_b200.dist import ShardedPipeline
            sp = ShardedPipeline(len(P.R), len(P.Q), P.L, P.ls)
            R2, Q2 = Rt.clone(), Qt.clone()
            for i in range(4):  # new input pointers at step 2: recapture -> re-exported handles
                sp.run(*((Rt, Qt) if i < 2 else (R2, Q2)))
                n = sp.finish()
                if rank == 0:
                    assert n == len(sp.merged)
                assert sp.p2p_ranks == 0  # every peer's run was read through its IPC mapping
            merged, n_local = sp.merged, len(sp.pl)
        else:
            gather = _staged_gather if backend == "gloo" else None
            kw = {"gather": gather} if gather else {}
            merged, local = find_mems_sharded(Rt, Qt, P.L, P.ls, **kw)
            n_local = len(local)
        if rank == 0:
            import oracle
            got = merged.numpy()
            want = oracle.mems(P.R, P.Q, P.L, P.ls)
            if mode == "pipeline":
                assert n == len(want)
            q.put(("ok", bool(np.array_equal(got, want)), len(want), n_local))
        if mode == "pipeline":
            sp.free()
    except Exception as e:  # pragma: no cover
        q.put(("err", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


def _spawn(world, cfg, scale, mode, backend):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cfg, scale, q, mode, backend)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(300)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
    res = q.get(timeout=10)
    assert res[0] == "ok" and res[1], res
    assert 0 < res[3] < res[2]  # rank 0 found only its shard


@pytest.mark.parametrize("mode", ["direct", "pipeline"])
@pytest.mark.parametrize("world,cfg,scale", [(2, "c1", 1.0), (3, "c2", 0.2)])
def test_sharded_find_gather_merge(world, cfg, scale, mode):
    _spawn(world, cfg, scale, mode, "gloo")


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="NCCL needs one GPU per rank (>= 2 GPUs)")
@pytest.mark.parametrize("mode", ["direct", "pipeline"])
def test_sharded_nccl(mode):
    """The NCCL data plane: count all_gather + send/recv (direct), control exchange +
    IPC-fused merge over NVLink (pipeline), one rank per GPU."""
    _spawn(min(torch.cuda.device_count(), 4), "c2", 0.2, mode, "nccl")
