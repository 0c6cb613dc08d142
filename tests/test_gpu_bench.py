"""bench.py on the GPU: the N = 1 line carries the contract's keys (roofline with D7
bytes, e2e, cpu_baseline, clocks, parity_sample, d9), and the N > 1 code path -- the
torchrun self-relaunch, per-rank shard pipelines, the IPC-fused gather + merge, the
max-over-ranks timing, e2e at N ranks -- runs end to end with two ranks sharing cuda:0
(gloo control plane; NCCL needs one GPU per rank) and reports the whole MEM set."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(args, env_extra=None, timeout=900):
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    env.update(env_extra or {})
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-3000:]
    return json.loads(lines[0])


def test_bench_single_gpu_line():
    d = _bench(["--config", "c2", "--steps", "5", "--warmup", "3"])
    assert d["n_gpus"] == 1 and d["config"]["mems"] == 89872
    for k in ("roofline", "e2e", "cpu_baseline", "clocks", "parity_sample", "d9", "gpu_launches"):
        assert k in d, k
    assert d["roofline"]["frac"] > 0 and d["roofline"]["bytes_model"].startswith("SURVEY")
    assert d["parity_sample"]["equal"]
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["gpu_launches"] > 0


def test_bench_two_ranks_path():
    d = _bench(["--gpus", "2", "--config", "c2", "--steps", "5", "--warmup", "3", "--no-cpu-baseline", "--no-d9"],
               {"GM_BENCH_BACKEND": "gloo", "GM_BENCH_SAME_DEVICE": "1"})
    assert d["n_gpus"] == 2 and d["config"]["mems"] == 89872
    assert d["value"] > 0 and "e2e" in d and d["e2e"]["h2d_bytes_per_step"] == 2 * (d["config"]["R_bp"] +
                                                                                   d["config"]["Q_bp"])
