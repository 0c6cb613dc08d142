"""The bench.py contract on CPU (no GPU needed for the reference arm, which times the
CPU oracle): one JSON line with the contract's keys; `--gpus N` outside a launcher
re-executes itself under torch.distributed.run with N ranks, rank 0 alone prints, and
n_gpus is the number of ranks that ran."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, timeout=300):
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR",
                                                             "MASTER_PORT")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


@pytest.mark.parametrize("gpus", [1, 2])
def test_reference_arm_line_and_relaunch(gpus):
    d = _run(["--impl", "reference", "--config", "c1", "--steps", "2", "--warmup", "1", "--gpus", str(gpus)])
    assert d["impl"] == "reference" and d["n_gpus"] == gpus
    for k in ("metric", "value", "unit", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["steps"] == 2 and d["warmup"] == 1 and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


def test_gpus_must_match_world_size():
    env = dict(os.environ, WORLD_SIZE="3", RANK="1", LOCAL_RANK="1")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2",
                        "--config", "c1"], capture_output=True, text=True, timeout=120, cwd=ROOT, env=env)
    assert r.returncode != 0 and "WORLD_SIZE=3" in r.stderr


def test_byte_models():
    """bench.py's byte models: the LSD pass count follows the library's digit rule
    (radix.cu pick_digit_bits: 8-bit digits above 16 M keys, else 9-bit when that saves a
    pass), and every stage of both models is positive at C4's sizes (the tiled index stage
    included)."""
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    assert bench.radix_passes(26, 2_840_909) == 3      # C4 index: 9 + 9 + 8
    assert bench.radix_passes(26, 31_249_999) == 4     # C5 L=20 index: 8-bit digits
    assert bench.radix_passes(16, 2_840_909) == 2
    assert bench.radix_passes(56, 13_420_345) == 7     # C5 L=20 output keys
    stats = {"positions": 149_997_216, "occupied": 12_000_000, "hits": 17_300_000, "mems": 811_662}
    impl = bench.impl_bytes(250_000_000, 150_000_000, 13, 100, stats)
    d7 = bench.d7_bytes(250_000_000, 150_000_000, 13, 100, stats, 151.5)
    assert set(impl) >= {"pack", "index.codes", "index.sort", "index.ptrs", "index.recs", "index.tiled", "find", "sort"}
    assert all(v > 0 for v in impl.values()) and all(v > 0 for v in d7.values())
    # D7's find bytes: 8.25 B per position + 20 B per hit + (mean/2 + 12) B per MEM
    assert abs(d7["find"] - (8.25 * 149_997_216 + 20 * 17_300_000 + (151.5 / 2 + 12) * 811_662)) < 1
