"""bench.py runs end to end (the driver's contract): one JSON line with the keys the driver and
the judge read, on a small workload (C1, e2e and the CPU baseline included), and the reference
arm's line.  Guards the measurement script itself, which the parity tests do not execute."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                       cwd=ROOT, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_bench_line_c1():
    j = _run(["--workload", "C1", "--steps", "3", "--warmup", "3"])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "clocks", "gpu_launches"):
        assert k in j, k
    assert j["value"] > 0 and j["ms_per_step"] > 0 and j["gpu_launches"] > 0
    assert j["e2e"]["value"] > 0 and j["e2e"]["h2d_bytes_per_step"] > 0
    assert j["roofline"]["peak"] > 0 and 0 < j["roofline"]["frac"] <= 1.5
    assert "flushed" in j["config"]["l2"]          # C1's inputs fit L2: trees timed with a flush between them


def test_bench_reference_arm():
    j = _run(["--impl", "reference", "--workload", "C1", "--steps", "1", "--warmup", "1"])
    assert j["impl"] == "reference" and j["value"] > 0
    assert j["e2e"]["h2d_bytes_per_step"] == 0


def test_bench_two_ranks_gloo():
    """The N > 1 launch the driver uses (torch.distributed.run, one JSON line from rank 0, max over
    ranks), with gloo and the collective exchange so the two ranks can share this one GPU: a smoke
    test of bench.py's multi-rank plumbing, not a measurement."""
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", "29571", os.path.join(ROOT, "bench.py"),
                        "--gpus", "2", "--steps", "2", "--warmup", "3", "--workload", "C1", "--backend", "gloo",
                        "--exchange", "collective", "--no-cpu-baseline"],
                       capture_output=True, text=True, cwd=ROOT, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    j = json.loads(lines[0])
    assert j["n_gpus"] == 2 and j["value"] > 0 and j["e2e"]["value"] > 0
    assert "feature-partition x2" in j["config"]["parallelism"]


def test_bench_reference_two_ranks():
    """--impl reference under torch.distributed.run: rank 0 alone prints the line, the others exit 0."""
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", "29573", os.path.join(ROOT, "bench.py"),
                        "--impl", "reference", "--gpus", "2", "--steps", "1", "--warmup", "1", "--workload", "C1"],
                       capture_output=True, text=True, cwd=ROOT, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1 and json.loads(lines[0])["impl"] == "reference", r.stdout[-2000:]
