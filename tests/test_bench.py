"""bench.py contract checks.  CPU: the --impl reference arm (oracle on host cores) prints
one valid JSON line, also under torchrun with 2 ranks (rank 1 exits 0 without work).
GPU: the main arm at a reduced size, at world size 1 and 2 (2 ranks sharing the one GPU
over gloo: exercises barrier / max-over-ranks / check-scalar SUM and weak scaling)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SMALL = ["--n-elem", "2048", "--blocks", "1", "--ref-elems", "256", "--tile", "8"]


def run(cmd, env=None, timeout=600):
    e = dict(os.environ)
    e.update(env or {})
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=timeout, env=e)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    return [json.loads(ln) for ln in lines]


def torchrun(n):
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
            "--master-addr", "127.0.0.1", "--master-port", str(29500 + os.getpid() % 1000)]


def test_reference_arm_json():
    out = run([sys.executable, "bench.py", "--impl", "reference", "--steps", "1", "--warmup", "0", *SMALL])
    assert len(out) == 1
    d = out[0]
    assert d["impl"] == "reference" and d["value"] > 0 and d["unit"] == "GFLOP/s"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["higher_is_better"] is True


def test_reference_arm_under_torchrun_prints_once():
    out = run(torchrun(2) + ["bench.py", "--impl", "reference", "--gpus", "2", "--steps", "1", "--warmup", "0", *SMALL])
    assert len(out) == 1 and out[0]["n_gpus"] == 2


@pytest.mark.gpu
def test_main_arm_world1():
    out = run([sys.executable, "bench.py", "--steps", "3", "--warmup", "3", *SMALL])
    d = out[0]
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "roofline", "cpu_baseline",
              "e2e", "clocks", "gpu_launches", "config"):
        assert k in d, k
    assert d["gpu_launches"] > 0 and d["roofline"]["frac"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0


@pytest.mark.gpu
def test_main_arm_world2_shared_gpu():
    out = run(torchrun(2) + ["bench.py", "--gpus", "2", "--steps", "3", "--warmup", "3", "--no-cpu", *SMALL],
              env={"BC_DIST_BACKEND": "gloo"})
    assert len(out) == 1
    d = out[0]
    assert d["n_gpus"] == 2 and d["scaling"] == "weak" and d["value"] > 0
