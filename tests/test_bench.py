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


def test_reference_arm_never_loads_the_product_library():
    """The oracle legs import only oracle / synthetic / accounting: after a full
    --impl reference run, libbarracuda.so is not mapped in the process (only liboracle)."""
    code = ("import runpy, sys; sys.argv = ['bench.py', '--impl', 'reference', '--steps', '1', '--warmup', '0', "
            + ", ".join(repr(a) for a in SMALL) + "]; runpy.run_path('bench.py', run_name='__main__'); "
            "maps = open('/proc/self/maps').read(); "
            "print('MAPPED', 'libbarracuda' in maps, 'liboracle' in maps)")
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    assert "MAPPED False True" in r.stdout, r.stdout[-500:]


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
    e = d["e2e"]
    assert e["d2h_bytes_per_step"] > e["h2d_bytes_per_step"] and e["sumsq_rel_diff_vs_device_step"] <= 1e-12
    assert e["host_results_match_device"]
    cb = d["cpu_baseline"]
    assert cb["gflops_1core"] > 0 and cb["cores_all"] >= 1 and cb["cpu_model"]
    assert d["fp64_peak_tflops"]["dmma"] > 1 and d["configs"]["cfg1_sumfact3d_p4_N64"]["us_per_call_graph"] > 0


@pytest.mark.gpu
def test_main_arm_world2_shared_gpu():
    out = run(torchrun(2) + ["bench.py", "--gpus", "2", "--steps", "3", "--warmup", "3", "--no-cpu", *SMALL],
              env={"BC_DIST_BACKEND": "gloo"})
    assert len(out) == 1
    d = out[0]
    assert d["n_gpus"] == 2 and d["scaling"] == "weak" and d["value"] > 0


@pytest.mark.gpu
def test_main_arm_world2_strong_shared_gpu():
    """Strong scaling: the global batch is split over the 2 ranks; the flops in `value`
    are the global step's (sum over ranks)."""
    out = run(torchrun(2) + ["bench.py", "--gpus", "2", "--steps", "3", "--warmup", "3", "--no-cpu", "--no-e2e",
                             "--scaling", "strong", *SMALL], env={"BC_DIST_BACKEND": "gloo"})
    d = out[0]
    assert d["scaling"] == "strong" and d["config"]["scaling"] == "strong" and d["value"] > 0
