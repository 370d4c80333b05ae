"""bench.py host logic on CPU: workloads and their per-rank grids (weak / strong), the autotune
candidate normal form, and --gpus handling (more GPUs than visible is an error; a launcher's
WORLD_SIZE must equal --gpus)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_workloads_weak_and_strong_grids():
    w = bench.Workload("weather", 1)
    assert w.desc.n == (512, 512, 128) and w.scaling == "weak" and w.global_npts == 512 * 512 * 128
    w4 = bench.Workload("weather", 4)
    assert w4.desc.n == (512, 512, 128) and w4.global_npts == 4 * 512 * 512 * 128
    k = bench.Workload("weak", 8)
    assert k.desc.n == (1024, 1024, 128) and k.global_npts == 8 * 1024 * 1024 * 128
    for world, (px, py) in ((1, (1, 1)), (2, (2, 1)), (4, (2, 2)), (8, (4, 2))):
        s = bench.Workload("stress", world)
        assert s.scaling == "strong" and s.desc.n == (768 // px, 768 // py, 768)
        assert s.global_npts == 768 ** 3                   # strong: the local grids partition 768^3
    assert bench.grid_for(8) == (4, 2)


def test_candidate_normal_form():
    assert bench.cand_norm(((32, 8, 64), 2, 1, 0, 0, 1)) == [[32, 8, 64], 2, 1, 0, 0, 1, 1, 1, 1]
    assert bench.cand_norm(((32, 8, 43), 3, 1, 0, -1, 1, 2, 0)) == [[32, 8, 43], 3, 1, 0, -1, 1, 2, 0, 1]
    kw = bench.cand_kw({"tile": (32, 8, 64)}, [[64, 4, 64], 2, 2, 1, -1, 0, 2, 0])
    assert kw["tile"] == (64, 4, 64) and kw["zunroll"] == 2 and kw["pblock"] == (2, 1) and kw["canvas_ld"] == 0


def test_gpus_flag_is_honoured():
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    env["CUDA_VISIBLE_DEVICES"] = ""
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1"],
                       capture_output=True, text=True, env=env, timeout=300)
    assert r.returncode != 0 and "CUDA device" in (r.stdout + r.stderr)
    env["WORLD_SIZE"] = "1"
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1"],
                       capture_output=True, text=True, env=env, timeout=300)
    assert r.returncode != 0 and "WORLD_SIZE=1 but --gpus 2" in (r.stdout + r.stderr)


def test_reference_arm_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--workload", "tiny",
                        "--steps", "2", "--warmup", "1"], capture_output=True, text=True, timeout=300)
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["value"] > 0 and line["cpu_baseline"]["kind"] == "oracle"
    assert line["e2e"]["h2d_bytes_per_step"] == 0
