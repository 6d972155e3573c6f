"""CPU tests of bench.py's host logic (no GPU): --gpus N fails loudly when fewer GPUs are
visible (never measures fewer GPUs than asked for), and the reference arm (the CPU oracle)
prints the contract line with the same `config` object the GPU arm uses."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, timeout=300):
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                          timeout=timeout, cwd=ROOT, env=env)


def test_gpus_more_than_visible_exits_with_enodev():
    import torch
    n = torch.cuda.device_count() + 1
    r = _run(["--gpus", str(max(n, 2)), "--steps", "1", "--warmup", "3", "--no-extras"])
    assert r.returncode == 2, r.stderr[-2000:]
    assert "JACOBI_ENODEV" in r.stderr
    assert r.stdout.strip() == ""  # no JSON line: nothing was measured


def test_reference_arm_line_and_shared_config():
    sys.path.insert(0, ROOT)
    import bench
    r = _run(["--impl", "reference", "--config", "c5b", "--steps", "1", "--warmup", "0", "--ref-iters", "1"])
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["unit"] == "Gcell-updates/s" and line["value"] > 0
    cfg = dict(bench.CONFIGS["c5b"])
    assert line["config"] == bench.workload_config(cfg, cfg["shape"], 1)
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] >= 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0


def test_reference_arm_weak_scaling_shape_follows_gpus():
    """C4 grows with N: 512 x 512 x (512 N) (R15); n_gpus reported as asked."""
    r = _run(["--impl", "reference", "--config", "c4", "--gpus", "2", "--steps", "1", "--warmup", "0",
              "--ref-iters", "1"], timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["n_gpus"] == 2 and line["config"]["shape_zyx"] == [1024, 512, 512]
    assert line["config"]["parallelism"] == "slab2"
