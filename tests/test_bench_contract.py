"""CPU checks of bench.py's driver contract (no GPU here): the reference arm's JSON line, the
reference arm on a non-zero rank, and the product arm failing loudly without a GPU (no CPU
fallback anywhere on the product path)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env=None, timeout=300):
    e = dict(os.environ)
    e.update(env or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], cwd=ROOT, env=e,
                          capture_output=True, text=True, timeout=timeout)


def test_reference_arm_json_line():
    r = _run(["--impl", "reference", "--steps", "1", "--warmup", "0"])
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["unit"] == "GFLOP/s" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["cpu_baseline"]["value"] == d["value"] and d["cpu_baseline"]["sample"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert "workload" in d["config"]


def test_reference_arm_other_ranks_exit_silently():
    r = _run(["--impl", "reference", "--gpus", "2", "--steps", "1", "--warmup", "0"],
             env={"RANK": "1", "WORLD_SIZE": "2", "LOCAL_RANK": "1"})
    assert r.returncode == 0 and r.stdout.strip() == ""


def test_product_arm_fails_loudly_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    r = _run(["--steps", "3", "--warmup", "3", "--no-cpu-baseline"])
    assert r.returncode != 0
    assert '"value"' not in r.stdout          # no number from a CPU fallback


def test_self_launch_without_torchrun():
    """`bench.py --gpus N` outside torchrun launches N ranks itself (torch.distributed.run,
    127.0.0.1 rendezvous); rank 0 alone prints one JSON line holding the max over ranks.  The
    CPU variant of the same launch path (--selftest-launch: gloo, no CUDA)."""
    r = _run(["--gpus", "2", "--selftest-launch"], timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["world_size"] == 2 and d["n_gpus"] == 2 and d["max_over_ranks"] == 2.0


def test_strong_scaling_grid_rule():
    """The documented strong-scaling process-grid rule (bench.choose_grid): maximise
    the interior fraction, then the fewest face bytes, then the larger Pt."""
    sys.path.insert(0, ROOT)
    import bench
    assert bench.choose_grid((48, 48, 48, 48), 1) == (1, 1, 1, 1)
    assert bench.choose_grid((48, 48, 48, 48), 2) == (1, 1, 1, 2)
    assert bench.choose_grid((48, 48, 48, 48), 4) == (1, 1, 1, 4)      # Lt = 12: 50% interior
    assert bench.choose_grid((48, 48, 48, 48), 8) == (1, 1, 2, 4)      # t8 (Lt = 6) has no interior site
    assert bench.interior_fraction((48, 48, 24, 12), (2, 3)) == 0.375
    assert bench.interior_fraction((48, 48, 48, 6), (3,)) == 0.0
