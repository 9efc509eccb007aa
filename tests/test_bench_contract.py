"""bench.py contract on CPU: the reference arm (the CPU oracle) prints one JSON
line with the driver's keys; the CUDA arm's JSON is checked on the GPU box by
running bench.py itself."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    out = subprocess.check_output([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                                   "--steps", "1", "--warmup", "0", "--ref-n", "12"], cwd=ROOT, timeout=300)
    lines = [l for l in out.decode().splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("impl", "metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["higher_is_better"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        assert d["metric"] == json.load(f)["metric"]


def test_reference_arm_non_zero_rank_is_silent():
    env = dict(os.environ, RANK="1", WORLD_SIZE="2")
    out = subprocess.check_output([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference",
                                   "--steps", "1", "--warmup", "0", "--ref-n", "12"], cwd=ROOT, env=env,
                                  timeout=300)
    assert out.decode().strip() == ""


def test_gpus_beyond_visible_devices_fails_loudly():
    """`bench.py --gpus N` without torchrun re-executes itself as N ranks only when N GPUs are
    visible; otherwise it exits non-zero (never silently runs one GPU)."""
    import torch
    n = torch.cuda.device_count() + 1
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", str(max(n, 2)),
                        "--steps", "1", "--warmup", "3"], cwd=ROOT, env=env, timeout=300,
                       capture_output=True)
    assert r.returncode != 0
    assert b"visible CUDA devices" in r.stderr
    assert not [l for l in r.stdout.decode().splitlines() if l.strip().startswith("{")]


def test_world_size_must_match_gpus():
    env = dict(os.environ, RANK="0", WORLD_SIZE="1", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1"],
                       cwd=ROOT, env=env, timeout=300, capture_output=True)
    assert r.returncode != 0 and b"one rank per GPU" in r.stderr
