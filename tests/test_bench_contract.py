"""bench.py contract on CPU: the reference arm (the fp64 oracle)
prints one JSON line with the driver's keys; non-zero ranks print nothing."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(extra_env=None, gpus=1):
    env = dict(os.environ)
    env.update({"POLYCONV_CPU_BASELINE_S": "0.5"})
    if extra_env:
        env.update(extra_env)
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "2",
                           "--warmup", "0", "--gpus", str(gpus)], capture_output=True, text=True, env=env,
                          timeout=600, cwd=ROOT)


def test_reference_arm_line():
    r = _run()
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for key in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
                "config", "cpu_baseline", "e2e", "impl"):
        assert key in d, key
    assert d["impl"] == "reference"
    assert d["unit"] == "TFLOP/s" and d["higher_is_better"] is True and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert d["config"]["workload"] == "resnet50_conv3x"


def test_reference_arm_nonzero_rank_silent():
    r = _run({"RANK": "1", "WORLD_SIZE": "2"}, gpus=2)
    assert r.returncode == 0, r.stderr[-2000:]
    assert not [l for l in r.stdout.splitlines() if l.strip().startswith("{")]


def test_gpus_must_match_world_size():
    """--gpus N under a launcher with another WORLD_SIZE is an error, not a silent 1-GPU run."""
    r = _run({"RANK": "0", "WORLD_SIZE": "2"}, gpus=4)
    assert r.returncode != 0
    assert "WORLD_SIZE" in (r.stderr + r.stdout)
