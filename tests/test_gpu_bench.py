"""bench.py as the driver calls it: `python bench.py --gpus N ...` with no
torchrun environment.  N > 1 spawns the ranks itself (one process per GPU;
on a 1-GPU box the ranks share the device over gloo, which validates the flow,
not the scaling), and rank 0 prints ONE JSON line carrying roofline,
cpu_baseline (the oracle, timed after the GPU work) and e2e at every N."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(*args, timeout=900):
    env = dict(os.environ)
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "PDL_DRY_RUN"):
        env.pop(k, None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *map(str, args)], capture_output=True,
                       text=True, timeout=timeout, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-3000:]
    return json.loads(lines[0])


def _common(line, n):
    assert line["n_gpus"] == n
    assert line["value"] > 0 and line["unit"] == "GFLOP/s"
    assert line["roofline"]["achieved"] and line["roofline"]["frac"] > 0
    cpu = line["cpu_baseline"]
    assert cpu and cpu["kind"] == "oracle" and cpu["cores"] >= 1 and cpu["value"] > 0
    e2e = line["e2e"]
    assert e2e and e2e["value"] > 0 and e2e["h2d_bytes_per_step"] > 0 and e2e["d2h_bytes_per_step"] > 0
    assert e2e["steps"] == line["steps"]
    assert line["gpu_launches"] >= line["steps"]


def test_bench_two_ranks_plain_invocation():
    line = _bench("--gpus", 2, "--config", "C3", "--steps", 3, "--warmup", 3, "--cpu-seconds", 2)
    _common(line, 2)
    assert line["config"]["parallelism"] == "block2d 1x2"
    if line["config"]["dist_backend"] == "gloo":
        assert "validates" in line["config"]["note"]


def test_bench_one_gpu_carries_the_fp32_leg():
    line = _bench("--gpus", 1, "--config", "C2", "--steps", 3, "--warmup", 3, "--cpu-seconds", 2, "--no-alt")
    _common(line, 1)
    for key, variant in (("f32_3xtf32", "3xtf32"), ("f32_tf32bf16", "tf32bf16")):
        f32 = line[key]
        assert f32["value"] > 0 and f32["roofline"]["frac"] > 0 and f32["e2e"]["value"] > 0
        assert "K2" in f32["roofline"]["kernel"] and f32["task_variant"].startswith(variant)


def test_bench_fp32_variants_main_line():
    for variant in ("default", "3xtf32"):
        line = _bench("--dtype", "f32", "--variant", variant, "--config", "C2", "--steps", 3, "--warmup", 3,
                      "--cpu-seconds", 1)
        _common(line, 1)
        want = "3xtf32" if variant == "3xtf32" else "tf32bf16"
        assert line["config"]["task_variant"].startswith(want)
        assert ("kind::f16" in line["roofline"]["kernel"]) == (want == "tf32bf16")
