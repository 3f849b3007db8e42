"""bench.py host logic on CPU: the reference arm (the oracle on host threads) prints the
contract's JSON line with the same metric / unit as our arm, and the source planning
of the multi-GPU modes covers the job exactly once (strong scaling) or per rank (weak)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_reference_arm_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "C1",
                        "--steps", "3", "--warmup", "1", "--cpu-threads", "2"],
                       capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [x for x in r.stdout.splitlines() if x.strip()]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["metric"] == bench.METRIC and d["unit"] == bench.UNIT
    assert d["value"] > 0 and d["steps"] == 3 and d["warmup"] == 1
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 2
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["config"]["workload"].startswith("C1")


def test_plan_sources_strong_weak_vertex():
    job = list(range(1000, 2024))
    for world in (1, 2, 8):
        blocks = [bench.plan_sources(job, r, world, "strong", "replicate") for r in range(world)]
        assert [x for b in blocks for x in b] == job
        assert all(len(b) == 1024 // world for b in blocks)
        for r in range(world):
            assert bench.plan_sources(job, r, world, "strong", "vertex") == job


def test_parse_args_defaults():
    a = bench.parse_args([])
    assert a.config == "C4" and a.scaling == "strong" and a.warmup >= 3 and a.steps >= 1
