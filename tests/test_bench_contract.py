"""bench.py's contract pieces that run without a GPU: the reference arm
prints one JSON line whose config dict is identical to the headline's (so the
driver's same_config holds), and a --gpus / WORLD_SIZE mismatch is an error
instead of a silently mislabelled line."""
from __future__ import annotations

import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(args, env_extra=None, timeout=600):
    env = dict(os.environ, **(env_extra or {}))
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                          timeout=timeout, env=env, cwd=ROOT)


def test_reference_arm_line_matches_the_headline_config():
    sys.path.insert(0, ROOT)
    import bench
    r = _bench(["--impl", "reference", "--steps", "1", "--warmup", "0"])
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["metric"] == bench.METRIC
    assert line["config"] == bench.headline_config(1)
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] >= 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0 and line["unit"] == "GFLOP/s" and line["value"] > 0
    r4 = _bench(["--impl", "reference", "--steps", "1", "--warmup", "0"], {"WORLD_SIZE": "4", "RANK": "0"})
    assert json.loads(r4.stdout.strip().splitlines()[-1])["config"] == bench.headline_config(4)
    r1 = _bench(["--impl", "reference", "--steps", "1", "--warmup", "0"], {"WORLD_SIZE": "4", "RANK": "1"})
    assert r1.returncode == 0 and r1.stdout.strip() == ""  # only rank 0 runs and prints


def test_gpus_mismatch_is_an_error():
    r = _bench(["--gpus", "2"], {"WORLD_SIZE": "1", "RANK": "0", "LOCAL_RANK": "0"}, timeout=120)
    assert r.returncode == 2 and "WORLD_SIZE=1" in r.stderr
