"""bench.py's launch contract on a box without enough GPUs (CPU only): `--gpus N`
without torchrun spawns N ranks itself and must fail loudly -- never time fewer
GPUs than asked -- and a WORLD_SIZE that disagrees with --gpus is an error."""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(args, env_extra=None):
    env = dict(os.environ, CUDA_VISIBLE_DEVICES="")
    env.pop("WORLD_SIZE", None)
    env.update(env_extra or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                          env=env, timeout=300)


def test_gpus_n_without_enough_gpus_fails_loudly():
    r = _bench(["--gpus", "2", "--steps", "1", "--warmup", "3"])
    assert r.returncode != 0
    assert "only 0 GPU(s) visible" in (r.stdout + r.stderr)


def test_world_size_must_match_gpus():
    r = _bench(["--gpus", "2", "--steps", "1", "--warmup", "3"], {"WORLD_SIZE": "1"})
    assert r.returncode != 0
    assert "WORLD_SIZE" in (r.stdout + r.stderr)


def test_warmup_below_three_rejected():
    r = _bench(["--warmup", "2"])
    assert r.returncode != 0 and "--warmup must be >= 3" in r.stderr


@pytest.mark.parametrize("cfg", ["C1"])
def test_reference_arm_runs_on_cpu(cfg):
    """The reference arm of this tier is the oracle: it runs without a GPU."""
    import json
    r = _bench(["--impl", "reference", "--config", cfg, "--steps", "1", "--warmup", "3"])
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["unit"] == "GStencil/s" and line["value"] > 0
    assert line["cpu_baseline"]["seconds_1_thread"] > 0 and line["cpu_baseline"]["cpu_model"]
