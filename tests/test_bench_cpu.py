"""bench.py host logic on CPU: the reference arm's JSON line (the oracle on the host cores), the
rank != 0 behaviour under torchrun, and the roofline helpers (per-unit figures of DESIGN.md 6.1)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def _run(args, env_extra=None):
    env = dict(os.environ)
    env.update(env_extra or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True,
                          text=True, env=env, timeout=600, cwd=ROOT)


def test_reference_arm_line_c1():
    r = _run(["--impl", "reference", "--config", "c1", "--steps", "2", "--warmup", "1"])
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "dtype", "config", "cpu_baseline", "e2e"):
        assert k in line, k
    assert line["impl"] == "reference"
    assert line["unit"] == "KOPS" and line["higher_is_better"] is True and line["value"] > 0
    assert line["steps"] == 2 and line["warmup"] == 1
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] >= 1
    assert line["cpu_baseline"]["value"] == line["value"]
    assert line["e2e"] == {"value": line["value"], "unit": "KOPS", "h2d_bytes_per_step": 0,
                           "d2h_bytes_per_step": 0}
    assert line["config"]["N"] == 4096 and line["config"]["L"] == 4


def test_reference_arm_other_ranks_are_silent():
    r = _run(["--impl", "reference", "--config", "c1", "--steps", "1", "--warmup", "0"],
             {"RANK": "1", "WORLD_SIZE": "2", "LOCAL_RANK": "1"})
    assert r.returncode == 0, r.stderr[-2000:]
    assert r.stdout.strip() == ""


def test_roofline_helpers():
    import bench
    n = 1 << 16
    # 256 u8 MACs per element per radix-16 stage: 4 stages for tensor, forward-only tc4
    assert bench.tensor_macs_per_transform("tensor", n, True) == 256.0 * n * 4
    assert bench.tensor_macs_per_transform("tc4", n, True) == 256.0 * n * 4
    assert bench.tensor_macs_per_transform("tc4", n, False) == 0.0
    assert bench.tensor_macs_per_transform("cuda", n, True) == 0.0
    assert bench.tensor_macs_per_transform("auto", n, False) == 0.0
    assert bench.tensor_macs_per_transform("tensor", 1 << 15, True) == 0.0
    pk, pk64, kind = bench.i8_peak()
    assert kind == "measured" and pk > pk64 > 0      # profiles/r02/peaks_i8.json is committed


# bench.py's configs c1..c4 are BASELINE.json configs[0..3] (N, L, ciphertexts; c1 is one polynomial)
@pytest.mark.parametrize("i,cfg,want", [(0, "c1", (12, 4, None)), (1, "c2", (16, 36, 1)), (2, "c3", (16, 36, 64)),
                                        (3, "c4", (17, 48, 32))])
def test_configs_match_baseline(i, cfg, want):
    import bench
    desc = json.load(open(os.path.join(ROOT, "BASELINE.json")))["configs"][i]
    assert bench.CONFIGS[cfg] == want
    logn, L, nct = want
    assert "N=2^%d" % logn in desc and "L=%d" % L in desc
    if nct is not None and nct > 1:
        assert "%d ciphertexts" % nct in desc
