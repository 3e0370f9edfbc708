"""bench.py output contract (the driver parses one JSON line): the reference arm on CPU
(the oracle on a small sample) and our arm on a B200 at a small size."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

BASE_KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
             "vs_baseline", "dtype", "data", "config"}


def _run(args, timeout=600):
    env = dict(os.environ, CUDA_VISIBLE_DEVICES=os.environ.get("CUDA_VISIBLE_DEVICES", ""))
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, cwd=ROOT, capture_output=True,
                         text=True, timeout=timeout, env=env)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0])


def test_reference_arm_line():
    d = _run(["--impl", "reference", "--steps", "2", "--warmup", "3", "--cpu-sample-bytes", str(4 << 20)])
    assert BASE_KEYS <= set(d)
    assert d["impl"] == "reference" and d["value"] > 0 and d["unit"] == "GB/s" and d["higher_is_better"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0


@pytest.mark.gpu
def test_our_arm_line_small():
    d = _run(["--config", "1", "--bytes", str(1 << 20), "--steps", "4", "--warmup", "3", "--no-cpu-baseline",
              "--e2e-steps", "2"])
    assert BASE_KEYS <= set(d)
    assert d["value"] > 0 and d["n_gpus"] == 1 and d["steps"] == 4 and d["warmup"] == 3
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["achieved"] > 0 and r["peak"] > 0 and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-3
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 1 << 20 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["gpu_launches"] > 0
    assert d["restore"]["ok"] and d["restart_import"]["ok"] and d["paper_throughput"]["ok"]
    assert set(d["clocks"]) >= {"sm_mhz", "sm_max_mhz", "reasons"}
    # resident lineage: pipelined calls timed, the one-call-at-a-time value beside them
    assert d["calls"].startswith("pipelined") and d["sync"]["value"] > 0 and d["sync"]["ms_per_step"] > 0


@pytest.mark.gpu
def test_our_arm_sync_flag():
    d = _run(["--config", "1", "--bytes", str(1 << 20), "--steps", "4", "--warmup", "3", "--no-cpu-baseline",
              "--e2e-steps", "1", "--sync"])
    assert d["calls"].startswith("one ckpt_checkpoint") and d["sync"] is None and d["value"] > 0


@pytest.mark.gpu
def test_our_arm_inplace_config5_form():
    """The in-place form bench.py uses for config 5 (16 GiB per GPU: the lineage does not fit
    in HBM), at a small size: one buffer mutated between steps outside the timed events."""
    d = _run(["--config", "5", "--bytes", str(64 << 20), "--inplace", "--steps", "3", "--warmup", "3",
              "--no-cpu-baseline"])
    assert BASE_KEYS <= set(d)
    assert d["value"] > 0 and d["n_gpus"] == 1 and d["config"]["buffer_bytes"] == 64 << 20
    assert "in place" in d["config"]["l2"] and d["calls"].startswith("one ckpt_checkpoint")
    assert d["restore"]["ok"] and d["paper_throughput"] is None and d["restart_import"] is None
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 64 << 20
    assert d["gpu_launches"] > 0
