"""bench.py's JSON-line contract.  CPU: the reference arm (the oracle, per the
task's tier rules), alone and under torchrun with two ranks (rank 0 alone
prints).  GPU: the main arm's keys on the tiny config."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BASE_KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
             "vs_baseline", "dtype", "data", "config"}


def _lines(cmd, env=None):
    out = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=600,
                         env=dict(os.environ, **(env or {})))
    assert out.returncode == 0, out.stderr[-3000:]
    return [json.loads(l) for l in out.stdout.splitlines() if l.startswith("{")]


def _check_reference(d, n_gpus):
    assert BASE_KEYS <= set(d) and d["impl"] == "reference"
    assert d["n_gpus"] == n_gpus and d["value"] > 0 and d["unit"] == "GB/s" and d["higher_is_better"] is True
    assert d["config"]["workload"] == "tiny" and d["dtype"] == "f32"
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == d["value"] and cb["sample"]
    assert d["e2e"] == {"value": d["value"], "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}


def test_reference_arm_line():
    lines = _lines([sys.executable, "bench.py", "--impl", "reference", "--config", "tiny", "--steps", "2",
                    "--warmup", "1", "--cpu-seconds", "1"])
    assert len(lines) == 1
    _check_reference(lines[0], 1)


def test_reference_arm_under_torchrun_prints_once():
    lines = _lines([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                    "--master-addr", "127.0.0.1", "--master-port", "29741", "bench.py", "--gpus", "2", "--impl",
                    "reference", "--config", "tiny", "--steps", "1", "--warmup", "1", "--cpu-seconds", "1"])
    assert len(lines) == 1
    _check_reference(lines[0], 2)


@pytest.mark.gpu
def test_main_arm_line_keys():
    lines = _lines([sys.executable, "bench.py", "--config", "tiny", "--steps", "5", "--warmup", "3",
                    "--cpu-seconds", "1"])
    assert len(lines) == 1
    d = lines[0]
    assert BASE_KEYS <= set(d) and d["n_gpus"] == 1 and d["warmup"] >= 3 and d["value"] > 0
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and r["peak"] > 0 and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-3
    assert {"value", "unit", "cores", "kind", "sample"} <= set(d["cpu_baseline"]) and d["cpu_baseline"]["kind"] == "oracle"
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] == 4 * 1048576 * 4 and e["d2h_bytes_per_step"] == 4 * 1048576
    assert e["roofline"]["bound"] == "pcie_h2d" and e["roofline"]["peak"] > 0 and 0 < e["roofline"]["frac"] < 1.5
    assert d["gpu_launches"] > 0 and {"sm_mhz", "sm_max_mhz", "reasons"} <= set(d["clocks"])
    assert d["parity"]["mismatched_words"] == 0 and d["parity"]["full_output_mismatched_words"] == 0
    assert d["parity"]["sha256_equal"] is True and d["switch"]["us_per_switch"] > 0
    ar = d["allreduce_only"]
    assert 0 < ar["ms"] <= ar["phase_step_ms"] and ar["ms"] <= d["ms_per_step"]
    n1 = d["next1"]                       # NEXT-1 leg: same bits, tail measured beside the copy step's
    assert n1["bits_equal_timed_step"] is True and n1["tail_ms"] > 0 and n1["copy_step_tail_ms"] > 0
