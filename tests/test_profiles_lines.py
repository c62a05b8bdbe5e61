"""The committed G = 1 bench lines (profiles/r02_bench_<config>_g1.json) keep the bench contract:
BASELINE's metric, the roofline / cpu_baseline / e2e / clocks objects, bit-exact parity, and the
tables in DESIGN.md and README.md are the ones scripts/bench_table.py generates from them."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CONFIGS = ["tiny", "resnet50", "vgg19", "bert_base", "swin_b"]


def _line(name):
    with open(os.path.join(ROOT, "profiles", f"r02_bench_{name}_g1.json")) as f:
        return json.load(f)


@pytest.mark.parametrize("name", CONFIGS)
def test_committed_line_keeps_the_contract(name):
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        metric = json.load(f)["metric"]
    d = _line(name)
    assert d["metric"] == metric and d["unit"] == "GB/s" and d["higher_is_better"] is True
    assert d["n_gpus"] == 1 and d["warmup"] >= 3 and d["steps"] >= 5 and d["value"] > 0
    assert d["config"]["workload"] == name and d["data"] == "synthetic" and d["vs_baseline"] is None
    r = d["roofline"]
    assert r["bound"] == "hbm" and r["unit"] == "GB/s" and abs(r["frac"] - r["achieved"] / r["peak"]) < 1e-3
    assert r["traffic"] is not None and r["traffic"] > 0
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] == 1 and cb["value"] > 0 and cb["sample"]
    e = d["e2e"]
    assert e["value"] > 0 and e["h2d_bytes_per_step"] > 0 and e["d2h_bytes_per_step"] > 0
    assert e["roofline"]["bound"] == "pcie_h2d"
    assert d["gpu_launches"] > 0
    c = d["clocks"]
    assert c["sm_mhz"] > 0.8 * c["sm_max_mhz"]
    assert not set(c["reasons"]) & {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"}
    p = d["parity"]
    assert p["mismatched_words"] == 0 and p["checked_elements"] > 0
    assert p["full_output_checked"] and p["full_output_mismatched_words"] == 0 and p["sha256_equal"] is True
    ar = d["allreduce_only"]
    assert 0 < ar["ms"] <= ar["phase_step_ms"] and ar["ms"] <= d["ms_per_step"]
    n1 = d["next1"]
    assert n1["bits_equal_timed_step"] is True and 0 < n1["tail_ms"] and 0 < n1["copy_step_tail_ms"]


def test_output_hash_is_the_oracles_where_checked_whole():
    for name in CONFIGS:
        d = _line(name)
        if d["parity"].get("full_output_checked"):
            assert d["output_sha256"] == d["parity"]["oracle_sha256"]


def test_tables_are_generated_from_the_lines():
    for kind, doc in (("design", "DESIGN.md"), ("readme", "README.md")):
        out = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "bench_table.py"), kind],
                             capture_output=True, text=True, check=True).stdout
        with open(os.path.join(ROOT, doc)) as f:
            text = f.read()
        for row in out.strip().splitlines()[2:]:
            cells = row.rstrip("|").rstrip()
            assert cells in text, f"{doc} lacks the generated row: {row}"
