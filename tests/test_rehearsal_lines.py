"""CPU: the committed N>1 bench lines (profiles/r02_rehearsal_same_gpu.jsonl: torchrun
--nproc-per-node G bench.py --rehearse-same-gpu, every rank on cuda:0) keep the G > 1 contract
(VERDICT r01 "next" #1/#2): allreduce_only is a phase-event time no longer than the step, its
roofline is the plan model (t_roof = max(HBM / HBM peak, NVLink / NVLink peak),
NVLink-bound where the plan says so), the schedule ladder and preflight are recorded, NVLink
counters sit beside the plan's bytes, and every G prints the G = 1 output hash (D1,
PAPER.md:763-772) with whole-output oracle parity."""
import json
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
def _g1_sha():
    """whole-output oracle SHA-256 of the committed G = 1 line of each workload"""
    out = {}
    for name in ("tiny", "resnet50", "vgg19", "bert_base", "swin_b"):
        with open(os.path.join(ROOT, "profiles", f"r02_bench_{name}_g1.json")) as f:
            d = json.load(f)
        assert d["parity"]["sha256_equal"]
        out[name] = d["output_sha256"]
    return out


G1_SHA = _g1_sha()


def _lines(name="r02_rehearsal_same_gpu.jsonl"):
    with open(os.path.join(ROOT, "profiles", name)) as f:
        return [json.loads(l) for l in f if l.strip()]


def _all_lines():
    # time-sliced processes, and the same under CUDA MPS (ranks running concurrently)
    return _lines() + _lines("r02_rehearsal_mps.jsonl")


@pytest.mark.parametrize("d", _all_lines(), ids=lambda d: d["run"])
def test_rehearsal_line_contract(d):
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        assert d["metric"] == json.load(f)["metric"]
    G = d["n_gpus"]
    assert G >= 2 and d["config"]["G"] == G and "rehearsal" in d["config"]
    ar = d["allreduce_only"]
    # part of the step: against the same replays' stash-start -> allreduce-done span (a rehearsal's
    # ranks time-slice one GPU, so separately timed replays are noise)
    assert 0 < ar["ms"] <= ar["phase_step_ms"], "allreduce_only is part of the step"
    assert "phase events" in ar["timing"] and "max over ranks" in ar["timing"]
    r = ar["roofline"]
    assert r["bound"] in ("nvlink", "hbm") and r["t_roof_ms"] > 0 and len(r["per_rank_MB"]) == G
    worst = max(r["per_rank_MB"], key=lambda c: max(c["hbm"] / r["peaks"]["hbm_gbps"],
                                                    max(c["nvl_in"], c["nvl_out"]) / r["peaks"]["nvlink_gbps"]))
    t_h = worst["hbm"] / r["peaks"]["hbm_gbps"]
    t_n = max(worst["nvl_in"], worst["nvl_out"]) / r["peaks"]["nvlink_gbps"]
    assert r["bound"] == ("nvlink" if t_n > t_h else "hbm")
    assert abs(r["t_roof_ms"] - max(t_h, t_n)) < 1e-3 * max(t_h, t_n) + 1e-4
    assert r["peaks"]["nvlink_gbps"] == 770.0 and "rehearsal" in r
    sch = d["schedule"]
    assert sch["ladder"][-1].get("ok") is True and len(sch["per_bucket"]) == d["config"]["buckets"]
    assert len(d["preflight"]) == G and {"device", "peer_access", "nvlink_links_active"} <= set(d["preflight"][0])
    nv = d["nvlink_counters"]
    assert len(nv["per_rank"]) == G and len(nv["plan_per_rank"]) == G
    for k in d["roofline_by_kernel"].values():
        if "rehearsal" in k:
            assert k["bound"] == "hbm"       # peer bytes never cross NVLink on one GPU
    p = d["parity"]
    assert p["mismatched_words"] == 0 and p["full_output_checked"] and p["full_output_mismatched_words"] == 0
    assert p["sha256_equal"] and d["output_sha256"] == G1_SHA[d["config"]["workload"]]
    assert "ring_crosscheck" in d


def test_fallback_ladder_recorded():
    """--simulate-peer-failure parity: the first rung fails the first-step oracle check on one
    rank, every rank moves to the next rung, and the line is still bit-exact."""
    d = [x for x in _lines() if x["run"].endswith("failparity")][0]
    lad = d["schedule"]["ladder"]
    assert "failed" in lad[0] and "first-step oracle check" in lad[0]["failed"] and lad[-1]["ok"] is True
    assert d["parity"]["full_output_mismatched_words"] == 0


def test_every_g_prints_the_same_hash():
    by = {}
    for d in _all_lines():
        by.setdefault(d["config"]["workload"], set()).add(d["output_sha256"])
    for w, hs in by.items():
        assert len(hs) == 1, w
