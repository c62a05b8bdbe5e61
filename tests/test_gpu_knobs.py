"""GPU: every environment knob libes reads (`grep getenv csrc/`) is run through
the oracle-parity probe in a fresh process (the knobs are read once, at load):
a knob may change speed, never bits.  ES_BARRIER_TIMEOUT_S is also checked for
its purpose: a peer that never arrives makes the device barrier trap (the
handle reports ES_ECUDA) instead of hanging the GPU.

Knobs: ES_NO_PDL=1 (no programmatic dependent launch), ES_STASH_EARLY=0 (no
early start of captured stashes), ES_FOLD_TMA=1 (TMA-staged fold, kept as the
measured-and-rejected design), ES_BARRIER_TIMEOUT_S (spin guard).
CUDA_DEVICE_MAX_CONNECTIONS is CUDA's own variable (es_peer_open reads it to
refuse more same-process peer ranks than hardware queues)."""
import os
import re
import subprocess
import sys

import pytest

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
PROBE = os.path.join(HERE, "knob_probe.py")

KNOBS = {"ES_NO_PDL": "1", "ES_STASH_EARLY": "0", "ES_FOLD_TMA": "1", "ES_BARRIER_TIMEOUT_S": "30"}


def _run(env_extra, mode, timeout=300):
    env = dict(os.environ, **env_extra)
    return subprocess.run([sys.executable, PROBE, mode], env=env, cwd=ROOT, capture_output=True, text=True,
                          timeout=timeout)


def test_knob_list_matches_the_library_sources():
    """CPU: the knobs tested here are exactly the ES_* variables libes reads."""
    names = set()
    csrc = os.path.join(ROOT, "paper_conf_sc_lixyszrljlllq23_b200", "csrc")
    for f in os.listdir(csrc):
        with open(os.path.join(csrc, f)) as fh:
            names |= set(re.findall(r'getenv\("([A-Z_0-9]+)"\)', fh.read()))
    assert names - {"CUDA_DEVICE_MAX_CONNECTIONS"} == set(KNOBS), names


@pytest.mark.gpu
@pytest.mark.parametrize("knob", sorted(KNOBS))
def test_knob_keeps_oracle_parity(knob):
    r = _run({knob: KNOBS[knob]}, "parity")
    assert r.returncode == 0 and "KNOB_PROBE_OK" in r.stdout, (knob, r.stdout[-2000:], r.stderr[-4000:])


@pytest.mark.gpu
def test_barrier_timeout_traps_instead_of_hanging():
    r = _run({"ES_BARRIER_TIMEOUT_S": "2"}, "stuck", timeout=120)
    assert r.returncode == 0 and "STUCK_TRAPPED" in r.stdout, (r.stdout[-2000:], r.stderr[-4000:])
