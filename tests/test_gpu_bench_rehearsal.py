"""bench.py's N>1 path (torchrun, barrier, max over ranks, rank-0 line, parity
regeneration of remote ESTs, e2e) rehearsed with two ranks on the one GPU this
build has: gloo process group, peer schedules over CUDA IPC (NCCL refuses two
ranks per GPU).  The reduced output's SHA-256 must equal the G = 1 run's --
placement invariance (D1) through the benchmark itself."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(args, nproc=1, port=29617):
    if nproc == 1:
        cmd = [sys.executable, os.path.join(ROOT, "bench.py")]
    else:
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
               "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.join(ROOT, "bench.py"),
               "--gpus", str(nproc), "--rehearse-same-gpu"]
    env = dict(os.environ, ES_BARRIER_TIMEOUT_S="60")
    out = subprocess.run(cmd + args, cwd=ROOT, capture_output=True, text=True, timeout=600, env=env)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0])


@pytest.mark.gpu
def test_bench_two_ranks_same_gpu_matches_g1():
    common = ["--config", "tiny", "--steps", "3", "--warmup", "3", "--no-cpu"]
    g1 = _bench(common + ["--no-e2e"])
    assert g1["parity"]["mismatched_words"] == 0 and g1["parity"]["full_output_mismatched_words"] == 0
    for i, sched in enumerate(["peer", "peer_chain"]):
        g2 = _bench(common + ["--sched", sched], nproc=2, port=29617 + i)
        assert g2["n_gpus"] == 2 and g2["config"]["G"] == 2 and "rehearsal" in g2["config"]
        assert g2["parity"]["mismatched_words"] == 0
        assert g2["output_sha256"] == g1["output_sha256"], sched
        assert g2["e2e"]["value"] > 0
        assert g2["next1"]["bits_equal_timed_step"] is True          # NEXT-1 at G = 2 on the bench path
        assert 0 < g2["allreduce_only"]["ms"] <= g2["ms_per_step"]
