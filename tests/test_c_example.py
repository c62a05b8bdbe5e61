"""The C ABI from plain C (examples/es_minimal.c): it compiles and links against
libes.so on CPU; on a GPU its result equals the oracle bit for bit."""
import os
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_sc_lixyszrljlllq23_b200")


def _build(tmp_path):
    exe = str(tmp_path / "es_minimal")
    subprocess.check_call(["gcc", "-O2", "-Wall", "-I", os.path.join(ROOT, "include"), "-I", "/usr/local/cuda/include",
                           os.path.join(ROOT, "examples", "es_minimal.c"), "-o", exe, "-L", PKG, "-les",
                           "-L", "/usr/local/cuda/lib64", "-lcudart", "-lm", f"-Wl,-rpath,{PKG}",
                           "-Wl,-rpath,/usr/local/cuda/lib64"])
    return exe


def test_c_example_builds_against_the_abi(tmp_path):
    from paper_conf_sc_lixyszrljlllq23_b200 import es
    es.lib()                                   # libes.so exists
    assert os.path.exists(_build(tmp_path))


@pytest.mark.gpu
def test_c_example_matches_oracle(tmp_path):
    import oracle
    exe = _build(tmp_path)
    out = str(tmp_path / "out.bin")
    subprocess.check_call([exe, out])
    got = np.fromfile(out, dtype=np.float32)
    L, N = 100003, 4
    i = np.arange(L, dtype=np.uint64)
    xs = [(((i * np.uint64(2654435761) + np.uint64(97 * k)) % np.uint64(2001)).astype(np.int64) - 1000)
          .astype(np.float32) * np.float32(0.001) for k in range(N)]
    want = oracle.reduce(xs, "f32")
    assert np.array_equal(got.view(np.uint32), want.view(np.uint32))
