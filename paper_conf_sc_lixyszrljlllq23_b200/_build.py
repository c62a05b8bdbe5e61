"""Builds libes.so in-tree: nvcc for sm_100a, -lineinfo, no fast-math.

The shared library travels to the GPU box with the repo snapshot (it is
git-ignored, not gpurun-ignored).  NCCL is resolved at run time with dlopen,
so only its header is needed here.
"""
import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libes.so")
ROOT = os.path.dirname(HERE)

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-lineinfo", "-O3", "-std=c++17",
    # R6: IEEE fp32 -- no fast-math, no FTZ, no FMA contraction in host code.
    "-ftz=false", "-prec-div=true", "-prec-sqrt=true", "-fmad=false",
    "-Xcompiler", "-fPIC,-Wall,-ffp-contract=off",
    "-shared",
]


def _nccl_include():
    try:
        import nvidia.nccl  # noqa: F401  (torch's bundled NCCL)
        base = os.path.dirname(sys.modules["nvidia.nccl"].__file__ or list(sys.modules["nvidia.nccl"].__path__)[0])
        if not os.path.isdir(os.path.join(base, "include")):
            base = list(sys.modules["nvidia.nccl"].__path__)[0]
        return os.path.join(base, "include")
    except Exception:
        for cand in glob.glob("/usr/include/nccl.h") + glob.glob("/usr/local/cuda/include/nccl.h"):
            return os.path.dirname(cand)
    raise RuntimeError("nccl.h not found (torch's nvidia-nccl package or /usr/include)")


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cpp")))


def needs_build():
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.h")) + [os.path.join(ROOT, "include", "es.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(verbose=False, force=False):
    if not force and not needs_build():
        return LIB
    nvcc = os.environ.get("NVCC", "nvcc")
    if not os.path.exists(nvcc) and os.path.exists("/usr/local/cuda/bin/nvcc"):
        nvcc = "/usr/local/cuda/bin/nvcc" if nvcc == "nvcc" and not _which("nvcc") else nvcc
    tmp = LIB + ".tmp"
    cmd = [nvcc] + NVCC_FLAGS + ["-I", _nccl_include(), "-I", os.path.join(ROOT, "include"),
                                "-o", tmp] + sources() + ["-ldl", "-lpthread"]
    if verbose:
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


def _which(x):
    for d in os.environ.get("PATH", "").split(os.pathsep):
        if os.path.exists(os.path.join(d, x)):
            return True
    return False


if __name__ == "__main__":
    print(build(verbose=True, force="--force" in sys.argv))
