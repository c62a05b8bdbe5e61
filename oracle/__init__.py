"""CPU oracle for EasyScale placement-invariant gradient aggregation.

TEST INFRASTRUCTURE.  Only ``tests/``, ``__graft_entry__.smoke()`` and the
``cpu_baseline`` / ``--impl reference`` legs of ``bench.py`` may import this
package.  The product path (``paper_conf_sc_lixyszrljlllq23_b200``) never
imports it and shares no code with it.

The arithmetic lives in ``es_oracle.c`` (plain C, -ffp-contract=off); this
module only marshals NumPy arrays into it.  ``switch_model.py`` is the
dictionary state machine for the context switch.

Pinned by tests/test_oracle_pins.py.
"""
import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

F32 = 0
BF16 = 1


def build():
    """Compile liboracle.so (gcc, -O2 -ffp-contract=off)."""
    subprocess.check_call(["make", "-s", "-C", _HERE])


def lib():
    global _lib
    if _lib is None:
        src = os.path.join(_HERE, "es_oracle.c")
        if not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
            build()
        L = ctypes.CDLL(_LIB_PATH)
        L.es_oracle_chunk_elems.restype = ctypes.c_int64
        L.es_oracle_chunk_elems.argtypes = [ctypes.c_int64, ctypes.c_int32, ctypes.c_int32]
        L.es_oracle_reduce.restype = ctypes.c_int
        L.es_oracle_reduce.argtypes = [ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                       ctypes.POINTER(ctypes.c_void_p), ctypes.c_int64, ctypes.c_int64,
                                       ctypes.c_void_p]
        L.es_oracle_reduce_ex.restype = ctypes.c_int
        L.es_oracle_reduce_ex.argtypes = [ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                          ctypes.c_uint32, ctypes.POINTER(ctypes.c_void_p), ctypes.c_int64,
                                          ctypes.c_int64, ctypes.c_void_p]
        L.es_oracle_philox4x32_10.restype = None
        L.es_oracle_philox4x32_10.argtypes = [ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32),
                                              ctypes.POINTER(ctypes.c_uint32)]
        L.es_oracle_dropout.restype = ctypes.c_int
        L.es_oracle_dropout.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64,
                                        ctypes.c_int32, ctypes.c_float, ctypes.c_uint64, ctypes.c_uint64]
        L.es_oracle_stash.restype = ctypes.c_int
        L.es_oracle_stash.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p, ctypes.c_int32,
                                      ctypes.c_int64]
        L.es_oracle_f32_to_bf16.restype = ctypes.c_uint16
        L.es_oracle_f32_to_bf16.argtypes = [ctypes.c_float]
        L.es_oracle_bf16_to_f32.restype = ctypes.c_float
        L.es_oracle_bf16_to_f32.argtypes = [ctypes.c_uint16]
        _lib = L
    return _lib


def _code(dtype):
    """'f32' / 'bf16' / numpy dtype -> oracle dtype code.  bf16 arrays are uint16 bit patterns."""
    if dtype in ("f32", F32) or dtype == np.float32:
        return F32
    if dtype in ("bf16", BF16) or dtype == np.uint16:
        return BF16
    raise ValueError(f"unsupported dtype {dtype!r}")


def chunk_elems(L, N, A=16):
    """Reading R1: C = A * ceil(ceil(L/N)/A)."""
    return int(lib().es_oracle_chunk_elems(int(L), int(N), int(A)))


def reduce(xs, dtype, L=None, A=16, first=0):
    """Canonical fold + 1/N post-scale (readings R1-R6, R13).

    ``xs``: list of N contiguous arrays (float32, or uint16 bf16 bit patterns),
    EST k's contribution to elements [first, first+len) of a bucket of ``L``
    elements (L defaults to first+len).  Returns an array of the same dtype.
    """
    code = _code(dtype)
    N = len(xs)
    xs = [np.ascontiguousarray(x) for x in xs]
    count = xs[0].size
    for x in xs:
        assert x.size == count and x.dtype == xs[0].dtype
    if L is None:
        L = first + count
    out = np.empty(count, dtype=xs[0].dtype)
    ptrs = (ctypes.c_void_p * N)(*[x.ctypes.data for x in xs])
    rc = lib().es_oracle_reduce(N, int(L), int(A), code, ptrs, int(first), int(count),
                                out.ctypes.data)
    if rc != 0:
        raise ValueError("es_oracle_reduce: bad arguments")
    return out


COMPAT_PREDIV, COMPAT_PREMUL, COMPAT_BF16HOP = 1, 2, 4


def reduce_ex(xs, dtype, compat, L=None, A=16, first=0):
    """NEXT-3 compatibility variants (pre-divide, pre-multiply, per-hop bf16
    rounding) in the same canonical order; compat=0 equals reduce()."""
    code = _code(dtype)
    N = len(xs)
    xs = [np.ascontiguousarray(x) for x in xs]
    count = xs[0].size
    if L is None:
        L = first + count
    out = np.empty(count, dtype=xs[0].dtype)
    ptrs = (ctypes.c_void_p * N)(*[x.ctypes.data for x in xs])
    rc = lib().es_oracle_reduce_ex(N, int(L), int(A), code, int(compat), ptrs, int(first), int(count),
                                   out.ctypes.data)
    if rc != 0:
        raise ValueError("es_oracle_reduce_ex: bad arguments")
    return out


def philox4x32_10(ctr, key):
    c = (ctypes.c_uint32 * 4)(*ctr)
    k = (ctypes.c_uint32 * 2)(*key)
    o = (ctypes.c_uint32 * 4)()
    lib().es_oracle_philox4x32_10(c, k, o)
    return list(o)


def dropout(x, dtype, p, seed, offset):
    """NEXT-4 per-EST dropout (see es_oracle.c).  Returns (y, mask)."""
    code = _code(dtype)
    x = np.ascontiguousarray(x)
    y = np.empty_like(x)
    mask = np.empty(x.size, np.uint8)
    rc = lib().es_oracle_dropout(x.ctypes.data, y.ctypes.data, mask.ctypes.data, x.size, code, float(p),
                                 int(seed), int(offset))
    if rc != 0:
        raise ValueError("es_oracle_dropout: bad arguments")
    return y, mask


def stash(src, src_dtype, dst_dtype):
    """Stash = cast into the slot dtype (identity / exact widening / RNE)."""
    s, d = _code(src_dtype), _code(dst_dtype)
    src = np.ascontiguousarray(src)
    out = np.empty(src.size, dtype=np.float32 if d == F32 else np.uint16)
    rc = lib().es_oracle_stash(src.ctypes.data, s, out.ctypes.data, d, src.size)
    if rc != 0:
        raise ValueError("es_oracle_stash: bad arguments")
    return out


def f32_to_bf16_bits(a):
    """fp32 array -> bf16 bit patterns (uint16), RNE."""
    return stash(np.asarray(a, dtype=np.float32), F32, BF16)


def bf16_bits_to_f32(a):
    return stash(np.asarray(a, dtype=np.uint16), BF16, F32)
