"""Thin ctypes binding of libes (include/es.h): same names, argument
marshalling only.  Every step of the hot path runs in libes's CUDA kernels;
nothing here computes.  PyTorch is used only for device memory, streams and
process groups.

If libes.so is missing this module raises on first use -- there is no CPU
fallback (the product path must fail loudly without its CUDA extension).
"""
import ctypes
import os

import numpy as np

from . import _build

ES_OK, ES_EINVAL, ES_ESTATE, ES_ENOMEM, ES_ECUDA, ES_ENCCL, ES_EUNSUPPORTED = range(7)
ES_F32, ES_BF16 = 0, 1
ES_STASH_COPY, ES_STASH_BORROW, ES_STASH_INPLACE = 0, 1, 2
ES_SCHED_AUTO, ES_SCHED_DIRECT, ES_SCHED_CHAIN, ES_SCHED_PEER, ES_SCHED_PEER_CHAIN, ES_SCHED_PEER_AUTO = range(6)
PEER_SCHEDS = (ES_SCHED_PEER, ES_SCHED_PEER_CHAIN, ES_SCHED_PEER_AUTO)
ES_TRANSPORT_NONE, ES_TRANSPORT_NCCL, ES_TRANSPORT_LOOPBACK = 0, 1, 2
ES_KERNEL_STASH, ES_KERNEL_FOLD, ES_KERNEL_SWAP, ES_KERNEL_DROPOUT, ES_KERNEL_GATHER, ES_KERNEL_BARRIER = range(6)
ES_OP_FIELDS = 10
ES_OP_FOLD, ES_OP_SEND, ES_OP_RECV, ES_OP_GROUP_BEGIN, ES_OP_GROUP_END, ES_OP_BARRIER, ES_OP_GATHER = range(1, 8)
ES_BUF_NONE, ES_BUF_SRC, ES_BUF_STAGE, ES_BUF_PART, ES_BUF_OUT, ES_BUF_RESULT, ES_BUF_PEER_PART = range(7)
ES_PEER_BLOB_BYTES = 128
ES_COMPAT_PREDIV, ES_COMPAT_PREMUL, ES_COMPAT_BF16_HOP = 1, 2, 4
ES_OPT_INCREMENTAL = 1
ES_OPT_PEER_ROUNDS = 2
ES_OPT_STASH_BACKGROUND = 4
ES_OPT_PEER_PUSH = 8

EXPORTED = [
    "es_workspace_bytes", "es_init", "es_destroy", "es_sync", "es_register_state", "es_init_state",
    "es_read_state", "es_switch_context", "es_stash_grad", "es_stash_grads", "es_stash_and_switch", "es_stash_fold_grads", "es_allreduce",
    "es_allreduce_many", "es_chunk_elems", "es_slot_ptr", "es_context_bytes", "es_export_context",
    "es_import_context", "es_dropout", "es_peer_blob", "es_peer_open",
    "es_plan_ops", "es_plan_incremental", "es_loopback_create", "es_loopback_destroy", "es_profile_enable",
    "es_profile_reset", "es_profile_query", "es_set_launch_override", "es_status_string",
    "es_last_error", "es_abi_version",
]


class EsError(RuntimeError):
    def __init__(self, status, fn, detail):
        self.status = status
        super().__init__(f"{fn}: status {status} ({detail})")


class es_bucket_desc(ctypes.Structure):
    _fields_ = [("numel", ctypes.c_uint64), ("dtype", ctypes.c_int)]


class es_config(ctypes.Structure):
    _fields_ = [
        ("N", ctypes.c_int32), ("G", ctypes.c_int32), ("rank", ctypes.c_int32),
        ("est_to_gpu", ctypes.POINTER(ctypes.c_int32)),
        ("buckets", ctypes.POINTER(es_bucket_desc)), ("n_buckets", ctypes.c_int32),
        ("chunk_align", ctypes.c_uint32),
        ("n_state", ctypes.c_int32), ("state_nbytes", ctypes.POINTER(ctypes.c_uint64)),
        ("transport", ctypes.c_int), ("comm", ctypes.c_void_p), ("sched", ctypes.c_int),
        ("compat", ctypes.c_uint32), ("options", ctypes.c_uint32),
    ]


_lib = None


def lib_path():
    return _build.LIB


def lib():
    """Loads libes.so (raises if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_build.LIB):
        raise RuntimeError(f"{_build.LIB} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = ctypes.CDLL(_build.LIB)
    st = ctypes.c_int
    P = ctypes.c_void_p
    i32, u32, u64, i64, sz = ctypes.c_int32, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int64, ctypes.c_size_t
    cfgp = ctypes.POINTER(es_config)
    sig = {
        "es_workspace_bytes": (st, [cfgp, ctypes.POINTER(sz)]),
        "es_init": (st, [cfgp, P, sz, ctypes.POINTER(P)]),
        "es_destroy": (st, [P]),
        "es_sync": (st, [P]),
        "es_register_state": (st, [P, i32, ctypes.POINTER(P)]),
        "es_init_state": (st, [P, i32, i32, P]),
        "es_read_state": (st, [P, i32, i32, P]),
        "es_switch_context": (st, [P, i32, P]),
        "es_stash_grad": (st, [P, i32, i32, P, ctypes.c_int, ctypes.c_int, P]),
        "es_allreduce": (st, [P, i32, P, P]),
        "es_stash_grads": (st, [P, i32, i32, ctypes.POINTER(i32), ctypes.POINTER(P), ctypes.POINTER(ctypes.c_int),
                                ctypes.c_int, P]),
        "es_allreduce_many": (st, [P, i32, ctypes.POINTER(i32), ctypes.POINTER(P), P]),
        "es_stash_and_switch": (st, [P, i32, i32, ctypes.POINTER(i32), ctypes.POINTER(P),
                                     ctypes.POINTER(ctypes.c_int), ctypes.c_int, i32, P]),
        "es_stash_fold_grads": (st, [P, i32, i32, ctypes.POINTER(i32), ctypes.POINTER(P),
                                     ctypes.POINTER(ctypes.c_int), ctypes.c_int, P]),
        "es_chunk_elems": (u64, [u64, i32, u32]),
        "es_slot_ptr": (st, [P, i32, i32, ctypes.POINTER(P)]),
        "es_dropout": (st, [P, P, P, P, u64, ctypes.c_int, ctypes.c_float, i32, P]),
        "es_peer_blob": (st, [P, P, sz]),
        "es_peer_open": (st, [P, P, sz]),
        "es_context_bytes": (st, [P, ctypes.POINTER(sz)]),
        "es_export_context": (st, [P, i32, P, sz, P]),
        "es_import_context": (st, [P, i32, P, sz, P]),
        "es_plan_ops": (st, [cfgp, i32, ctypes.POINTER(i64), sz, ctypes.POINTER(sz), ctypes.POINTER(i32)]),
        "es_plan_incremental": (st, [cfgp, i32, ctypes.POINTER(i64), sz, ctypes.POINTER(sz)]),
        "es_loopback_create": (st, [i32, ctypes.POINTER(P)]),
        "es_loopback_destroy": (st, [P]),
        "es_profile_enable": (st, [P, i32]),
        "es_profile_reset": (st, [P]),
        "es_profile_query": (st, [P, ctypes.c_int, ctypes.POINTER(u64), ctypes.POINTER(ctypes.c_double),
                                  ctypes.POINTER(u64)]),
        "es_set_launch_override": (st, [P, i32, i32]),
        "es_status_string": (ctypes.c_char_p, [st]),
        "es_last_error": (ctypes.c_char_p, []),
        "es_abi_version": (i32, []),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


def _check(status, fn):
    if status != ES_OK:
        raise EsError(status, fn, lib().es_last_error().decode(errors="replace"))


class Config:
    """Owns an es_config and the host arrays it points to."""

    def __init__(self, N, G, rank, est_to_gpu, buckets, chunk_align=16, state_nbytes=(),
                 transport=ES_TRANSPORT_NONE, comm=None, sched=ES_SCHED_AUTO, compat=0, options=0):
        self.N, self.G, self.rank = int(N), int(G), int(rank)
        self.est_to_gpu = list(int(g) for g in est_to_gpu)
        self.buckets = [(int(n), int(d)) for n, d in buckets]
        self._map = (ctypes.c_int32 * len(self.est_to_gpu))(*self.est_to_gpu)
        self._bk = (es_bucket_desc * len(self.buckets))(*[es_bucket_desc(n, d) for n, d in self.buckets])
        self._sn = (ctypes.c_uint64 * max(len(state_nbytes), 1))(*state_nbytes)
        self.state_nbytes = list(state_nbytes)
        self.c = es_config(self.N, self.G, self.rank, self._map, self._bk, len(self.buckets), int(chunk_align),
                           len(state_nbytes), self._sn, int(transport), comm, int(sched), int(compat),
                           int(options))

    def ptr(self):
        return ctypes.byref(self.c)


# ---- same-name wrappers -------------------------------------------------------

def es_workspace_bytes(cfg):
    n = ctypes.c_size_t()
    _check(lib().es_workspace_bytes(cfg.ptr(), ctypes.byref(n)), "es_workspace_bytes")
    return n.value


def es_init(cfg, workspace_ptr, nbytes):
    h = ctypes.c_void_p()
    _check(lib().es_init(cfg.ptr(), ctypes.c_void_p(workspace_ptr), nbytes, ctypes.byref(h)), "es_init")
    return h


def es_destroy(h):
    _check(lib().es_destroy(h), "es_destroy")


def es_sync(h):
    _check(lib().es_sync(h), "es_sync")


def es_register_state(h, live_ptrs):
    arr = (ctypes.c_void_p * max(len(live_ptrs), 1))(*live_ptrs)
    _check(lib().es_register_state(h, len(live_ptrs), arr), "es_register_state")


def es_init_state(h, est, idx, data):
    buf = ctypes.create_string_buffer(bytes(data), len(data))
    _check(lib().es_init_state(h, est, idx, buf), "es_init_state")


def es_read_state(h, est, idx, nbytes):
    buf = ctypes.create_string_buffer(nbytes)
    _check(lib().es_read_state(h, est, idx, buf), "es_read_state")
    return buf.raw


def es_switch_context(h, est, stream):
    _check(lib().es_switch_context(h, est, ctypes.c_void_p(stream)), "es_switch_context")


def es_stash_grad(h, est, bucket, grad_ptr, grad_dtype, mode, stream):
    _check(lib().es_stash_grad(h, est, bucket, ctypes.c_void_p(grad_ptr), grad_dtype, mode,
                               ctypes.c_void_p(stream)), "es_stash_grad")


def es_allreduce(h, bucket, out_ptr, stream):
    _check(lib().es_allreduce(h, bucket, ctypes.c_void_p(out_ptr), ctypes.c_void_p(stream)), "es_allreduce")


def es_stash_grads(h, est, buckets, grad_ptrs, grad_dtypes, mode, stream):
    n = len(buckets)
    b = (ctypes.c_int32 * max(n, 1))(*buckets)
    g = (ctypes.c_void_p * max(n, 1))(*grad_ptrs)
    d = (ctypes.c_int * max(n, 1))(*grad_dtypes)
    _check(lib().es_stash_grads(h, est, n, b, g, d, mode, ctypes.c_void_p(stream)), "es_stash_grads")


def es_stash_and_switch(h, est, buckets, grad_ptrs, grad_dtypes, mode, next_est, stream):
    n = len(buckets)
    b = (ctypes.c_int32 * max(n, 1))(*buckets)
    g = (ctypes.c_void_p * max(n, 1))(*grad_ptrs)
    d = (ctypes.c_int * max(n, 1))(*grad_dtypes)
    _check(lib().es_stash_and_switch(h, est, n, b, g, d, mode, next_est, ctypes.c_void_p(stream)),
           "es_stash_and_switch")


def es_stash_fold_grads(h, est, buckets, grad_ptrs, grad_dtypes, mode, stream):
    n = len(buckets)
    b = (ctypes.c_int32 * max(n, 1))(*buckets)
    g = (ctypes.c_void_p * max(n, 1))(*grad_ptrs)
    d = (ctypes.c_int * max(n, 1))(*grad_dtypes)
    _check(lib().es_stash_fold_grads(h, est, n, b, g, d, mode, ctypes.c_void_p(stream)), "es_stash_fold_grads")


def es_allreduce_many(h, buckets, out_ptrs, stream):
    n = len(buckets)
    b = (ctypes.c_int32 * max(n, 1))(*buckets)
    o = (ctypes.c_void_p * max(n, 1))(*out_ptrs)
    _check(lib().es_allreduce_many(h, n, b, o, ctypes.c_void_p(stream)), "es_allreduce_many")


def es_slot_ptr(h, est, bucket):
    p = ctypes.c_void_p()
    _check(lib().es_slot_ptr(h, est, bucket, ctypes.byref(p)), "es_slot_ptr")
    return p.value


def es_context_bytes(h):
    n = ctypes.c_size_t()
    _check(lib().es_context_bytes(h, ctypes.byref(n)), "es_context_bytes")
    return n.value


def es_export_context(h, est, stream):
    n = es_context_bytes(h)
    buf = ctypes.create_string_buffer(n)
    _check(lib().es_export_context(h, est, buf, n, ctypes.c_void_p(stream)), "es_export_context")
    return buf.raw


def es_import_context(h, est, blob, stream):
    buf = ctypes.create_string_buffer(bytes(blob), len(blob))
    _check(lib().es_import_context(h, est, buf, len(blob), ctypes.c_void_p(stream)), "es_import_context")


def es_dropout(h, x_ptr, y_ptr, mask_ptr, n, dtype, p, state_idx, stream):
    _check(lib().es_dropout(h, ctypes.c_void_p(x_ptr), ctypes.c_void_p(y_ptr), ctypes.c_void_p(mask_ptr), n, dtype,
                            float(p), state_idx, ctypes.c_void_p(stream)), "es_dropout")


def es_peer_blob(h):
    buf = ctypes.create_string_buffer(ES_PEER_BLOB_BYTES)
    _check(lib().es_peer_blob(h, buf, ES_PEER_BLOB_BYTES), "es_peer_blob")
    return buf.raw


def es_peer_open(h, blobs):
    data = b"".join(blobs)
    buf = ctypes.create_string_buffer(data, len(data))
    _check(lib().es_peer_open(h, buf, len(data)), "es_peer_open")


def es_chunk_elems(L, N, A=16):
    return int(lib().es_chunk_elems(L, N, A))


def es_plan_ops(cfg, bucket):
    """-> (int64 array [n_ops, ES_OP_FIELDS], sched)."""
    n = ctypes.c_size_t()
    sched = ctypes.c_int32()
    _check(lib().es_plan_ops(cfg.ptr(), bucket, None, 0, ctypes.byref(n), ctypes.byref(sched)), "es_plan_ops")
    ops = np.zeros((max(n.value, 1), ES_OP_FIELDS), dtype=np.int64)
    _check(lib().es_plan_ops(cfg.ptr(), bucket, ops.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)), n.value,
                             ctypes.byref(n), ctypes.byref(sched)), "es_plan_ops")
    return ops[: n.value], sched.value


def es_plan_incremental(cfg, bucket):
    """-> int64 array [n_rows, 5]: (c, first, q, lo, hi) per chunk with an incremental prefix."""
    n = ctypes.c_size_t()
    _check(lib().es_plan_incremental(cfg.ptr(), bucket, None, 0, ctypes.byref(n)), "es_plan_incremental")
    rows = np.zeros((max(n.value, 1), 5), dtype=np.int64)
    _check(lib().es_plan_incremental(cfg.ptr(), bucket, rows.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                     n.value, ctypes.byref(n)), "es_plan_incremental")
    return rows[: n.value]


def es_loopback_create(G):
    w = ctypes.c_void_p()
    _check(lib().es_loopback_create(G, ctypes.byref(w)), "es_loopback_create")
    return w


def es_loopback_destroy(w):
    _check(lib().es_loopback_destroy(w), "es_loopback_destroy")


def es_profile_enable(h, on):
    _check(lib().es_profile_enable(h, 1 if on else 0), "es_profile_enable")


def es_profile_reset(h):
    _check(lib().es_profile_reset(h), "es_profile_reset")


def es_profile_query(h, kind):
    """-> (launches, ms, algorithmic bytes)."""
    n, b = ctypes.c_uint64(), ctypes.c_uint64()
    ms = ctypes.c_double()
    _check(lib().es_profile_query(h, kind, ctypes.byref(n), ctypes.byref(ms), ctypes.byref(b)), "es_profile_query")
    return n.value, ms.value, b.value


def es_set_launch_override(h, blocks, threads):
    _check(lib().es_set_launch_override(h, blocks, threads), "es_set_launch_override")


def es_status_string(s):
    return lib().es_status_string(s).decode()


def es_last_error():
    return lib().es_last_error().decode(errors="replace")


def es_abi_version():
    return int(lib().es_abi_version())
