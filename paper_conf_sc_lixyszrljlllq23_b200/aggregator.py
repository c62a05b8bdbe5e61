"""Torch-facing wrapper of the libes C ABI (marshalling only).

``Aggregator`` is one rank's handle: it allocates the workspace with
PyTorch's allocator (the library never calls cudaMalloc), passes tensor
pointers and the current CUDA stream through, and keeps the host-side
mirror of torch's Philox generator state per EST (reading R12).
"""
import torch

from . import es

DTYPES = {torch.float32: es.ES_F32, torch.bfloat16: es.ES_BF16, "f32": es.ES_F32, "bf16": es.ES_BF16,
          es.ES_F32: es.ES_F32, es.ES_BF16: es.ES_BF16}
TORCH_DTYPES = {es.ES_F32: torch.float32, es.ES_BF16: torch.bfloat16}


def _stream(stream):
    if stream is None:
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, torch.cuda.Stream):
        return stream.cuda_stream
    return int(stream)


def nccl_comm_ptr(group=None):
    """ncclComm_t of a torch ProcessGroupNCCL (after at least one collective)."""
    import torch.distributed as dist
    group = group or dist.group.WORLD
    backend = group._get_backend(torch.device("cuda"))
    return int(backend._comm_ptr())


class Aggregator:
    """One rank of the placement-invariant EST gradient aggregator.

    buckets: list of (numel, dtype) with dtype torch.float32/bfloat16 or 'f32'/'bf16'.
    """

    def __init__(self, N, G, rank, est_to_gpu, buckets, chunk_align=16, state_nbytes=(),
                 transport=None, comm=None, sched=es.ES_SCHED_AUTO, device=None, compat=0, options=0):
        if transport is None:
            transport = es.ES_TRANSPORT_NONE if G == 1 else es.ES_TRANSPORT_NCCL
        self.buckets = [(int(n), DTYPES[d]) for n, d in buckets]
        self.cfg = es.Config(N, G, rank, est_to_gpu, self.buckets, chunk_align, tuple(state_nbytes),
                             transport, comm, sched, compat, options)
        self.N, self.G, self.rank = N, G, rank
        self.local_ests = [e for e in range(N) if est_to_gpu[e] == rank]
        self.device = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.ws_bytes = es.es_workspace_bytes(self.cfg)
        self.workspace = torch.empty(max(self.ws_bytes, 256), dtype=torch.uint8, device=self.device)
        if self.workspace.data_ptr() % 256:
            raise RuntimeError("workspace not 256-byte aligned")
        with torch.cuda.device(self.device):
            self.h = es.es_init(self.cfg, self.workspace.data_ptr(), self.workspace.numel())
        self._live = None
        self._gen = None
        self._philox = {}
        self._cur = None

    # ---- context state -------------------------------------------------------------
    def register_state(self, tensors):
        """Live per-EST context buffers (Philox record, BN running stats), in
        the order of state_nbytes."""
        self._live = list(tensors)
        es.es_register_state(self.h, [t.data_ptr() for t in self._live])

    def init_state(self, est, idx, data):
        if isinstance(data, torch.Tensor):
            data = data.detach().cpu().contiguous().view(torch.uint8).numpy().tobytes()
        es.es_init_state(self.h, est, idx, data)

    def read_state(self, est, idx):
        return es.es_read_state(self.h, est, idx, self.cfg.state_nbytes[idx])

    def attach_generator(self, gen, seeds):
        """Keep torch generator `gen` in step with the running EST: EST k
        starts from manual_seed(seeds[k]) with offset 0 (D0 fixed seeds,
        PAPER.md:751-757)."""
        self._gen = gen
        self._philox = {k: (int(seeds[k]), 0) for k in self.local_ests}

    def switch(self, est, stream=None):
        es.es_switch_context(self.h, est, _stream(stream))
        self._mirror_generator(est)

    def _mirror_generator(self, est):
        if self._gen is not None and est != self._cur:
            if self._cur is not None:
                self._philox[self._cur] = (self._gen.initial_seed(), self._gen.get_offset())
            seed, off = self._philox[est]
            self._gen.manual_seed(seed)
            self._gen.set_offset(off)
        self._cur = est

    # ---- stash / aggregate ------------------------------------------------------------
    def stash(self, est, bucket, grad, mode=es.ES_STASH_COPY, stream=None):
        es.es_stash_grad(self.h, est, bucket, grad.data_ptr(), DTYPES[grad.dtype], mode, _stream(stream))

    def stash_many(self, est, buckets, grads, mode=es.ES_STASH_COPY, stream=None):
        """All of EST `est`'s buckets in one call (one multi-segment launch)."""
        es.es_stash_grads(self.h, est, list(buckets), [g.data_ptr() for g in grads],
                          [DTYPES[g.dtype] for g in grads], mode, _stream(stream))

    def stash_and_switch(self, est, buckets, grads, next_est, mode=es.ES_STASH_COPY, stream=None):
        """EST `est` finished its local step: stash its buckets and switch to
        `next_est` in one launch."""
        es.es_stash_and_switch(self.h, est, list(buckets), [g.data_ptr() for g in grads],
                               [DTYPES[g.dtype] for g in grads], mode, next_est, _stream(stream))
        self._mirror_generator(next_est)

    def stash_fold(self, est, buckets, grads, mode=es.ES_STASH_COPY, stream=None):
        """NEXT-1: fold EST `est` into the running partials now, stash the rest."""
        es.es_stash_fold_grads(self.h, est, list(buckets), [g.data_ptr() for g in grads],
                               [DTYPES[g.dtype] for g in grads], mode, _stream(stream))

    def allreduce_many(self, buckets, outs, stream=None):
        es.es_allreduce_many(self.h, list(buckets), [o.data_ptr() for o in outs], _stream(stream))
        return outs

    def allreduce(self, bucket, out, stream=None):
        es.es_allreduce(self.h, bucket, out.data_ptr(), _stream(stream))
        return out

    def new_out(self, bucket):
        n, d = self.buckets[bucket]
        return torch.empty(n, dtype=TORCH_DTYPES[d], device=self.device)

    # ---- peer memory (ES_SCHED_PEER) ----------------------------------------------------
    def peer_blob(self):
        return es.es_peer_blob(self.h)

    def peer_open(self, blobs):
        """blobs: every rank's peer_blob(), in rank order."""
        es.es_peer_open(self.h, list(blobs))

    def peer_connect(self, group=None):
        """All-gather the peer blobs over torch.distributed and map the peers."""
        import torch.distributed as dist
        blobs = [None] * self.G
        dist.all_gather_object(blobs, self.peer_blob(), group=group)
        self.peer_open(blobs)

    # ---- per-EST dropout (NEXT-4) ---------------------------------------------------------
    def dropout(self, x, p, state_idx=0, with_mask=False, stream=None):
        """Dropout of the running EST from its device Philox record."""
        y = torch.empty_like(x)
        mask = torch.empty(x.numel(), dtype=torch.uint8, device=x.device) if with_mask else None
        es.es_dropout(self.h, x.data_ptr(), y.data_ptr(), mask.data_ptr() if mask is not None else 0, x.numel(),
                      DTYPES[x.dtype], p, state_idx, _stream(stream))
        return (y, mask) if with_mask else y

    # ---- zero-copy slots / elastic resume (NEXT-2) ------------------------------------
    def slot(self, est, bucket):
        """Tensor view of local EST `est`'s slot for `bucket` (bind gradients here,
        then stash with ES_STASH_INPLACE: no bytes move)."""
        ptr = es.es_slot_ptr(self.h, est, bucket)
        n, d = self.buckets[bucket]
        off = ptr - self.workspace.data_ptr()
        esz = 2 if d == es.ES_BF16 else 4
        return self.workspace[off:off + n * esz].view(TORCH_DTYPES[d])

    def export_context(self, est, stream=None):
        return es.es_export_context(self.h, est, _stream(stream))

    def import_context(self, est, blob, stream=None):
        es.es_import_context(self.h, est, blob, _stream(stream))

    def sync(self):
        es.es_sync(self.h)

    # ---- instrumentation -------------------------------------------------------------
    def profile(self, on=True):
        es.es_profile_enable(self.h, on)

    def profile_reset(self):
        es.es_profile_reset(self.h)

    def profile_query(self, kind):
        return es.es_profile_query(self.h, kind)

    def set_launch_override(self, blocks, threads):
        es.es_set_launch_override(self.h, blocks, threads)

    def close(self):
        if getattr(self, "h", None) is not None:
            es.es_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
