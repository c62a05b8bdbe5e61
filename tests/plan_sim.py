"""Host replay of libes's plan (schedule simulator).

For each rank, the op list the GPU path executes is exported through the C
ABI (es_plan_ops, host-only) and replayed here with NumPy float32 folds and
an in-process mailbox (or a torch.distributed gloo transport).  This checks
the planner -- chunk coverage, canonical order of every segment, message
matching, staging and partial buffers -- for any G and mapping without a
GPU.  Test infrastructure only."""
import collections

import numpy as np
import torch

from paper_conf_sc_lixyszrljlllq23_b200 import es


def widen(a):
    a = np.asarray(a)
    if a.dtype == np.float32:
        return a
    return (a.astype(np.uint32) << 16).view(np.float32)


def narrow(a32, dtype):
    if dtype == "f32":
        return a32.astype(np.float32)
    return torch.from_numpy(np.ascontiguousarray(a32, dtype=np.float32)).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)


class RankExec:
    """Replays one rank's plan.  xs[b][e] is EST e's bucket b (only local ESTs used)."""

    def __init__(self, N, G, rank, mapping, buckets, xs, A=16, sched=es.ES_SCHED_AUTO):
        self.N, self.G, self.g, self.map, self.A = N, G, rank, list(mapping), A
        self.buckets = buckets
        self.xs = xs
        cfg = es.Config(N, G, rank, mapping, [(L, es.ES_F32 if d == "f32" else es.ES_BF16) for L, d in buckets], A,
                        sched=sched)
        self.plans = [es.es_plan_ops(cfg, b) for b in range(len(buckets))]
        self.sched = sched
        self.out = [np.zeros(L, np.float32 if d == "f32" else np.uint16) for L, d in buckets]
        self.result = [np.zeros(L, np.float32 if d == "f32" else np.uint16) for L, d in buckets]   # PEER
        self.peer_parts = {}        # PEER_CHAIN: byte offset -> (lo, fp32 partial), read by the next GPU
        self.world = [self]
        self.nbar = 0
        self.b = 0
        self.pc = 0
        self.stage = {}
        self.parts = {}
        self.group = None
        self.log = collections.Counter()

    def done(self):
        return self.b >= len(self.buckets)

    def _src(self, e, lo, hi):
        b = self.b
        if self.map[e] == self.g or self.plans[b][1] in (es.ES_SCHED_PEER, es.ES_SCHED_PEER_CHAIN):
            return self.xs[b][e][lo:hi]          # local slot, or (PEER) the owner's slot over NVLink
        slo, arr = self.stage[e]
        assert slo <= lo and hi <= slo + arr.size, "staging does not cover the fold range"
        return arr[lo - slo:hi - slo]

    def _fold(self, f):
        lo, hi, e0, m, ink, inid, outk, outid = (int(v) for v in f[1:9])
        L, d = self.buckets[self.b]
        C = es.es_chunk_elems(L, self.N, self.A)
        if e0 < 0:
            assert m == self.N
            pieces = []
            c0, c1 = lo // C, (hi - 1) // C
            for c in range(c0, c1 + 1):
                a, z = max(lo, c * C), min(hi, (c + 1) * C)
                pieces.append((a, z, [(c + j) % self.N for j in range(1, self.N + 1)]))
        else:
            order = [(e0 + j) % self.N for j in range(m)]
            assert all(self.map[e] == self.g for e in order), "chain segment uses a non-local EST"
            c = lo // C
            assert lo == c * C and hi == min(L, (c + 1) * C), "chain segment is not one chunk"
            want = [(c + j) % self.N for j in range(1, self.N + 1)]
            assert order == want[want.index(order[0]):want.index(order[0]) + m], "segment not in canonical order"
            pieces = [(lo, hi, order)]
        for a, z, order in pieces:
            if ink == es.ES_BUF_PART:
                plo, parr = self.parts[inid]
                acc = parr[a - plo:z - plo].copy()
                rest = order
            elif ink == es.ES_BUF_PEER_PART:      # producer rank inid, byte offset f[9]
                plo, parr = self.world[inid].peer_parts[int(f[9])]
                acc = parr[a - plo:z - plo].copy()
                rest = order
            else:
                acc = widen(self._src(order[0], a, z)).copy()
                rest = order[1:]
            for e in rest:
                acc = (acc + widen(self._src(e, a, z))).astype(np.float32)
            if outk == es.ES_BUF_RESULT:
                r = np.float32(1) / np.float32(self.N)
                self.result[self.b][a:z] = narrow(acc * r, d)
            elif outk == es.ES_BUF_PART and self.plans[self.b][1] == es.ES_SCHED_PEER_CHAIN:
                self.peer_parts[outid] = (lo, acc.copy())
            elif outk == es.ES_BUF_PART:
                if outid not in self.parts:
                    self.parts[outid] = (lo, np.zeros(hi - lo, np.float32))
                plo, parr = self.parts[outid]
                parr[a - plo:z - plo] = acc
            else:
                r = np.float32(1) / np.float32(self.N)
                self.out[self.b][a:z] = narrow(acc * r, d)
        self.log["fold"] += 1

    def _payload(self, f):
        lo, hi, peer, kind, bid = (int(v) for v in f[1:6])
        if kind == es.ES_BUF_SRC:
            assert self.map[bid] == self.g
            return self.xs[self.b][bid][lo:hi].copy()
        if kind == es.ES_BUF_PART:
            plo, parr = self.parts[bid]
            return parr[lo - plo:hi - plo].copy()
        if kind == es.ES_BUF_OUT:
            return self.out[self.b][lo:hi].copy()
        raise AssertionError("bad send buffer kind")

    def _deliver(self, f, data):
        lo, hi, peer, kind, bid = (int(v) for v in f[1:6])
        assert data.size == hi - lo, "message size mismatch"
        if kind == es.ES_BUF_STAGE:
            self.stage[bid] = (lo, data)
        elif kind == es.ES_BUF_PART:
            self.parts[bid] = (lo, data.astype(np.float32))
        elif kind == es.ES_BUF_OUT:
            self.out[self.b][lo:hi] = data
        else:
            raise AssertionError("bad recv buffer kind")

    def run(self, transport):
        """Advance until blocked or done.  Returns True if progress was made."""
        progressed = False
        while not self.done():
            ops, _ = self.plans[self.b]
            if self.pc >= len(ops):
                self.b += 1
                self.pc = 0
                self.stage, self.parts = {}, {}
                # peer_parts survive until every rank passed the next barrier; keep them (offsets are reused
                # per bucket, and a bucket's consumers read them before the bucket's next barrier)
                progressed = True
                continue
            f = ops[self.pc]
            op = int(f[0])
            if op == es.ES_OP_FOLD:
                self._fold(f)
                self.pc += 1
            elif op == es.ES_OP_BARRIER:
                if not transport.barrier(self):
                    return progressed
                self.pc += 1
            elif op == es.ES_OP_GATHER:
                lo, hi, owner = int(f[1]), int(f[2]), int(f[3])
                self.out[self.b][lo:hi] = transport.ranks[owner].result[self.b][lo:hi]
                self.pc += 1
            elif op == es.ES_OP_GROUP_BEGIN:
                end = self.pc + 1
                while int(ops[end][0]) != es.ES_OP_GROUP_END:
                    end += 1
                body = ops[self.pc + 1:end]
                if not transport.group(self, body):
                    return progressed
                self.pc = end + 1
            else:
                raise AssertionError(f"unexpected op {op} outside a group")
            progressed = True
        return progressed


class Mailbox:
    """In-process transport: NCCL-like per-(src, dst) FIFO matching."""

    def __init__(self, ranks=()):
        self.q = collections.defaultdict(collections.deque)
        self.posted = {}
        self.ranks = list(ranks)
        self.arrived = collections.Counter()

    def barrier(self, ex):
        """PEER barrier: passes once every rank has arrived at its n-th barrier."""
        key = ex.nbar
        if not getattr(ex, "_at_barrier", False):
            self.arrived[key] += 1
            ex._at_barrier = True
        if self.arrived[key] < len(self.ranks):
            return False
        ex._at_barrier = False
        ex.nbar += 1
        return True

    def group(self, ex, body):
        key = (ex.g, ex.b, ex.pc)
        if key not in self.posted:
            for f in body:
                if int(f[0]) == es.ES_OP_SEND:
                    self.q[(ex.g, int(f[3]))].append((int(f[1]), int(f[2]), ex._payload(f)))
            self.posted[key] = 0
        recvs = [f for f in body if int(f[0]) == es.ES_OP_RECV]
        i = self.posted[key]
        while i < len(recvs):
            f = recvs[i]
            q = self.q[(int(f[3]), ex.g)]
            if not q:
                self.posted[key] = i
                return False
            lo, hi, data = q.popleft()
            assert (lo, hi) == (int(f[1]), int(f[2])), "send/recv ranges do not match"
            ex._deliver(f, data)
            i += 1
        del self.posted[key]
        return True


def simulate(N, G, mapping, buckets, xs, A=16, sched=es.ES_SCHED_AUTO):
    ranks = [RankExec(N, G, g, mapping, buckets, xs, A, sched) for g in range(G)]
    for r in ranks:
        r.world = ranks
    box = Mailbox(ranks)
    while not all(r.done() for r in ranks):
        if not any(r.run(box) for r in ranks if not r.done()):
            raise AssertionError("deadlock: no rank can progress")
    assert all(not q for q in box.q.values()), "unreceived messages"
    return ranks
