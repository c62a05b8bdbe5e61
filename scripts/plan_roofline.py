"""Multi-GPU roofline of the ACTUAL plans (host-only, no GPU).

For every BASELINE config, G and schedule, export each rank's op list through
the C ABI (es_plan_ops) and count, per rank: bytes received over NVLink
(RECV ops, peer reads of PEER folds / chain partials, GATHER of remote
shards) and HBM bytes (fold reads/writes, staging writes, gathers).  The step
time bound is the slowest rank's max(HBM / 6.54 TB/s, NVLink / 0.77 TB/s);
chain rounds are separated by barriers, so for CHAIN / PEER_CHAIN the bound
is summed over rounds; the "pipelined" columns are the default executors
(PEER_CHAIN: k_fold_pipe's per-tile flags; CHAIN over NCCL: chain_pipelined's
tile wavefront on two streams), where every fold round and transfer overlaps
and only the all-gather follows.  Stash bytes are excluded (SURVEY 8(d):
allreduce only).  Writes profiles/r02_plan_roofline.md.

  python scripts/plan_roofline.py [out.md]
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads  # noqa: E402

HBM = 6455.6e9          # MEASURED_PEAKS hbm_gbs (copy), round 2
NVL = 770e9             # B200_PROFILING.md measured peer copy per direction
SCHEDS = {"direct": es.ES_SCHED_DIRECT, "chain": es.ES_SCHED_CHAIN, "peer": es.ES_SCHED_PEER,
          "peer_chain": es.ES_SCHED_PEER_CHAIN}


def rank_costs(name, G, kind, sched, push=False):
    """-> list over ranks of list over phases of (hbm_bytes, nvlink_in_bytes).
    push (ES_OPT_PEER_PUSH, PEER only): every owner's fold also writes its shard into each peer's
    RESULT area, so a rank's fold phase receives the other shards over NVLink and its gather
    phase is a local RESULT -> out copy."""
    c = workloads.config(name)
    N = c["N"]
    m = workloads.mapping(N, G, kind)
    buckets = [(n, es.ES_F32 if d == "f32" else es.ES_BF16) for n, d in c["buckets"]]
    out = []
    for g in range(G):
        cfg = es.Config(N, G, g, m, buckets, sched=sched)
        phases = {}
        for b, (L, dt) in enumerate(buckets):
            esz = 2 if dt == es.ES_BF16 else 4
            ops, _ = es.es_plan_ops(cfg, b)
            ph = 0
            for f in ops:
                op = int(f[0])
                if op in (es.ES_OP_BARRIER, es.ES_OP_GROUP_END):
                    ph += 1
                    continue
                hb, nv = phases.get(ph, (0, 0))
                lo, hi = int(f[1]), int(f[2])
                n = hi - lo
                if op == es.ES_OP_FOLD:
                    srcs = N if int(f[3]) < 0 else int(f[4])
                    remote = 0
                    if int(f[3]) < 0 and sched == es.ES_SCHED_PEER:
                        remote = sum(1 for e in range(N) if m[e] != g)
                    hb += n * esz * (srcs - remote)                        # local contributions
                    nv += n * esz * remote                                  # peer slots over NVLink
                    if int(f[5]) == es.ES_BUF_PART:
                        hb += n * 4
                    elif int(f[5]) == es.ES_BUF_PEER_PART:
                        nv += n * 4
                    hb += n * (4 if int(f[7]) == es.ES_BUF_PART else esz)   # write
                    if push and sched == es.ES_SCHED_PEER and int(f[7]) != es.ES_BUF_PART:
                        # the other owners' pushes land here in the same phase: L - own shard
                        nv += (L - n) * esz
                        hb += (L - n) * esz
                elif op == es.ES_OP_RECV:
                    w = 4 if int(f[4]) == es.ES_BUF_PART else esz
                    nv += n * w
                    hb += n * w
                elif op == es.ES_OP_GATHER and push and sched == es.ES_SCHED_PEER:
                    hb += 2 * n * esz                                       # own RESULT -> out
                elif op == es.ES_OP_GATHER:
                    if int(f[3]) != g:
                        nv += n * esz
                    hb += n * esz * (2 if int(f[3]) == g else 1)
                phases[ph] = (hb, nv)
        out.append(phases)
    return out


def bound_ms(costs):
    keys = sorted({k for r in costs for k in r})
    t = 0.0
    for k in keys:
        t += max(max(r[k][0] / HBM, r[k][1] / NVL) if k in r else 0.0 for r in costs)
    return t * 1e3


def bound_ms_pipelined(costs):
    """PEER_CHAIN as k_fold_pipe runs it: every fold round of a rank overlaps
    (per-tile flags, no barrier between rounds), so the folds are one phase;
    the gathers (the last phase) follow the closing barrier."""
    last = max(k for r in costs for k in r)
    merged = []
    for r in costs:
        hb = sum(v[0] for k, v in r.items() if k < last)
        nv = sum(v[1] for k, v in r.items() if k < last)
        merged.append({0: (hb, nv), 1: r.get(last, (0, 0))})
    return bound_ms(merged)


def next1_tail_saving(name, G, kind, sched):
    """NEXT-1 (es_plan_incremental): per rank, the end-of-step fold reads that move to the stashes
    -- q contributions per element of each row, less the fp32 partial read instead -- as a share of
    that rank's end-of-step fold reads; returns the slowest rank's (max fold bytes) saving."""
    c = workloads.config(name)
    N = c["N"]
    m = workloads.mapping(N, G, kind)
    buckets = [(n, es.ES_F32 if d == "f32" else es.ES_BF16) for n, d in c["buckets"]]
    worst = None
    for g in range(G):
        cfg = es.Config(N, G, g, m, buckets, sched=sched, options=es.ES_OPT_INCREMENTAL)
        fold = saved = 0
        for b, (L, dt) in enumerate(buckets):
            esz = 2 if dt == es.ES_BF16 else 4
            ops, _ = es.es_plan_ops(cfg, b)
            for f in ops:
                if int(f[0]) == es.ES_OP_FOLD:
                    fold += (int(f[2]) - int(f[1])) * esz * (N if int(f[3]) < 0 else int(f[4]))
            for _c, _first, q, lo, hi in es.es_plan_incremental(cfg, b).tolist():
                saved += (hi - lo) * (q * esz - 4)
        if worst is None or fold > worst[0]:
            worst = (fold, saved)
    return worst[1] / worst[0] if worst and worst[0] else 0.0


def main(path):
    rows = ["# Multi-GPU roofline of the exported plans (allreduce only; HBM 6.46 TB/s, NVLink 0.77 TB/s)\n",
            "Per phase (between groups / barriers), the slowest rank's max(HBM, NVLink) time, summed.\n",
            "peer_chain = rounds separated by barriers (ES_OPT_PEER_ROUNDS); pipelined = the default k_fold_pipe step "
            "(all rounds overlapped through per-tile flags, then the gather).\n",
            "peer push = ES_OPT_PEER_PUSH (the gather fused into the fold as NVLink stores): the same ingress bytes "
            "per rank move into the fold phase, so the bandwidth bound does not drop; what it removes is the "
            "gather's remote loads and one phase boundary (not modelled here).\n",
            "chain pipelined = CHAIN over NCCL as chain_pipelined runs it (tile wavefront: every round's folds "
            "and transfers overlapped, then the all-gather group).\n",
            "NEXT-1 = the share of the slowest rank's end-of-step fold reads that es_stash_fold_grads moves to the "
            "stashes (es_plan_incremental rows: q contributions per element, less the fp32 partial read), under "
            "the AUTO schedule.\n",
            "| config | G | mapping | direct ms | chain ms (rounds) | chain pipelined ms | peer ms | peer push ms | "
            "peer_chain ms | peer_chain pipelined ms | AUTO picks | max NVLink in / rank MB (direct, chain) | "
            "NEXT-1 tail reads moved |",
            "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    cases = [("resnet50", G, "contiguous") for G in (2, 4, 8)] + [("vgg19", G, "contiguous") for G in (2, 4, 8)] + \
        [("bert_base", 8, "contiguous"), ("bert_base", 8, "round_robin")] + \
        [("swin_b", G, "contiguous") for G in (2, 4, 8)]
    for name, G, kind in cases:
        res = {k: rank_costs(name, G, kind, v) for k, v in SCHEDS.items()}
        res["peer_push"] = rank_costs(name, G, kind, es.ES_SCHED_PEER, push=True)
        c = workloads.config(name)
        cfg = es.Config(c["N"], G, 0, workloads.mapping(c["N"], G, kind),
                        [(n, es.ES_F32 if d == "f32" else es.ES_BF16) for n, d in c["buckets"]])
        picks = sorted({es.es_plan_ops(cfg, b)[1] for b in range(len(c["buckets"]))})
        pick = "/".join({1: "direct", 2: "chain"}[p] for p in picks)
        nvd = max(sum(ph[1] for ph in r.values()) for r in res["direct"]) / 1e6
        nvc = max(sum(ph[1] for ph in r.values()) for r in res["chain"]) / 1e6
        rows.append(f"| {name} | {G} | {kind} | {bound_ms(res['direct']):.3f} | {bound_ms(res['chain']):.3f} | "
                    f"{bound_ms_pipelined(res['chain']):.3f} | "
                    f"{bound_ms(res['peer']):.3f} | {bound_ms(res['peer_push']):.3f} | {bound_ms(res['peer_chain']):.3f} | "
                    f"{bound_ms_pipelined(res['peer_chain']):.3f} | {pick} | {nvd:.0f}, {nvc:.0f} | "
                    f"{100 * next1_tail_saving(name, G, kind, es.ES_SCHED_AUTO):.0f} % |")
    g1 = ", ".join(f"{n} {100 * next1_tail_saving(n, 1, 'contiguous', es.ES_SCHED_AUTO):.0f} %"
                   for n in ("resnet50", "vgg19", "bert_base", "swin_b"))
    rows.append(f"\nNEXT-1 tail reads moved at G = 1 (same measure): {g1}.")
    text = "\n".join(rows) + "\n"
    with open(path, "w") as f:
        f.write(text)
    print(text)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "r02_plan_roofline.md"))
