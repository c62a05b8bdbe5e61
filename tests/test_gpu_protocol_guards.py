"""GPU: protocol guards of the C ABI.

* es_export_context refuses (ES_ESTATE) an EST whose bucket is being folded
  incrementally (NEXT-1, COPY mode): its slot holds only the chunks that wait
  for the wrap, the rest lives in the fp32 partials; exporting it would write
  stale bytes marked as stashed (R17: a context is the EST's whole gradient).
  EST 0 and a BORROWed EST are exportable; import refuses to bypass partials.
* es_peer_open refuses (ES_EINVAL) blobs from ranks whose plan differs (options,
  schedule, mapping...): mismatched executors would wait on barriers the others
  never reach or gather results nobody pushed.
"""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_sc_lixyszrljlllq23_b200 import es

from gpu_util import Aggregator, assert_bits_equal, from_dev, to_dev

pytestmark = pytest.mark.gpu


def test_export_refuses_partially_folded_slot():
    """NEXT-1 (es_stash_fold_grads) at G = 1, N = 4: EST 0 opens chunk 3's partial (its
    sequence 0, 1, 2, 3 starts there), EST 1 folds into chunk 3 and opens chunk 0's, EST 2 folds
    into both (chunk 1's one-EST prefix is not worth a partial); EST 3, the last local EST, folds
    nothing and its COPY slot holds its whole gradient."""
    N, L = 4, 100003
    agg = Aggregator(N, 1, 0, [0] * N, [(L, "f32")], options=es.ES_OPT_INCREMENTAL)
    rng = np.random.default_rng(5)
    xs = [(rng.standard_normal(L) * 1e-2).astype(np.float32) for _ in range(N)]
    d = [to_dev(x) for x in xs]
    agg.stash_fold(0, [0], [d[0]], es.ES_STASH_COPY)
    agg.stash_fold(1, [0], [d[1]], es.ES_STASH_COPY)
    for e in (0, 1):                                          # partly folded: the slot is not the gradient
        with pytest.raises(es.EsError) as ei:
            agg.export_context(e)
        assert ei.value.status == es.ES_ESTATE
    agg.stash_fold(2, [0], [d[2]], es.ES_STASH_COPY)
    agg.stash_fold(3, [0], [d[3]], es.ES_STASH_COPY)
    blob3 = agg.export_context(3)                             # nothing folded: exportable
    with pytest.raises(es.EsError) as ei:                     # importing would bypass the partials
        agg.import_context(3, blob3)
    assert ei.value.status == es.ES_ESTATE
    out = agg.new_out(0)
    agg.allreduce(0, out)                                     # the refused calls changed nothing
    torch.cuda.synchronize()
    assert_bits_equal(from_dev(out), oracle.reduce(xs, "f32"), "incremental after refused export")
    blob = np.frombuffer(blob3, dtype=np.uint8)
    assert blob[-L * 4:].tobytes() == xs[3].tobytes()        # no context buffers: the bucket ends the blob
    agg.close()


def test_peer_open_refuses_mismatched_plans():
    N, G = 4, 2
    m = [0, 0, 1, 1]
    world = es.es_loopback_create(G)
    a0 = Aggregator(N, G, 0, m, [(4096, "f32")], transport=es.ES_TRANSPORT_LOOPBACK, comm=world.value,
                    sched=es.ES_SCHED_PEER)
    a1 = Aggregator(N, G, 1, m, [(4096, "f32")], transport=es.ES_TRANSPORT_LOOPBACK, comm=world.value,
                    sched=es.ES_SCHED_PEER, options=es.ES_OPT_PEER_PUSH)
    blobs = [a0.peer_blob(), a1.peer_blob()]
    for a in (a0, a1):
        with pytest.raises(es.EsError) as ei:
            a.peer_open(blobs)
        assert ei.value.status == es.ES_EINVAL
        assert "plan differs" in str(ei.value)
    a0.close()
    a1.close()
    es.es_loopback_destroy(world)
