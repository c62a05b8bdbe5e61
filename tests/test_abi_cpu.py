"""CPU: the C-ABI library loads, exports every symbol include/es.h declares,
and its host-only entry points (sizing, planner export, argument checks)
behave as documented.  No compute calls are made without a GPU."""
import ctypes
import os
import re
import subprocess

import pytest

from paper_conf_sc_lixyszrljlllq23_b200 import es, workloads

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "es.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(es_[a-z0-9_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    names = _declared()
    assert len(names) >= 20
    lib = es.lib()
    for n in names:
        assert hasattr(lib, n), f"libes.so lacks {n}"
    out = subprocess.run(["nm", "-D", "--defined-only", es.lib_path()], capture_output=True, text=True).stdout
    for n in names:
        assert re.search(rf"\bT {n}\b", out), f"{n} not exported as text symbol"
    assert set(names) == set(es.EXPORTED)


def test_binding_names_match_c_abi():
    for n in _declared():
        if n not in ("es_status_string", "es_last_error"):
            assert hasattr(es, n), f"binding lacks {n}"


def test_library_built_for_sm100a():
    out = subprocess.run(["cuobjdump", "--list-elf", es.lib_path()], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_abi_version_and_status_strings():
    assert es.es_abi_version() == 1
    for s in range(7):
        assert es.es_status_string(s).startswith("ES_")


def test_chunk_elems_matches_hand_table():
    assert es.es_chunk_elems(1000003, 12) == 83344
    assert es.es_chunk_elems(2049000, 8) == 256128
    assert es.es_chunk_elems(1 << 20, 4) == 262144
    assert es.es_chunk_elems(0, 4) == 0


@pytest.mark.parametrize("bad", [
    dict(N=0), dict(N=1025), dict(G=0), dict(G=5), dict(rank=2), dict(map=[0, 0, 0, 0]),
    dict(map=[0, 1, 2, 0]), dict(buckets=[(1 << 31, es.ES_F32)]), dict(buckets=[(10, 7)]), dict(A=12),
    dict(sched=9), dict(states=[0]), dict(compat=8), dict(compat=3),
])
def test_config_validation(bad):
    N = bad.get("N", 4)
    G = bad.get("G", 2)
    m = bad.get("map", [0, 0, 1, 1][:max(N, 0)] if N == 4 else [0] * max(N, 0))
    cfg = es.Config(N, G, bad.get("rank", 0), m, bad.get("buckets", [(100, es.ES_F32)]), bad.get("A", 16),
                    bad.get("states", ()), sched=bad.get("sched", 0), compat=bad.get("compat", 0))
    with pytest.raises(es.EsError) as e:
        es.es_workspace_bytes(cfg)
    assert e.value.status == es.ES_EINVAL
    assert es.es_last_error()


def test_workspace_layout_sizes():
    c = workloads.config("resnet50")
    cfg = es.Config(8, 1, 0, [0] * 8, [(n, es.ES_F32) for n, _ in c["buckets"]],
                    state_nbytes=workloads.state_nbytes())
    nb = es.es_workspace_bytes(cfg)
    slot = sum((n * 4 + 255) // 256 * 256 for n, _ in c["buckets"])
    assert slot * 8 <= nb <= slot * 8 + 8 * 300000                  # slots + state slots + tables
    cfg2 = es.Config(8, 2, 0, workloads.mapping(8, 2), [(n, es.ES_F32) for n, _ in c["buckets"]])
    assert es.es_workspace_bytes(cfg2) > slot * 4                     # 4 local slots + staging/partials


def test_init_rejects_null_workspace_without_touching_cuda():
    cfg = es.Config(4, 1, 0, [0] * 4, [(100, es.ES_F32)])
    with pytest.raises(es.EsError) as e:
        es.es_init(cfg, 0, 1 << 20)
    assert e.value.status == es.ES_EINVAL
    with pytest.raises(es.EsError) as e:
        es.es_init(es.Config(4, 2, 0, [0, 0, 1, 1], [(100, es.ES_F32)]), 0, 1 << 20)   # G>1 without comm
    assert e.value.status == es.ES_EINVAL


def test_null_handle_calls():
    L = es.lib()
    assert L.es_sync(None) == es.ES_EINVAL
    assert L.es_destroy(None) == es.ES_EINVAL
    assert L.es_allreduce(None, 0, None, None) == es.ES_EINVAL
    assert L.es_stash_grad(None, 0, 0, None, 0, 0, None) == es.ES_EINVAL
    assert L.es_switch_context(None, 0, None) == es.ES_EINVAL


def test_loopback_world_lifecycle():
    w = es.es_loopback_create(4)
    es.es_loopback_destroy(w)
    with pytest.raises(es.EsError):
        es.es_loopback_create(0)


def test_product_path_has_no_oracle_or_cpu_fallback():
    """The product package never imports the oracle and has no CPU compute path."""
    pkg = os.path.join(ROOT, "paper_conf_sc_lixyszrljlllq23_b200")
    for fn in os.listdir(pkg):
        if fn.endswith(".py"):
            src = open(os.path.join(pkg, fn)).read()
            assert "import oracle" not in src and "from oracle" not in src, fn
    for fn in os.listdir(os.path.join(pkg, "csrc")):
        src = open(os.path.join(pkg, "csrc", fn)).read()
        assert "es_oracle" not in src and "oracle/" not in src, fn
