"""C-ABI checks that need no GPU: the library loads, exports every symbol
include/granii.h declares, validates arguments, and its host-side partition
helper agrees bit-exactly with the oracle's (O2)."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle as O
from paper_conf_cgo_lenadorasgytm26_b200 import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def G():
    from paper_conf_cgo_lenadorasgytm26_b200 import build
    build.build()
    from paper_conf_cgo_lenadorasgytm26_b200 import granii
    return granii


def declared_symbols():
    hdr = open(os.path.join(ROOT, "include", "granii.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)
    return sorted(set(re.findall(r"\b(granii_[a-z_0-9]+)\s*\(", hdr)))


def test_every_declared_symbol_is_exported(G):
    lib = ctypes.CDLL(G.LIB_PATH)
    syms = declared_symbols()
    assert len(syms) >= 20
    for s in syms:
        assert hasattr(lib, s), f"{s} declared in granii.h but not exported"
    assert set(syms) == set(G.EXPORTED), "binding and header disagree"


def test_version_and_errors_without_gpu(G):
    assert "sm_100a" in G.granii_version()
    lib = ctypes.CDLL(G.LIB_PATH)
    lib.granii_graph_query.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
    assert lib.granii_graph_query(None, None) == G.ERR_INVALID_ARG
    assert "NULL" in G.granii_last_error()
    lib.granii_gemm_workspace_size.argtypes = [ctypes.c_int64] * 3 + [ctypes.c_uint32, ctypes.c_void_p]
    assert lib.granii_gemm_workspace_size(-1, 2, 3, 0, None) == G.ERR_INVALID_ARG


def test_constants_match_oracle(G):
    assert (G.ADD_SELF_LOOPS, G.SYMMETRIZE) == (O.ADD_SELF_LOOPS, O.SYMMETRIZE)
    assert G.GCN_COMPS == O.GCN_COMPS and G.GAT_COMPS == O.GAT_COMPS


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_partition_bounds_bit_exact(G, world):
    n = 500
    s, d = synth.chung_lu(n, 4000, 2.3, seed=5)
    rp, _ = O.csr_build(n, s, d, O.SYMMETRIZE | O.ADD_SELF_LOOPS)
    assert np.array_equal(G.granii_partition_bounds(rp, world), O.partition(rp, world))


def test_compute_without_device_fails_loudly(G):
    import torch
    if torch.cuda.is_available():
        pytest.skip("has a GPU")
    with pytest.raises(G.GraniiError) as e:
        G.granii_graph_csr_create(4, torch.zeros(1, dtype=torch.int32), torch.zeros(1, dtype=torch.int32))
    assert e.value.status == G.ERR_CUDA
