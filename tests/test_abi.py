"""The C-ABI library loads and exports every symbol include/lfqs.h declares (no GPU needed)."""
import ctypes as C
import os
import re

import pytest

import paper_conf_cgo_tarabkhahdds25_b200 as L
from paper_conf_cgo_tarabkhahdds25_b200 import build as B

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "lfqs.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(lfqs_\w+)\s*\(", src)))


@pytest.fixture(scope="module")
def lib():
    B.build()
    return L.lib()


def test_header_declares_the_binding_exports():
    assert declared_functions() == sorted(L.EXPORTS)


def test_library_exports_every_declared_symbol(lib):
    for name in declared_functions():
        assert hasattr(lib, name), name


def test_abi_version_and_struct_layout(lib):
    assert lib.lfqs_abi_version() == 1
    assert C.sizeof(L.LfqsGate) == 72
    assert L.LfqsGate.control_mask.offset == 32
    assert L.LfqsGate.matrix.offset == 64


def test_kernels_are_sm100a(lib):
    """The .so carries sm_100a SASS (cross-compiled here; no GPU needed)."""
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", L.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_no_device_fails_loudly(lib):
    """Without a GPU every call that needs one returns LFQS_ERR_CUDA -- never a CPU fallback."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(L.LfqsError) as e:
        L.State.create(4)
    assert e.value.status == -3


def test_null_handle_is_rejected(lib):
    with pytest.raises(L.LfqsError) as e:
        L.lfqs_synchronize(None)
    assert e.value.status == -1
    assert b"NULL" in lib.lfqs_last_error()


def test_jit_precompile_host_only(lib):
    """LFQS_FUSE_JIT: the pass compiler plans and compiles every fused pass on the
    host (nvPTXCompiler, no device); a second call hits the cache."""
    import time

    import workloads as W
    n = 16
    gates = W.qft(n) + W.random_layered(n, 3, seed=1)
    t0 = time.time()
    k = L.lfqs_jit_precompile(n, gates, "jit")
    t1 = time.time()
    assert k >= 2
    assert L.lfqs_jit_precompile(n, gates, "jit") == k
    assert time.time() - t1 < max(0.5, t1 - t0)
    assert L.lfqs_jit_precompile(n, gates, "jit+phase") >= 2
    assert L.lfqs_jit_precompile(n, gates, "jit", c64=True) == k
    with pytest.raises(L.LfqsError):
        L.lfqs_jit_precompile(n, gates, True)  # FUSE_JIT missing


def test_jit_precompile_small_n_launches_nothing(lib):
    """Below the smallest fused tile (n < 8) the schedule falls back to per-gate kernels;
    lfqs_jit_precompile is host-only, so it must count those passes without launching
    anything (no device here: a launch would fail the call)."""
    import workloads as W
    for n in (1, 3, 7):
        gates = W.random_gate_list(n, 20, seed=n)
        k = L.lfqs_jit_precompile(n, gates, "jit")   # one pass per non-identity gate
        assert len(gates) - 3 <= k <= len(gates), (n, k)


def test_fused_coefficient_budget_counts_merged_gates(lib):
    """A pass of 1-target gates that build_program merges into dense U2 matrices (4
    coefficients each, e.g. X followed by H on the same qubit) must stay inside the
    program's coefficient budget: the planner budgets every 1-target gate at 4
    (ADVICE r1).  Host-only: plan + compile, no launch."""
    import workloads as W
    n = 14
    gates = []
    for rep in range(24):   # 24 x 64 = 1536 coefficients
        gates.append(W.Gate("UNITARY3", (3, 4, 5), (), (), W.haar_unitary(3, rep)))
    for rep in range(14):   # X(0) H(0) merge into one U2: 4 coefficients (budgeted 0 + 1 before)
        gates += [W.CNOT(1, 0), W.Gate("X", (0,)), W.Gate("H", (0,))]
    assert L.lfqs_jit_precompile(n, gates, "jit") >= 2


@pytest.mark.parametrize("n", [12, 20])
def test_jit_compiles_merged_programs(lib, n):
    """Host-only: every fused pass of circuits exercising the 2-target merges (controlled
    gates in 4x4 form, diagonals acting outside the tile, same-pair products) generates PTX
    that ptxas accepts (a dense merged gate on a qubit outside the tile would not)."""
    import workloads as W
    for s in range(3):
        for g in (W.random_gate_list(n, 300, seed=s, max_controls=2),
                  W.sycamore_like(2, n // 2, 6, seed=s), W.random_layered(n, 6, seed=s),
                  W.qft(n) + W.grover(n, 5, 1)):
            for mode in ("jit", "jit+phase"):
                assert L.lfqs_jit_precompile(n, g, mode) >= 1
