"""LFQS_FUSE_PHASE: runs of diagonal gates inside a fused pass merged into per-tile
phase tables (include/lfqs.h).  The merged product is the same diagonal (Eq. 3,
PAPER.md:142) -- diagonal matrices commute -- rounded in a different order, so the
bar is the BASELINE.json north_star tolerance for non-exact results: max abs
amplitude error <= 1e-12 against the oracle (reading R21)."""
import math

import numpy as np
import pytest

import oracle as O
import workloads as W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def L():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import paper_conf_cgo_tarabkhahdds25_b200 as lib
    lib.lib()
    return lib


def diag_heavy(n, count, seed):
    """Seeded circuit of mostly diagonal gates on random qubits: one-entry (Z, S, T,
    PHASE, CZ, CPhase, multi-controlled), two-entry (RZ), diagonal UNITARY2/3 (all
    entries != 1), with an occasional H / X / SWAP between the runs."""
    rng = W.SplitMix64(seed)
    out = []
    kinds = ["Z", "S", "T", "TDG", "PHASE", "RZ", "RZ", "PHASE", "UNITARY2", "UNITARY3",
             "PHASE", "H", "X", "SWAP"]
    while len(out) < count:
        kind = kinds[rng.below(len(kinds))]
        m = W.ARITY[kind]
        perm = list(range(n))
        for i in range(n - 1, 0, -1):
            j = rng.below(i + 1)
            perm[i], perm[j] = perm[j], perm[i]
        nc = rng.below(min(3, n - m) + 1)
        targets = tuple(perm[:m])
        controls = tuple(sorted(perm[m:m + nc]))
        params = tuple(rng.angle() for _ in range(W.NPARAMS[kind]))
        mat = None
        if kind.startswith("UNITARY"):
            mat = np.diag(np.exp(1j * np.array([rng.angle() for _ in range(1 << m)])))
        out.append(W.Gate(kind, targets, controls, params, mat))
    return out


def _run(L, n, psi, gates, fuse, tile=None, low=None, c64=False, split=None):
    with L.State.create(n, c64=c64) as st:
        if split is not None:
            st.set_option(L.OPT_FUSE_PHASE_SPLIT, split)
        if tile:
            st.set_option(L.OPT_FUSE_TILE_QUBITS, tile)
        if low:
            st.set_option(L.OPT_FUSE_LOW_QUBITS, low)
        st.copy_in(psi)
        c0 = st.launches()
        st.run_circuit(gates, fuse=fuse)
        out = st.copy_out()
        return out, st.launches() - c0


@pytest.mark.parametrize("split", [0, 1])
@pytest.mark.parametrize("low", [5, 7])
@pytest.mark.parametrize("tile", [8, 10, 12])
@pytest.mark.parametrize("n", [12, 17])
def test_phase_tables_diag_heavy(L, n, tile, low, split):
    """split: LFQS_OPT_FUSE_PHASE_SPLIT (tile-invariant and tile-dependent diagonals in
    separate tables) -- a different rounding order, the same bar."""
    psi = W.random_state(n, 31 * n + tile)
    gates = diag_heavy(n, 400, seed=n * 100 + tile + low)
    ref = O.run_circuit(n, gates, psi.copy())
    got, passes = _run(L, n, psi, gates, "phase", tile, low, split=split)
    jit, _ = _run(L, n, psi, gates, "jit+phase", tile, low, split=split)
    assert np.array_equal(got, jit)  # compiled == interpreted, bit for bit
    assert np.max(np.abs(got - ref)) <= 1e-12
    exact, passes_exact = _run(L, n, psi, gates, True, tile, low)
    assert np.max(np.abs(got - exact)) <= 1e-12
    assert passes <= passes_exact


@pytest.mark.parametrize("n", [10, 16, 20])
def test_phase_tables_qft_closed_form(L, n):
    x = (0x9E3779B97F4A7C15 >> (64 - n)) | 1
    """QFT rows make separable tables (every member a CPhase on one table bit besides the
    common target bit): built from per-bit factors, interpreter == compiled bit for bit."""
    with L.State.create(n) as st:
        st.init_basis(x)
        st.run_circuit(W.qft(n), fuse="phase")
        a = st.copy_out()
        st.init_basis(x)
        st.run_circuit(W.qft(n), fuse="jit+phase")
        b = st.copy_out()
    assert np.array_equal(a, b)
    y = np.arange(1 << n, dtype=np.int64)
    ref = np.exp(2j * np.pi * ((x * y) % (1 << n)) / (1 << n)) / np.sqrt(1 << n)
    assert np.max(np.abs(a - ref)) <= 1e-12


def test_phase_tables_qpe_and_mixed(L):
    n = 15
    psi = W.random_state(n, 4)
    for gates in (W.qpe(n - 1, 0x1A5), W.random_gate_list(n, 300, seed=11, max_controls=2),
                  W.random_layered(n, 8, seed=3), W.grover(n, 999, 2),
                  W.qft(n) + W.qft_inverse(n)):
        ref = O.run_circuit(n, gates, psi.copy())
        got, _ = _run(L, n, psi, gates, "phase")
        assert np.max(np.abs(got - ref)) <= 1e-12


def test_phase_tables_c64(L):
    n = 14
    psi = W.random_state(n, 8)
    psi32 = psi.astype(np.complex64).astype(np.complex128)
    gates = diag_heavy(n, 200, seed=5) + W.qft(n)
    ref = O.run_circuit(n, gates, psi32.copy())
    got, _ = _run(L, n, psi32, gates, "phase", c64=True)
    assert np.max(np.abs(got - ref)) <= 2e-5


def test_phase_tables_virtual_partition(L):
    """The sharded planner folds global-qubit diagonals into rank-local ones; the
    fused local segments then merge them into tables."""
    n = 14
    psi = W.random_state(n, 9)
    gates = diag_heavy(n, 300, seed=77) + W.qft(n)
    ref = O.run_circuit(n, gates, psi.copy())
    for world in (2, 4):
        with L.State.virtual(n, world) as st:
            st.copy_in(psi)
            st.run_circuit(gates, fuse="phase")
            assert np.max(np.abs(st.copy_out() - ref)) <= 1e-12


def test_phase_flag_rejected_alone_is_harmless(L):
    """FUSE_PHASE without FUSE_LOW is accepted and has no effect (no fused passes)."""
    n = 8
    psi = W.random_state(n, 1)
    gates = diag_heavy(n, 50, seed=1)
    a, k = _run(L, n, psi, gates, L.FUSE_PHASE)
    b, k0 = _run(L, n, psi, gates, False)
    assert np.array_equal(a, b) and k == k0
    assert math.isfinite(float(np.abs(a).sum()))


@pytest.mark.parametrize("c64", [False, True])
@pytest.mark.parametrize("tile", [8, 12])
def test_hoisted_table_factors(L, tile, c64):
    """Phase-table members decided by the tile index alone (QFT's CPhase rows to qubits
    outside the tile; controlled diagonals with controls outside the tile) form a per-tile
    factor the pass compiler computes once per tile (one thread, after a barrier) and the
    interpreter per entry -- the same products in the same order, so compiled == interpreted
    bit for bit; within the tolerance of the oracle."""
    n = 18
    psi = W.random_state(n, 8)
    x = 0x2B3C5
    gates = W.qft(n) + W.qpe(n - 1, x) + diag_heavy(n, 300, 3)
    ref = O.run_circuit(n, gates, psi.copy())
    a, _ = _run(L, n, psi, gates, "phase", tile=tile, c64=c64)
    b, _ = _run(L, n, psi, gates, "jit+phase", tile=tile, c64=c64)
    assert np.array_equal(a, b)
    assert np.max(np.abs(b - ref)) <= (2e-5 if c64 else 1e-12)
