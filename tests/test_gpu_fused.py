"""Fused low-qubit staging (LFQS_FUSE_LOW) == unfused per-gate semantics and == oracle.

Permutation/diagonal gates use the same formulas fused or not, so circuits made
only of them must agree bit-exactly; dense gates within 1e-12."""
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


def _run(L, n, psi, gates, fuse, tile=None, reorder=1, merge=None):
    with L.State.create(n) as st:
        st.set_option(L.OPT_FUSE_REORDER, reorder)
        if merge is not None:
            st.set_option(L.OPT_FUSE_MERGE_COMMUTING, merge)
        if tile:
            st.set_option(L.OPT_FUSE_TILE_QUBITS, tile)
        st.copy_in(psi)
        c0 = st.launches()
        st.run_circuit(gates, fuse=fuse)
        out = st.copy_out()
        return out, st.launches() - c0


@pytest.mark.parametrize("reorder", [0, 1])
@pytest.mark.parametrize("tile", [6, 9, 12, 13])
@pytest.mark.parametrize("n", [8, 14, 17])
def test_fused_random_circuit(L, n, tile, reorder):
    psi = W.random_state(n, n + tile)
    gates = W.random_gate_list(n, 250, seed=7 * n + tile, max_controls=2)
    ref = O.run_circuit(n, gates, psi.copy())
    got, launches = _run(L, n, psi, gates, True, tile, reorder)
    assert np.max(np.abs(got - ref)) <= 1e-12
    unf, _ = _run(L, n, psi, gates, False)
    assert np.max(np.abs(got - unf)) <= 1e-12
    exact = [g for g in gates if g.exact]
    a, _ = _run(L, n, psi, exact, True, tile, reorder)
    b, _ = _run(L, n, psi, exact, False)
    assert np.array_equal(a, b)
    # diagonal gates are never reordered among themselves: a diagonal-only circuit
    # (QFT's controlled phases included) stays bit-identical to the oracle
    diag = [g for g in gates if W.KIND_CLASS[g.kind] == "diag"] + \
        [g for g in W.qft(n) if g.kind == "PHASE"]
    a, _ = _run(L, n, psi, diag, True, tile, reorder)
    assert np.array_equal(a, O.run_circuit(n, diag, psi.copy()))


@pytest.mark.parametrize("tma", [0, 256])
@pytest.mark.parametrize("low", [5, 7, 12])
def test_fused_general_tiles(L, low, tma):
    """Tiles = qubits [0, low) + qubits claimed by the gates (NEXT-1); chunks moved by
    TMA bulk copies (tma=256) or by direct register loads/stores (tma=0)."""
    n = 18
    psi = W.random_state(n, low)
    gates = W.random_gate_list(n, 200, seed=100 + low, max_controls=2) + W.qft(n) + \
        W.random_layered(n, 4, seed=low)
    ref = O.run_circuit(n, gates, psi.copy())
    with L.State.create(n) as st:
        st.set_option(L.OPT_FUSE_LOW_QUBITS, low)
        st.set_option(L.OPT_FUSE_TMA_MAX_CHUNKS, tma)
        st.copy_in(psi)
        c0 = st.launches()
        st.run_circuit(gates, fuse=True)
        passes = st.launches() - c0
        got = st.copy_out()
    assert np.max(np.abs(got - ref)) <= 1e-12
    assert passes < len(gates) // 3
    exact = [g for g in gates if g.exact]
    with L.State.create(n) as st:
        st.set_option(L.OPT_FUSE_LOW_QUBITS, low)
        st.copy_in(psi)
        st.run_circuit(exact, fuse=True)
        assert np.array_equal(st.copy_out(), O.run_circuit(n, exact, psi.copy()))


def test_fusion_reduces_passes_qft(L):
    n, x = 20, 0xBEEF1
    gates = W.qft(n)
    with L.State.create(n) as st:
        st.init_basis(x)
        c0 = st.launches()
        st.run_circuit(gates, fuse=True)
        launches = st.launches() - c0
        a = st.copy_out()
    y = np.arange(1 << n, dtype=np.int64)
    ref = np.exp(2j * np.pi * ((x * y) % (1 << n)) / (1 << n)) / np.sqrt(1 << n)
    assert np.max(np.abs(a - ref)) <= 1e-12
    assert launches < len(gates) // 4, (launches, len(gates))


def test_fused_layered_and_grover(L):
    n = 16
    psi = W.random_state(n, 3)
    for gates in (W.random_layered(n, 10, seed=5), W.grover(n, 12345, 2), W.ghz(n)):
        ref = O.run_circuit(n, gates, psi.copy())
        got, _ = _run(L, n, psi, gates, True)
        assert np.max(np.abs(got - ref)) <= 1e-12


@pytest.mark.parametrize("fuse", [True, "phase", "jit", "jit+phase"])
@pytest.mark.parametrize("tile", [9, 12])
def test_merge_commuting_1q_runs(L, fuse, tile):
    """LFQS_OPT_FUSE_MERGE_COMMUTING: same-qubit 1-target gates separated by gates on
    other qubits merge into one matrix (Grover's H and X layers, VQE's RY and RZ
    layers); the result changes by rounding only, and exact-class circuits never merge."""
    n = 14
    psi = W.random_state(n, 5 + tile)
    gates = (W.grover(n, 0x2A7D, 1) + W.vqe_ansatz(n, 2, seed=3) +
             W.random_gate_list(n, 200, seed=tile, max_controls=2))
    ref = O.run_circuit(n, gates, psi.copy())
    a, ka = _run(L, n, psi, gates, fuse, tile, merge=1)
    b, kb = _run(L, n, psi, gates, fuse, tile, merge=0)
    assert ka == kb
    assert np.max(np.abs(a - ref)) <= 1e-12
    assert np.max(np.abs(b - ref)) <= 1e-12
    exact = [g for g in gates if g.exact]
    c, _ = _run(L, n, psi, exact, fuse, tile, merge=1)
    if fuse in (True, "jit"):
        assert np.array_equal(c, O.run_circuit(n, exact, psi.copy()))


@pytest.mark.parametrize("tma", [0, 256])
@pytest.mark.parametrize("low", [6, 7])
def test_fused_lane_bit_dense_1q(L, low, tma):
    """Dense 1-target gates on lane bits (tile bits 0-4: shuffle path) for every
    register specialisation -- H, Ry (real), Rx (real diagonal, imaginary
    off-diagonal), U3 / UNITARY1 (general) -- uncontrolled and controlled on lane,
    register and out-of-tile qubits; commuting merges off so each gate keeps its own
    kind.  Interpreted fused passes vs the oracle, and vs the compiled passes
    (identical arithmetic, so bit-identical)."""
    n = 14
    rng = np.random.default_rng(1000 + low + tma)
    u = W.haar_unitary(1, 77)
    gates = []
    for t in range(5):
        for ctl in [(), ((t + 1) % 5,), (9,), (13,), ((t + 2) % 5, 10)]:
            th = rng.uniform(-np.pi, np.pi, 3)
            gates += [W.Gate("H", (t,), ctl), W.Gate("RY", (t,), ctl, (th[0],)),
                      W.Gate("RX", (t,), ctl, (th[1],)), W.Gate("U3", (t,), ctl, tuple(th)),
                      W.Gate("UNITARY1", (t,), ctl, matrix=u)]
    psi = W.random_state(n, 31 + low)
    ref = O.run_circuit(n, gates, psi.copy())
    out = {}
    for fuse in (True, "jit"):
        with L.State.create(n) as st:
            st.set_option(L.OPT_FUSE_LOW_QUBITS, low)
            st.set_option(L.OPT_FUSE_TMA_MAX_CHUNKS, tma)
            st.set_option(L.OPT_FUSE_MERGE_COMMUTING, 0)
            st.copy_in(psi)
            st.run_circuit(gates, fuse=fuse)
            out[fuse] = st.copy_out()
    assert np.max(np.abs(out[True] - ref)) <= 1e-12
    assert np.array_equal(out[True], out["jit"])


def _merge2q_cases(n):
    """Every shape the 2-target merge handles, and some it must refuse."""
    U = lambda s: W.haar_unitary(1, s)  # noqa: E731
    U4 = lambda s: W.haar_unitary(2, s)  # noqa: E731
    fsim = W.fsim(np.pi / 2, np.pi / 6)
    g = []
    g += [W.Gate("UNITARY2", (3, 7), (), (), U4(1)), W.Gate("UNITARY1", (3,), (), (), U(2)),
          W.Gate("H", (7,)), W.Gate("RX", (7,), (), (0.4,))]           # 1q after a U4 (both)
    g += [W.Gate("U3", (1,), (), (0.3, 0.2, 0.1)), W.Gate("RY", (9,), (), (1.1,)),
          W.Gate("T", (4,)), W.Gate("UNITARY2", (9, 1), (), (), fsim)]  # 1q before fSim
    g += [W.Gate("UNITARY2", (9, 1), (), (), fsim),                     # same pair, reversed
          W.Gate("UNITARY2", (1, 9), (), (), U4(3))]
    g += [W.Gate("SWAP", (2, 5)), W.Gate("H", (5,)), W.Gate("H", (2,))]  # SWAP absorbs 1q
    g += [W.Gate("UNITARY2", (0, 6), (8,), (), U4(4)),                  # same controls
          W.Gate("UNITARY1", (6,), (8,), (), U(5)),
          W.Gate("UNITARY1", (0,), (), (), U(6))]                       # different controls
    g += [W.Gate("UNITARY2", (10, 11), (), (), U4(7)), W.CNOT(2, 10),   # blocked by CNOT
          W.Gate("H", (10,)), W.Gate("H", (11,))]
    g += W.sycamore_like(2, n // 2, 4, seed=8)
    return g


@pytest.mark.parametrize("fuse", [True, "jit", "jit+phase"])
def test_merge_2q_matches_oracle_and_unmerged(L, fuse):
    """LFQS_OPT_FUSE_MERGE_2Q: dense 1-target gates folded into neighbouring 2-target gates
    (both orders, SWAP, same-pair products, controlled) equal the oracle within 1e-12 and
    the unmerged fused run within rounding; the interpreter and the pass compiler agree
    bit for bit; permutation / diagonal circuits stay bit-exact."""
    n = 12
    psi = W.random_state(n, 17)
    gates = _merge2q_cases(n)
    ref = O.run_circuit(n, gates, psi.copy())
    outs = {}
    for m2 in (0, 1):
        with L.State.create(n) as st:
            st.set_option(L.OPT_FUSE_MERGE_2Q, m2)
            st.copy_in(psi)
            st.run_circuit(gates, fuse=fuse)
            outs[m2] = st.copy_out()
        assert np.max(np.abs(outs[m2] - ref)) <= 1e-12, m2
    assert np.max(np.abs(outs[0] - outs[1])) <= 1e-13
    if fuse == "jit":
        with L.State.create(n) as st:  # interpreter with the same merges
            st.copy_in(psi)
            st.run_circuit(gates, fuse=True)
            assert np.array_equal(st.copy_out(), outs[1])
    exact = [W.Gate("SWAP", (2, 5)), W.CNOT(5, 2), W.Gate("X", (2,)), W.Gate("SWAP", (5, 2)),
             W.CZ(1, 3), W.Gate("S", (5,))] * 5
    with L.State.create(n) as st:
        st.copy_in(psi)
        st.run_circuit(exact, fuse=fuse)
        assert np.array_equal(st.copy_out(), O.run_circuit(n, exact, psi.copy()))


@pytest.mark.parametrize("c64", [False, True])
@pytest.mark.parametrize("n", [12, 16, 21])
def test_bitperm_pass(n, c64):
    """LFQS_OPT_FUSE_PERM: a fused run ending in >= 3 SWAPs whose composition is an
    involution (QFT's bit reversal, disjoint SWAPs) applies them as one bit-permutation
    pass.  Moves only: an exact circuit with such a tail is bit-identical with the pass on
    and off and to the oracle; QFT within tolerance, compiled == interpreted; a cyclic SWAP
    chain (not an involution) falls back to the tile passes."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    psi = W.random_state(n, 77 + n)
    rev = [W.Gate("SWAP", (q, n - 1 - q)) for q in range(n // 2)]
    exact = [g for g in W.random_gate_list(n, 120, seed=n, max_controls=2) if g.exact]
    cases = {"rev": exact + rev,
             "pairs": exact + [W.Gate("SWAP", (0, 7)), W.Gate("SWAP", (3, n - 2)),
                               W.Gate("SWAP", (1, 9)), W.Gate("SWAP", (2, n - 1)),
                               W.Gate("SWAP", (4, 6))],
             "cycle": exact + [W.Gate("SWAP", (0, 5)), W.Gate("SWAP", (5, 9)),
                               W.Gate("SWAP", (9, n - 1))]}
    tol = 0.0
    for name, gates in cases.items():
        ref = O.run_circuit(n, gates, psi.copy())
        outs = []
        for perm in (0, 1):
            for fuse in (True, "jit"):
                with L.State.create(n, c64=c64) as st:
                    st.set_option(L.OPT_FUSE_PERM, perm)
                    st.copy_in(psi)
                    st.run_circuit(gates, fuse=fuse)
                    outs.append(st.copy_out())
        for o in outs[1:]:
            assert np.array_equal(o, outs[0]), name
        if not c64:
            assert np.array_equal(outs[0], ref), name
    qft = W.qft(n)
    ref = O.run_circuit(n, qft, psi.copy())
    res = {}
    for perm in (0, 1):
        for fuse in ("phase", "jit+phase"):
            with L.State.create(n, c64=c64) as st:
                st.set_option(L.OPT_FUSE_PERM, perm)
                st.copy_in(psi)
                st.run_circuit(qft, fuse=fuse)
                res[perm, fuse] = st.copy_out()
            assert np.max(np.abs(res[perm, fuse] - ref)) <= (2e-5 if c64 else 1e-12)
    assert np.array_equal(res[1, "phase"], res[1, "jit+phase"])


def test_bitperm_inside_circuit():
    """A SWAP run inside a circuit (an inverse QFT's leading bit reversal in QPE) is split
    out as a permutation pass only when that saves passes; either way the result equals the
    run without permutation passes within tolerance, and exact circuits stay bit-exact."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    n = 17
    psi = W.random_state(n, 5)
    rev = [W.Gate("SWAP", (q, n - 1 - q)) for q in range(n // 2)]
    exact = [g for g in W.random_gate_list(n, 100, seed=3, max_controls=1) if g.exact]
    for gates, bitexact in ((W.qpe(n - 1, 0x5A5A), False), (exact + rev + exact, True),
                            (W.qft(n) + W.random_layered(n, 2, seed=1) + W.qft_inverse(n), False)):
        ref = O.run_circuit(n, gates, psi.copy())
        outs = []
        for perm in (0, 1):
            with L.State.create(n) as st:
                st.set_option(L.OPT_FUSE_PERM, perm)
                st.copy_in(psi)
                st.run_circuit(gates, fuse="jit+phase" if not bitexact else "jit")
                outs.append(st.copy_out())
        for o in outs:
            if bitexact:
                assert np.array_equal(o, ref)
            else:
                assert np.max(np.abs(o - ref)) <= 1e-12
