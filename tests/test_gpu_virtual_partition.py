"""The distributed planner on one GPU: `world` shards in one allocation with the
same remap / exchange / rank-predicate logic as the NCCL path.
Partition invariance: P = 1, 2, 4, 8 give the same state (SURVEY §8(c) invariants)."""
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


def _run(L, n, world, psi, gates):
    st = L.State.create(n) if world == 1 else L.State.virtual(n, world)
    with st:
        st.copy_in(psi)
        st.run_circuit(gates)
        probs = st.measure_probs([n - 1, 0, n - 2])
        return st.copy_out(), probs


@pytest.mark.parametrize("world", [2, 4, 8])
def test_partition_invariance_random_circuit(L, world):
    n = 12
    psi = W.random_state(n, 21)
    gates = W.random_gate_list(n, 200, seed=world, max_controls=2)
    ref = O.run_circuit(n, gates, psi.copy())
    one, p1 = _run(L, n, 1, psi, gates)
    many, pw = _run(L, n, world, psi, gates)
    assert np.max(np.abs(many - ref)) <= 1e-12
    assert np.max(np.abs(many - one)) <= 1e-13
    np.testing.assert_allclose(pw, O.probs(n, ref, [n - 1, 0, n - 2]), rtol=1e-12)
    exact = [g for g in gates if g.exact]
    a, _ = _run(L, n, world, psi, exact)
    b, _ = _run(L, n, 1, psi, exact)
    assert np.array_equal(a, b)


@pytest.mark.parametrize("world", [2, 8])
def test_global_qubit_cases(L, world):
    """(i) global controls, (ii) diagonal on global targets, (iii) dense/perm on global
    targets (remap), SWAP(global, local) relabel, canonicalisation at copy-out."""
    n = 10
    p = world.bit_length() - 1
    hi = list(range(n - p, n)) if p > 1 else [n - 1, n - 2]  # n-2 is local when p = 1
    psi = W.random_state(n, 5)
    gates = [
        W.Gate("H", (hi[-1],)), W.CNOT(hi[0], 2), W.CZ(hi[-1], 3), W.CPHASE(1, hi[0], 0.7),
        W.Gate("RZ", (hi[-1],), (), (1.1,)), W.Gate("SWAP", (hi[0], 0)), W.Gate("X", (hi[-1],), (4,)),
        W.Gate("UNITARY2", (hi[-1], 0), (), (), W.haar_unitary(2, 8)),
        W.Gate("UNITARY3", (hi[0], 5, hi[-1]), (), (), W.haar_unitary(3, 9)),
        W.Gate("UNITARY2", (hi[0], hi[-1]), (2,), (), np.diag(np.exp(1j * np.arange(4.0)))),
        W.TOFFOLI(hi[0], 1, hi[-1]), W.mcz(n), W.Gate("SWAP", (hi[0], hi[-1])),
    ]
    ref = O.run_circuit(n, gates, psi.copy())
    got, _ = _run(L, n, world, psi, gates)
    assert np.max(np.abs(got - ref)) <= 1e-12


@pytest.mark.parametrize("world", [2, 4, 8])
def test_virtual_partition_fused(L, world):
    """Distributed run with Belady remaps and fused local segments == oracle."""
    n = 16
    psi = W.random_state(n, 77)
    gates = W.random_gate_list(n, 150, seed=3 * world, max_controls=2) + W.qft(n) + \
        W.random_layered(n, 3, seed=world)
    ref = O.run_circuit(n, gates, psi.copy())
    with L.State.virtual(n, world) as st:
        st.copy_in(psi)
        st.run_circuit(gates, fuse=True)
        got = st.copy_out()
    assert np.max(np.abs(got - ref)) <= 1e-12
    exact = [g for g in gates if g.exact]
    with L.State.virtual(n, world) as st:
        st.copy_in(psi)
        st.run_circuit(exact, fuse=True)
        assert np.array_equal(st.copy_out(), O.run_circuit(n, exact, psi.copy()))


def test_virtual_qft_and_ghz(L):
    n, x = 14, 9001
    with L.State.virtual(n, 4) as st:
        st.init_basis(x)
        st.run_circuit(W.qft(n))
        a = st.copy_out()
        y = np.arange(1 << n)
        ref = np.exp(2j * np.pi * ((x * y) % (1 << n)) / (1 << n)) / np.sqrt(1 << n)
        assert np.max(np.abs(a - ref)) <= 1e-12
        st.init_basis(0)
        st.run_circuit(W.ghz(n))
        a = st.copy_out()
        assert a[0] == np.sqrt(0.5) and a[-1] == np.sqrt(0.5) and np.count_nonzero(a) == 2


@pytest.mark.parametrize("world", [2, 4])
def test_global_x_relabel_measure(L, world):
    """X on global qubits is a relabel (no exchange); probabilities, sampling and
    collapse read the flips, and copy_out materialises them."""
    n = 12
    psi = W.random_state(n, 33)
    gates = [W.Gate("X", (n - 1,)), W.Gate("X", (n - 2,)), W.CNOT(n - 1, 0),
             W.Gate("T", (n - 2,)), W.Gate("X", (n - 1,)), W.Gate("X", (n - 1,))]
    ref = O.run_circuit(n, gates, psi.copy())
    qs = [n - 1, 0, n - 2]
    with L.State.virtual(n, world) as st:
        st.copy_in(psi)
        e0 = st.exchange_stats()[0]
        st.run_circuit(gates)
        assert st.exchange_stats()[0] == e0  # relabels only
        p = st.measure_probs(qs)
        np.testing.assert_allclose(p, O.probs(n, ref, qs), rtol=0, atol=1e-14)
        u = np.array([0.05, 0.3, 0.61, 0.97])
        np.testing.assert_array_equal(st.sample(qs, u), O.measure_sample(n, ref, qs, u))
        pr = st.collapse(qs, 5)
        want = ref.copy()
        wp = O.measure_collapse(n, want, qs, 5)
        assert abs(pr - wp) <= 1e-14
        got = st.copy_out()
    assert np.max(np.abs(got - want)) <= 1e-13
