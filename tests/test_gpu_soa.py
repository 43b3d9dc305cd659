"""Structure-of-arrays states (LFQS_STATE_SOA, NEXT-4: the paper's AOS/SOA layout study,
PAPER.md §6.6, lines 501-505 / 605-613).  Same bar as the AOS kernels (BASELINE.json
north_star): permutation and diagonal gates bit-exact against the oracle, dense gates
max abs error <= 1e-12; probabilities bit-identical to an AOS state with the same
amplitudes (same reduction order)."""
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


@pytest.mark.parametrize("n", [1, 3, 7, 12])
def test_soa_every_kind_vs_oracle(L, n):
    psi = W.random_state(n, 40 + n)
    gates = W.random_gate_list(n, 120, seed=n, max_targets=min(3, n), max_controls=2)
    with L.State.create(n, soa=True) as st:
        for g in gates:
            st.copy_in(psi)
            st.apply(g)
            got = st.copy_out()
            ref = O.apply_gate(n, g, psi.copy())
            if g.exact:
                assert np.array_equal(got, ref), g.label()
            else:
                assert np.max(np.abs(got - ref)) <= 1e-12, g.label()


def test_soa_circuit_probs_and_init(L):
    n = 14
    psi = W.random_state(n, 5)
    gates = W.random_gate_list(n, 300, seed=9, max_controls=2) + W.qft(n)
    ref = O.run_circuit(n, gates, psi.copy())
    with L.State.create(n, soa=True) as s, L.State.create(n) as a:
        s.copy_in(psi)
        s.run_circuit(gates)
        got = s.copy_out()
        assert np.max(np.abs(got - ref)) <= 1e-12
        a.copy_in(got)
        for qs in ([], [0], [3, 11], list(range(10)), list(range(12))):
            assert np.array_equal(s.measure_probs(qs), a.measure_probs(qs))
        s.init_basis(12345)
        b = s.copy_out()
        assert b[12345] == 1 and np.count_nonzero(b) == 1
        s.init_random(77)
        a.init_random(77)
        assert np.array_equal(s.copy_out(), a.copy_out())
        u = np.linspace(0.01, 0.99, 64)
        assert np.array_equal(s.sample([1, 2, 5], u), a.sample([1, 2, 5], u))
        assert s.collapse([4], 1) == a.collapse([4], 1)
        assert np.array_equal(s.copy_out(), a.copy_out())


def test_soa_rejects_fusion_and_sharding(L):
    with L.State.create(10, soa=True) as st:
        with pytest.raises(L.LfqsError):
            st.run_circuit(W.qft(10), fuse=True)
    with pytest.raises(L.LfqsError):
        L.lfqs_state_create_ex(10, 2, 0, None, L.STATE_SOA)


def test_soa_c64(L):
    n = 12
    psi = W.random_state(n, 3).astype(np.complex64).astype(np.complex128)
    gates = W.random_gate_list(n, 100, seed=3, max_controls=1)
    with L.State.create(n, c64=True, soa=True) as st:
        st.copy_in(psi)
        st.run_circuit(gates)
        assert np.max(np.abs(st.copy_out() - O.run_circuit(n, gates, psi.copy()))) <= 2e-5
