"""Sampling and projective collapse (P:122 measurement, P:154 mid-circuit) vs the oracle."""
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


@pytest.mark.parametrize("world", [1, 4])
def test_sample_matches_oracle(L, world):
    n = 14
    psi = O.run_circuit(n, W.random_layered(n, 4, seed=9), W.basis_state(n, 0))
    u = np.random.default_rng(5).random(4000)
    st = L.State.create(n) if world == 1 else L.State.virtual(n, world)
    with st:
        st.copy_in(psi)
        for qs in ([0], [13, 2], [5, 0, 12, 7], list(range(10))):
            got = st.sample(qs, u)
            ref = O.measure_sample(n, psi, qs, u)
            # identical draws give identical outcomes except when a draw lands within
            # rounding of a CDF boundary (probability ~1e-15 per shot)
            assert np.mean(got == ref) >= 0.999
            assert np.sum(got != ref) <= 1


@pytest.mark.parametrize("world", [1, 2, 8])
def test_collapse_matches_oracle(L, world):
    n = 13
    psi0 = W.random_state(n, 11)  # every outcome has nonzero probability
    for qs, outcome in (([0], 1), ([12, 3], 2), ([1, 11, 6, 9], 0b1011)):
        ref = psi0.copy()
        p_ref = O.measure_collapse(n, ref, qs, outcome)
        st = L.State.create(n) if world == 1 else L.State.virtual(n, world)
        with st:
            st.copy_in(psi0)
            if world > 1:  # leave the qubit map non-identity first (remaps + relabel)
                st.run_circuit([W.Gate("H", (n - 1,)), W.Gate("H", (n - 1,)),
                                W.Gate("SWAP", (n - 1, 0)), W.Gate("SWAP", (n - 1, 0))])
            p = st.collapse(qs, outcome)
            got = st.copy_out()
        assert abs(p - p_ref) <= 1e-14
        assert np.max(np.abs(got - ref)) <= 1e-12
        zero = np.flatnonzero(ref == 0)
        assert np.all(got[zero] == 0)


def test_collapse_ghz_and_errors(L):
    n = 20
    with L.State.create(n) as st:
        st.run_circuit(W.ghz(n))
        p = st.collapse([7], 0)
        assert abs(p - 0.5) < 1e-15
        a = st.copy_out(0, 2)
        assert abs(a[0] - 1.0) < 1e-15 and a[1] == 0
        assert abs(st.norm2() - 1.0) < 1e-14
        with pytest.raises(L.LfqsError):
            st.collapse([7], 1)  # probability 0 now
