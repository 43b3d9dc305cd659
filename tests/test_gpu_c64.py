"""complex64 states (NEXT-4 precision variant) vs the complex128 oracle.

Inputs are rounded to complex64 first; the oracle applies the same gates in
complex128 to those rounded inputs.  Permutation gates only move values, so
they must match exactly; everything else within fp32 rounding.
"""
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


def _c64(psi):
    return psi.astype(np.complex64)


@pytest.mark.parametrize("n", [7, 13])
def test_single_gates_c64(L, n):
    psi32 = _c64(W.random_amplitudes(3 + n, 0, 1 << n))
    psi = psi32.astype(np.complex128)
    with L.State.create(n, c64=True) as st:
        for g in W.random_gate_list(n, 120, seed=n, max_controls=2):
            st.copy_in(psi32)
            st.apply(g)
            got = st.copy_out_c64().astype(np.complex128)
            ref = O.apply_gate(n, g, psi.copy())
            if g.kind in ("X", "Y", "SWAP"):
                assert np.array_equal(got, ref), g.label()
            else:
                assert np.max(np.abs(got - ref)) <= 4e-6, g.label()


@pytest.mark.parametrize("fuse", [False, True])
def test_circuit_c64(L, fuse):
    n = 15
    psi32 = _c64(W.random_state(n, 8))
    psi = psi32.astype(np.complex128)
    gates = W.random_gate_list(n, 200, seed=2, max_controls=2) + W.qft(n)
    ref = O.run_circuit(n, gates, psi.copy())
    with L.State.create(n, c64=True) as st:
        st.copy_in(psi32)
        st.run_circuit(gates, fuse=fuse)
        got = st.copy_out()
        p = st.measure_probs([0, 7, 14])
    assert np.max(np.abs(got - ref)) <= 2e-5
    np.testing.assert_allclose(p, O.probs(n, ref, [0, 7, 14]), atol=2e-6)


def test_virtual_partition_c64(L):
    n = 14
    psi32 = _c64(W.random_state(n, 4))
    psi = psi32.astype(np.complex128)
    gates = W.random_gate_list(n, 150, seed=9, max_controls=2)
    ref = O.run_circuit(n, gates, psi.copy())
    with L.State.virtual(n, 4, c64=True) as st:
        st.copy_in(psi32)
        st.run_circuit(gates, fuse=True)
        got = st.copy_out()
    assert np.max(np.abs(got - ref)) <= 2e-5


def test_ghz_c64_closed_form(L):
    n = 24
    with L.State.create(n, c64=True) as st:
        st.run_circuit(W.ghz(n))
        a = st.copy_out_c64()
    s = np.float32(np.sqrt(np.float32(0.5)))
    assert a[0] == np.complex64(a[0]) and abs(a[0].real - np.sqrt(0.5)) < 1e-7
    assert a[-1] == a[0] and np.count_nonzero(a) == 2


def test_wrap_torch_complex64(L):
    import torch
    n = 10
    psi32 = _c64(W.random_state(n, 1))
    t = torch.from_numpy(psi32.copy()).cuda()
    with L.State.wrap(t) as st:
        assert st.c64
        st.apply(W.Gate("H", (3,)))
        st.synchronize()
    ref = O.apply_gate(n, W.Gate("H", (3,)), psi32.astype(np.complex128))
    assert np.max(np.abs(t.cpu().numpy().astype(np.complex128) - ref)) <= 1e-7
