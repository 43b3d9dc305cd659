"""Captured circuits (lfqs_circuit_compile / _launch): a CUDA-graph replay of the
circuit runner (Eq. 3) must equal lfqs_run_circuit bit for bit (same
kernels, same arguments) and the oracle within the usual bounds."""
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


def config0_gates(n=10, seed=0x1F5):
    """BASELINE configs[0]: H and Rz on every qubit, CNOT on every ordered pair,
    Toffoli on every (c1 < c2, t)."""
    rng = W.SplitMix64(seed)
    g = [W.Gate("H", (t,)) for t in range(n)]
    g += [W.Gate("RZ", (t,), (), ((rng.next_u64() >> 11) * 2.0 ** -53 * 2 * np.pi,)) for t in range(n)]
    g += [W.CNOT(c, t) for c in range(n) for t in range(n) if c != t]
    g += [W.TOFFOLI(a, b, t) for a in range(n) for b in range(a + 1, n) for t in range(n)
          if t not in (a, b)]
    return g


@pytest.mark.parametrize("fuse", [False, True])
def test_graph_equals_run_circuit(L, fuse):
    n = 10
    psi = W.random_state(n, 3)
    gates = config0_gates(n)
    with L.State.create(n) as a, L.State.create(n) as b:
        a.copy_in(psi)
        b.copy_in(psi)
        with b.compile(gates, fuse=fuse) as c:
            assert c.kernels >= 1
            np.testing.assert_array_equal(b.copy_out(), psi)  # compile runs nothing
            k0 = b.launches()
            for _ in range(2):
                a.run_circuit(gates, fuse=fuse)
                c.launch()
            assert b.launches() - k0 == 2 * c.kernels
            got, ref = b.copy_out(), a.copy_out()
    assert np.array_equal(got, ref)
    want = O.run_circuit(n, gates + gates, psi.copy())
    assert np.max(np.abs(got - want)) <= 1e-12


def test_graph_exact_circuit_bit_exact_vs_oracle(L):
    n = 12
    psi = W.random_state(n, 5)
    gates = [g for g in W.random_gate_list(n, 300, seed=4, max_controls=2) if g.exact]
    with L.State.create(n) as st:
        st.copy_in(psi)
        with st.compile(gates) as c:
            c.launch()
        got = st.copy_out()
    assert np.array_equal(got, O.run_circuit(n, gates, psi.copy()))


@pytest.mark.parametrize("world", [2, 4])
def test_graph_virtual_partition(L, world):
    n = 12
    psi = W.random_state(n, 6)
    gates = W.random_gate_list(n, 150, seed=world, max_controls=2) + W.qft(n)
    with L.State.virtual(n, world) as st:
        st.copy_in(psi)
        with st.compile(gates, fuse=True) as c:
            c.launch()
            c.launch()
        got = st.copy_out()
    want = O.run_circuit(n, gates + gates, psi.copy())
    assert np.max(np.abs(got - want)) <= 1e-12


def test_graph_on_torch_stream(L):
    import torch
    n = 14
    s = torch.cuda.Stream()
    gates = W.qft(n)
    x = 12345
    with L.State.create(n, stream=s) as st:
        st.init_basis(x)
        with st.compile(gates, fuse=True) as c:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            c.launch()
            e1.record(s)
            torch.cuda.synchronize()
            assert e0.elapsed_time(e1) > 0
        got = st.copy_out()
    k = np.arange(1 << n)
    want = np.exp(2j * np.pi * ((x * k) % (1 << n)) / (1 << n)) / np.sqrt(2.0 ** n)
    assert np.max(np.abs(got - want)) <= 1e-13


def test_graph_rejects_bad_gate(L):
    with L.State.create(6) as st:
        with pytest.raises(L.LfqsError):
            st.compile([W.Gate("H", (9,))])
        st.apply(W.Gate("H", (0,)))  # the state is still usable after a failed compile
        assert abs(st.norm2() - 1.0) < 1e-15
