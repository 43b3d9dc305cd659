"""lfqs_run_circuit_streamed: the whole-state upload overlapped with the circuit prefix
that stays inside the upload pieces (Eq. 1: a gate below the piece bits acts on every
piece independently).  Without fusion it must equal lfqs_copy_in + lfqs_run_circuit bit for
bit, for every piece count and prefixes of any length (empty, partial, the whole circuit);
with fusion the prefix and the rest are fused separately (different pass boundaries), so
dense results agree within rounding and permutation/diagonal circuits stay exact."""
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


def _plain(L, n, psi, gates, fuse):
    with L.State.create(n) as st:
        st.copy_in(psi)
        st.run_circuit(gates, fuse=fuse)
        return st.copy_out()


def _streamed(L, n, psi, gates, fuse, cb, max_prefix=0):
    with L.State.create(n) as st:
        st.set_option(L.OPT_STREAM_MAX_PREFIX, max_prefix)
        st.init_basis(0)
        st.run_circuit_streamed(psi, gates, fuse=fuse, chunk_bits=cb)
        return st.copy_out()


@pytest.mark.parametrize("fuse", [False, True, "jit+phase"])
@pytest.mark.parametrize("cb", [0, 1, 3, 5])
def test_streamed_equals_copy_in_then_run(L, cb, fuse):
    n = 16
    psi = np.ascontiguousarray(W.random_state(n, 11 + cb))
    low = W.random_gate_list(n - 5, 120, seed=cb, max_controls=2)  # inside every piece
    gates = low + W.random_gate_list(n, 150, seed=cb + 1, max_controls=2) + W.qft(n)
    a = _plain(L, n, psi, gates, fuse)
    b = _streamed(L, n, psi, gates, fuse, cb)
    if fuse is False or cb == 0:
        assert np.array_equal(a, b)
    else:
        assert np.max(np.abs(a - b)) <= 1e-12
    assert np.max(np.abs(b - O.run_circuit(n, gates, psi.copy()))) <= 1e-12
    if fuse is True:
        exact = [g for g in gates if g.exact]
        assert np.array_equal(_streamed(L, n, psi, exact, fuse, cb),
                              O.run_circuit(n, exact, psi.copy()))


def test_streamed_edge_prefixes(L):
    n = 14
    psi = np.ascontiguousarray(W.random_state(n, 5))
    only_low = W.random_gate_list(n - 3, 80, seed=2)
    starts_high = [W.Gate("H", (n - 1,))] + only_low
    for gates in (only_low, starts_high, []):
        for cb in (2, 3):
            for mp in (0, 1, 17):  # LFQS_OPT_STREAM_MAX_PREFIX
                assert np.array_equal(_plain(L, n, psi, gates, False),
                                      _streamed(L, n, psi, gates, False, cb, mp))


def test_streamed_sweep_configs1_shape(L):
    """The bench's e2e call: the configs[1] sweep (18 kinds x n targets) at small n."""
    n = 15
    psi = np.ascontiguousarray(W.random_state(n, 9))
    gates = [g for _, g in W.sweep_gates(n)]
    assert np.array_equal(_plain(L, n, psi, gates, False), _streamed(L, n, psi, gates, False, 3))


def test_streamed_rejects_bad_args(L):
    with L.State.create(10) as st:
        with pytest.raises(L.LfqsError):
            st.run_circuit_streamed(np.zeros(1 << 10, np.complex128), [], chunk_bits=9)
    with L.State.virtual(10, 2) as st:
        with pytest.raises(L.LfqsError):
            st.run_circuit_streamed(np.zeros(1 << 10, np.complex128), [], chunk_bits=1)
