"""Global-qubit exchanges overlapped with local work (BASELINE
north_star "overlapped with local work on separate streams"), on the single-GPU virtual
partition: the exchange is split into 2^c parts by the top c local qubits, moved on an
exchange stream while the neighbouring local ops run part by part (state.cu
overlapped_exchange).  Unfused runs apply exactly the same kernels per amplitude as the
serial path, and fused runs launch exactly the serial run's passes block by block, so
both are bit-identical to serial exchanges; all are held to the oracle (<= 1e-12;
permutation/diagonal circuits bit-exact)."""
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


def _run(L, n, world, psi, gates, fuse, bits, ctas=0):
    with L.State.virtual(n, world) as st:
        st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, bits)
        st.set_option(L.OPT_EXCHANGE_CTAS, ctas)
        st.copy_in(psi)
        x0 = st.exchange_stats()[0]
        st.run_circuit(gates, fuse=fuse)
        nx = st.exchange_stats()[0] - x0
        out = st.copy_out()
        probs = st.measure_probs([n - 1, 1])
    return out, probs, nx


@pytest.mark.parametrize("world", [2, 4, 8])
def test_overlap_unfused_bit_identical_to_serial(L, world):
    """The plan does not depend on the chunk bits (the planner always keeps the top two
    local positions free), so chunk bits 0 (serial exchanges), 1, 2 (default), 3 (an
    exchange at position n_local - 3 falls back to serial) and a grid-limited swap kernel
    all run the same plan; unfused they apply the same kernels per amplitude: bit-identical."""
    n = 14
    psi = W.random_state(n, 31 + world)
    gates = (W.random_gate_list(n, 160, seed=70 + world, max_controls=2) + W.qft(n) +
             W.random_layered(n, 3, seed=world))
    ref = O.run_circuit(n, gates, psi.copy())
    serial, ps, nx0 = _run(L, n, world, psi, gates, False, 0)
    assert nx0 > 0
    assert np.max(np.abs(serial - ref)) <= 1e-12
    for bits, ctas in ((2, 0), (2, 8), (1, 0), (3, 3)):
        out, probs, nx = _run(L, n, world, psi, gates, False, bits, ctas)
        assert nx == nx0
        assert np.array_equal(out, serial), (bits, ctas)
        assert np.array_equal(probs, ps), (bits, ctas)


@pytest.mark.parametrize("fuse", [True, "jit", "jit+phase"])
@pytest.mark.parametrize("world", [2, 8])
def test_overlap_fused_vs_oracle(L, world, fuse):
    n = 16
    psi = W.random_state(n, 9)
    gates = W.random_gate_list(n, 200, seed=world, max_controls=2) + W.qft(n)
    ref = O.run_circuit(n, gates, psi.copy())
    exact = [g for g in W.random_gate_list(n, 300, seed=world + 1, max_controls=2) if g.exact]
    ref_exact = O.run_circuit(n, exact, psi.copy())
    serial = None
    for bits in (0, 2, 3):
        out, probs, _ = _run(L, n, world, psi, gates, fuse, bits)
        assert np.max(np.abs(out - ref)) <= 1e-12, bits
        np.testing.assert_allclose(probs, O.probs(n, ref, [n - 1, 1]), rtol=1e-12, atol=1e-15)
        if serial is None:
            serial = out
        else:  # the overlapped run launches the serial run's passes, block by block
            assert np.array_equal(out, serial), bits
        if fuse != "jit+phase":
            out, _, _ = _run(L, n, world, psi, exact, fuse, bits)
            assert np.array_equal(out, ref_exact), bits


@pytest.mark.parametrize("fuse", [True, "jit", "jit+phase"])
@pytest.mark.parametrize("world,n,tile", [(4, 20, 12), (2, 16, 8), (8, 17, 8)])
def test_chunk_select_bit_identical(L, world, n, tile, fuse):
    """LFQS_OPT_EXCHANGE_CHUNK_SELECT: each exchange's chunk qubits are chosen among the
    local qubits at or above the tile size (fixed bits of the fused passes' tile index,
    strided blocks for the swap kernels), and consecutive exchanges sharing them are
    chained block by block.  The passes are the serial run's: bit-identical to serial
    exchanges and to the top-qubit blocks, within 1e-12 of the oracle; strided and
    chained exchanges do occur."""
    psi = W.random_state(n, 5 + world)
    gates = (W.qft(n) + W.random_layered(n, 3, seed=world) +
             W.random_gate_list(n, 120, seed=world, max_controls=2) + W.ghz(n))
    ref = O.run_circuit(n, gates, psi.copy())
    outs, stats = {}, {}
    for bits, sel, ctas, rate in ((0, 1, 0, 0), (2, 0, 0, 0), (2, 1, 0, 0), (3, 1, 8, 0),
                                  (1, 1, 0, 0), (2, 1, 0, 200)):
        with L.State.virtual(n, world) as st:
            st.set_option(L.OPT_FUSE_TILE_QUBITS, tile)
            st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, bits)
            st.set_option(L.OPT_EXCHANGE_CHUNK_SELECT, sel)
            st.set_option(L.OPT_EXCHANGE_CTAS, ctas)
            st.set_option(L.OPT_EXCHANGE_RATE_GBS, rate)
            st.copy_in(psi)
            st.run_circuit(gates, fuse=fuse)
            outs[bits, sel, rate] = st.copy_out()
            stats[bits, sel, rate] = st.overlap_stats()
    serial = outs[0, 1, 0]
    assert np.max(np.abs(serial - ref)) <= 1e-12
    for k, o in outs.items():
        assert np.array_equal(o, serial), (k, stats[k])
    assert stats[0, 1, 0]["overlapped"] == 0
    st2 = stats[2, 1, 0]
    assert st2["overlapped"] > 0 and st2["block_passes"] > 0 and st2["strided"] > 0, st2
    assert stats[2, 0, 0]["strided"] == 0


def test_chunk_select_chains_exchanges(L):
    """Consecutive exchanges whose run between them leaves the chunk qubits unmixed run as
    a pipeline (part v of the second exchange starts when part v of the run is done): QFT
    on 8 shards takes the Hadamards of its three global qubits one after another, with only
    the swapped-in qubit mixed (and phase tables) between the exchanges."""
    n, world = 18, 8
    psi = W.random_state(n, 4)
    gates = W.qft(n) + W.random_gate_list(n, 100, seed=11, max_controls=1)
    ref = O.run_circuit(n, gates, psi.copy())
    with L.State.virtual(n, world) as st:
        st.set_option(L.OPT_FUSE_TILE_QUBITS, 8)
        st.copy_in(psi)
        st.run_circuit(gates, fuse="jit+phase")
        got = st.copy_out()
        stats = st.overlap_stats()
        st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, 0)
        st.copy_in(psi)
        st.run_circuit(gates, fuse="jit+phase")
        serial = st.copy_out()
    assert np.max(np.abs(got - ref)) <= 1e-12
    assert np.array_equal(got, serial)
    assert stats["overlapped"] > 0 and stats["chained"] > 0, stats


def test_overlap_graph_capture_and_per_gate_apply(L):
    """The exchange stream forks from and joins the capturing stream (lfqs_circuit_compile
    on a virtual partition), and per-gate lfqs_apply_gate overlaps its own exchange."""
    n, world = 14, 4
    psi = W.random_state(n, 77)
    gates = W.qft(n) + W.random_gate_list(n, 60, seed=2, max_controls=1)
    ref = O.run_circuit(n, gates, psi.copy())
    with L.State.virtual(n, world) as st:
        st.set_option(L.OPT_EXCHANGE_CTAS, 16)
        st.copy_in(psi)
        with st.compile(gates) as c:
            c.launch()
            got = st.copy_out()
        assert np.max(np.abs(got - ref)) <= 1e-12
        st.copy_in(psi)
        for g in gates:
            st.apply(g)
        assert np.max(np.abs(st.copy_out() - ref)) <= 1e-12


def test_pass_count(L):
    """lfqs_state_pass_count: one per single-gate kernel or fused pass; a pass run block by
    block around an overlapped exchange counts once (the per-pass roofline denominator)."""
    n = 14
    gates = W.random_gate_list(n, 50, seed=3, max_controls=1)
    with L.State.create(n) as st:
        p0 = st.passes()
        st.run_circuit(gates)
        assert st.passes() - p0 == len([g for g in gates if g.kind != "I"])
        p0, l0 = st.passes(), st.launches()
        st.run_circuit(gates, fuse="jit")
        assert 2 <= st.passes() - p0 <= st.launches() - l0
    for bits in (0, 2):
        with L.State.virtual(n, 4) as st:
            st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, bits)
            st.run_circuit(W.qft(n), fuse="jit")
            if bits == 0:
                serial = st.passes()
            else:
                assert st.passes() == serial


def test_exchange_options_validated(L):
    with L.State.virtual(10, 2) as st:
        for opt, bad in ((L.OPT_EXCHANGE_CHUNK_BITS, 4), (L.OPT_EXCHANGE_CHUNK_BITS, -1),
                         (L.OPT_EXCHANGE_CTAS, -1), (L.OPT_EXCHANGE_CTAS, 1 << 20)):
            with pytest.raises(L.LfqsError) as e:
                st.set_option(opt, bad)
            assert e.value.status == -1
        st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, 3)  # n_local = 9: 9 - 3 >= 4, still valid
        st.set_option(L.OPT_EXCHANGE_CTAS, 1)
        psi = W.random_state(10, 3)
        st.copy_in(psi)
        gates = W.qft(10)
        st.run_circuit(gates)
        assert np.max(np.abs(st.copy_out() - O.run_circuit(10, gates, psi.copy()))) <= 1e-12


def test_chunk_select_complex64(L):
    """Strided exchange blocks on a complex64 virtual partition (8-byte amplitudes in the
    swap kernels' fixed-bit indexing and the fused passes' tile-index insertions): the same
    bits as serial exchanges, within single-precision tolerance of the oracle."""
    n, world = 17, 4
    psi = W.random_state(n, 12)
    gates = W.qft(n) + W.random_layered(n, 3, seed=9)
    ref = O.run_circuit(n, gates, psi.copy())
    outs, strided = {}, 0
    for bits, rate in ((0, 0), (2, 0), (3, 300)):
        with L.State.virtual(n, world, c64=True) as st:
            st.set_option(L.OPT_FUSE_TILE_QUBITS, 8)
            st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, bits)
            st.set_option(L.OPT_EXCHANGE_RATE_GBS, rate)
            st.copy_in(psi)
            st.run_circuit(gates, fuse="jit+phase")
            outs[bits] = st.copy_out()
            strided += st.overlap_stats()["strided"]
    assert np.max(np.abs(outs[0] - ref)) <= 1e-5
    assert np.array_equal(outs[2], outs[0]) and np.array_equal(outs[3], outs[0])
    assert strided > 0


@pytest.mark.parametrize("world", [2, 8])
def test_canonicalize_fused(L, world):
    """LFQS_OPT_CANON_FUSE: the SWAP passes that restore the canonical map run fused (a run
    of them in one tile pass) with their exchanges overlapped -- moves only, so copy_out is
    bit-identical to one pass per SWAP, in fewer passes."""
    n = 18
    psi = W.random_state(n, 41)
    gates = W.qft(n) + W.random_gate_list(n, 60, seed=6, max_controls=1)
    ref = O.run_circuit(n, gates, psi.copy())
    outs, canon_passes = {}, {}
    for cf in (0, 1):
        with L.State.virtual(n, world) as st:
            st.set_option(L.OPT_CANON_FUSE, cf)
            st.set_option(L.OPT_FUSE_TILE_QUBITS, 10)
            st.copy_in(psi)
            st.run_circuit(gates, fuse="jit+phase")
            p0 = st.passes()
            outs[cf] = st.copy_out()  # canonicalises
            canon_passes[cf] = st.passes() - p0
    assert np.array_equal(outs[0], outs[1])
    assert np.max(np.abs(outs[1] - ref)) <= 1e-12
    assert canon_passes[1] <= canon_passes[0], canon_passes
