"""LFQS_FUSE_JIT: every fused pass compiled into its own kernel (csrc/jit.cpp).

The pass compiler emits the interpreting kernel's arithmetic op by op (same
formulas, FMA/rounding order and tile/register transitions), so a compiled pass
must equal the interpreted pass BIT FOR BIT on every circuit, tile geometry and
precision; against the oracle the usual bar holds (permutation/diagonal circuits
exact, otherwise max abs error <= 1e-12, BASELINE.json north_star)."""
import numpy as np
import pytest

import oracle as O
import workloads as W
from tests.test_gpu_phase import diag_heavy

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def L():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import paper_conf_cgo_tarabkhahdds25_b200 as lib
    lib.lib()
    return lib


def _run(L, n, psi, gates, fuse, tile=None, low=None, c64=False, reorder=1, threads=256,
         lane_move=None, greedy=None, lane_reg2=None, pool=None, partial=None):
    with L.State.create(n, c64=c64) as st:
        if partial is not None:
            st.set_option(L.OPT_JIT_PARTIAL_RT, partial)
        if pool is not None:
            st.set_option(L.OPT_JIT_LANE_POOL, pool)
        if lane_reg2 is not None:
            st.set_option(L.OPT_JIT_LANE_REG2, lane_reg2)
        if greedy is not None:
            st.set_option(L.OPT_JIT_GREEDY_PLACE, greedy)
        st.set_option(L.OPT_FUSE_REORDER, reorder)
        st.set_option(L.OPT_JIT_THREADS, threads)
        if lane_move is not None:
            st.set_option(L.OPT_JIT_LANE_MOVE, lane_move)
        if tile:
            st.set_option(L.OPT_FUSE_TILE_QUBITS, tile)
        if low:
            st.set_option(L.OPT_FUSE_LOW_QUBITS, low)
        st.copy_in(psi)
        c0 = st.launches()
        st.run_circuit(gates, fuse=fuse)
        return st.copy_out(), st.launches() - c0


def _mixed(n, seed):
    return (W.random_gate_list(n, 220, seed=seed, max_controls=2) + W.qft(n) +
            W.random_layered(n, 4, seed=seed) + diag_heavy(n, 120, seed + 1))


@pytest.mark.parametrize("reorder", [0, 1])
@pytest.mark.parametrize("low", [5, 7])
@pytest.mark.parametrize("tile", [8, 10, 12])
@pytest.mark.parametrize("n", [13, 17])
def test_jit_equals_interpreter(L, n, tile, low, reorder):
    psi = W.random_state(n, 7 * n + tile + low)
    gates = _mixed(n, 1000 + 13 * n + tile + low)
    a, ka = _run(L, n, psi, gates, True, tile, low, reorder=reorder)
    b, kb = _run(L, n, psi, gates, "jit", tile, low, reorder=reorder)
    assert ka == kb
    assert np.array_equal(a, b)
    ref = O.run_circuit(n, gates, psi.copy())
    assert np.max(np.abs(b - ref)) <= 1e-12


@pytest.mark.parametrize("threads", [0, 128, 256, 512])
@pytest.mark.parametrize("tile", [9, 10, 12])
@pytest.mark.parametrize("n", [13, 16])
def test_jit_512_threads_equals_interpreter(L, n, tile, threads):
    """Compiled passes with 128 / 256 / 512 threads per CTA or chosen per pass (0, the
    default; LFQS_OPT_JIT_THREADS): a different thread/register placement of the same
    per-amplitude arithmetic."""
    psi = W.random_state(n, 3 * n + tile)
    gates = _mixed(n, 2000 + n + tile)
    a, _ = _run(L, n, psi, gates, True, tile)
    b, _ = _run(L, n, psi, gates, "jit", tile, threads=threads)
    assert np.array_equal(a, b)
    c, _ = _run(L, n, psi, gates, "phase", tile)
    d, _ = _run(L, n, psi, gates, "jit+phase", tile, threads=threads)
    assert np.array_equal(c, d)


@pytest.mark.parametrize("c64", [False, True])
@pytest.mark.parametrize("threads", [128, 256, 512])
@pytest.mark.parametrize("tile", [9, 12])
@pytest.mark.parametrize("greedy,pool", [(0, 0), (1, 0), (1, 1)])
@pytest.mark.parametrize("lane_move", [0, 1])
def test_jit_placement_variants_equal_interpreter(L, lane_move, greedy, pool, tile, threads, c64):
    """Tile-bit placement variants of the compiled passes: LFQS_OPT_JIT_LANE_MOVE (lane
    tile bits 3-4, complex64: 4, move into register positions and keep the interpreter's
    lane formulas there) and LFQS_OPT_JIT_GREEDY_PLACE (multi-bit remaps) -- all
    bit-identical to the interpreted pass on lane-heavy and layered circuits (Grover,
    layered, Sycamore-like)."""
    n = 15
    psi = W.random_state(n, 31 + tile)
    if c64:
        psi = psi.astype(np.complex64).astype(np.complex128)
    gates = (W.grover(n, 0x1A5B, 1) + W.random_layered(n, 5, seed=tile) +
             W.sycamore_like(3, 5, 4, seed=threads) + W.random_gate_list(n, 150, seed=9, max_controls=2))
    a, _ = _run(L, n, psi, gates, True, tile, c64=c64)
    b, _ = _run(L, n, psi, gates, "jit", tile, c64=c64, threads=threads, lane_move=lane_move,
                greedy=greedy, pool=pool)
    assert np.array_equal(a, b)
    c, _ = _run(L, n, psi, gates, "phase", tile, c64=c64)
    d, _ = _run(L, n, psi, gates, "jit+phase", tile, c64=c64, threads=threads,
                lane_move=lane_move, greedy=greedy, pool=pool)
    assert np.array_equal(c, d)
    tol = 2e-5 if c64 else 1e-12
    assert np.max(np.abs(b - O.run_circuit(n, gates, psi.copy()))) <= tol


@pytest.mark.parametrize("c64", [False, True])
@pytest.mark.parametrize("tile", [9, 10, 12])
@pytest.mark.parametrize("lane_reg2,pool,partial", [(0, 0, 1), (1, 0, 1), (1, 1, 1), (1, 0, 0),
                                                    (1, 1, 0)])
def test_jit_lane_register_2q_equals_interpreter(L, lane_reg2, pool, partial, tile, c64):
    """LFQS_OPT_JIT_LANE_REG2: SWAP / 2-target dense gates with one target on a lane
    bit and the other register-held run by shuffles in registers -- bit-identical to
    the interpreter's shared-memory op (2-target gates on every placement, with
    controls, Sycamore-like fSim layers); with and without the lane pool and partial
    round trips (LFQS_OPT_JIT_PARTIAL_RT)."""
    n = 14
    psi = W.random_state(n, 5 * tile + 1)
    if c64:
        psi = psi.astype(np.complex64).astype(np.complex128)
    gates = (W.random_gate_list(n, 300, seed=tile, max_targets=2, max_controls=2) +
             W.sycamore_like(2, 7, 6, seed=tile) + W.random_layered(n, 4, seed=tile) +
             W.random_gate_list(n, 100, seed=tile + 1, max_targets=3, max_controls=1))
    a, _ = _run(L, n, psi, gates, True, tile, c64=c64)
    b, _ = _run(L, n, psi, gates, "jit", tile, c64=c64, lane_reg2=lane_reg2, pool=pool,
                partial=partial)
    assert np.array_equal(a, b)
    tol = 2e-5 if c64 else 1e-12
    assert np.max(np.abs(b - O.run_circuit(n, gates, psi.copy()))) <= tol


@pytest.mark.parametrize("tile", [9, 12])
def test_jit_phase_equals_interpreter_phase(L, tile):
    n = 16
    psi = W.random_state(n, 99)
    gates = _mixed(n, 5) + W.qpe(n - 1, 0x2B3) + diag_heavy(n, 300, 17)
    a, _ = _run(L, n, psi, gates, "phase", tile)
    b, _ = _run(L, n, psi, gates, "jit+phase", tile)
    assert np.array_equal(a, b)
    assert np.max(np.abs(b - O.run_circuit(n, gates, psi.copy()))) <= 1e-12


def test_jit_exact_classes_bit_exact_vs_oracle(L):
    n = 15
    psi = W.random_state(n, 3)
    exact = [g for g in _mixed(n, 44) if g.exact]
    got, _ = _run(L, n, psi, exact, "jit")
    assert np.array_equal(got, O.run_circuit(n, exact, psi.copy()))


def test_jit_c64(L):
    n = 14
    psi = W.random_state(n, 8).astype(np.complex64).astype(np.complex128)
    gates = _mixed(n, 8)
    a, _ = _run(L, n, psi, gates, True, c64=True)
    b, _ = _run(L, n, psi, gates, "jit", c64=True)
    assert np.array_equal(a, b)
    assert np.max(np.abs(b - O.run_circuit(n, gates, psi.copy()))) <= 2e-5


def test_jit_macro_closed_forms(L):
    n = 20
    x = 0xABCDE
    with L.State.create(n) as st:
        for fuse in ("jit", "jit+phase"):
            st.init_basis(x)
            st.run_circuit(W.qft(n), fuse=fuse)
            a = st.copy_out()
            y = np.arange(1 << n, dtype=np.int64)
            ref = np.exp(2j * np.pi * ((x * y) % (1 << n)) / (1 << n)) / np.sqrt(1 << n)
            assert np.max(np.abs(a - ref)) <= 1e-12
            st.init_basis(0)
            st.run_circuit(W.ghz(n), fuse=fuse)
            g = st.copy_out()
            assert g[0] == np.sqrt(0.5) and g[-1] == np.sqrt(0.5)
            assert np.count_nonzero(g) == 2


def test_jit_virtual_partition_and_graph(L):
    """The sharded planner's fused local segments and captured circuits run the
    compiled passes too."""
    n = 14
    psi = W.random_state(n, 12)
    gates = _mixed(n, 21)
    ref = O.run_circuit(n, gates, psi.copy())
    for world in (2, 4):
        with L.State.virtual(n, world) as st:
            st.copy_in(psi)
            st.run_circuit(gates, fuse="jit")
            assert np.max(np.abs(st.copy_out() - ref)) <= 1e-12
    with L.State.create(n) as st:
        st.copy_in(psi)
        with st.compile(gates, fuse="jit") as c:
            c.launch()
        assert np.max(np.abs(st.copy_out() - ref)) <= 1e-12


def test_jit_precompile_then_run(L):
    n = 18
    gates = W.random_layered(n, 6, seed=2)
    k = L.lfqs_jit_precompile(n, gates, "jit")
    psi = W.random_state(n, 2)
    got, passes = _run(L, n, psi, gates, "jit")
    assert passes == k
    assert np.max(np.abs(got - O.run_circuit(n, gates, psi.copy()))) <= 1e-12


@pytest.mark.parametrize("c64", [False, True])
@pytest.mark.parametrize("fuse", ["jit", "jit+phase"])
def test_h_scale_folding(L, fuse, c64):
    """LFQS_OPT_FUSE_H_SCALE: a pass's unpredicated Hadamards compute unscaled butterflies
    and one of them carries (1/sqrt 2)^k.  Compiled == interpreted bit for bit with the
    folding on and off; within the dense tolerance of the oracle and of the unfolded pass
    (QFT, Grover and an H layer: passes with many Hadamards, controlled H left alone)."""
    n = 14
    psi = W.random_state(n, 21)
    gates = (W.qft(n) + W.grover(n, 1234, 1) + [W.Gate("H", (q,)) for q in range(n)] +
             [W.Gate("H", (3,), (9,)), W.Gate("H", (10,), (2, 5))] +
             W.random_gate_list(n, 80, seed=5, max_controls=2))
    ref = O.run_circuit(n, gates, psi.copy())
    tol = 1e-5 if c64 else 1e-12
    interp = True if fuse == "jit" else "phase"  # the interpreter of the same passes
    outs = {}
    for hs in (0, 1):
        for f in (interp, fuse):
            with L.State.create(n, c64=c64) as st:
                st.set_option(L.OPT_FUSE_H_SCALE, hs)
                st.copy_in(psi)
                st.run_circuit(gates, fuse=f)
                outs[hs, f] = st.copy_out()
            assert np.max(np.abs(outs[hs, f] - ref)) <= tol, (hs, f)
    for hs in (0, 1):  # interpreter == pass compiler
        assert np.array_equal(outs[hs, interp], outs[hs, fuse]), hs
    assert not np.array_equal(outs[0, fuse], outs[1, fuse])  # the folding did change the passes


@pytest.mark.parametrize("c64", [False, True])
@pytest.mark.parametrize("fuse", ["jit", "jit+phase"])
def test_phase_extraction(L, fuse, c64):
    """LFQS_OPT_FUSE_PHASE_EXTRACT: dense 1-target gates that are a global phase times a
    4-operation form (sqrt X = e^{i pi/4} Rx(pi/2), sqrt Y = e^{i pi/4} Ry(pi/2), phased
    Rx / Ry) run in that form with the phases carried by one other gate of the pass.
    Compiled == interpreted bit for bit with the extraction on and off; within the dense
    tolerance of the oracle (Sycamore-like cycles, random layered, controlled sqrt X left
    alone)."""
    n = 15
    psi = W.random_state(n, 33)
    sx = np.exp(1j * np.pi / 4) * np.array([[1, -1j], [-1j, 1]]) / np.sqrt(2)
    ph = np.exp(0.37j) * np.array([[np.cos(0.4), -np.sin(0.4)], [np.sin(0.4), np.cos(0.4)]])
    gates = (W.sycamore_like(3, 5, 6, seed=2) + W.random_layered(n, 3, seed=4) +
             [W.Gate("UNITARY1", (q,), (), (), ph if q % 2 else sx) for q in range(n)] +
             [W.Gate("UNITARY1", (3,), (7,), (), sx), W.Gate("UNITARY1", (9,), (), (), ph)])
    ref = O.run_circuit(n, gates, psi.copy())
    tol = 2e-5 if c64 else 1e-12
    interp = True if fuse == "jit" else "phase"
    outs = {}
    for pe in (0, 1):
        for f in (interp, fuse):
            with L.State.create(n, c64=c64) as st:
                st.set_option(L.OPT_FUSE_PHASE_EXTRACT, pe)
                st.copy_in(psi)
                st.run_circuit(gates, fuse=f)
                outs[pe, f] = st.copy_out()
            assert np.max(np.abs(outs[pe, f] - ref)) <= tol, (pe, f)
    for pe in (0, 1):
        assert np.array_equal(outs[pe, interp], outs[pe, fuse]), pe
    assert not np.array_equal(outs[0, fuse], outs[1, fuse])


def test_qft33_full_size_sampled(L):
    """configs[2] at full size in the bench's launch configuration (compiled passes + phase
    tables: folded Hadamard scales, hoisted table factors, the bit-permutation pass for the
    final SWAPs): QFT(33)|x> against its closed form e^{2 pi i x y / 2^33} / 2^16.5 on
    sampled amplitudes (the state does not fit the host oracle), and the norm."""
    import torch
    n = 33
    free = torch.cuda.mem_get_info()[0]
    if free < (16 << n) + (4 << 30):
        pytest.skip("needs a 128 GiB state")
    x = 0x1A2B3C4D5 & ((1 << n) - 1)
    rng = np.random.default_rng(3)
    idx = np.unique(np.concatenate([rng.integers(0, 1 << n, 200), [0, 1, (1 << n) - 1]]))
    with L.State.create(n) as st:
        st.init_basis(x)
        st.run_circuit(W.qft(n), fuse="jit+phase")
        got = np.array([st.copy_out(int(k), 1)[0] for k in idx])
        norm = st.norm2()
    ref = np.exp(2j * np.pi * ((x * idx.astype(object)) % (1 << n)).astype(np.float64) / (1 << n)) \
        / np.sqrt(2.0 ** n)
    assert np.max(np.abs(got - ref)) <= 1e-12
    assert abs(norm - 1.0) <= 1e-12
