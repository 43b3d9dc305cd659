"""GPU (C-ABI) vs oracle parity -- the first gate.

Bar (BASELINE.json north_star): permutation and diagonal gates bit-exact
(IEEE == per component); everything else max |diff| <= 1e-12 per amplitude;
norm drift <= 1e-12 per 1000 gates.  Every input is seeded; nothing expected
comes from the CUDA path.
"""
import math

import numpy as np
import pytest

import oracle as O
import workloads as W

pytestmark = pytest.mark.gpu

TOL = 1e-12


@pytest.fixture(scope="module")
def L():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import paper_conf_cgo_tarabkhahdds25_b200 as lib
    lib.lib()
    return lib


def _cmp(got, ref, exact, label=""):
    if exact:
        bad = np.flatnonzero((got.real != ref.real) | (got.imag != ref.imag))
        assert bad.size == 0, f"{label}: {bad.size} amplitudes differ, first at {bad[:5]}: " \
                              f"{got[bad[:3]]} vs {ref[bad[:3]]}"
    else:
        err = np.max(np.abs(got - ref)) if got.size else 0.0
        assert err <= TOL, f"{label}: max abs err {err:.3e}"


def _gpu_apply(L, n, psi, gates, fuse=False, shuffle=True):
    with L.State.create(n) as st:
        st.set_option(L.OPT_LOWQ_SHUFFLE, int(shuffle))
        st.copy_in(psi)
        st.run_circuit(gates, fuse=fuse)
        return st.copy_out()


# ---------------------------------------------------------------------------
# configs[0]: 10-qubit micro gates, every qubit index, tiers A and B
# ---------------------------------------------------------------------------

def test_config0_micro_gates_every_index(L):
    n = 10
    psi = W.random_state(n, 0x1F5)
    gates = W.micro_gates_10q(n)
    with L.State.create(n) as st:
        for g in gates:
            st.copy_in(psi)
            st.apply(g)
            got = st.copy_out()
            ref_b = O.apply_gate(n, g, psi.copy())
            exact = g.exact
            _cmp(got, ref_b, exact, g.label())
            if g.kind in ("H", "RZ") or (len(g.controls) == 1 and g.targets[0] in (0, 9)):
                _cmp(got, O.apply_dense(n, g, psi), exact, g.label() + " tierA")


@pytest.mark.parametrize("shuffle", [True, False])
@pytest.mark.parametrize("n", [7, 10, 13])
def test_every_kind_every_placement(L, n, shuffle):
    """Single gates of every kind on random targets/controls, fresh state each."""
    rng = np.random.default_rng(1000 + n)
    psi = W.random_amplitudes(77 + n, 0, 1 << n)
    with L.State.create(n) as st:
        st.set_option(L.OPT_LOWQ_SHUFFLE, int(shuffle))
        for g in W.random_gate_list(n, 150, seed=n * 31 + shuffle, max_controls=3):
            st.copy_in(psi)
            st.apply(g)
            _cmp(st.copy_out(), O.apply_gate(n, g, psi.copy()), g.exact, g.label())
        for t in range(n):  # every low/high target for the pair kernels, with controls
            for kind in ("X", "Y", "H", "RX", "U3", "Z", "T", "RZ"):
                params = tuple(rng.uniform(0, 2 * math.pi, W.NPARAMS[kind]))
                ctrl = tuple(q for q in (t + 3, t + 5) if q < n)[: rng.integers(0, 3)]
                g = W.Gate(kind, (t,), ctrl, params)
                st.copy_in(psi)
                st.apply(g)
                _cmp(st.copy_out(), O.apply_gate(n, g, psi.copy()), g.exact, g.label())


@pytest.mark.parametrize("n", [3, 5, 11])
def test_two_and_three_target_dense_all_orders(L, n):
    """Eq. 5: non-adjacent 2q gates in both target orders; 3q gates, with qubit 0."""
    rng = np.random.default_rng(n)
    psi = W.random_amplitudes(5, 0, 1 << n)
    with L.State.create(n) as st:
        pairs = [(a, b) for a in range(n) for b in range(n) if a != b]
        for (a, b) in pairs[:: max(1, len(pairs) // 40)]:
            for kind in ("UNITARY2", "SWAP"):
                mat = W.haar_unitary(2, a * 100 + b) if kind == "UNITARY2" else None
                g = W.Gate(kind, (a, b), (), (), mat)
                st.copy_in(psi)
                st.apply(g)
                _cmp(st.copy_out(), O.apply_gate(n, g, psi.copy()), g.exact, g.label())
        if n >= 3:
            for _ in range(20):
                t = tuple(int(x) for x in rng.choice(n, 3, replace=False))
                g = W.Gate("UNITARY3", t, (), (), W.haar_unitary(3, int(rng.integers(1 << 30))))
                st.copy_in(psi)
                st.apply(g)
                _cmp(st.copy_out(), O.apply_gate(n, g, psi.copy()), False, g.label())


@pytest.mark.parametrize("n", [12, 16])
def test_random_circuits_vs_oracle(L, n):
    """Eq. 3: a seeded circuit of every kind, run through lfqs_run_circuit."""
    psi = W.random_state(n, 99 + n)
    gates = W.random_gate_list(n, 300, seed=n, max_controls=2)
    ref = O.run_circuit(n, gates, psi.copy())
    got = _gpu_apply(L, n, psi, gates)
    _cmp(got, ref, False, f"circuit n={n}")
    exact_only = [g for g in gates if g.exact]
    _cmp(_gpu_apply(L, n, psi, exact_only), O.run_circuit(n, exact_only, psi.copy()), True,
         "perm/diag circuit")


def test_ragged_and_edge_cases(L):
    """n = 1..6 (smaller than a warp / tile), MC-Z (n-1 controls), identity, diagonal UNITARY."""
    for n in range(1, 7):
        psi = W.random_amplitudes(n, 0, 1 << n)
        gs = [W.Gate("H", (n - 1,)), W.Gate("I", (0,)), W.Gate("T", (0,))]
        if n > 1:
            gs += [W.mcz(n), W.Gate("UNITARY2", (0, n - 1), (), (),
                                    np.diag(np.exp(1j * np.arange(4.0)))), W.CNOT(n - 1, 0)]
        for g in gs:
            got = _gpu_apply(L, n, psi, [g])
            _cmp(got, O.apply_gate(n, g, psi.copy()), g.exact or g.kind == "UNITARY2", g.label())


# ---------------------------------------------------------------------------
# Full size (BASELINE configs[1], n = 30, bench launch configuration): sampled
# ---------------------------------------------------------------------------

def test_full_size_sampled_n30(L):
    """At n = 30 (16 GiB) the oracle computes sampled output groups one by one from the
    same counter-based input (workloads.random_amplitudes_at): every gate kind and class of
    the bench sweep on targets 0, 1, 4, 5, 17, 29 (incl. the line-shaped sparse-touch
    kernels: Toffoli on controls {1, 2}, controls / one-entry diagonals on qubit 1)."""
    n, seed = 30, 0xC0FFEE
    rng = np.random.default_rng(30)
    sweep = dict()
    for cls, g in W.sweep_gates(n):
        if g.targets[0] in (0, 1, 4, 5, 17, 29):
            sweep.setdefault((cls, g.kind, len(g.controls), g.targets[0]), g)
    with L.State.create(n) as st:
        for key, g in sorted(sweep.items(), key=lambda kv: str(kv[0])):
            st.init_random(seed)
            st.apply(g)
            tm = sum(1 << t for t in g.targets)
            m = len(g.targets)
            bases = rng.integers(0, 1 << n, 24, dtype=np.uint64) & np.uint64(~tm & ((1 << n) - 1))
            idx = np.unique(np.array([int(b) | sum(((j >> (m - 1 - s)) & 1) << t
                                                   for s, t in enumerate(g.targets))
                                      for b in bases for j in range(1 << m)], dtype=np.uint64))
            ref = O.apply_gate_sparse(n, g, idx, W.random_amplitudes_at(seed, idx))
            got = np.array([st.copy_out(int(k), 1)[0] for k in idx])
            _cmp(got, ref, g.exact, f"n=30 {g.label()}")


# ---------------------------------------------------------------------------
# Measurement, closed forms, invariants
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("n", [4, 12, 20])
def test_measure_probs_vs_oracle(L, n):
    psi = W.random_state(n, n)
    with L.State.create(n) as st:
        st.copy_in(psi)
        for qs in ([], [0], [n - 1], [1, 3], [2, 0, n - 1], list(range(min(n, 10)))):
            got = st.measure_probs(qs)
            ref = O.probs(n, psi, qs)
            np.testing.assert_allclose(got, ref, rtol=1e-13, atol=1e-16)
            assert np.array_equal(got, st.measure_probs(qs))  # deterministic


@pytest.mark.parametrize("n,world", [(11, 1), (16, 1), (21, 1), (16, 4)])
def test_measure_probs_many_qubits_one_pass(L, n, world):
    """11..20 measured qubits (two-level binning: the 10 lowest positions in the shared
    histogram, the rest select subspaces), in caller order, including lane bits, vs the
    oracle's pairwise sums; deterministic; also through a virtual partition."""
    psi = W.random_state(n, 3 * n)
    rng = np.random.default_rng(n)
    cases = [list(range(min(n, 20))), list(range(n - 1, max(-1, n - 21), -1)),
             [int(x) for x in rng.permutation(n)[:min(n, 20)]],
             [int(x) for x in rng.permutation(n)[:11]]]
    st = L.State.create(n) if world == 1 else L.State.virtual(n, world)
    with st:
        st.copy_in(psi)
        if world > 1:
            st.run_circuit([W.Gate("X", (n - 1,)), W.Gate("X", (n - 1,))])  # flip + unflip
        for qs in cases:
            got = st.measure_probs(qs)
            ref = O.probs(n, psi, qs)
            np.testing.assert_allclose(got, ref, rtol=1e-13, atol=1e-17, err_msg=str(qs))
            assert np.array_equal(got, st.measure_probs(qs))


def test_measure_probs_20_qubits_costs_one_pass(L):
    """n = 28, 20 measured qubits: one read pass (not 2^10 filtered passes):
    the 20-qubit measurement costs at most ~2x the 1-qubit one (same bytes read)."""
    import time
    n = 28
    with L.State.create(n) as st:
        st.init_random(5)
        for qs in ([3], list(range(4, 24))):
            st.measure_probs(qs)  # warm-up (scratch allocation)
        t = {}
        for key, qs in (("one", [3]), ("twenty", list(range(4, 24)))):
            t0 = time.perf_counter()
            for _ in range(5):
                st.measure_probs(qs)
            t[key] = (time.perf_counter() - t0) / 5
        assert t["twenty"] <= 2.5 * t["one"] + 2e-3, t


@pytest.mark.parametrize("n", [8, 20, 26])
def test_ghz_and_uniform_closed_forms(L, n):
    with L.State.create(n) as st:
        st.run_circuit(W.ghz(n))
        a = st.copy_out()
        s2 = math.sqrt(0.5)
        assert a[0] == s2 and a[-1] == s2 and np.count_nonzero(a) == 2
        st.init_basis(0)
        st.run_circuit([W.Gate("H", (q,)) for q in range(n)])
        a = st.copy_out()
        assert np.all(a == a[0]) and abs(a[0].real - 2.0 ** (-n / 2)) <= n * np.spacing(2.0 ** (-n / 2))


@pytest.mark.parametrize("n,x", [(10, 777), (18, 123457)])
def test_qft_closed_form(L, n, x):
    with L.State.create(n) as st:
        st.init_basis(x)
        st.run_circuit(W.qft(n))
        a = st.copy_out()
    y = np.arange(1 << n, dtype=np.int64)
    ref = np.exp(2j * np.pi * ((x * y) % (1 << n)) / (1 << n)) / math.sqrt(1 << n)
    assert np.max(np.abs(a - ref)) <= 1e-12


def test_grover_closed_form(L):
    n, k, w = 12, 5, 0b101101110001
    with L.State.create(n) as st:
        st.run_circuit(W.grover(n, w, k))
        a = st.copy_out()
    th = math.asin(2.0 ** (-n / 2))
    ref = np.full(1 << n, (-1) ** k * math.cos((2 * k + 1) * th) / math.sqrt((1 << n) - 1))
    ref[w] = (-1) ** k * math.sin((2 * k + 1) * th)
    assert np.max(np.abs(a - ref)) <= 1e-12


def test_norm_drift_1000_gates(L):
    n = 20
    gates = W.random_layered(n, 34, seed=3)[:1000]
    with L.State.create(n) as st:
        st.init_random(5)
        n0 = st.norm2()
        st.run_circuit(gates)
        assert abs(st.norm2() / n0 - 1.0) <= 1e-12


# ---------------------------------------------------------------------------
# Boundary behaviour
# ---------------------------------------------------------------------------

def test_wrap_torch_tensor_and_stream(L):
    import torch
    n = 12
    psi = W.random_state(n, 4)
    t = torch.from_numpy(psi.copy()).cuda()
    s = torch.cuda.Stream()
    with L.State.wrap(t, stream=s) as st:
        g = W.Gate("U3", (3,), (7,), (0.1, 0.2, 0.3))
        st.apply(g)
        st.synchronize()
    _cmp(t.cpu().numpy(), O.apply_gate(n, g, psi.copy()), False, "wrap")


@pytest.mark.parametrize("dtype,bad,good", [("complex128", 1, 2), ("complex64", 1, 2),
                                             ("complex64", 3, 4)])
def test_wrap_rejects_underaligned_views(L, dtype, bad, good):
    """The wrap contract is as wide as the narrowest kernel access (two amplitudes per
    vector access: 32 B complex128, 16 B complex64): a torch view offset by an odd
    number of amplitudes is LFQS_ERR_INVALID_ARG, not a misaligned-address fault; a view
    at the next aligned offset works and matches the oracle."""
    import torch
    n = 9
    dt = getattr(torch, dtype)
    base = torch.zeros((1 << n) + 8, dtype=dt, device="cuda")
    with pytest.raises(L.LfqsError) as e:
        L.State.wrap(base[bad:bad + (1 << n)])
    assert e.value.status == -1 and "aligned" in str(e.value)
    psi = W.random_state(n, 12)
    if dtype == "complex64":
        psi = psi.astype(np.complex64)
    view = base[good:good + (1 << n)]
    view.copy_(torch.from_numpy(psi))
    g = W.Gate("U3", (0,), (4,), (0.3, -0.2, 0.9))
    with L.State.wrap(view) as st:
        st.apply(g)
        st.apply(W.Gate("T", (0,)))
        st.synchronize()
    ref = O.apply_gate(n, W.Gate("T", (0,)), O.apply_gate(n, g, psi.astype(np.complex128)))
    tol = 1e-12 if dtype == "complex128" else 2e-6
    assert np.max(np.abs(view.cpu().numpy().astype(np.complex128) - ref)) <= tol
    assert torch.count_nonzero(base[:good]) == 0     # nothing written outside the view
    assert torch.count_nonzero(base[good + (1 << n):]) == 0


def test_invalid_arguments_raise(L):
    with L.State.create(5) as st:
        for bad in [dict(kind="H", targets=(5,)), dict(kind="X", targets=(1,), controls=(1,)),
                    dict(kind="SWAP", targets=(1, 1)), dict(kind="RX", targets=(0,)),
                    dict(kind="UNITARY1", targets=(0,))]:
            with pytest.raises(L.LfqsError) as e:
                st.apply_gate(**bad)
            assert e.value.status == -1
        with pytest.raises(L.LfqsError):
            st.measure_probs(list(range(5)) + [0])
        with pytest.raises(L.LfqsError):
            st.copy_out(30, 5)
    with pytest.raises(L.LfqsError) as e:
        L.State.create(36 + 1)
    assert e.value.status == -1


def test_kernel_launch_accounting(L):
    with L.State.create(14) as st:
        c0 = st.launches()
        st.run_circuit([W.Gate("H", (q,)) for q in range(14)])
        assert st.launches() - c0 == 14


@pytest.mark.parametrize("fuse", [False, True])
def test_table1_workloads_vs_oracle(L, fuse):
    """QPE (closed form), VQE ansatz and Sycamore-like circuits (Table 1)."""
    for n, gates in ((13, W.qpe(12, 2901)), (14, W.vqe_ansatz(14, 4, seed=3)),
                     (15, W.sycamore_like(3, 5, 12, seed=4))):
        psi = W.basis_state(n, 0)
        ref = O.run_circuit(n, gates, psi.copy())
        got = _gpu_apply(L, n, psi, gates, fuse=fuse)
        assert np.max(np.abs(got - ref)) <= 1e-12
    with L.State.create(13) as st:
        st.run_circuit(W.qpe(12, 2901), fuse=fuse)
        assert abs(st.measure_probs(list(range(12)))[2901] - 1.0) < 1e-12


# ---------------------------------------------------------------------------
# Dense 4x4 / 8x8 gates with every target in qubits 1..5 (coalesced lane-group
# kernel, LFQS_OPT_LANE_GROUP): same terms in the same order as the group kernel
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("c64", [False, True])
@pytest.mark.parametrize("n", [8, 9, 13])
def test_lane_group_dense_low_targets(L, n, c64):
    psi = W.random_state(n, 77 + n)
    if c64:
        psi = psi.astype(np.complex64).astype(np.complex128)
    cases = []
    for ts in [(1, 2), (2, 1), (1, 5), (5, 3), (4, 2), (1, 2, 3), (3, 1, 5), (5, 4, 2)]:
        m = len(ts)
        U = W.haar_unitary(m, sum(ts) + 7 * m)
        kind = "UNITARY2" if m == 2 else "UNITARY3"
        free = [q for q in range(n) if q not in ts]
        for ctrl in [(), (0,), (free[-1],), (free[1], free[-1]), (6,) if 6 in free else ()]:
            cases.append(W.Gate(kind, ts, tuple(ctrl), (), U))
    tol = 4e-6 if c64 else TOL
    for g in cases:
        ref = O.apply_gate(n, g, psi.copy())
        outs = []
        for lg in (2, 0):
            with L.State.create(n, c64=c64) as st:
                st.set_option(L.OPT_LANE_GROUP, lg)
                st.copy_in(psi)
                st.apply(g)
                outs.append(st.copy_out())
        assert np.array_equal(outs[0], outs[1]), g  # forced lane-group == group kernel
        assert np.max(np.abs(outs[0] - ref)) <= tol, g


# ---------------------------------------------------------------------------
# Maximum sizes on one B200 (180 GB HBM3e): n = 33 complex128 and n = 34 complex64,
# 128 GiB each (BASELINE configs[2]); sampled outputs against the sparse oracle and
# closed forms
# ---------------------------------------------------------------------------

def _free_gib():
    import torch
    free, _ = torch.cuda.mem_get_info()
    return free / 2 ** 30


def test_maximum_size_n33_c128(L):
    if _free_gib() < 132:
        pytest.skip("needs 128 GiB of free device memory")
    n, seed = 33, 0x5EED33
    rng = np.random.default_rng(33)
    s2 = math.sqrt(0.5)
    top = (1 << n) - 1
    with L.State.create(n) as st:
        # single gates on the top qubit / spanning the whole index range vs the sparse oracle
        for g in [W.Gate("H", (n - 1,)), W.Gate("UNITARY2", (0, n - 1), (), (), W.haar_unitary(2, 9)),
                  W.TOFFOLI(n - 2, 1, n - 1), W.CPHASE(n - 1, 0, 0.7), W.Gate("U3", (16,), (n - 1,),
                                                                            (0.3, 1.1, -0.4))]:
            st.init_random(seed)
            st.apply(g)
            tm = sum(1 << t for t in g.targets)
            m = len(g.targets)
            bases = rng.integers(0, 1 << n, 16, dtype=np.uint64) & np.uint64(~tm & top)
            idx = np.unique(np.array([int(b) | sum(((j >> (m - 1 - s)) & 1) << t
                                                   for s, t in enumerate(g.targets))
                                      for b in bases for j in range(1 << m)], dtype=np.uint64))
            ref = O.apply_gate_sparse(n, g, idx, W.random_amplitudes_at(seed, idx))
            got = np.array([st.copy_out(int(k), 1)[0] for k in idx])
            _cmp(got, ref, g.exact, f"n=33 {g.label()}")
        # GHZ(33), compiled fused passes: two amplitudes of exactly 1/sqrt(2), zeros elsewhere
        st.init_basis(0)
        st.run_circuit(W.ghz(n), fuse="jit")
        assert st.copy_out(0, 1)[0] == s2 and st.copy_out(top, 1)[0] == s2
        for k in rng.integers(1, top, 32):
            assert st.copy_out(int(k), 1)[0] == 0
        assert st.measure_probs([]).sum() == 2 * (s2 * s2)  # |M_SQRT1_2|^2 = 0.5 + 1.1e-16
        # QFT(33)|x>, compiled passes with phase tables: closed form on sampled amplitudes
        x = 0x1F2E3D4C5 & top
        st.init_basis(x)
        st.run_circuit(W.qft(n), fuse="jit+phase")
        ys = [0, 1, top] + [int(v) for v in rng.integers(0, 1 << n, 61)]
        got = np.array([st.copy_out(y, 1)[0] for y in ys])
        ref = np.array([np.exp(2j * np.pi * ((x * y) % (1 << n)) / (1 << n)) for y in ys]) \
            / math.sqrt(2.0 ** n)
        assert np.max(np.abs(got - ref)) <= 1e-12


def test_maximum_size_n34_c64(L):
    if _free_gib() < 132:
        pytest.skip("needs 128 GiB of free device memory")
    n = 34
    top = (1 << n) - 1
    with L.State.create(n, c64=True) as st:
        st.init_basis(0)
        st.run_circuit(W.ghz(n), fuse="jit")
        s2 = float(np.float32(math.sqrt(0.5)))
        assert st.copy_out(0, 1)[0] == s2 and st.copy_out(top, 1)[0] == s2
        rng = np.random.default_rng(34)
        for k in rng.integers(1, top, 32):
            assert st.copy_out(int(k), 1)[0] == 0
