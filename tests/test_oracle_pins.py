"""Pins for the CPU oracle against what the paper and mathematics fix (no GPU).

Each test names the passage it pins.  "P:N" = /root/reference/PAPER.md line N.
A plausible oracle bug (dropped term, wrong sign/index, transposed operand, wrong
bit order, wrong control projection) fails at least one of these; see DESIGN.md §3.
"""
import cmath
import itertools
import math

import numpy as np
import pytest
import scipy.linalg

import oracle as O
import workloads as W
from tests._tensor_ref import apply_tensor
from tests.conftest import read_golden

S2 = math.sqrt(0.5)  # correctly rounded 1/sqrt(2) (reading R4)


# --------------------------------------------------------------------------
# Gate table
# --------------------------------------------------------------------------

def _parse_entry(tok, sym):
    tok = tok.strip()
    if tok in sym:
        return sym[tok]
    return {"i": 1j, "-i": -1j, "e^{i pi/4}": cmath.exp(1j * math.pi / 4)}.get(tok, None) \
        if tok in ("i", "-i", "e^{i pi/4}") else complex(int(tok))


def _golden_fig1():
    out = {}
    for ln in read_golden("fig1_gates.txt"):
        name, scale, rows = [x.strip() for x in ln.split("|")]
        out[name] = (scale, [r.split() if "e^{" not in r else _split_keep(r) for r in rows.split(";")])
    return out


def _split_keep(row):
    toks, cur = [], ""
    for part in row.split(" "):
        if cur:
            cur += " " + part
            if "}" in part:
                toks.append(cur); cur = ""
        elif part.startswith("e^{") and "}" not in part:
            cur = part
        else:
            toks.append(part)
    return toks


def test_fig1_gate_matrices():
    """Fig. 1 literal entries, P:103-116 (X, Y, Z, H, T, I, SWAP, CNOT, CU)."""
    fig = _golden_fig1()
    rng = np.random.default_rng(5)
    u = W.haar_unitary(1, 77)
    sym = {f"u{r}{c}": u[r, c] for r in range(2) for c in range(2)}
    for name, (scale, rows) in fig.items():
        ref = np.array([[_parse_entry(t, sym) for t in r] for r in rows], dtype=np.complex128)
        if scale == "1/sqrt2":
            ref = ref / math.sqrt(2.0)
        if name in ("X", "Y", "Z", "H", "T", "I", "SWAP"):
            got = O.gate_matrix(W.Gate(name, (0,) if name != "SWAP" else (1, 0)))
        elif name == "CNOT":  # control = first (Kronecker-left) qubit = bit 1
            got = O.dense_kron(2, W.CNOT(1, 0))
        elif name == "CU":
            got = O.dense_kron(2, W.Gate("UNITARY1", (0,), (1,), (), u))
        assert got.shape == ref.shape, name
        np.testing.assert_allclose(got, ref, rtol=0, atol=2.3e-16 if name in ("H", "T") else 0,
                                   err_msg=name)


def _rand_params(kind, rng):
    return tuple(rng.uniform(-7, 7) for _ in range(W.NPARAMS[kind]))


def _pauli():
    X = np.array([[0, 1], [1, 0]], dtype=complex)
    Y = np.array([[0, -1j], [1j, 0]])
    Z = np.array([[1, 0], [0, -1]], dtype=complex)
    return X, Y, Z


@pytest.mark.parametrize("theta", [0.0, 0.3, -1.7, 2 * math.pi - 0.01, 5.5])
def test_rotation_gates_are_matrix_exponentials(theta):
    """Rx/Ry/Rz = exp(-i theta P/2) (N&C [27]; reading R7), Phase = diag(1, e^{i phi})."""
    X, Y, Z = _pauli()
    for kind, P in (("RX", X), ("RY", Y), ("RZ", Z)):
        got = O.gate_matrix(W.Gate(kind, (0,), (), (theta,)))
        np.testing.assert_allclose(got, scipy.linalg.expm(-0.5j * theta * P), atol=2e-15)
    got = O.gate_matrix(W.Gate("PHASE", (0,), (), (theta,)))
    np.testing.assert_allclose(got, np.diag([1, cmath.exp(1j * theta)]), atol=2e-16)


def test_u3_decomposition_and_discrete_gate_relations():
    """U3(t,p,l) = e^{i(p+l)/2} Rz(p) Ry(t) Rz(l); T^2 = S, S^2 = Z, H Z H = X, Tdg = T^dagger."""
    rng = np.random.default_rng(11)
    g = lambda k, *p: O.gate_matrix(W.Gate(k, (0,), (), p))
    for _ in range(20):
        t, p, l = rng.uniform(-7, 7, 3)
        ref = cmath.exp(0.5j * (p + l)) * g("RZ", p) @ g("RY", t) @ g("RZ", l)
        np.testing.assert_allclose(g("U3", t, p, l), ref, atol=3e-15)
    np.testing.assert_allclose(g("T") @ g("T"), g("S"), atol=3e-16)
    np.testing.assert_allclose(g("S") @ g("S"), g("Z"), atol=0)
    np.testing.assert_allclose(g("H") @ g("Z") @ g("H"), g("X"), atol=3e-16)
    np.testing.assert_allclose(g("TDG"), g("T").conj().T, atol=0)
    np.testing.assert_allclose(g("SDG"), g("S").conj().T, atol=0)
    X, Y, Z = _pauli()
    np.testing.assert_array_equal(g("Y"), Y)
    np.testing.assert_allclose(g("PHASE", math.pi / 4), g("T"), atol=2e-16)


def test_every_kind_is_unitary():
    """U U^dagger = I (gates are unitary, preserve the inner product)."""
    rng = np.random.default_rng(3)
    for kind in O.KINDS:
        m = W.ARITY[kind]
        mat = W.haar_unitary(m, 100 + m) if kind.startswith("UNITARY") else None
        for _ in range(5):
            U = O.gate_matrix(W.Gate(kind, tuple(range(m)), (), _rand_params(kind, rng), mat))
            np.testing.assert_allclose(U @ U.conj().T, np.eye(1 << m), atol=1e-15, err_msg=kind)


# --------------------------------------------------------------------------
# Embedding (Eq. 1, Eq. 4, Eq. 5) and the dense builders
# --------------------------------------------------------------------------

def _symbolic_u4():
    """4x4 matrix with 16 distinct entries, so the pattern identifies each u_rc."""
    return np.array([[complex(r * 4 + c + 1, 0.5 + r - 2 * c) for c in range(4)] for r in range(4)])


def test_g02_worked_matrix():
    """Eq. 5 worked matrix G_{0,2}: paper qubits 0 and 2 = bits 2 and 0."""
    U = _symbolic_u4()
    sym = {f"u{r}{c}": U[r, c] for r in range(4) for c in range(4)}
    ref = np.array([[sym.get(t, 0) if t != "0" else 0 for t in ln.split()]
                    for ln in read_golden("g02_matrix.txt")], dtype=np.complex128)
    g = W.Gate("UNITARY2", (2, 0), (), (), U)
    np.testing.assert_array_equal(O.dense_kron(3, g), ref)
    np.testing.assert_array_equal(O.dense_definition(3, g), ref)


@pytest.mark.parametrize("gap", [0, 1, 2, 3])
def test_eq4_swap_route_equals_eq5(gap):
    """Eq. 4 == Eq. 5 and the 2N-SWAP equivalence for gap N, exactly."""
    n = gap + 3
    U = _symbolic_u4()
    for lo in range(n - gap - 1):
        hi = lo + gap + 1
        for tg in ((hi, lo), (lo, hi)):
            for ctrl in ((), tuple(q for q in range(n) if q not in tg)[:1]):
                g = W.Gate("UNITARY2", tg, ctrl, (), U)
                A = O.dense_swap_route(n, g)
                B = O.dense_kron(n, g)
                np.testing.assert_array_equal(A, B)


def test_definition_builder_equals_kron_builder():
    """Definition (entrywise) == Fig.-5 Kronecker construction, every kind/placement (exact)."""
    rng = np.random.default_rng(21)
    for n in (1, 2, 3, 4, 5):
        for kind in O.KINDS:
            m = W.ARITY[kind]
            if m > n:
                continue
            for _ in range(6):
                qs = rng.permutation(n)
                nc = rng.integers(0, n - m + 1)
                mat = W.haar_unitary(m, int(rng.integers(1 << 30))) if kind.startswith("UNITARY") else None
                g = W.Gate(kind, tuple(int(x) for x in qs[:m]),
                           tuple(int(x) for x in qs[m:m + nc]), _rand_params(kind, rng), mat)
                np.testing.assert_array_equal(O.dense_kron(n, g), O.dense_definition(n, g),
                                              err_msg=g.label())


def test_sdql_example1_mvdot():
    """SDQL Example 1: M . V = {0 -> m0 v0 + m1 v2, 1 -> m2 v1 + m3 v2}."""
    rng = np.random.default_rng(8)
    m = rng.normal(size=4) + 1j * rng.normal(size=4)
    v = rng.normal(size=3) + 1j * rng.normal(size=3)
    lines = {ln.split("|")[0].strip(): ln.split("|")[1].strip() for ln in read_golden("sdql_example1.txt")}
    env = {"m0": m[0], "m1": m[1], "m2": m[2], "m3": m[3], "v0": v[0], "v1": v[1], "v2": v[2]}
    V = np.array([env.get(t, 0) if t != "0" else 0 for t in lines["V"].split()], dtype=complex)
    Mrows = [[env.get(t, 0) if t != "0" else 0 for t in r.split()] for r in lines["M"].split(";")]
    M4 = np.zeros((4, 4), dtype=complex)
    M4[:2] = np.array(Mrows)
    out = O.dense_matvec(M4, V)
    expect = [eval(e, {}, env) for e in lines["OUT"].split(";")]
    np.testing.assert_allclose(out[:2], expect, rtol=1e-15)
    assert np.all(out[2:] == 0)


def test_hadamard_index_map_fig14():
    """Fig. 14 / Fig. 3b index map id1 = rR + 2 rL Rs, id2 = id1 + Rs."""
    for ln in read_golden("hadamard_fig14.txt"):
        head, pairs = ln.split("|")
        kv = dict(x.split("=") for x in head.split())
        n, i, q = int(kv["n"]), int(kv["i"]), int(kv["q"])
        assert q == n - 1 - i                            # reading R1
        Ls, Rs = 1 << i, 1 << (n - 1 - i)               # reading R3: L qubits before, R after
        want = [tuple(int(x) for x in p.split()) for p in pairs.split(";")]
        formula = [(rR + 2 * rL * Rs, rR + 2 * rL * Rs + Rs) for rL in range(Ls) for rR in range(Rs)]
        assert formula == want
        G = O.dense_kron(n, W.Gate("H", (q,)))
        for id1, id2 in want:   # H couples exactly these pairs with sq2r*(s1 +- s2)
            assert G[id1, id1] == S2 and G[id1, id2] == S2 and G[id2, id1] == S2 and G[id2, id2] == -S2
        assert np.count_nonzero(G) == 4 * len(want)


def _all_gate_cases(n, rng, per_kind=4):
    for kind in O.KINDS:
        m = W.ARITY[kind]
        if m > n:
            continue
        for _ in range(per_kind):
            qs = rng.permutation(n)
            nc = int(rng.integers(0, n - m + 1))
            mat = W.haar_unitary(m, int(rng.integers(1 << 30))) if kind.startswith("UNITARY") else None
            yield W.Gate(kind, tuple(int(x) for x in qs[:m]), tuple(int(x) for x in qs[m:m + nc]),
                         _rand_params(kind, rng), mat)


@pytest.mark.parametrize("n", [1, 2, 3, 5, 7])
def test_tier_a_equals_tier_b_value_exact(n):
    """Tier A (dense matvec, ascending sum incl. zeros) == tier B (index loop).

    Value-exact whenever both sums visit the nonzero terms in the same order: always
    for the diagonal/permutation classes (one nonzero term per row), and for dense
    gates whose targets are listed MSB-first (local order == global order).  A dense
    gate with targets in another order sums the same terms in another order: 1e-15.
    """
    rng = np.random.default_rng(100 + n)
    psi = W.random_state(n, 42 + n)
    for g in _all_gate_cases(n, rng):
        a = O.apply_dense(n, g, psi)
        b = O.apply_gate(n, g, psi.copy())
        if g.exact or list(g.targets) == sorted(g.targets, reverse=True):
            assert np.array_equal(a, b), g.label()
        else:
            np.testing.assert_allclose(a, b, rtol=0, atol=1e-15, err_msg=g.label())


@pytest.mark.parametrize("n", [3, 4, 6, 9])
def test_oracle_matches_tensor_contraction(n):
    """Tier B (and A for small n) vs an independent tensordot route (_tensor_ref)."""
    rng = np.random.default_rng(200 + n)
    psi = W.random_state(n, 7 * n)
    for g in _all_gate_cases(n, rng, per_kind=3):
        M = O.gate_matrix(g)
        ref = apply_tensor(n, M, g.targets, g.controls, psi)
        b = O.apply_gate(n, g, psi.copy())
        np.testing.assert_allclose(b, ref, rtol=0, atol=4e-16, err_msg=g.label())
        if n <= 6:
            np.testing.assert_allclose(O.apply_dense(n, g, psi), ref, rtol=0, atol=4e-16)


def test_numpy_kron_brute_force():
    """Single-target embedding vs numpy.kron(I_L, kron(M, I_R)) -- the paper's naive NumPy
    baseline -- for n <= 8."""
    rng = np.random.default_rng(9)
    for n in range(1, 9):
        psi = W.random_state(n, n)
        for t in range(n):
            kind = ["H", "RX", "U3", "Y", "T"][t % 5]
            g = W.Gate(kind, (t,), (), _rand_params(kind, rng))
            G = np.kron(np.kron(np.eye(1 << (n - 1 - t)), O.gate_matrix(g)), np.eye(1 << t))
            np.testing.assert_allclose(O.apply_gate(n, g, psi.copy()), G @ psi, atol=5e-16)


def test_circuit_is_ordered_product_eq3():
    """Eq. 3: the circuit acts as G_D ... G_1 (gate 1 applied first)."""
    n = 5
    gates = W.random_gate_list(n, 12, seed=4)
    psi = W.random_state(n, 3)
    P = np.eye(1 << n, dtype=complex)
    for g in gates:
        P = O.dense_kron(n, g) @ P
    np.testing.assert_allclose(O.run_circuit(n, gates, psi.copy()), P @ psi, atol=2e-15)


def test_dense_matmul_is_eq3_product():
    """oracle_dense_matmul (the exported C = A.B, Eq. 3): (a) the oracle's product of
    two gate matrices, applied with the oracle's mvdot, equals applying the two gates one
    after the other by tier B (G_2 G_1 -- a transposed operand or swapped order fails);
    (b) it equals numpy's matmul (an independent library routine) on random complex
    matrices, non-commuting ones included; (c) I.A = A.I = A value-exactly."""
    rng = np.random.default_rng(31)
    n = 4
    psi = W.random_state(n, 8)
    gates = W.random_gate_list(n, 10, seed=12, max_controls=2)
    for g1, g2 in zip(gates[:-1], gates[1:]):
        G = O.dense_matmul(O.dense_kron(n, g2), O.dense_kron(n, g1))
        seq = O.apply_gate(n, g2, O.apply_gate(n, g1, psi.copy()))
        np.testing.assert_allclose(O.dense_matvec(G, psi), seq, rtol=0, atol=2e-15,
                                   err_msg=f"{g1.label()} then {g2.label()}")
    for dim in (1, 2, 3, 8, 16):
        A = rng.standard_normal((dim, dim)) + 1j * rng.standard_normal((dim, dim))
        B = rng.standard_normal((dim, dim)) + 1j * rng.standard_normal((dim, dim))
        np.testing.assert_allclose(O.dense_matmul(A, B), A @ B, rtol=0, atol=1e-13 * dim)
        I = np.eye(dim, dtype=complex)
        assert np.array_equal(O.dense_matmul(I, A), A) and np.array_equal(O.dense_matmul(A, I), A)
    X, Z = O.gate_matrix(W.Gate("X", (0,))), O.gate_matrix(W.Gate("Z", (0,)))
    assert np.array_equal(O.dense_matmul(Z, X), np.array([[0, 1], [-1, 0]], dtype=complex))
    assert np.array_equal(O.dense_matmul(X, Z), np.array([[0, -1], [1, 0]], dtype=complex))


def _omp_cases(n, rng):
    """Every kind, every target placement class (low/high/straddling, both orders) and
    0-3 controls (low, high, mixed) at size n."""
    for kind in O.KINDS:
        m = W.ARITY[kind]
        if m > n:
            continue
        for nc in range(0, min(3, n - m) + 1):
            for _ in range(3):
                qs = [int(x) for x in rng.permutation(n)]
                mat = (W.haar_unitary(m, int(rng.integers(1 << 30)))
                       if kind.startswith("UNITARY") else None)
                yield W.Gate(kind, tuple(qs[:m]), tuple(qs[m:m + nc]), _rand_params(kind, rng), mat)
        # extremes: targets on the lowest / highest bits, controls at the other end
        lo = tuple(range(m)); hi = tuple(range(n - 1, n - 1 - m, -1))
        for tg, cq in ((lo, tuple(range(n - 1, n - 1 - min(3, n - m), -1))),
                       (hi, tuple(range(min(3, n - m))))):
            mat = W.haar_unitary(m, 5) if kind.startswith("UNITARY") else None
            yield W.Gate(kind, tg, cq, _rand_params(kind, rng), mat)


@pytest.mark.parametrize("threads", [1, 3, "all"])
def test_omp_tier_b_equals_serial_tier_b(threads):
    """oracle_apply_gate_omp (the OpenMP parallel-for of the P:465-467 pattern, which times
    every cpu_baseline and --impl reference number) equals oracle_apply_gate bit for bit:
    every kind, target/control placement and 0-3 controls, n = 1..12, on 1 thread, an odd
    thread count (uneven static chunks) and every host core.  A race, a dropped or doubled
    group, or a chunk-boundary bug changes at least one amplitude."""
    rng = np.random.default_rng(77)
    t = O.omp_max_threads() if threads == "all" else threads
    before = O.omp_max_threads()
    O.omp_set_threads(t)
    try:
        assert O.omp_max_threads() == t
        for n in (1, 2, 3, 5, 8, 12):
            psi = W.random_state(n, 1000 + n)
            for g in _omp_cases(n, rng):
                a = O.apply_gate(n, g, psi.copy())
                b = O.apply_gate(n, g, psi.copy(), omp=True)
                assert np.array_equal(a.view(np.float64), b.view(np.float64)), (n, g.label())
        # the bench's own sweep at a size where every thread owns many groups
        n = 16
        psi = W.random_state(n, 99)
        a, b = psi.copy(), psi.copy()
        for _, g in W.sweep_gates(n)[::5]:
            O.apply_gate(n, g, a)
            O.apply_gate(n, g, b, omp=True)
        assert np.array_equal(a.view(np.float64), b.view(np.float64))
    finally:
        O.omp_set_threads(before)


# --------------------------------------------------------------------------
# Closed forms (circuits of Table 1, readings R10-R12)
# --------------------------------------------------------------------------

@pytest.mark.parametrize("n", [1, 4, 8, 12])
def test_hadamard_all_uniform(n):
    """H^{(x)n}|0> = 2^{-n/2} sum |k>: all amplitudes bit-identical, within n ulp."""
    psi = W.basis_state(n, 0)
    O.run_circuit(n, [W.Gate("H", (q,)) for q in range(n)], psi)
    assert np.all(psi == psi[0]) and np.all(psi.imag == 0)
    assert abs(psi[0].real - 2.0 ** (-n / 2)) <= n * np.spacing(2.0 ** (-n / 2))


@pytest.mark.parametrize("n", [2, 5, 11, 16])
def test_ghz_closed_form(n):
    """GHZ (Table 1; reading R11): 1/sqrt2 at |0..0> and |1..1>, exactly, zero elsewhere."""
    psi = W.basis_state(n, 0)
    O.run_circuit(n, W.ghz(n), psi)
    ref = np.zeros(1 << n, dtype=complex)
    ref[0] = ref[-1] = S2
    assert np.array_equal(psi, ref)


@pytest.mark.parametrize("n,x", [(3, 5), (5, 19), (8, 200), (10, 777)])
def test_qft_closed_form(n, x):
    """QFT|x> = 2^{-n/2} sum_y e^{2 pi i x y / 2^n}|y> (Table 1 QFT; reading R10)."""
    psi = W.basis_state(n, x)
    O.run_circuit(n, W.qft(n), psi)
    y = np.arange(1 << n)
    ref = np.exp(2j * np.pi * ((x * y) % (1 << n)) / (1 << n)) / math.sqrt(1 << n)
    np.testing.assert_allclose(psi, ref, atol=1e-13)


@pytest.mark.parametrize("n,k", [(4, 1), (6, 3), (9, 5)])
def test_grover_closed_form(n, k):
    """Grover after k iterations (Table 1; reading R12): a_w = (-1)^k sin((2k+1) th)."""
    w = (0b1011011011 * 37) % (1 << n)
    psi = W.basis_state(n, 0)
    O.run_circuit(n, W.grover(n, w, k), psi)
    th = math.asin(2.0 ** (-n / 2))
    sgn = (-1) ** k
    ref = np.full(1 << n, sgn * math.cos((2 * k + 1) * th) / math.sqrt((1 << n) - 1), dtype=complex)
    ref[w] = sgn * math.sin((2 * k + 1) * th)
    np.testing.assert_allclose(psi, ref, atol=1e-12)


def test_norm_and_inverse_circuit():
    """Unitarity: norm preserved; C followed by C^dagger returns the start state."""
    n = 10
    gates = W.random_layered(n, 6, seed=7)
    psi0 = W.random_state(n, 99)
    psi = O.run_circuit(n, gates, psi0.copy())
    assert abs(O.probs(n, psi)[0] - 1.0) < 1e-13
    inv = [W.Gate("UNITARY%d" % len(g.targets), g.targets, g.controls, (), O.gate_matrix(g).conj().T)
           for g in reversed(gates)]
    O.run_circuit(n, inv, psi)
    np.testing.assert_allclose(psi, psi0, atol=1e-13)


# --------------------------------------------------------------------------
# Measurement, sparse tier B, generator
# --------------------------------------------------------------------------

def test_probs_pairwise_and_marginals():
    """probs(Q) (P:122 measurement): bins = exact-rounded sums (fsum) within ~1 ulp-scale."""
    n = 11
    psi = W.random_state(n, 5)
    p2 = np.abs(psi) ** 2
    assert abs(O.probs(n, psi)[0] - math.fsum(p2)) <= 4e-16
    for qs in ([0], [10], [3, 7], [9, 0, 4], [1, 2, 3, 4, 5]):
        got = O.probs(n, psi, qs)
        k = np.arange(1 << n)
        v = sum(((k >> q) & 1) << s for s, q in enumerate(qs))
        for b in range(1 << len(qs)):
            assert abs(got[b] - math.fsum(p2[v == b])) <= 4e-16
    b = W.basis_state(n, 0b10110011101)
    assert O.probs(n, b, [0, 2, 9])[0b011] == 1.0   # bits 0, 2, 9 of the index = 1, 1, 0


def test_sparse_tier_b_matches_full():
    """oracle_apply_gate_sparse == oracle_apply_gate on the sampled groups."""
    n = 12
    rng = np.random.default_rng(17)
    psi = W.random_amplitudes(3, 0, 1 << n)
    for g in _all_gate_cases(n, rng, per_kind=2):
        full = O.apply_gate(n, g, psi.copy())
        tm = sum(1 << t for t in g.targets)
        base = rng.integers(0, 1 << n, 7) & ~tm
        idx = sorted({int(b) | sum(((j >> (len(g.targets) - 1 - s)) & 1) << t
                                   for s, t in enumerate(g.targets))
                      for b in base for j in range(1 << len(g.targets))})
        idx = np.array(idx, dtype=np.uint64)
        got = O.apply_gate_sparse(n, g, idx, psi[idx.astype(np.int64)])
        assert np.array_equal(got, full[idx.astype(np.int64)]), g.label()


def test_counter_generator_matches_workloads():
    """The oracle's C SplitMix64 == workloads (numpy) == reference vectors."""
    r = W.SplitMix64(1234567)
    assert [r.next_u64() for _ in range(3)] == [6457827717110365317, 3203168211198807973,
                                                9817491932198370423]
    a = O.fill_random(0xBEEF, 1000, 4096)
    assert np.array_equal(a, W.random_amplitudes(0xBEEF, 1000, 4096))
    idx = np.array([0, 5, 1 << 33, (1 << 35) + 17], dtype=np.uint64)
    for i, k in enumerate(idx):
        assert W.random_amplitudes_at(0xBEEF, idx)[i] == O.fill_random(0xBEEF, int(k), 1)[0]


def test_oracle_rejects_bad_gates():
    n = 4
    for g in (W.Gate("H", (4,)), W.Gate("X", (1,), (1,)), W.Gate("SWAP", (2, 2))):
        with pytest.raises(ValueError):
            O.apply_gate(n, g, W.random_state(n, 1))


# --------------------------------------------------------------------------
# Remaining Table-1 workloads (NEXT-2): QPE closed form, inverse QFT, inputs
# --------------------------------------------------------------------------

@pytest.mark.parametrize("t,m", [(3, 5), (6, 37), (9, 300)])
def test_qpe_exact_phase_closed_form(t, m):
    """QPE (Table 1; reading R18): with phase m/2^t the counting register is |m>
    with probability 1 and the eigenstate qubit stays |1>."""
    n = t + 1
    psi = W.basis_state(n, 0)
    O.run_circuit(n, W.qpe(t, m), psi)
    p = O.probs(n, psi, list(range(t)))
    assert abs(p[m] - 1.0) < 1e-12
    assert abs(O.probs(n, psi, [t])[1] - 1.0) < 1e-12


def test_qft_inverse_undoes_qft():
    n = 7
    psi0 = W.random_state(n, 8)
    psi = O.run_circuit(n, W.qft(n) + W.qft_inverse(n), psi0.copy())
    np.testing.assert_allclose(psi, psi0, atol=1e-14)


def test_sycamore_inputs_are_the_named_gates():
    """Input sanity: sqrt(X)^2 = X, sqrt(Y)^2 = Y, sqrt(W)^2 = W; fSim unitary."""
    gates = W.sycamore_like(2, 3, 8, seed=1)
    X = np.array([[0, 1], [1, 0]]); Y = np.array([[0, -1j], [1j, 0]])
    targets = {"X": X, "Y": Y, "W": (X + Y) / np.sqrt(2)}
    seen = set()
    for g in gates:
        if g.kind == "UNITARY1":
            sq = g.matrix @ g.matrix
            name = [k for k, v in targets.items() if np.allclose(sq, v, atol=1e-15)]
            assert len(name) == 1
            seen.add(name[0])
        else:
            np.testing.assert_allclose(g.matrix @ g.matrix.conj().T, np.eye(4), atol=1e-15)
    assert seen == {"X", "Y", "W"}


# --------------------------------------------------------------------------
# Measurement: sampling and collapse (reading R15)
# --------------------------------------------------------------------------

def test_sampling_inverse_cdf_and_statistics():
    """Uniform 2-qubit state: u in the v-th quarter -> outcome v exactly; a biased
    state's sample frequencies follow its probabilities (chi-square)."""
    n = 2
    psi = O.run_circuit(n, [W.Gate("H", (0,)), W.Gate("H", (1,))], W.basis_state(n, 0))
    u = (np.arange(4) + 0.5) / 4
    assert list(O.measure_sample(n, psi, [0, 1], u)) == [0, 1, 2, 3]
    assert list(O.measure_sample(n, psi, [1, 0], u)) == [0, 1, 2, 3]
    n = 6
    psi = O.run_circuit(n, W.random_layered(n, 3, seed=2), W.basis_state(n, 0))
    p = O.probs(n, psi, [1, 4])
    rng = np.random.default_rng(0)
    shots = 200000
    counts = np.bincount(O.measure_sample(n, psi, [1, 4], rng.random(shots)).astype(int),
                         minlength=4)
    chi2 = float(np.sum((counts - shots * p) ** 2 / (shots * p)))
    assert chi2 < 16.27  # 3 dof, p = 0.001
    b = W.basis_state(n, 0b101101)
    assert set(O.measure_sample(n, b, [0, 2, 5], rng.random(50))) == {7}  # bits 0, 2, 5 all 1
    assert set(O.measure_sample(n, b, [1, 4, 2], rng.random(50))) == {4}  # bits 1, 4, 2 = 0, 0, 1


def test_collapse_closed_forms():
    """GHZ: measuring qubit 0 as 1 leaves |1..1> exactly (P = 1/2); collapse keeps norm 1
    and equals the renormalised projection of the state."""
    n = 5
    psi = O.run_circuit(n, W.ghz(n), W.basis_state(n, 0))
    p = O.measure_collapse(n, psi, [0], 1)
    assert abs(p - 0.5) <= 2.3e-16  # |M_SQRT1_2|^2 = 0.5 + 1 ulp
    ref = np.zeros(1 << n, dtype=complex)
    ref[-1] = 1.0
    np.testing.assert_allclose(psi, ref, atol=2e-16)
    psi0 = W.random_state(7, 3)
    psi = psi0.copy()
    p = O.measure_collapse(7, psi, [2, 5], 0b10)
    k = np.arange(1 << 7)
    keep = (((k >> 2) & 1) == 0) & (((k >> 5) & 1) == 1)
    proj = np.where(keep, psi0, 0)
    assert abs(p - np.sum(np.abs(proj) ** 2)) < 1e-15
    np.testing.assert_allclose(psi, proj / np.sqrt(p), atol=1e-15)
    assert abs(O.probs(7, psi)[0] - 1.0) < 1e-14
