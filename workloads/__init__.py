"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NONE of the method's arithmetic (no gate matrices, no state
update, no reduction): it only draws random numbers and writes down circuits as
lists of gate *descriptions* (kind name, qubits, angles).  Both sides -- the CPU
oracle under ``oracle/`` and the CUDA library under
``paper_conf_cgo_tarabkhahdds25_b200/`` -- turn a description into a matrix with
their own, independent gate tables.

Conventions (DESIGN.md "Readings" R1, R2, R10-R13):

* qubit q = bit position q of the amplitude index (little-endian).  The paper's
  Kronecker-left qubit i is q = n-1-i (Eq. 1; verified on the
  G_{0,2} worked matrix).
* targets[0] is the most significant bit of a gate's local index (Eq. 5's q1,
  PAPER.md:284-291; Fig. 1's CNOT/CU).
* controls act on the all-ones subspace.

Random numbers: SplitMix64 (Steele, Lea, Flood 2014).  Output #i (0-based) of a
generator seeded with ``seed`` is ``mix(seed + (i+1) * 0x9E3779B97F4A7C15)``, so
the stream is counter-based: the CUDA library's device-side state initialiser
(``lfqs_state_init_random``) and the oracle's C helper each implement the same
formula and can produce any amplitude independently.  Amplitude k of a random
state takes outputs #2k (real) and #2k+1 (imag), mapped to [-1, 1) by
``u = (x >> 11) * 2**-53 * 2 - 1``.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field
from typing import List, Optional, Sequence, Tuple

import numpy as np

GOLDEN = 0x9E3779B97F4A7C15
_M64 = (1 << 64) - 1

# ----------------------------------------------------------------------------
# SplitMix64
# ----------------------------------------------------------------------------

def splitmix64_mix_scalar(z: int) -> int:
    z &= _M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


def splitmix64_stream(seed: int, start: int, count: int) -> np.ndarray:
    """Outputs #start .. #start+count-1 of SplitMix64(seed) as uint64 (vectorised)."""
    with np.errstate(over="ignore"):
        i = np.arange(start + 1, start + 1 + count, dtype=np.uint64)
        z = np.uint64(seed & _M64) + i * np.uint64(GOLDEN)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def u01_from_bits(x: np.ndarray) -> np.ndarray:
    """uint64 -> float64 in [0, 1) with 53 random bits."""
    return (x >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)


class SplitMix64:
    """Sequential SplitMix64 for drawing circuit structure and angles."""

    def __init__(self, seed: int):
        self.state = seed & _M64

    def next_u64(self) -> int:
        self.state = (self.state + GOLDEN) & _M64
        return splitmix64_mix_scalar(self.state)

    def uniform(self) -> float:
        return (self.next_u64() >> 11) * (2.0 ** -53)

    def angle(self) -> float:
        """Angle in [0, 2*pi) (reading R13)."""
        return self.uniform() * 2.0 * math.pi

    def below(self, m: int) -> int:
        return self.next_u64() % m


# ----------------------------------------------------------------------------
# States
# ----------------------------------------------------------------------------

def random_amplitudes(seed: int, start: int, count: int) -> np.ndarray:
    """Amplitudes start..start+count-1 of the counter-based random state (unnormalised).

    Re/im uniform in [-1, 1) -- no denormals, no zeros except with probability 2^-53.
    """
    bits = splitmix64_stream(seed, 2 * start, 2 * count)
    u = u01_from_bits(bits) * 2.0 - 1.0
    return u[0::2] + 1j * u[1::2]


def random_amplitudes_at(seed: int, index: np.ndarray) -> np.ndarray:
    """Amplitudes at arbitrary global indices (for sampled parity at full size)."""
    index = np.asarray(index, dtype=np.uint64)
    out = np.empty(index.shape, dtype=np.complex128)
    with np.errstate(over="ignore"):
        for c, part in ((0, "re"), (1, "im")):
            z = np.uint64(seed & _M64) + (np.uint64(2) * index + np.uint64(c + 1)) * np.uint64(GOLDEN)
            z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
            z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
            z = z ^ (z >> np.uint64(31))
            u = u01_from_bits(z) * 2.0 - 1.0
            if c == 0:
                out.real = u
            else:
                out.imag = u
    return out


def random_state(n: int, seed: int, normalize: bool = True) -> np.ndarray:
    """Seeded random n-qubit state (complex128, AOS order).  Normalised with math.fsum."""
    a = random_amplitudes(seed, 0, 1 << n)
    if normalize:
        nrm = math.sqrt(math.fsum((a.real * a.real + a.imag * a.imag).tolist()))
        a = a / nrm
    return a


def basis_state(n: int, index: int) -> np.ndarray:
    a = np.zeros(1 << n, dtype=np.complex128)
    a[index] = 1.0
    return a


# ----------------------------------------------------------------------------
# Gate descriptions
# ----------------------------------------------------------------------------

#: kind name -> number of targets
ARITY = {
    "I": 1, "X": 1, "Y": 1, "Z": 1, "H": 1, "S": 1, "SDG": 1, "T": 1, "TDG": 1,
    "RX": 1, "RY": 1, "RZ": 1, "PHASE": 1, "U3": 1,
    "SWAP": 2,
    "UNITARY1": 1, "UNITARY2": 2, "UNITARY3": 3,
}
#: kind name -> number of angle parameters
NPARAMS = {k: 0 for k in ARITY}
NPARAMS.update({"RX": 1, "RY": 1, "RZ": 1, "PHASE": 1, "U3": 3})
#: how the paper's sparsity classes (§4.6) partition the kinds.
#: Used only to label workloads and pick tolerances in tests.
KIND_CLASS = {
    "I": "diag", "Z": "diag", "S": "diag", "SDG": "diag", "T": "diag", "TDG": "diag",
    "RZ": "diag", "PHASE": "diag",
    "X": "perm", "Y": "perm", "SWAP": "perm",
    "H": "dense", "RX": "dense", "RY": "dense", "U3": "dense",
    "UNITARY1": "dense", "UNITARY2": "dense", "UNITARY3": "dense",
}


@dataclass(frozen=True)
class Gate:
    kind: str
    targets: Tuple[int, ...]
    controls: Tuple[int, ...] = ()
    params: Tuple[float, ...] = ()
    matrix: Optional[np.ndarray] = field(default=None, compare=False)

    def __post_init__(self):
        if self.kind not in ARITY:
            raise ValueError(f"unknown gate kind {self.kind}")

    @property
    def qubits(self) -> Tuple[int, ...]:
        return tuple(self.targets) + tuple(self.controls)

    @property
    def exact(self) -> bool:
        """True when GPU and oracle must agree bit-exactly (permutation / diagonal class)."""
        return KIND_CLASS[self.kind] in ("diag", "perm")

    def label(self) -> str:
        c = f"c{list(self.controls)}" if self.controls else ""
        return f"{self.kind}{c}{list(self.targets)}"


def CNOT(c: int, t: int) -> Gate:
    return Gate("X", (t,), (c,))


def CZ(c: int, t: int) -> Gate:
    return Gate("Z", (t,), (c,))


def CPHASE(c: int, t: int, phi: float) -> Gate:
    return Gate("PHASE", (t,), (c,), (phi,))


def TOFFOLI(c1: int, c2: int, t: int) -> Gate:
    return Gate("X", (t,), (c1, c2))


# ----------------------------------------------------------------------------
# Random unitaries (inputs for UNITARY1/2/3)
# ----------------------------------------------------------------------------

def haar_unitary(m: int, seed: int) -> np.ndarray:
    """Seeded Haar-random 2^m x 2^m unitary: QR of a complex Gaussian matrix (Box-Muller)."""
    d = 1 << m
    bits = splitmix64_stream(seed, 0, 4 * d * d)
    u1 = u01_from_bits(bits[0::2])
    u2 = u01_from_bits(bits[1::2])
    r = np.sqrt(-2.0 * np.log1p(-u1))  # 1-u1 in (0,1]
    g = r * np.cos(2 * np.pi * u2) + 1j * r * np.sin(2 * np.pi * u2)
    z = (g[0::2] + 1j * g[1::2]).reshape(d, d) / math.sqrt(2.0)
    q, rr = np.linalg.qr(z)
    ph = np.diag(rr) / np.abs(np.diag(rr))
    return np.ascontiguousarray(q * ph[None, :])


# ----------------------------------------------------------------------------
# Circuits (readings R10-R13)
# ----------------------------------------------------------------------------

def ghz(n: int) -> List[Gate]:
    """H(0) then CNOT(q -> q+1) for q = 0..n-2 (reading R11; Table 1 GHZ)."""
    return [Gate("H", (0,))] + [CNOT(q, q + 1) for q in range(n - 1)]


def qft(n: int, with_swaps: bool = True) -> List[Gate]:
    """Textbook QFT in bit positions (reading R10; Table 1 QFT).

    for q = n-1..0: H(q); for k = q-1..0: CPhase(pi/2^(q-k)) control k target q;
    then SWAP(q, n-1-q) for q < n/2.  Maps |x> to 2^(-n/2) sum_y e^{2 pi i x y / 2^n} |y>.
    """
    g: List[Gate] = []
    for q in range(n - 1, -1, -1):
        g.append(Gate("H", (q,)))
        for k in range(q - 1, -1, -1):
            g.append(CPHASE(k, q, math.pi / (1 << (q - k))))
    if with_swaps:
        for q in range(n // 2):
            g.append(Gate("SWAP", (q, n - 1 - q)))
    return g


def qft_inverse(n: int, with_swaps: bool = True) -> List[Gate]:
    """QFT^dagger: the QFT gate list reversed with negated phases (H, SWAP self-inverse)."""
    out = []
    for g in reversed(qft(n, with_swaps)):
        out.append(Gate(g.kind, g.targets, g.controls, tuple(-p for p in g.params)))
    return out


def qpe(t: int, m: int) -> List[Gate]:
    """Quantum phase estimation (Table 1 QPE; reading R18).

    Counting register = qubits 0..t-1, eigenstate qubit = t, prepared in |1>
    (X), U = Phase(2 pi m / 2^t) with eigenvalue e^{2 pi i m/2^t} on |1>.
    H on the counting qubits, controlled-U^(2^j) = CPhase(2 pi m 2^j / 2^t)
    (control j, target t), then QFT^dagger on the counting register.  With the
    exact phase m/2^t the counting register ends in |m> with probability 1.
    """
    g: List[Gate] = [Gate("X", (t,))] + [Gate("H", (q,)) for q in range(t)]
    for j in range(t):
        g.append(CPHASE(j, t, 2.0 * math.pi * ((m << j) % (1 << t)) / (1 << t)))
    g += qft_inverse(t)
    return g


def vqe_ansatz(n: int, layers: int, seed: int) -> List[Gate]:
    """Hardware-efficient VQE ansatz (Table 1 VQE; reading R19): per layer
    RY(theta) RZ(theta) on every qubit, then a CNOT ladder q -> q+1; angles seeded."""
    rng = SplitMix64(seed)
    g: List[Gate] = []
    for _ in range(layers):
        for q in range(n):
            g.append(Gate("RY", (q,), (), (rng.angle(),)))
            g.append(Gate("RZ", (q,), (), (rng.angle(),)))
        g += [CNOT(q, q + 1) for q in range(n - 1)]
    return g


def fsim(theta: float, phi: float) -> np.ndarray:
    """fSim(theta, phi) two-qubit gate (Sycamore coupler; reading R20)."""
    c, s = math.cos(theta), math.sin(theta)
    return np.array([[1, 0, 0, 0], [0, c, -1j * s, 0], [0, -1j * s, c, 0],
                     [0, 0, 0, complex(math.cos(phi), -math.sin(phi))]], dtype=np.complex128)


def sycamore_like(rows: int, cols: int, cycles: int, seed: int) -> List[Gate]:
    """Sycamore-style random circuit on a rows x cols grid (GSC; reading R20):
    each cycle a random single-qubit gate from {sqrt X, sqrt Y, sqrt W} per qubit (never
    repeating on a qubit), then fSim(pi/2, pi/6) on one of four coupler patterns
    (horizontal even/odd, vertical even/odd) in the order A B C D C D A B.  Qubit
    (r, c) = bit r*cols + c.  The paper's exact coupler layout is not given: parity of
    this circuit against the paper's instances is unpinned."""
    n = rows * cols
    rng = SplitMix64(seed)
    # sqrt(P) = e^{i pi/4} (I - i P) / sqrt 2 for P in {X, Y, W = (X + Y)/sqrt 2}
    X = np.array([[0, 1], [1, 0]], dtype=complex)
    Y = np.array([[0, -1j], [1j, 0]])
    sx = np.exp(1j * math.pi / 4) * (np.eye(2) - 1j * X) / math.sqrt(2)
    sy = np.exp(1j * math.pi / 4) * (np.eye(2) - 1j * Y) / math.sqrt(2)
    Wm = (X + Y) / math.sqrt(2)
    sw = np.exp(1j * math.pi / 4) * (np.eye(2) - 1j * Wm) / math.sqrt(2)
    singles = [sx, sy, sw]
    patterns = []
    for kind in ("h0", "h1", "v0", "v1"):
        pairs = []
        for r in range(rows):
            for c in range(cols):
                if kind[0] == "h" and c + 1 < cols and c % 2 == int(kind[1]):
                    pairs.append((r * cols + c, r * cols + c + 1))
                if kind[0] == "v" and r + 1 < rows and r % 2 == int(kind[1]):
                    pairs.append((r * cols + c, (r + 1) * cols + c))
        patterns.append(pairs)
    order = [0, 1, 2, 3, 2, 3, 0, 1]
    F = fsim(math.pi / 2, math.pi / 6)
    last = [-1] * n
    g: List[Gate] = []
    for cyc in range(cycles):
        for q in range(n):
            k = rng.below(3)
            while k == last[q]:
                k = rng.below(3)
            last[q] = k
            g.append(Gate("UNITARY1", (q,), (), (), singles[k]))
        for (a, b) in patterns[order[cyc % 8]]:
            g.append(Gate("UNITARY2", (a, b), (), (), F))
    return g


def mcz(n: int) -> Gate:
    """Z on qubit 0 controlled by qubits 1..n-1 (flips the sign of |1...1>)."""
    return Gate("Z", (0,), tuple(range(1, n)))


def grover(n: int, marked: int, iterations: int) -> List[Gate]:
    """Grover search from |0..0> (reading R12; Table 1 Grover)."""
    g: List[Gate] = [Gate("H", (q,)) for q in range(n)]
    zeros = [q for q in range(n) if not (marked >> q) & 1]
    for _ in range(iterations):
        g += [Gate("X", (q,)) for q in zeros]
        g.append(mcz(n))
        g += [Gate("X", (q,)) for q in zeros]
        g += [Gate("H", (q,)) for q in range(n)]
        g += [Gate("X", (q,)) for q in range(n)]
        g.append(mcz(n))
        g += [Gate("X", (q,)) for q in range(n)]
        g += [Gate("H", (q,)) for q in range(n)]
    return g


_LAYER_1Q = ("H", "RX", "RY", "RZ", "U3", "S", "T")


def random_layered(n: int, depth: int, seed: int) -> List[Gate]:
    """Seeded brickwork circuit standing in for RQC (reading R13).

    Layer l: one random 1q gate per qubit from {H, Rx, Ry, Rz, U3, S, T} (angles
    U[0, 2pi)), then CZ (even l) or CNOT (odd l) on bricks (q, q+1), q = l mod 2.
    """
    rng = SplitMix64(seed)
    g: List[Gate] = []
    for layer in range(depth):
        for q in range(n):
            kind = _LAYER_1Q[rng.below(len(_LAYER_1Q))]
            params = tuple(rng.angle() for _ in range(NPARAMS[kind]))
            g.append(Gate(kind, (q,), (), params))
        for q in range(layer % 2, n - 1, 2):
            g.append(CZ(q, q + 1) if layer % 2 == 0 else CNOT(q, q + 1))
    return g


def random_gate_list(n: int, count: int, seed: int, max_targets: int = 3,
                     max_controls: int = 2) -> List[Gate]:
    """Seeded mix of every kind on random distinct qubits (parity fuzzing)."""
    rng = SplitMix64(seed)
    kinds = sorted(ARITY)
    out: List[Gate] = []
    while len(out) < count:
        kind = kinds[rng.below(len(kinds))]
        m = ARITY[kind]
        if m > min(max_targets, n):
            continue
        perm = list(range(n))
        for i in range(n - 1, 0, -1):  # Fisher-Yates
            j = rng.below(i + 1)
            perm[i], perm[j] = perm[j], perm[i]
        nc = rng.below(min(max_controls, n - m) + 1)
        targets = tuple(perm[:m])
        controls = tuple(sorted(perm[m:m + nc]))
        params = tuple(rng.angle() for _ in range(NPARAMS[kind]))
        mat = haar_unitary(m, rng.next_u64()) if kind.startswith("UNITARY") else None
        out.append(Gate(kind, targets, controls, params, mat))
    return out


# ----------------------------------------------------------------------------
# BASELINE.json workloads
# ----------------------------------------------------------------------------

def micro_gates_10q(n: int = 10, seed: int = 0x1F5) -> List[Gate]:
    """configs[0]: H(t), Rz(t) for all t; CNOT(c,t) for all c != t; Toffoli(c1<c2, t) all distinct.

    Each gate is applied to a fresh copy of the same seeded state ("Individual Gates").
    """
    rng = SplitMix64(seed ^ 0xA5A5)
    g: List[Gate] = []
    for t in range(n):
        g.append(Gate("H", (t,)))
        g.append(Gate("RZ", (t,), (), (rng.angle(),)))
    for c in range(n):
        for t in range(n):
            if c != t:
                g.append(CNOT(c, t))
    for c1 in range(n):
        for c2 in range(c1 + 1, n):
            for t in range(n):
                if t not in (c1, c2):
                    g.append(TOFFOLI(c1, c2, t))
    return g


def sweep_gates(n: int, seed: int = 0x5EED) -> List[Tuple[str, Gate]]:
    """configs[1]: every gate class x every target qubit (SURVEY.md §8(d) row [1]).

    Returns (class_label, gate) pairs.  18 gates per target qubit.
    """
    rng = SplitMix64(seed)
    out: List[Tuple[str, Gate]] = []
    for t in range(n):
        t1, t2, t15 = (t + 1) % n, (t + 2) % n, (t + 15) % n
        if t15 in (t, t1):
            t15 = (t + n // 2 + 1) % n
        a = rng.angle
        out += [
            ("diag", Gate("Z", (t,))),
            ("diag", Gate("S", (t,))),
            ("diag", Gate("T", (t,))),
            ("diag", Gate("RZ", (t,), (), (a(),))),
            ("diag", Gate("PHASE", (t,), (), (a(),))),
            ("diag", CZ(t1, t)),
            ("diag", CPHASE(t1, t, a())),
            ("perm", Gate("X", (t,))),
            ("perm", Gate("Y", (t,))),
            ("perm", CNOT(t1, t)),
            ("perm", Gate("SWAP", (t, t1))),
            ("perm", TOFFOLI(t1, t2, t)),
            ("dense1", Gate("H", (t,))),
            ("dense1", Gate("RX", (t,), (), (a(),))),
            ("dense1", Gate("RY", (t,), (), (a(),))),
            ("dense1", Gate("U3", (t,), (), (a(), a(), a()))),
            ("dense2", Gate("UNITARY2", (t, t1), (), (), haar_unitary(2, rng.next_u64()))),
            ("dense2", Gate("UNITARY2", (t, t15), (), (), haar_unitary(2, rng.next_u64()))),
        ]
    return out


def algorithmic_bytes(g: Gate, n: int) -> float:
    """SURVEY.md §8(d) algorithmic bytes of one gate pass (accounting, not arithmetic).

    32 B per touched amplitude (16 read + 16 written).  Exception (§8(d)): when the
    touched/untouched split falls on bit 0 -- qubit 0 is a control, a one-entry
    diagonal (Z/S/T/Phase...) targets qubit 0, or a SWAP involves qubit 0 -- every
    32-byte DRAM sector holds one touched and one untouched amplitude, so the pass
    reads 32 B and writes 16 B per touched amplitude (24 * 2^n for Z on qubit 0).
    """
    t = touched_amplitudes(g, n)
    one_entry_diag = g.kind in ("Z", "S", "SDG", "T", "TDG", "PHASE")
    split0 = (0 in g.controls) or (one_entry_diag and 0 in g.targets) or \
        (g.kind == "SWAP" and 0 in g.targets)
    return 48.0 * t if split0 else 32.0 * t


def touched_amplitudes(g: Gate, n: int) -> int:
    """Amplitudes a gate reads+writes when only the changed subspace is touched
    (PAPER.md:495 in-place update "eliminate unnecessary calculations").  Used for
    algorithmic bytes = 32 B x touched amps."""
    c = len(g.controls)
    if g.kind in ("Z", "S", "SDG", "T", "TDG", "PHASE", "I"):
        return 0 if g.kind == "I" else 1 << (n - c - 1)
    if g.kind == "SWAP":
        return 1 << (n - c - 1)
    return 1 << (n - c)


def dram_line_bytes(g: Gate, n: int) -> float:
    """DRAM cost of one per-gate pass at the memory's access granularity (accounting only).

    Measured with tools/probe_sparse.cu on B200 (profiles/r02_probe_sparse.md): DRAM reads
    whole 128-B lines whatever part of a line is requested (reading 1 sector in 4 takes as
    long as reading them all), and a line whose writes cover fewer than two 32-B sectors
    costs as much as writing two (1-sector-in-4 writes run at half the rate of
    1-sector-in-2 writes).  So a line holding any touched amplitude costs 128 B of reads
    plus max(64, 32 * touched sectors) B of writes; the kernels widen touched amplitudes to
    whole 32-B sectors (bit-0 neighbours).  This is the floor for gates whose touched set
    is sparser than a line (controls / one-entry diagonals on qubits 0-2), where SURVEY
    §8(d)'s touched bytes undercount; for line-dense gates it equals algorithmic_bytes.
    """
    if g.kind == "I":
        return 0.0
    one_entry = g.kind in ("Z", "S", "SDG", "T", "TDG", "PHASE")
    fixed = {c: 1 for c in g.controls}
    if one_entry:
        fixed[g.targets[0]] = 1
    high_fixed = [b for b in fixed if b >= 3]
    swap_hi = [t for t in g.targets if t >= 3] if g.kind == "SWAP" else []
    line_types = 1 << len(swap_hi)
    rd = wr = 0.0
    for lt in range(line_types):
        hib = {t: (lt >> i) & 1 for i, t in enumerate(swap_hi)}
        sectors = set()
        for low in range(8):
            def bit(q):
                return (low >> q) & 1 if q < 3 else hib.get(q, 1)
            ok = all(bit(b) == v for b, v in fixed.items() if b < 3)
            if g.kind == "SWAP":
                ok = ok and bit(g.targets[0]) != bit(g.targets[1])
            if ok:
                sectors.add(low >> 1)
        if sectors:
            rd += 128.0
            wr += max(64.0, 32.0 * len(sectors))
    lines = 2.0 ** (n - 3) / line_types / 2.0 ** len(high_fixed)
    return lines * (rd + wr)
