"""ctypes wrapper around the C oracle (oracle/oracle.c).

TEST INFRASTRUCTURE: only tests/, ``__graft_entry__.smoke()`` and bench.py's
``cpu_baseline`` / ``--impl reference`` legs may import this module.  The CUDA
product path never imports it and shares no code with it.

The oracle is the plain definition S_out = G . S_in (Eq. 2) with
G = I_L (x) M (x) I_R (Eq. 1) / Eq. 5 plus controls
(PAPER.md:110-114, 312); see oracle/oracle.h for the conventions and DESIGN.md
§3 for the pins.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from typing import Iterable, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

KINDS = ["I", "X", "Y", "Z", "H", "S", "SDG", "T", "TDG", "RX", "RY", "RZ", "PHASE", "U3",
         "SWAP", "UNITARY1", "UNITARY2", "UNITARY3"]
KIND_ID = {k: i for i, k in enumerate(KINDS)}


class OracleGate(C.Structure):
    _fields_ = [
        ("kind", C.c_int32), ("n_targets", C.c_int32), ("n_controls", C.c_int32),
        ("_pad0", C.c_int32), ("targets", C.c_int32 * 3), ("_pad1", C.c_int32),
        ("control_mask", C.c_uint64), ("params", C.c_double * 3),
        ("matrix", C.POINTER(C.c_double)),
    ]


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (-O2 -ffp-contract=off, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
                               "-fPIC", "-shared", "-Wall", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        dp = C.POINTER(C.c_double)
        gp = C.POINTER(OracleGate)
        L.oracle_gate_matrix.argtypes = [gp, C.POINTER(C.c_int), dp]
        for f in ("oracle_dense_definition", "oracle_dense_kron", "oracle_dense_swap_route"):
            getattr(L, f).argtypes = [C.c_int, gp, dp]
        L.oracle_dense_matvec.argtypes = [C.c_int, dp, dp, dp]
        L.oracle_dense_matvec.restype = None
        L.oracle_dense_matmul.argtypes = [C.c_int64, dp, dp, dp]
        L.oracle_dense_matmul.restype = None
        L.oracle_kron.argtypes = [C.c_int64, C.c_int64, dp, C.c_int64, C.c_int64, dp, dp]
        L.oracle_kron.restype = None
        L.oracle_apply_gate.argtypes = [C.c_int, gp, dp]
        L.oracle_apply_gate_omp.argtypes = [C.c_int, gp, dp]
        L.oracle_run_circuit.argtypes = [C.c_int, gp, C.c_size_t, dp]
        L.oracle_apply_gate_sparse.argtypes = [C.c_int, gp, C.c_size_t,
                                               C.POINTER(C.c_uint64), dp]
        L.oracle_probs.argtypes = [C.c_int, dp, C.POINTER(C.c_int), C.c_int, dp]
        L.oracle_measure_sample.argtypes = [C.c_int, dp, C.POINTER(C.c_int), C.c_int, dp,
                                            C.c_size_t, C.POINTER(C.c_uint64)]
        L.oracle_measure_collapse.argtypes = [C.c_int, dp, C.POINTER(C.c_int), C.c_int,
                                              C.c_uint64, dp]
        L.oracle_fill_random.argtypes = [C.c_uint64, C.c_uint64, C.c_uint64, dp]
        L.oracle_fill_random.restype = None
        L.oracle_omp_max_threads.restype = C.c_int
        L.oracle_omp_set_threads.argtypes = [C.c_int]
        L.oracle_omp_set_threads.restype = None
        _lib = L
    return _lib


def _dp(a: np.ndarray):
    return a.ctypes.data_as(C.POINTER(C.c_double))


class _Marshalled:
    """Keeps the matrix buffers alive for the duration of a call."""

    def __init__(self, gates):
        gates = list(gates)
        self.arr = (OracleGate * max(1, len(gates)))()
        self.keep = []
        for i, g in enumerate(gates):
            o = self.arr[i]
            o.kind = KIND_ID[g.kind]
            o.n_targets = len(g.targets)
            o.n_controls = len(g.controls)
            for s, t in enumerate(g.targets):
                o.targets[s] = t
            mask = 0
            for c in g.controls:
                mask |= 1 << c
            o.control_mask = mask
            for s, p in enumerate(g.params):
                o.params[s] = p
            if g.matrix is not None:
                mtx = np.ascontiguousarray(np.asarray(g.matrix, dtype=np.complex128))
                self.keep.append(mtx)
                o.matrix = mtx.view(np.float64).ctypes.data_as(C.POINTER(C.c_double))
        self.n = len(gates)

    def ptr(self, i=0):
        return C.pointer(self.arr[i]) if i == 0 else C.cast(
            C.addressof(self.arr) + i * C.sizeof(OracleGate), C.POINTER(OracleGate))


def _check(rc, what):
    if rc != 0:
        raise ValueError(f"oracle: {what} rejected its arguments (rc={rc})")


def gate_matrix(g) -> np.ndarray:
    m = _Marshalled([g])
    out = np.zeros(128, dtype=np.float64)
    mm = C.c_int(0)
    _check(lib().oracle_gate_matrix(m.ptr(), C.byref(mm), _dp(out)), "gate_matrix")
    d = 1 << mm.value
    return out[: 2 * d * d].view(np.complex128).reshape(d, d).copy()


def dense_definition(n: int, g) -> np.ndarray:
    m = _Marshalled([g])
    G = np.zeros((1 << n, 1 << n), dtype=np.complex128)
    _check(lib().oracle_dense_definition(n, m.ptr(), _dp(G.view(np.float64))), "dense_definition")
    return G


def dense_kron(n: int, g) -> np.ndarray:
    m = _Marshalled([g])
    G = np.zeros((1 << n, 1 << n), dtype=np.complex128)
    _check(lib().oracle_dense_kron(n, m.ptr(), _dp(G.view(np.float64))), "dense_kron")
    return G


def dense_swap_route(n: int, g) -> np.ndarray:
    m = _Marshalled([g])
    G = np.zeros((1 << n, 1 << n), dtype=np.complex128)
    _check(lib().oracle_dense_swap_route(n, m.ptr(), _dp(G.view(np.float64))), "dense_swap_route")
    return G


def dense_matvec(G: np.ndarray, v: np.ndarray) -> np.ndarray:
    G = np.ascontiguousarray(G, dtype=np.complex128)
    v = np.ascontiguousarray(v, dtype=np.complex128)
    n = int(v.size).bit_length() - 1
    out = np.zeros_like(v)
    lib().oracle_dense_matvec(n, _dp(G.view(np.float64)), _dp(v.view(np.float64)),
                              _dp(out.view(np.float64)))
    return out


def dense_matmul(A: np.ndarray, B: np.ndarray) -> np.ndarray:
    A = np.ascontiguousarray(A, dtype=np.complex128)
    B = np.ascontiguousarray(B, dtype=np.complex128)
    out = np.zeros_like(A)
    lib().oracle_dense_matmul(A.shape[0], _dp(A.view(np.float64)), _dp(B.view(np.float64)),
                              _dp(out.view(np.float64)))
    return out


def kron(A: np.ndarray, B: np.ndarray) -> np.ndarray:
    A = np.ascontiguousarray(A, dtype=np.complex128)
    B = np.ascontiguousarray(B, dtype=np.complex128)
    out = np.zeros((A.shape[0] * B.shape[0], A.shape[1] * B.shape[1]), dtype=np.complex128)
    lib().oracle_kron(A.shape[0], A.shape[1], _dp(A.view(np.float64)), B.shape[0], B.shape[1],
                      _dp(B.view(np.float64)), _dp(out.view(np.float64)))
    return out


def apply_dense(n: int, g, state: np.ndarray, builder: str = "kron") -> np.ndarray:
    """Tier A: build the 2^n x 2^n matrix and multiply (n <= 12)."""
    G = dense_kron(n, g) if builder == "kron" else dense_definition(n, g)
    return dense_matvec(G, state)


def apply_gate(n: int, g, state: np.ndarray, omp: bool = False) -> np.ndarray:
    """Tier B in place on a complex128 array (returned for convenience)."""
    assert state.dtype == np.complex128 and state.flags.c_contiguous and state.size == 1 << n
    m = _Marshalled([g])
    f = lib().oracle_apply_gate_omp if omp else lib().oracle_apply_gate
    _check(f(n, m.ptr(), _dp(state.view(np.float64))), f"apply_gate({g.label()})")
    return state


def run_circuit(n: int, gates: Sequence, state: np.ndarray) -> np.ndarray:
    assert state.dtype == np.complex128 and state.flags.c_contiguous and state.size == 1 << n
    m = _Marshalled(gates)
    if m.n:
        _check(lib().oracle_run_circuit(n, m.ptr(), m.n, _dp(state.view(np.float64))),
               "run_circuit")
    return state


def apply_gate_sparse(n: int, g, idx: np.ndarray, amps: np.ndarray) -> np.ndarray:
    idx = np.ascontiguousarray(idx, dtype=np.uint64)
    amps = np.ascontiguousarray(amps, dtype=np.complex128).copy()
    m = _Marshalled([g])
    _check(lib().oracle_apply_gate_sparse(n, m.ptr(), idx.size,
                                          idx.ctypes.data_as(C.POINTER(C.c_uint64)),
                                          _dp(amps.view(np.float64))), "apply_gate_sparse")
    return amps


def probs(n: int, state: np.ndarray, qubits: Sequence[int] = ()) -> np.ndarray:
    q = (C.c_int * max(1, len(qubits)))(*qubits)
    out = np.zeros(1 << len(qubits), dtype=np.float64)
    _check(lib().oracle_probs(n, _dp(np.ascontiguousarray(state).view(np.float64)), q,
                              len(qubits), _dp(out)), "probs")
    return out


def measure_sample(n: int, state: np.ndarray, qubits: Sequence[int], u) -> np.ndarray:
    q = (C.c_int * max(1, len(qubits)))(*qubits)
    u = np.ascontiguousarray(u, dtype=np.float64)
    out = np.zeros(u.size, dtype=np.uint64)
    _check(lib().oracle_measure_sample(n, _dp(np.ascontiguousarray(state).view(np.float64)), q,
                                       len(qubits), _dp(u), u.size,
                                       out.ctypes.data_as(C.POINTER(C.c_uint64))), "measure_sample")
    return out


def measure_collapse(n: int, state: np.ndarray, qubits: Sequence[int], outcome: int):
    """In place on a complex128 array; returns P(outcome)."""
    q = (C.c_int * max(1, len(qubits)))(*qubits)
    p = C.c_double(0.0)
    _check(lib().oracle_measure_collapse(n, _dp(state.view(np.float64)), q, len(qubits), outcome,
                                         C.byref(p)), "measure_collapse")
    return p.value


def fill_random(seed: int, start: int, count: int) -> np.ndarray:
    out = np.empty(count, dtype=np.complex128)
    lib().oracle_fill_random(seed, start, count, _dp(out.view(np.float64)))
    return out


def omp_max_threads() -> int:
    return int(lib().oracle_omp_max_threads())


def omp_set_threads(threads: int) -> None:
    lib().oracle_omp_set_threads(int(threads))
