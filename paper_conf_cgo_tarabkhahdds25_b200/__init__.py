"""Thin Python binding of liblfqs.so (include/lfqs.h) -- argument marshalling only.

Every step of gate application, measurement and exchange runs in the CUDA
library; this module only converts Python/numpy/torch arguments into the C ABI.
There is no CPU fallback: if liblfqs.so is missing or no CUDA device is
usable, calls raise :class:`LfqsError`.

The module-level functions carry the C names (``lfqs_apply_gate`` ...); the
:class:`State` class is a convenience wrapper over them.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import Iterable, Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# LFQS_LIBRARY: load another build of the same library (A/B timing in tools/).
LIB_PATH = os.environ.get("LFQS_LIBRARY") or os.path.join(_HERE, "liblfqs.so")

KINDS = ["I", "X", "Y", "Z", "H", "S", "SDG", "T", "TDG", "RX", "RY", "RZ", "PHASE", "U3",
         "SWAP", "UNITARY1", "UNITARY2", "UNITARY3"]
KIND_ID = {k: i for i, k in enumerate(KINDS)}
NPARAMS = {k: 0 for k in KINDS}
NPARAMS.update({"RX": 1, "RY": 1, "RZ": 1, "PHASE": 1, "U3": 3})

FUSE_NONE = 0
FUSE_LOW = 1
FUSE_PHASE = 2  # with FUSE_LOW: diagonal runs merged into per-tile phase tables (include/lfqs.h)
FUSE_JIT = 4  # with FUSE_LOW: each fused pass compiled into its own kernel (include/lfqs.h)
OPT_LOWQ_SHUFFLE = 1
OPT_FUSE_TILE_QUBITS = 2
OPT_ITEMS_PER_THREAD = 3
OPT_WIDE256 = 4
OPT_FUSE_LOW_QUBITS = 5
OPT_FUSE_TMA_MAX_CHUNKS = 6
OPT_FUSE_REORDER = 7
OPT_JIT_THREADS = 8
OPT_JIT_LANE_MOVE = 9
OPT_FUSE_MERGE_COMMUTING = 10
OPT_JIT_GREEDY_PLACE = 11
OPT_LANE_GROUP = 12
OPT_JIT_LANE_REG2 = 13
OPT_JIT_LANE_POOL = 14
OPT_JIT_PARTIAL_RT = 15
OPT_FUSE_PHASE_SPLIT = 16
OPT_STREAM_MAX_PREFIX = 17
OPT_L2_FETCH_GRANULARITY = 18
OPT_LINE_READS = 19
OPT_EXCHANGE_CHUNK_BITS = 20
OPT_EXCHANGE_CTAS = 21
OPT_FUSE_MERGE_2Q = 22
OPT_EXCHANGE_CHUNK_SELECT = 23
OPT_EXCHANGE_RATE_GBS = 24
OPT_FUSE_H_SCALE = 25
OPT_FUSE_PHASE_EXTRACT = 26
OPT_CANON_FUSE = 27
OPT_FUSE_PERM = 28
OPT_EXCHANGE_WIDE = 29

STATUS = {0: "OK", -1: "INVALID_ARG", -2: "OUT_OF_MEMORY", -3: "CUDA", -4: "NCCL",
          -5: "UNSUPPORTED"}
#: Every symbol include/lfqs.h declares (checked by tests/test_abi.py).
EXPORTS = [
    "lfqs_state_create", "lfqs_state_wrap", "lfqs_state_destroy", "lfqs_state_set_stream",
    "lfqs_dist_unique_id", "lfqs_state_create_dist", "lfqs_state_create_virtual",
    "lfqs_state_init_basis", "lfqs_state_init_random", "lfqs_copy_in", "lfqs_copy_out",
    "lfqs_apply_gate", "lfqs_run_circuit", "lfqs_measure_probs", "lfqs_synchronize",
    "lfqs_state_info", "lfqs_kernel_launches", "lfqs_set_option", "lfqs_last_error",
    "lfqs_state_pass_count",
    "lfqs_abi_version", "lfqs_plan_circuit", "lfqs_measure_sample", "lfqs_measure_collapse",
    "lfqs_state_create_ex", "lfqs_state_wrap_ex", "lfqs_copy_in_c64", "lfqs_copy_out_c64",
    "lfqs_circuit_compile", "lfqs_circuit_launch", "lfqs_circuit_destroy",
    "lfqs_state_create_p2p", "lfqs_state_p2p_handle", "lfqs_state_p2p_attach",
    "lfqs_state_exchange_stats", "lfqs_jit_precompile", "lfqs_run_circuit_streamed",
    "lfqs_state_overlap_stats",
]
P2P_HANDLE_BYTES = 256
STATE_C64 = 1
STATE_SOA = 2  # structure-of-arrays planes (include/lfqs.h, NEXT-4 layout study)


class LfqsError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"lfqs {STATUS.get(status, status)}: {msg}")
        self.status = status


class LfqsGate(C.Structure):
    """Mirror of lfqs_gate (72 bytes)."""
    _fields_ = [
        ("kind", C.c_int32), ("n_targets", C.c_int32), ("n_controls", C.c_int32),
        ("_pad0", C.c_int32), ("targets", C.c_int32 * 3), ("_pad1", C.c_int32),
        ("control_mask", C.c_uint64), ("params", C.c_double * 3),
        ("matrix", C.POINTER(C.c_double)),
    ]


assert C.sizeof(LfqsGate) == 72

PLAN_LOCAL = 0
PLAN_EXCHANGE = 1


class LfqsPlanOp(C.Structure):
    """Mirror of lfqs_plan_op."""
    _fields_ = [("kind", C.c_int32), ("l", C.c_int32), ("g", C.c_int32), ("_pad", C.c_int32),
                ("gate", LfqsGate), ("matrix", C.c_double * 128)]


_lib = None


def lib():
    """Load liblfqs.so (fails loudly if the CUDA extension was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: build it with "
                              "`python -m paper_conf_cgo_tarabkhahdds25_b200.build`")
        L = C.CDLL(LIB_PATH)
        vp, dp, u64 = C.c_void_p, C.POINTER(C.c_double), C.c_uint64
        ip = C.POINTER(C.c_int)
        sig = {
            "lfqs_state_create": [C.c_int, C.c_int, vp, C.POINTER(vp)],
            "lfqs_state_wrap": [C.c_int, C.c_int, vp, vp, C.POINTER(vp)],
            "lfqs_state_destroy": [vp],
            "lfqs_state_set_stream": [vp, vp],
            "lfqs_dist_unique_id": [C.POINTER(C.c_uint8)],
            "lfqs_state_create_dist": [C.c_int, C.c_int, C.c_int, C.POINTER(C.c_uint8), C.c_int, vp,
                                       C.POINTER(vp)],
            "lfqs_state_create_virtual": [C.c_int, C.c_int, C.c_int, vp, C.POINTER(vp)],
            "lfqs_state_init_basis": [vp, u64],
            "lfqs_state_init_random": [vp, u64],
            "lfqs_copy_in": [vp, u64, u64, dp],
            "lfqs_copy_out": [vp, u64, u64, dp],
            "lfqs_apply_gate": [vp, C.c_int, ip, C.c_int, ip, C.c_int, dp, C.c_int, dp],
            "lfqs_run_circuit": [vp, C.POINTER(LfqsGate), C.c_size_t, C.c_uint32],
            "lfqs_run_circuit_streamed": [vp, dp, C.POINTER(LfqsGate), C.c_size_t, C.c_uint32,
                                          C.c_int],
            "lfqs_circuit_compile": [vp, C.POINTER(LfqsGate), C.c_size_t, C.c_uint32,
                                     C.POINTER(vp), C.POINTER(u64)],
            "lfqs_circuit_launch": [vp],
            "lfqs_state_create_p2p": [C.c_int, C.c_int, C.c_int, C.c_int, vp, C.c_uint32,
                                      C.POINTER(vp)],
            "lfqs_state_p2p_handle": [vp, C.POINTER(C.c_uint8)],
            "lfqs_state_p2p_attach": [vp, C.POINTER(C.c_uint8)],
            "lfqs_state_exchange_stats": [vp, C.POINTER(u64), C.POINTER(u64)],
            "lfqs_state_overlap_stats": [vp, C.POINTER(u64), C.POINTER(u64), C.POINTER(u64),
                                         C.POINTER(u64)],
            "lfqs_circuit_destroy": [vp],
            "lfqs_measure_probs": [vp, ip, C.c_int, dp, C.c_size_t],
            "lfqs_synchronize": [vp],
            "lfqs_state_info": [vp, ip, ip, ip, ip, C.POINTER(vp)],
            "lfqs_kernel_launches": [vp, C.POINTER(u64)],
            "lfqs_state_pass_count": [vp, C.POINTER(u64)],
            "lfqs_set_option": [vp, C.c_int, C.c_int64],
            "lfqs_state_create_ex": [C.c_int, C.c_int, C.c_int, vp, C.c_uint32, C.POINTER(vp)],
            "lfqs_state_wrap_ex": [C.c_int, C.c_int, vp, vp, C.c_uint32, C.POINTER(vp)],
            "lfqs_copy_in_c64": [vp, u64, u64, C.POINTER(C.c_float)],
            "lfqs_copy_out_c64": [vp, u64, u64, C.POINTER(C.c_float)],
            "lfqs_measure_sample": [vp, ip, C.c_int, dp, C.c_size_t, C.POINTER(u64)],
            "lfqs_measure_collapse": [vp, ip, C.c_int, u64, dp],
            "lfqs_plan_circuit": [C.c_int, C.c_int, C.c_int, C.POINTER(LfqsGate), C.c_size_t,
                                  C.c_int, C.POINTER(LfqsPlanOp), C.c_size_t,
                                  C.POINTER(C.c_size_t)],
            "lfqs_jit_precompile": [C.c_int, C.c_int, C.POINTER(LfqsGate), C.c_size_t, C.c_uint32,
                                    C.POINTER(u64)],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = C.c_int
        L.lfqs_last_error.restype = C.c_char_p
        L.lfqs_last_error.argtypes = []
        L.lfqs_abi_version.restype = C.c_int
        L.lfqs_abi_version.argtypes = []
        _lib = L
    return _lib


def _check(rc: int):
    if rc != 0:
        raise LfqsError(rc, lib().lfqs_last_error().decode())


def _dp(a: np.ndarray):
    return a.ctypes.data_as(C.POINTER(C.c_double))


def _ints(xs: Sequence[int]):
    xs = list(xs)
    return (C.c_int * max(1, len(xs)))(*xs), len(xs)


CUDA_STREAM_LEGACY = 0x1  # cudaStreamLegacy


def _stream_handle(stream) -> Optional[int]:
    """Accept None (library-owned stream), an int handle, or a torch.cuda.Stream.

    torch's default stream has handle 0; it is passed as cudaStreamLegacy so that
    the library's work is ordered with torch's (a NULL handle would mean "make
    your own stream")."""
    if stream is None:
        return None
    h = stream if isinstance(stream, int) else int(stream.cuda_stream)
    return h if h != 0 else CUDA_STREAM_LEGACY


# ---- C-named thin wrappers ---------------------------------------------------

def lfqs_state_create(n_qubits: int, device: int = 0, stream=None) -> int:
    h = C.c_void_p()
    _check(lib().lfqs_state_create(n_qubits, device, _stream_handle(stream), C.byref(h)))
    return h.value


def lfqs_state_wrap(n_qubits: int, device: int, dev_ptr: int, stream=None) -> int:
    h = C.c_void_p()
    _check(lib().lfqs_state_wrap(n_qubits, device, dev_ptr, _stream_handle(stream), C.byref(h)))
    return h.value


def lfqs_state_create_ex(n_qubits: int, world: int = 1, device: int = 0, stream=None,
                         flags: int = 0) -> int:
    h = C.c_void_p()
    _check(lib().lfqs_state_create_ex(n_qubits, world, device, _stream_handle(stream), flags,
                                      C.byref(h)))
    return h.value


def lfqs_state_wrap_ex(n_qubits: int, device: int, dev_ptr: int, stream=None, flags: int = 0) -> int:
    h = C.c_void_p()
    _check(lib().lfqs_state_wrap_ex(n_qubits, device, dev_ptr, _stream_handle(stream), flags,
                                    C.byref(h)))
    return h.value


def lfqs_copy_in_c64(h: int, offset: int, amps: np.ndarray):
    a = np.ascontiguousarray(amps, dtype=np.complex64)
    _check(lib().lfqs_copy_in_c64(h, offset, a.size, a.view(np.float32).ctypes.data_as(
        C.POINTER(C.c_float))))


def lfqs_copy_out_c64(h: int, offset: int, count: int, out: Optional[np.ndarray] = None):
    if out is None:
        out = np.empty(count, dtype=np.complex64)
    assert out.dtype == np.complex64 and out.flags.c_contiguous and out.size >= count
    _check(lib().lfqs_copy_out_c64(h, offset, count, out.view(np.float32).ctypes.data_as(
        C.POINTER(C.c_float))))
    return out


def lfqs_state_create_virtual(n_qubits: int, world: int, device: int = 0, stream=None) -> int:
    h = C.c_void_p()
    _check(lib().lfqs_state_create_virtual(n_qubits, world, device, _stream_handle(stream),
                                           C.byref(h)))
    return h.value


def lfqs_dist_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    _check(lib().lfqs_dist_unique_id(buf))
    return bytes(buf)


def lfqs_state_create_p2p(n_qubits: int, rank: int, world: int, device: int, stream=None,
                          flags: int = 0) -> int:
    h = C.c_void_p()
    _check(lib().lfqs_state_create_p2p(n_qubits, rank, world, device, _stream_handle(stream),
                                       flags, C.byref(h)))
    return h.value


def lfqs_state_p2p_handle(h: int) -> bytes:
    buf = (C.c_uint8 * P2P_HANDLE_BYTES)()
    _check(lib().lfqs_state_p2p_handle(h, buf))
    return bytes(buf)


def lfqs_state_p2p_attach(h: int, blobs: bytes):
    buf = (C.c_uint8 * len(blobs)).from_buffer_copy(blobs)
    _check(lib().lfqs_state_p2p_attach(h, buf))


def lfqs_state_create_dist(n_qubits: int, rank: int, world: int, uid: bytes, device: int,
                           stream=None) -> int:
    h = C.c_void_p()
    buf = (C.c_uint8 * 128)(*uid)
    _check(lib().lfqs_state_create_dist(n_qubits, rank, world, buf, device,
                                        _stream_handle(stream), C.byref(h)))
    return h.value


def lfqs_state_destroy(h: int):
    _check(lib().lfqs_state_destroy(h))


def lfqs_state_init_basis(h: int, index: int):
    _check(lib().lfqs_state_init_basis(h, index))


def lfqs_state_init_random(h: int, seed: int):
    _check(lib().lfqs_state_init_random(h, seed))


def lfqs_copy_in(h: int, offset: int, amps: np.ndarray):
    a = np.ascontiguousarray(amps, dtype=np.complex128)
    _check(lib().lfqs_copy_in(h, offset, a.size, _dp(a.view(np.float64))))


def lfqs_copy_out(h: int, offset: int, count: int, out: Optional[np.ndarray] = None) -> np.ndarray:
    if out is None:
        out = np.empty(count, dtype=np.complex128)
    assert out.dtype == np.complex128 and out.flags.c_contiguous and out.size >= count
    _check(lib().lfqs_copy_out(h, offset, count, _dp(out.view(np.float64))))
    return out


def _matrix_ptr(matrix, keep: list):
    if matrix is None:
        return None
    m = np.ascontiguousarray(np.asarray(matrix, dtype=np.complex128))
    keep.append(m)
    return _dp(m.view(np.float64))


def lfqs_apply_gate(h: int, kind, targets: Sequence[int], controls: Sequence[int] = (),
                    params: Sequence[float] = (), matrix=None):
    k = KIND_ID[kind] if isinstance(kind, str) else int(kind)
    t, nt = _ints(targets)
    c, nc = _ints(controls)
    p = (C.c_double * max(1, len(params)))(*params)
    keep: list = []
    _check(lib().lfqs_apply_gate(h, k, t, nt, c, nc, p, len(params), _matrix_ptr(matrix, keep)))


def marshal_gates(gates: Iterable):
    """workloads.Gate-like objects -> (ctypes LfqsGate array, keep-alive list)."""
    gates = list(gates)
    arr = (LfqsGate * max(1, len(gates)))()
    keep: list = []
    for i, g in enumerate(gates):
        o = arr[i]
        o.kind = KIND_ID[g.kind]
        o.n_targets = len(g.targets)
        o.n_controls = len(g.controls)
        for s, t in enumerate(g.targets):
            o.targets[s] = t
        mask = 0
        for q in g.controls:
            mask |= 1 << q
        o.control_mask = mask
        for s, x in enumerate(g.params):
            o.params[s] = x
        if g.matrix is not None:
            o.matrix = _matrix_ptr(g.matrix, keep)
    return arr, len(gates), keep


def lfqs_run_circuit(h: int, gates, flags: int = FUSE_NONE):
    if isinstance(gates, tuple) and len(gates) == 3 and isinstance(gates[1], int):
        arr, n, keep = gates  # pre-marshalled
    else:
        arr, n, keep = marshal_gates(gates)
    _check(lib().lfqs_run_circuit(h, arr, n, flags))


def lfqs_run_circuit_streamed(h: int, host: np.ndarray, gates, flags: int = FUSE_NONE,
                              chunk_bits: int = 3):
    """host: the whole state, a C-contiguous complex128 array (page-locked for overlap);
    it must stay alive and unchanged until the next synchronising call."""
    assert host.dtype == np.complex128 and host.flags.c_contiguous
    if isinstance(gates, tuple) and len(gates) == 3 and isinstance(gates[1], int):
        arr, n, keep = gates
    else:
        arr, n, keep = marshal_gates(gates)
    _check(lib().lfqs_run_circuit_streamed(h, _dp(host.view(np.float64)), arr, n, flags,
                                           chunk_bits))


def lfqs_circuit_compile(h: int, gates, flags: int = FUSE_NONE):
    """Captures the circuit into a CUDA graph; returns (circuit handle, kernels per launch)."""
    if isinstance(gates, tuple) and len(gates) == 3 and isinstance(gates[1], int):
        arr, n, keep = gates
    else:
        arr, n, keep = marshal_gates(gates)
    out, k = C.c_void_p(), C.c_uint64()
    _check(lib().lfqs_circuit_compile(h, arr, n, flags, C.byref(out), C.byref(k)))
    return out.value, k.value


def fuse_flags(fuse) -> int:
    """fuse: False -> FUSE_NONE, True -> FUSE_LOW, "phase" -> FUSE_LOW | FUSE_PHASE,
    "jit" -> FUSE_LOW | FUSE_JIT, "jit+phase" -> all three, or an int."""
    if isinstance(fuse, str):
        return {"phase": FUSE_LOW | FUSE_PHASE, "jit": FUSE_LOW | FUSE_JIT,
                "jit+phase": FUSE_LOW | FUSE_JIT | FUSE_PHASE}[fuse]
    if isinstance(fuse, bool):
        return FUSE_LOW if fuse else FUSE_NONE
    return int(fuse)


def lfqs_jit_precompile(n_qubits: int, gates, fuse="jit", c64: bool = False) -> int:
    """Compiles the fused passes of `gates` for LFQS_FUSE_JIT ahead of time (host only,
    no device needed); returns the number of passes of the plan."""
    arr, n, keep = gates if (isinstance(gates, tuple) and len(gates) == 3) else marshal_gates(gates)
    k = C.c_uint64()
    _check(lib().lfqs_jit_precompile(n_qubits, int(c64), arr, n, fuse_flags(fuse), C.byref(k)))
    return k.value


def lfqs_circuit_launch(c: int):
    _check(lib().lfqs_circuit_launch(c))


def lfqs_circuit_destroy(c: int):
    _check(lib().lfqs_circuit_destroy(c))


class Circuit:
    """A circuit captured once (CUDA graph) and replayed by launch()."""

    def __init__(self, state: "State", gates, fuse: bool = False):
        self.state = state  # keeps the state alive
        self.h, self.kernels = lfqs_circuit_compile(state.h, gates, fuse_flags(fuse))

    def launch(self):
        lfqs_circuit_launch(self.h)

    def close(self):
        if self.h:
            lfqs_circuit_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def lfqs_measure_probs(h: int, qubits: Sequence[int] = ()) -> np.ndarray:
    q, nq = _ints(qubits)
    out = np.zeros(1 << nq, dtype=np.float64)
    _check(lib().lfqs_measure_probs(h, q, nq, _dp(out), out.size))
    return out


def lfqs_measure_sample(h: int, qubits: Sequence[int], uniforms) -> np.ndarray:
    """Outcomes (uint64) of len(uniforms) shots; uniforms in [0, 1) are the caller's draws."""
    q, nq = _ints(qubits)
    u = np.ascontiguousarray(uniforms, dtype=np.float64)
    out = np.zeros(u.size, dtype=np.uint64)
    _check(lib().lfqs_measure_sample(h, q, nq, _dp(u), u.size,
                                     out.ctypes.data_as(C.POINTER(C.c_uint64))))
    return out


def lfqs_measure_collapse(h: int, qubits: Sequence[int], outcome: int) -> float:
    """Projects onto `outcome` of the measured qubits and renormalises; returns P(outcome)."""
    q, nq = _ints(qubits)
    p = C.c_double(0.0)
    _check(lib().lfqs_measure_collapse(h, q, nq, outcome, C.byref(p)))
    return p.value


def lfqs_synchronize(h: int):
    _check(lib().lfqs_synchronize(h))


def lfqs_state_info(h: int) -> dict:
    n, nl, r, w = C.c_int(), C.c_int(), C.c_int(), C.c_int()
    p = C.c_void_p()
    _check(lib().lfqs_state_info(h, C.byref(n), C.byref(nl), C.byref(r), C.byref(w), C.byref(p)))
    return {"n_qubits": n.value, "n_local": nl.value, "rank": r.value, "world": w.value,
            "dev_ptr": p.value}


def lfqs_kernel_launches(h: int) -> int:
    c = C.c_uint64()
    _check(lib().lfqs_kernel_launches(h, C.byref(c)))
    return c.value


def lfqs_set_option(h: int, option: int, value: int):
    _check(lib().lfqs_set_option(h, option, value))


def lfqs_state_set_stream(h: int, stream=None):
    _check(lib().lfqs_state_set_stream(h, _stream_handle(stream)))


class PlanGate:
    """A LOCAL plan op's gate (duck-typed like workloads.Gate: kind/targets/controls/params/matrix)."""

    def __init__(self, kind, targets, controls, matrix):
        self.kind, self.targets, self.controls, self.matrix = kind, targets, controls, matrix
        self.params = ()

    def label(self):
        return f"{self.kind}c{list(self.controls)}{list(self.targets)}"


def lfqs_plan_circuit(n_qubits: int, world: int, rank: int, gates, canonicalize: bool = True,
                      wide: bool = False):
    """Host-only planner query (no GPU).  Returns a list of
    ("local", PlanGate) and ("exchange", l, g) tuples for `rank` (include/lfqs.h).
    wide: the device / P2P transports' exchange window (LFQS_PLAN_WIDE)."""
    arr, n, keep = marshal_gates(gates)
    need = C.c_size_t(0)
    flags = int(bool(canonicalize)) | (2 if wide else 0)
    rc = lib().lfqs_plan_circuit(n_qubits, world, rank, arr, n, flags, None, 0,
                                 C.byref(need))
    if rc != 0 and need.value == 0:
        _check(rc)
    ops = (LfqsPlanOp * max(1, need.value))()
    _check(lib().lfqs_plan_circuit(n_qubits, world, rank, arr, n, flags, ops,
                                   need.value, C.byref(need)))
    out = []
    for i in range(need.value):
        o = ops[i]
        if o.kind == PLAN_EXCHANGE:
            out.append(("exchange", o.l, o.g))
            continue
        m = o.gate.n_targets
        d = 1 << m
        mat = np.array(o.matrix[: 2 * d * d]).view(np.complex128).reshape(d, d).copy()
        ctrl = tuple(q for q in range(64) if (o.gate.control_mask >> q) & 1)
        out.append(("local", PlanGate(KINDS[o.gate.kind], tuple(o.gate.targets[:m]), ctrl, mat)))
    return out


# ---- convenience class ----------------------------------------------------------

class State:
    """An n-qubit state vector on a B200 (complex128 by default, complex64 with c64=True),
    on one GPU, a virtual partition of one GPU, or sharded across ranks."""

    def __init__(self, handle: int, n_qubits: int, c64: bool = False):
        self.h = handle
        self.n = n_qubits
        self.c64 = c64

    @classmethod
    def create(cls, n_qubits: int, device: int = 0, stream=None, c64: bool = False,
               soa: bool = False) -> "State":
        if c64 or soa:
            flags = (STATE_C64 if c64 else 0) | (STATE_SOA if soa else 0)
            return cls(lfqs_state_create_ex(n_qubits, 1, device, stream, flags), n_qubits, c64)
        return cls(lfqs_state_create(n_qubits, device, stream), n_qubits)

    @classmethod
    def wrap(cls, tensor, stream=None) -> "State":
        """Borrow a contiguous torch.complex128 (or complex64) CUDA tensor of 2^n elements."""
        import torch
        assert tensor.is_cuda and tensor.is_contiguous()
        assert tensor.dtype in (torch.complex128, torch.complex64)
        n = int(tensor.numel()).bit_length() - 1
        assert tensor.numel() == 1 << n
        c64 = tensor.dtype == torch.complex64
        st = cls(lfqs_state_wrap_ex(n, tensor.device.index, tensor.data_ptr(), stream,
                                    STATE_C64 if c64 else 0), n, c64)
        st._tensor = tensor
        return st

    @classmethod
    def virtual(cls, n_qubits: int, world: int, device: int = 0, stream=None,
                c64: bool = False) -> "State":
        if c64:
            return cls(lfqs_state_create_ex(n_qubits, world, device, stream, STATE_C64),
                       n_qubits, True)
        return cls(lfqs_state_create_virtual(n_qubits, world, device, stream), n_qubits)

    @classmethod
    def distributed(cls, n_qubits: int, rank: int, world: int, uid: bytes, device: int,
                    stream=None) -> "State":
        return cls(lfqs_state_create_dist(n_qubits, rank, world, uid, device, stream), n_qubits)

    @classmethod
    def p2p(cls, n_qubits: int, rank: int, world: int, device: int = 0, stream=None,
            c64: bool = False, group=None) -> "State":
        """One rank of a peer-memory (CUDA IPC) sharded state; collective over the
        torch.distributed group (any backend), which carries the 256-byte handles."""
        import torch.distributed as dist
        h = lfqs_state_create_p2p(n_qubits, rank, world, device, stream, STATE_C64 if c64 else 0)
        st = cls(h, n_qubits, c64)
        blobs = [None] * world
        dist.all_gather_object(blobs, lfqs_state_p2p_handle(h), group=group)
        lfqs_state_p2p_attach(h, b"".join(blobs))
        return st

    def close(self):
        if self.h:
            lfqs_state_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def init_basis(self, index: int = 0):
        lfqs_state_init_basis(self.h, index)

    def init_random(self, seed: int):
        lfqs_state_init_random(self.h, seed)

    def copy_in(self, amps: np.ndarray, offset: int = 0):
        """complex128 input (converted for complex64 states) or complex64 input (raw)."""
        if self.c64 and getattr(amps, "dtype", None) == np.complex64:
            lfqs_copy_in_c64(self.h, offset, amps)
        else:
            lfqs_copy_in(self.h, offset, amps)

    def copy_out(self, offset: int = 0, count: Optional[int] = None, out=None) -> np.ndarray:
        """complex128 array (complex64 states are widened); see copy_out_c64 for raw."""
        if count is None:
            count = (1 << self.n) - offset
        return lfqs_copy_out(self.h, offset, count, out)

    def copy_out_c64(self, offset: int = 0, count: Optional[int] = None, out=None) -> np.ndarray:
        if count is None:
            count = (1 << self.n) - offset
        return lfqs_copy_out_c64(self.h, offset, count, out)

    def apply_gate(self, kind, targets, controls=(), params=(), matrix=None):
        lfqs_apply_gate(self.h, kind, targets, controls, params, matrix)

    def apply(self, g):
        lfqs_apply_gate(self.h, g.kind, g.targets, g.controls, g.params, g.matrix)

    def run_circuit(self, gates, fuse=False):
        """fuse: False (one pass per gate), True (FUSE_LOW, exact for permutation/diagonal
        gates) or "phase" (FUSE_LOW | FUSE_PHASE)."""
        lfqs_run_circuit(self.h, gates, fuse_flags(fuse))

    def run_circuit_streamed(self, host: np.ndarray, gates, fuse=False, chunk_bits: int = 3):
        """Upload of this process's part of the state from `host` (the whole state on one
        GPU, this rank's shard when sharded) overlapped with the circuit
        (lfqs_run_circuit_streamed)."""
        lfqs_run_circuit_streamed(self.h, host, gates, fuse_flags(fuse), chunk_bits)

    def compile(self, gates, fuse: bool = False) -> Circuit:
        return Circuit(self, gates, fuse)

    def measure_probs(self, qubits: Sequence[int] = ()) -> np.ndarray:
        return lfqs_measure_probs(self.h, qubits)

    def sample(self, qubits: Sequence[int], uniforms) -> np.ndarray:
        return lfqs_measure_sample(self.h, qubits, uniforms)

    def collapse(self, qubits: Sequence[int], outcome: int) -> float:
        return lfqs_measure_collapse(self.h, qubits, outcome)

    def norm2(self) -> float:
        return float(self.measure_probs(())[0])

    def synchronize(self):
        lfqs_synchronize(self.h)

    def info(self) -> dict:
        return lfqs_state_info(self.h)

    def exchange_stats(self):
        """(exchanges issued, bytes sent per rank and direction), cumulative."""
        a, b = C.c_uint64(), C.c_uint64()
        _check(lib().lfqs_state_exchange_stats(self.h, C.byref(a), C.byref(b)))
        return a.value, b.value

    def overlap_stats(self) -> dict:
        """Cumulative overlapped-exchange accounting (lfqs_state_overlap_stats)."""
        v = [C.c_uint64() for _ in range(4)]
        _check(lib().lfqs_state_overlap_stats(self.h, *[C.byref(x) for x in v]))
        return dict(zip(("overlapped", "block_passes", "strided", "chained"),
                        (x.value for x in v)))

    def launches(self) -> int:
        return lfqs_kernel_launches(self.h)

    def passes(self) -> int:
        """State passes run so far (fused passes + single-gate kernels; lfqs_state_pass_count)."""
        c = C.c_uint64()
        _check(lib().lfqs_state_pass_count(self.h, C.byref(c)))
        return int(c.value)

    def set_option(self, option: int, value: int):
        lfqs_set_option(self.h, option, value)

    def set_stream(self, stream=None):
        lfqs_state_set_stream(self.h, stream)
