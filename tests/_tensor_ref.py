"""An independent route to S_out = G . S_in used to pin the oracle (tests only).

Instead of building I_L (x) M (x) I_R (the oracle's route) this views the state
as an n-way tensor with one axis per qubit and contracts M with the target axes
(numpy.tensordot), restricted to the control = 1 slice.  A mistake in the
oracle's bit/Kronecker ordering, its Eq.-5 block slicing or its control
projection gives a different answer here.

Axis convention: reshape(2,)*n in C order, so axis i holds bit n-1-i (the
paper's qubit i).  targets[0] is the MSB of M's local index.
"""
import numpy as np


def apply_tensor(n, M, targets, controls, psi):
    m = len(targets)
    T = np.asarray(psi, dtype=np.complex128).reshape((2,) * n).copy()
    ctrl_axes = {n - 1 - c: 1 for c in controls}
    idx = tuple(1 if ax in ctrl_axes else slice(None) for ax in range(n))
    sub = T[idx]                                   # control axes removed
    remaining = [ax for ax in range(n) if ax not in ctrl_axes]
    tgt_axes = [remaining.index(n - 1 - t) for t in targets]
    Mt = np.asarray(M, dtype=np.complex128).reshape((2,) * (2 * m))
    # contract M's input indices (last m) with the target axes, in targets order
    res = np.tensordot(Mt, sub, axes=(list(range(m, 2 * m)), tgt_axes))
    # res axes: M output indices (targets order) followed by the untouched axes
    others = [ax for ax in range(sub.ndim) if ax not in tgt_axes]
    order = [None] * sub.ndim
    for s, ax in enumerate(tgt_axes):
        order[ax] = s
    for r, ax in enumerate(others):
        order[ax] = m + r
    sub_new = np.transpose(res, order)
    T[idx] = sub_new
    return T.reshape(-1)
