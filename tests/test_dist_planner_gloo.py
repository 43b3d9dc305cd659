"""Multi-process (gloo, CPU) test of the distributed planner's host logic.

Each rank asks the product planner (lfqs_plan_circuit, the same C++ code the
NCCL path executes) for its ops, applies LOCAL ops to its shard with the oracle
(n_local qubits) and performs EXCHANGE ops as real send/recv of half-shards with
its partner over torch.distributed (gloo).  The gathered state must equal the
oracle applied to the whole state.  No GPU is involved.
"""
import os
import socket
import tempfile

import numpy as np
import pytest

import workloads as W


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _circuits(n):
    hi = [n - 1, n - 2]
    return {
        "random": W.random_gate_list(n, 120, seed=11, max_controls=2),
        "qft": W.qft(n),
        "ghz": W.ghz(n),
        "globals": [
            W.Gate("H", (hi[0],)), W.CNOT(hi[1], 1), W.CZ(hi[0], 2), W.CPHASE(0, hi[1], 0.4),
            W.Gate("RZ", (hi[0],), (), (0.9,)), W.Gate("SWAP", (hi[1], 3)), W.Gate("Y", (hi[0],), (2,)),
            W.Gate("UNITARY2", (hi[0], 0), (), (), W.haar_unitary(2, 3)),
            W.Gate("UNITARY3", (hi[1], 4, hi[0]), (1,), (), W.haar_unitary(3, 4)),
            W.Gate("UNITARY2", (hi[1], hi[0]), (), (), np.diag(np.exp(1j * np.arange(4.0)))),
            W.TOFFOLI(hi[0], hi[1], 0), W.mcz(n), W.Gate("SWAP", (hi[0], hi[1])),
            W.Gate("X", (hi[1],)),
        ],
        "exact": [g for g in W.random_gate_list(n, 150, seed=5, max_controls=3) if g.exact],
    }


def _worker(rank, world, port, n, outdir):
    import torch
    import torch.distributed as dist

    import oracle as O
    import paper_conf_cgo_tarabkhahdds25_b200 as L

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    nl = n - (world.bit_length() - 1)
    psi = W.random_state(n, 123)
    results = {}
    for name, gates in _circuits(n).items():
        shard = psi[rank << nl:(rank + 1) << nl].copy()
        ops = L.lfqs_plan_circuit(n, world, rank, gates, canonicalize=True)
        n_ex = 0
        for op in ops:
            if op[0] == "local":
                O.apply_gate(nl, op[1], shard)
            else:
                _, l, g = op
                j = g - nl
                b = (rank >> j) & 1
                partner = rank ^ (1 << j)
                idx = np.flatnonzero(((np.arange(1 << nl) >> l) & 1) == 1 - b)
                send = torch.from_numpy(shard[idx].copy())
                recv = torch.empty_like(send)
                req = dist.isend(send, partner)
                dist.recv(recv, partner)
                req.wait()
                shard[idx] = recv.numpy()
                n_ex += 1
        parts = [torch.zeros(1 << nl, dtype=torch.complex128) for _ in range(world)]
        dist.all_gather(parts, torch.from_numpy(shard))
        full = np.concatenate([p.numpy() for p in parts])
        results[name] = (full, n_ex)
    if rank == 0:
        np.savez(os.path.join(outdir, "out.npz"),
                 **{k: v[0] for k, v in results.items()},
                 **{k + "_ex": v[1] for k, v in results.items()})
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_planner_with_gloo_exchanges(world):
    import torch.multiprocessing as mp

    import oracle as O
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    from paper_conf_cgo_tarabkhahdds25_b200 import build as B
    B.build()
    L.lib()
    n = 9
    with tempfile.TemporaryDirectory() as d:
        mp.start_processes(_worker, args=(world, _free_port(), n, d), nprocs=world,
                           start_method="spawn", join=True)
        out = np.load(os.path.join(d, "out.npz"))
        psi = W.random_state(n, 123)
        for name, gates in _circuits(n).items():
            ref = O.run_circuit(n, gates, psi.copy())
            got = out[name]
            if name == "exact":
                assert np.array_equal(got, ref), name
            else:
                assert np.max(np.abs(got - ref)) <= 1e-12, name
        # QFT: every CPhase on a global qubit is communication-free (rank-folded diagonal);
        # only the H gates on global qubits and the canonicalisation move data.
        assert out["qft_ex"] <= 3 * (world.bit_length() - 1) + 2 * (world.bit_length() - 1)
        assert out["globals_ex"] >= 1


def test_plan_single_rank_is_the_circuit():
    """world = 1: the plan is the circuit itself, one LOCAL op per non-identity gate."""
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    gates = W.random_gate_list(6, 40, seed=2)
    ops = L.lfqs_plan_circuit(6, 1, 0, gates)
    assert all(o[0] == "local" for o in ops)
    assert len(ops) == sum(1 for g in gates if g.kind != "I")


def test_plan_rejects_bad_world():
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    with pytest.raises(L.LfqsError):
        L.lfqs_plan_circuit(6, 3, 0, W.ghz(6))
    with pytest.raises(L.LfqsError):
        L.lfqs_plan_circuit(6, 2, 2, W.ghz(6))
