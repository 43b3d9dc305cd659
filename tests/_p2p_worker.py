"""Worker of tests/test_gpu_p2p.py: one rank of a peer-memory (CUDA IPC) sharded
state.  All ranks share cuda:0 (IPC works between processes on one device), so the
NVLink P2P exchange kernel, the device-side flag barriers and the rank-ordered
probability reduction run for real on the single test GPU."""
import os
import traceback

import numpy as np


def worker(rank, world, port, n, seed, out_q):
    try:
        import torch
        import torch.distributed as dist

        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        import oracle as O
        import paper_conf_cgo_tarabkhahdds25_b200 as L
        import workloads as W

        nl = n - (world.bit_length() - 1)
        lo, hi = rank << nl, (rank + 1) << nl
        report = {}
        psi = W.random_state(n, seed)
        gates = W.random_gate_list(n, 160, seed=seed + 11, max_controls=2) + W.qft(n)
        exact = [g for g in W.random_gate_list(n, 200, seed=seed + 12, max_controls=2) if g.exact]
        ref = O.run_circuit(n, gates, psi.copy())
        ref_exact = O.run_circuit(n, exact, psi.copy())
        qs = [0, n // 2, n - 1]
        for key, fuse in ((0, False), (1, True), (2, "jit")):
            with L.State.p2p(n, rank, world) as st:
                st.copy_in(psi)
                st.run_circuit(gates, fuse=fuse)
                got = st.copy_out()[lo:hi]
                err = float(np.max(np.abs(got - ref[lo:hi])))
                p = st.measure_probs(qs)
                perr = float(np.max(np.abs(p - O.probs(n, ref, qs))))
                report[f"fuse{key}"] = (err, perr)
                st.copy_in(psi)
                st.run_circuit(exact, fuse=fuse)
                report[f"exact{key}"] = bool(np.array_equal(st.copy_out()[lo:hi],
                                                                   ref_exact[lo:hi]))
                st.synchronize()
        # exchanges overlapped with local work (chunk bits 2, the default; also with a
        # grid-limited swap kernel) vs serial exchanges (chunk bits 0): the same plan and
        # the same kernels per amplitude, so the same bits
        outs = []
        for bits, ctas in ((0, 0), (2, 0), (2, 8)):
            with L.State.p2p(n, rank, world) as st:
                st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, bits)
                st.set_option(L.OPT_EXCHANGE_CTAS, ctas)
                st.copy_in(psi)
                st.run_circuit(gates)
                outs.append(st.copy_out()[lo:hi])
        report["overlap"] = (all(np.array_equal(outs[0], o) for o in outs[1:]),
                             float(np.max(np.abs(outs[1] - ref[lo:hi]))))
        # fused (compiled) passes with the chunk qubits chosen per exchange (strided blocks
        # below the top qubits: fixed tile-index bits, swap kernels with fixed bits; the
        # choice is made from the plan, so every rank picks the same blocks) vs top-qubit
        # blocks vs serial exchanges: the same passes, so the same bits
        nf = 16
        lf, hf = rank << (nf - (world.bit_length() - 1)), (rank + 1) << (nf - (world.bit_length() - 1))
        psif = W.random_state(nf, seed + 3)
        # gates controlled on the global qubits make the ranks' pass lists differ (a
        # rank whose control bit is 0 drops them), while their blocks must still agree
        gf = (W.qft(nf) + W.random_layered(nf, 3, seed=seed) +
              W.random_gate_list(nf, 80, seed=seed, max_controls=2) +
              [W.Gate("RX", (q,), (nf - 1,), (0.3 + q,)) for q in range(4, 12)] +
              [W.Gate("H", (nf - 2,))] +
              [W.Gate("RY", (q,), (nf - 1,), (0.7 * q,)) for q in range(0, 12, 2)] +
              [W.Gate("H", (nf - 1,))])
        reff = O.run_circuit(nf, gf, psif.copy())
        outs, strided = [], 0
        for bits, sel, ctas in ((0, 1, 0), (2, 0, 0), (2, 1, 0), (2, 1, 8)):
            with L.State.p2p(nf, rank, world) as st:
                st.set_option(L.OPT_FUSE_TILE_QUBITS, 8)
                st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, bits)
                st.set_option(L.OPT_EXCHANGE_CHUNK_SELECT, sel)
                st.set_option(L.OPT_EXCHANGE_CTAS, ctas)
                st.copy_in(psif)
                st.run_circuit(gf, fuse="jit")
                outs.append(st.copy_out()[lf:hf])
                strided += st.overlap_stats()["strided"] if sel else 0
        report["overlap_fused"] = (all(np.array_equal(outs[0], o) for o in outs[1:]),
                                   float(np.max(np.abs(outs[0] - reff[lf:hf]))), strided)
        # one gate at a time through lfqs_apply_gate (planner per gate, exchanges included)
        with L.State.p2p(n, rank, world) as st:
            st.copy_in(psi)
            for g in gates[:60]:
                st.apply(g)
            want = O.run_circuit(n, gates[:60], psi.copy())
            report["apply"] = float(np.max(np.abs(st.copy_out()[lo:hi] - want[lo:hi])))
        # lfqs_run_circuit_streamed on the sharded state: this rank's shard uploaded in
        # pieces, the piece-local prefix run per piece, the rest through the planner
        low = W.random_gate_list(nl - 2, 60, seed=seed + 13, max_controls=1)
        sg = low + gates
        want = O.run_circuit(n, sg, psi.copy())
        with L.State.p2p(n, rank, world) as st:
            st.copy_in(psi)
            st.run_circuit(sg)
            plain = st.copy_out()[lo:hi]
            st.init_basis(0)
            st.run_circuit_streamed(np.ascontiguousarray(psi[lo:hi]), sg, chunk_bits=2)
            streamed = st.copy_out()[lo:hi]
            report["streamed"] = (bool(np.array_equal(plain, streamed)),
                                  float(np.max(np.abs(streamed - want[lo:hi]))))
        dist.barrier()
        dist.destroy_process_group()
        out_q.put((rank, "ok", report))
    except Exception:
        out_q.put((rank, "error", traceback.format_exc()))
