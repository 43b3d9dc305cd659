"""Small-n workload for compute-sanitizer (memcheck / racecheck / synccheck):
every kernel family once -- class kernels, shuffle path, fused TMA and direct
tiles (incl. smem ops), compiled passes (LFQS_FUSE_JIT, with phase tables, 256 and
512 threads, placement variants), the lane-group kernel, SOA kernels, virtual-partition exchange, probabilities, collapse.

    compute-sanitizer --tool racecheck python tools/sanitize_run.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402


def main():
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    n = 14
    gates = W.random_gate_list(n, 120, seed=1, max_controls=2) + W.qft(n) + \
        W.random_layered(n, 3, seed=2) + W.sycamore_like(2, 7, 4, seed=3)
    with L.State.create(n) as st:
        st.init_random(1)
        st.set_option(L.OPT_LOWQ_SHUFFLE, 1)
        st.run_circuit(gates[:120])
        st.set_option(L.OPT_LOWQ_SHUFFLE, 0)
        for tma in (256, 0):
            st.set_option(L.OPT_FUSE_TMA_MAX_CHUNKS, tma)
            st.run_circuit(gates, fuse=True)
        for threads in (256, 512):
            st.set_option(L.OPT_JIT_THREADS, threads)
            st.run_circuit(gates, fuse="jit")
            st.run_circuit(gates, fuse="jit+phase")
        st.set_option(L.OPT_JIT_THREADS, 256)
        for lm, gr in ((1, 1), (0, 0)):  # placement variants of the compiled passes
            st.set_option(L.OPT_JIT_LANE_MOVE, lm)
            st.set_option(L.OPT_JIT_GREEDY_PLACE, gr)
            st.run_circuit(gates, fuse="jit")
        # lane-group kernel: dense 4x4 / 8x8 with targets in qubits 1..5
        U2, U3 = W.haar_unitary(2, 5), W.haar_unitary(3, 6)
        st.run_circuit([W.Gate("UNITARY2", (1, 2), (), (), U2),
                        W.Gate("UNITARY2", (5, 3), (0, 11), (), U2),
                        W.Gate("UNITARY3", (1, 2, 3), (), (), U3),
                        W.Gate("UNITARY3", (4, 1, 5), (7,), (), U3)])
        # line-shaped reads: fixed bits on qubits 1 / 2 (controls, one-entry diagonals)
        st.run_circuit([W.TOFFOLI(1, 2, 5), W.TOFFOLI(1, 2, 0), W.CZ(1, 2), W.Gate("S", (1,)),
                        W.CNOT(2, 9), W.Gate("T", (2,), (7,))])
        st.measure_probs([0, 3, 13])
        st.measure_probs(list(range(12)))
        st.measure_probs(list(range(13, -1, -1)))  # 14 qubits: two-level binning
        st.sample([1, 2], np.linspace(0, 0.99, 7))
        st.collapse([5], 1)
        st.synchronize()
    with L.State.create(n, soa=True) as st:
        st.init_random(3)
        st.run_circuit(gates)
        st.measure_probs([0, 1])
        st.collapse([0], 0)
    with L.State.virtual(n, 4) as st:  # exchanges overlapped with passes (exchange stream)
        st.init_random(2)
        st.run_circuit(gates, fuse=True)
        st.set_option(L.OPT_EXCHANGE_CTAS, 8)  # grid-limited swap kernel
        st.run_circuit(gates, fuse="jit")
        st.run_circuit(gates[:80])
        st.copy_out(0, 16)
        st.measure_probs(list(range(n)))
    # chunk qubits chosen per exchange (strided blocks: fixed tile-index bits, swap kernels
    # with fixed bits), chained exchanges, the paced swap kernel
    with L.State.virtual(16, 4) as st:
        st.init_random(5)
        st.set_option(L.OPT_FUSE_TILE_QUBITS, 8)
        g16 = W.qft(16) + W.random_layered(16, 3, seed=4)
        st.run_circuit(g16, fuse="jit+phase")
        st.set_option(L.OPT_EXCHANGE_RATE_GBS, 200)
        st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, 3)
        st.run_circuit(g16, fuse=True)
        assert st.overlap_stats()["strided"] > 0
        st.measure_probs([0, 15])
    print("sanitize workload done")


if __name__ == "__main__":
    main()
