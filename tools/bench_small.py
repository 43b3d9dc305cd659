"""BASELINE configs[0]: the 10-qubit micro-benchmark gates (H and Rz on every qubit,
CNOT on every ordered pair, Toffoli on every (c1 < c2, t): 470 gates) on one GPU --
launch-bound, so it reports the ways of issuing them:

  apply    one lfqs_apply_gate call per gate from Python (ctypes)
  run      lfqs_run_circuit, one kernel per gate (LFQS_FUSE_NONE)
  graph    the same launches captured once in a CUDA graph (lfqs_circuit_launch)
  fused    lfqs_run_circuit with LFQS_FUSE_LOW (the 16 KiB state is one tile)
  fgraph   the fused program captured in a CUDA graph
  jit      lfqs_run_circuit with LFQS_FUSE_LOW | LFQS_FUSE_JIT (compiled passes; compile
           done once before timing, reported as jit_compile_s)
  jgraph   the compiled passes captured in a CUDA graph
  oracle   the oracle, tier B, one host thread

    python tools/bench_small.py [--n 10] [--reps 50]
Prints one JSON object per mode (gates/s, us per gate).
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402
from test_gpu_graph import config0_gates  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=10)
    ap.add_argument("--reps", type=int, default=50)
    args = ap.parse_args()
    import torch
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    n, reps = args.n, args.reps
    gates = config0_gates(n)
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    arr = L.marshal_gates(gates)
    psi = W.random_state(n, 1)

    def timed(fn, reps_):
        fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record(s)
        for _ in range(reps_):
            fn()
        e1.record(s)
        torch.cuda.synchronize()
        wall = time.perf_counter() - t0
        return max(e0.elapsed_time(e1) / 1e3, wall) / reps_  # host-bound modes: wall clock

    with L.State.create(n, stream=s) as st:
        st.copy_in(psi)
        res = {}
        res["apply"] = timed(lambda: [st.apply(g) for g in gates], max(2, reps // 10))
        res["run"] = timed(lambda: L.lfqs_run_circuit(st.h, arr, L.FUSE_NONE), reps)
        with st.compile(arr) as c:
            res["graph"] = timed(c.launch, reps)
            kern = c.kernels
        res["fused"] = timed(lambda: L.lfqs_run_circuit(st.h, arr, L.FUSE_LOW), reps)
        with st.compile(arr, fuse=True) as c:
            res["fgraph"] = timed(c.launch, reps)
            fkern = c.kernels
        t0 = time.perf_counter()
        L.lfqs_jit_precompile(n, arr, "jit")
        jit_s = time.perf_counter() - t0
        res["jit"] = timed(lambda: L.lfqs_run_circuit(st.h, arr, L.FUSE_LOW | L.FUSE_JIT), reps)
        with st.compile(arr, fuse="jit") as c:
            res["jgraph"] = timed(c.launch, reps)
    from bench import oracle_circuit_time  # bench.py's cpu_baseline leg
    res["oracle"] = oracle_circuit_time(n, gates, psi)
    for mode, t in res.items():
        print(json.dumps({"config": "configs[0]", "n": n, "gates": len(gates), "mode": mode,
                          "s_per_circuit": t, "us_per_gate": t / len(gates) * 1e6,
                          "gates_per_s": len(gates) / t,
                          "kernels": kern if mode == "graph" else fkern if mode in ("fgraph", "jgraph") else None,
                          "jit_compile_s": jit_s if mode in ("jit", "jgraph") else None,
                          "host_threads": 1 if mode == "oracle" else None}), flush=True)


if __name__ == "__main__":
    main()
