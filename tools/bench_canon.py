"""Cost of restoring the canonical qubit map after a sharded circuit (State::canonicalize:
local SWAP passes + exchanges), fused (LFQS_OPT_CANON_FUSE = 1) vs one pass per SWAP, on a
virtual partition of one GPU.   python tools/bench_canon.py --n 32 --world 4 --circuit qft
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=32)
    ap.add_argument("--world", type=int, default=4)
    ap.add_argument("--circuit", default="qft")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--rate", type=int, default=0)
    ap.add_argument("--ctas", type=int, default=0)
    args = ap.parse_args()
    import torch
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    n = args.n
    gates = {"qft": W.qft(n), "random": W.random_layered(n, 20, seed=7),
             "grover": W.grover(n, 12345, 1)}[args.circuit]
    arr = L.marshal_gates(gates)
    flags = L.FUSE_LOW | L.FUSE_JIT | L.FUSE_PHASE
    with L.State.virtual(n, args.world, 0) as st:
        st.set_option(L.OPT_EXCHANGE_CTAS, args.ctas)
        st.set_option(L.OPT_EXCHANGE_RATE_GBS, args.rate)
        for cf in (0, 1, 0, 1):
            st.set_option(L.OPT_CANON_FUSE, cf)
            best_c, best_t = 1e30, 1e30
            for r in range(args.reps + 1):
                st.init_basis(0)
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                L.lfqs_run_circuit(st.h, arr, flags)
                st.synchronize()
                t1 = time.perf_counter()
                x0, p0 = st.exchange_stats()[0], st.passes()
                st.copy_out(0, 1)  # canonicalises
                t2 = time.perf_counter()
                if r > 0:
                    best_c, best_t = min(best_c, t2 - t1), min(best_t, t2 - t0)
                nx, npass = st.exchange_stats()[0] - x0, st.passes() - p0
            print(json.dumps({"circuit": args.circuit, "n": n, "world": args.world,
                              "canon_fuse": cf, "canon_ms": round(best_c * 1e3, 3),
                              "run_plus_canon_ms": round(best_t * 1e3, 3),
                              "canon_exchanges": nx, "canon_passes": npass}), flush=True)


if __name__ == "__main__":
    main()
