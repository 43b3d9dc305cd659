"""Launch a few representative gates for ncu / quick per-gate timing.

    python tools/profile_gates.py --n 28 --reps 3 [--time] [--no-shuffle]
        [--gates H:2,H:20,X:0,Z:15,RZ:3,SWAP:1/20,U2:0/7,CX:1/0,CCX:1/2/5,U3q:0/4/9]

Gate spec: KIND:t (1 target), U2:a/b, U3q:a/b/c, SWAP:a/b, CX:c/t, CCX:c1/c2/t, CZ:c/t.
With --time, prints per-gate mean ms and algorithmic GB/s from CUDA events.
"""
import argparse
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402

DEFAULT = ("H:2,H:20,X:0,X:3,X:20,Y:7,RX:12,Z:15,Z:0,T:0,S:1,PHASE:6,RZ:0,RZ:3,RZ:20,CZ:0/9,"
           "CZ:3/9,SWAP:1/20,SWAP:0/20,SWAP:12/20,U2:0/7,U2:20/25,U2:7/0,CX:1/0,CX:0/29,CX:10/11,"
           "CCX:1/2/5,CCX:0/1/20,CCX:20/21/5,U3q:0/4/9,U3q:20/25/28")


def parse(spec, n):
    out = []
    for tok in spec.split(","):
        k, a = tok.split(":")
        q = [int(x) for x in a.split("/")]
        if k == "U2":
            out.append(W.Gate("UNITARY2", tuple(q), (), (), W.haar_unitary(2, 1)))
        elif k == "U3q":
            out.append(W.Gate("UNITARY3", tuple(q), (), (), W.haar_unitary(3, 2)))
        elif k == "SWAP":
            out.append(W.Gate("SWAP", tuple(q)))
        elif k == "CX":
            out.append(W.CNOT(q[0], q[1]))
        elif k == "CZ":
            out.append(W.CZ(q[0], q[1]))
        elif k == "CCX":
            out.append(W.TOFFOLI(q[0], q[1], q[2]))
        else:
            out.append(W.Gate(k, (q[0],), (), tuple(0.3 + i for i in range(W.NPARAMS[k]))))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=28)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--gates", default=DEFAULT)
    ap.add_argument("--time", action="store_true")
    ap.add_argument("--no-shuffle", action="store_true")
    ap.add_argument("--no-wide", action="store_true")
    ap.add_argument("--lane-group", type=int, default=1,
                    help="LFQS_OPT_LANE_GROUP (0 never, 1 default, 2 every low dense 4x4/8x8)")
    ap.add_argument("--l2-fetch", type=int, default=-1,
                    help="LFQS_OPT_L2_FETCH_GRANULARITY in bytes (-1: leave the device default)")
    ap.add_argument("--c64", action="store_true", help="complex64 state")
    ap.add_argument("--line-reads", type=int, default=-1,
                    help="LFQS_OPT_LINE_READS (0/1; -1: library default)")
    ap.add_argument("--soa", action="store_true", help="structure-of-arrays state (NEXT-4 layout study)")
    ap.add_argument("--ipt", type=int, default=0, help="groups per thread for pair gates (0=default)")
    args = ap.parse_args()
    import torch
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    gates = parse(args.gates, args.n)
    ab = 8 if args.c64 else 16
    with L.State.create(args.n, 0, stream=s, c64=args.c64, soa=args.soa) as st:
        st.set_option(L.OPT_LOWQ_SHUFFLE, 0 if args.no_shuffle else 1)
        st.set_option(L.OPT_WIDE256, 0 if args.no_wide else 1)
        st.set_option(L.OPT_ITEMS_PER_THREAD, args.ipt)
        st.set_option(L.OPT_LANE_GROUP, args.lane_group)
        if args.line_reads >= 0:
            st.set_option(L.OPT_LINE_READS, args.line_reads)
        if args.l2_fetch >= 0:
            st.set_option(L.OPT_L2_FETCH_GRANULARITY, args.l2_fetch)
        st.init_random(7)
        for g in gates:
            st.apply(g)  # warm-up
        torch.cuda.synchronize()
        for g in gates:
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(args.reps + 1)]
            for r in range(args.reps):
                ev[r].record(s)
                st.apply(g)
            ev[-1].record(s)
            torch.cuda.synchronize()
            if args.time:
                ms = [ev[r].elapsed_time(ev[r + 1]) for r in range(args.reps)]
                alg = W.algorithmic_bytes(g, args.n) * ab / 16
                print(f"{g.label():28s} mean {np.mean(ms):8.3f} ms  min {np.min(ms):8.3f} ms  "
                      f"alg {alg / np.min(ms) / 1e6:8.1f} GB/s  conv {2 * ab * 2 ** args.n / np.min(ms) / 1e6:8.1f} GB/s",
                      flush=True)


if __name__ == "__main__":
    main()
