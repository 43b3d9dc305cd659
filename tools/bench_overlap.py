"""Exchange/compute overlap on one GPU: a virtual partition into `world` shards
runs a circuit with serial exchanges (LFQS_OPT_EXCHANGE_CHUNK_BITS = 0) and overlapped
ones (2^c blocks on a high-priority exchange stream while the neighbouring local passes run
block by block; LFQS_OPT_EXCHANGE_CHUNK_SELECT picks the chunk qubits per exchange).  The
exchange swap kernel is grid-limited (`--ctas`) and optionally paced (`--rate`, GB/s per
direction per shard pair): what an exchange over NVLink looks like to the GPU -- a
link-bound transfer that leaves most SMs and most of the HBM bandwidth to the passes.

Pacing ratio: on P real GPUs every rank runs its own shard's passes (time C) and all shard
pairs exchange at once at the link rate R; the virtual partition runs the P shards' passes
back to back (P * C) and its P/2 pair exchanges one after another, so the virtual swap at
R/2 per pair keeps exchange time : pass time equal to the real one (R = 900 GB/s NVLink 5
-> --rate 450).  The same circuit on an unsharded state (world = 1) gives the local work
alone.

    python tools/bench_overlap.py --n 32 --world 4 --circuit qft --ctas 64 --rate 450

Prints one JSON object per (ctas, rate, chunk bits, select): ms, exchanges, the overlap
accounting (lfqs_state_overlap_stats), the exposed exchange time (ms - unsharded ms) and
the fraction of the serial exchange time hidden by overlapping.
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
    ap.add_argument("--mode", default="jit+phase")
    ap.add_argument("--ctas", default="64")
    ap.add_argument("--bits", default="0,2,3")
    ap.add_argument("--select", default="0,1", help="LFQS_OPT_EXCHANGE_CHUNK_SELECT values")
    ap.add_argument("--tile", type=int, default=12)
    ap.add_argument("--rate", default="450", help="LFQS_OPT_EXCHANGE_RATE_GBS values (0: unpaced)")
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    import torch
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    n = args.n
    x = int(W.SplitMix64(n).next_u64() & ((1 << n) - 1))
    gates = {"qft": W.qft(n), "random": W.random_layered(n, 20, seed=7),
             "grover": W.grover(n, x, 1), "ghz": W.ghz(n)}[args.circuit]
    flags = {"unfused": L.FUSE_NONE, "fused": L.FUSE_LOW, "jit": L.FUSE_LOW | L.FUSE_JIT,
             "jit+phase": L.FUSE_LOW | L.FUSE_JIT | L.FUSE_PHASE}[args.mode]
    arr = L.marshal_gates(gates)

    def timed(st):
        best = 1e30
        for r in range(args.reps + 1):
            st.init_basis(x if args.circuit == "qft" else 0)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            L.lfqs_run_circuit(st.h, arr, flags)
            e1.record(s)
            torch.cuda.synchronize()
            if r > 0:
                best = min(best, e0.elapsed_time(e1))
        return best

    with L.State.create(n, 0, stream=s) as st:
        if flags & L.FUSE_JIT:
            L.lfqs_jit_precompile(n, arr, flags)
        t1 = timed(st)
    print(json.dumps({"circuit": args.circuit, "mode": args.mode, "n": n, "world": 1,
                      "ms": round(t1, 3)}), flush=True)
    with L.State.virtual(n, args.world, 0, stream=s) as st:
        if flags & L.FUSE_JIT:  # compile every pass shape outside the timed region
            st.set_option(L.OPT_FUSE_TILE_QUBITS, args.tile)
            for b in [int(v) for v in args.bits.split(",")]:
                st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, b)
                st.init_basis(0)
                L.lfqs_run_circuit(st.h, arr, flags)
            torch.cuda.synchronize()
        st.set_option(L.OPT_FUSE_TILE_QUBITS, args.tile)
        for ctas, rate in [(int(v), int(r)) for v in args.ctas.split(",")
                           for r in args.rate.split(",")]:
            st.set_option(L.OPT_EXCHANGE_CTAS, ctas)
            st.set_option(L.OPT_EXCHANGE_RATE_GBS, rate)
            serial = None
            for b in [int(v) for v in args.bits.split(",")]:
                for sel in ([1] if b == 0 else [int(v) for v in args.select.split(",")]):
                    st.set_option(L.OPT_EXCHANGE_CHUNK_BITS, b)
                    st.set_option(L.OPT_EXCHANGE_CHUNK_SELECT, sel)
                    x0 = st.exchange_stats()[0]
                    o0 = st.overlap_stats()
                    t = timed(st)
                    nx = (st.exchange_stats()[0] - x0) // (args.reps + 1)
                    o1 = st.overlap_stats()
                    ov = {k: (o1[k] - o0[k]) // (args.reps + 1) for k in o1}
                    rec = {"circuit": args.circuit, "mode": args.mode, "n": n,
                           "world": args.world, "exchange_ctas": ctas, "rate_gbs": rate,
                           "chunk_bits": b,
                           "chunk_select": sel, "ms": round(t, 3), "exchanges": int(nx),
                           "overlap": ov, "unsharded_ms": round(t1, 3),
                           "exposed_exchange_ms": round(t - t1, 3)}
                    if b == 0:
                        serial = t
                    elif serial is not None and serial > t1:
                        rec["hidden_frac"] = round((serial - t) / (serial - t1), 3)
                    print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()
