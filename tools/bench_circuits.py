"""Macro benchmarks (BASELINE.json configs[2]-[3] shapes on one GPU): QFT, GHZ, Grover,
random layered circuits at n qubits, fused and unfused, with closed-form checks on
sampled amplitudes (n >= 31 does not fit the host oracle).

    python tools/bench_circuits.py --n 30 [--circuits qft,ghz,grover,random] [--reps 2]
Prints one JSON object per (circuit, mode).
"""
import argparse
import json
import math
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402
from bench import oracle_circuit_prefix, peaks  # noqa: E402  (bench.py's cpu_baseline leg)


def sample_idx(n, count, seed):
    rng = np.random.default_rng(seed)
    return np.unique(np.concatenate([rng.integers(0, 1 << n, count), [0, (1 << n) - 1]]))


def check(name, n, st, meta):
    idx = sample_idx(n, 64, 1)
    got = np.array([st.copy_out(int(k), 1)[0] for k in idx])
    if name == "qft":
        x = meta["x"]
        ref = np.exp(2j * np.pi * ((x * idx.astype(object)) % (1 << n)).astype(np.float64) / (1 << n)) \
            / math.sqrt(2.0 ** n)
    elif name == "ghz":
        ref = np.where((idx == 0) | (idx == (1 << n) - 1), math.sqrt(0.5), 0.0).astype(complex)
    elif name == "qpe":
        m = meta["m"]
        p = st.measure_probs(list(range(min(n - 1, 20))))
        return {"max_abs_err": float(abs(p[m & ((1 << min(n - 1, 20)) - 1)] - 1.0))}
    elif name == "grover":
        k, w = meta["k"], meta["w"]
        th = math.asin(2.0 ** (-n / 2))
        ref = np.full(idx.shape, (-1) ** k * math.cos((2 * k + 1) * th) / math.sqrt(2.0 ** n - 1),
                      dtype=complex)
        ref[idx == w] = (-1) ** k * math.sin((2 * k + 1) * th)
    else:
        return {"norm2": st.norm2()}
    return {"max_abs_err": float(np.max(np.abs(got - ref)))}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=30)
    ap.add_argument("--circuits", default="qft,ghz,grover,random,qpe,vqe,sycamore")
    ap.add_argument("--modes", default="fused,jit,jit+phase,unfused",
                    help="fused = FUSE_LOW (exact), phase = FUSE_LOW|FUSE_PHASE, jit = "
                         "FUSE_LOW|FUSE_JIT, jit+phase, unfused")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--tile", type=int, default=0)
    ap.add_argument("--low", type=int, default=0)
    ap.add_argument("--reorder", type=int, default=1)
    ap.add_argument("--jit-threads", type=int, default=0,
                    help="LFQS_OPT_JIT_THREADS (0: per pass, the library default; 128/256/512)")
    ap.add_argument("--lane-move", type=int, default=-1,
                    help="LFQS_OPT_JIT_LANE_MOVE (0/1; -1: library default)")
    ap.add_argument("--phase-split", type=int, default=-1,
                    help="LFQS_OPT_FUSE_PHASE_SPLIT (0/1; -1: library default)")
    ap.add_argument("--partial-rt", type=int, default=-1,
                    help="LFQS_OPT_JIT_PARTIAL_RT (0/1; -1: library default)")
    ap.add_argument("--pool", type=int, default=-1,
                    help="LFQS_OPT_JIT_LANE_POOL (0/1; -1: library default)")
    ap.add_argument("--lane-reg2", type=int, default=-1,
                    help="LFQS_OPT_JIT_LANE_REG2 (0/1; -1: library default)")
    ap.add_argument("--greedy", type=int, default=-1,
                    help="LFQS_OPT_JIT_GREEDY_PLACE (0/1; -1: library default)")
    ap.add_argument("--merge", type=int, default=-1,
                    help="LFQS_OPT_FUSE_MERGE_COMMUTING (0/1; -1: library default)")
    ap.add_argument("--merge2q", type=int, default=-1,
                    help="LFQS_OPT_FUSE_MERGE_2Q (0/1; -1: library default)")
    ap.add_argument("--perm", type=int, default=-1,
                    help="LFQS_OPT_FUSE_PERM (0/1; -1: library default)")
    ap.add_argument("--pextract", type=int, default=-1,
                    help="LFQS_OPT_FUSE_PHASE_EXTRACT (0/1; -1: library default)")
    ap.add_argument("--hscale", type=int, default=-1,
                    help="LFQS_OPT_FUSE_H_SCALE (0/1; -1: library default)")
    ap.add_argument("--c64", action="store_true", help="complex64 state (NEXT-4)")
    ap.add_argument("--world", type=int, default=1,
                    help="virtual partition into this many shards (the sharded planner and "
                         "exchange kernels on one GPU)")
    ap.add_argument("--tma", type=int, default=-1, help="max chunks moved by TMA (-1: default)")
    ap.add_argument("--oracle-s", type=float, default=0.0,
                    help="time the CPU oracle (tier B, OpenMP on all host cores) on a prefix of "
                         "each circuit for about this many seconds (SURVEY 8(d): oracle beside "
                         "the GPU; 0 = off)")
    args = ap.parse_args()
    import torch
    import paper_conf_cgo_tarabkhahdds25_b200 as L
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    n = args.n
    x = int(W.SplitMix64(n).next_u64() & ((1 << n) - 1))
    w = int(W.SplitMix64(n + 1).next_u64() & ((1 << n) - 1))
    circuits = {
        "qft": (W.qft(n), lambda st: st.init_basis(x), {"x": x}),
        "ghz": (W.ghz(n), lambda st: st.init_basis(0), {}),
        "grover": (W.grover(n, w, 2), lambda st: st.init_basis(0), {"k": 2, "w": w}),
        "random": (W.random_layered(n, 20, seed=7), lambda st: st.init_basis(0), {}),
        "qpe": (W.qpe(n - 1, x >> 1), lambda st: st.init_basis(0), {"m": x >> 1}),
        "vqe": (W.vqe_ansatz(n, 4, seed=5), lambda st: st.init_basis(0), {}),
        "sycamore": (W.sycamore_like(5, n // 5, 14, seed=6) if n % 5 == 0 else
                     W.sycamore_like(n // 6, 6, 14, seed=6) + [W.Gate("H", (q,)) for q in
                                                            range((n // 6) * 6, n)],
                     lambda st: st.init_basis(0), {}),
        # light programs: fused-pass memory efficiency (one H per qubit; X pairs)
        "hlayer": ([W.Gate("H", (q,)) for q in range(n)], lambda st: st.init_basis(0), {}),
        "xlow": ([W.Gate("X", (0,)), W.Gate("X", (1,))], lambda st: st.init_basis(0), {}),
        # QFT's final bit reversal alone (one bit-permutation pass, LFQS_OPT_FUSE_PERM)
        "bitrev": ([W.Gate("SWAP", (q, n - 1 - q)) for q in range(n // 2)],
                   lambda st: st.init_basis(0), {}),
        "xhigh": ([W.Gate("X", (n - 1,)), W.Gate("X", (n - 5,))], lambda st: st.init_basis(0), {}),
    }
    ab = 8 if args.c64 else 16
    peak, peak_src = peaks()
    st_ = (L.State.create(n, 0, stream=s, c64=args.c64) if args.world == 1 else
           L.State.virtual(n, args.world, 0, stream=s, c64=args.c64))
    with st_ as st:
        if args.tile:
            st.set_option(L.OPT_FUSE_TILE_QUBITS, args.tile)
        if args.low:
            st.set_option(L.OPT_FUSE_LOW_QUBITS, args.low)
        if args.tma >= 0:
            st.set_option(L.OPT_FUSE_TMA_MAX_CHUNKS, args.tma)
        st.set_option(L.OPT_FUSE_REORDER, args.reorder)
        st.set_option(L.OPT_JIT_THREADS, args.jit_threads)
        if args.phase_split >= 0:
            st.set_option(L.OPT_FUSE_PHASE_SPLIT, args.phase_split)
        if args.partial_rt >= 0:
            st.set_option(L.OPT_JIT_PARTIAL_RT, args.partial_rt)
        if args.pool >= 0:
            st.set_option(L.OPT_JIT_LANE_POOL, args.pool)
        if args.lane_reg2 >= 0:
            st.set_option(L.OPT_JIT_LANE_REG2, args.lane_reg2)
        if args.greedy >= 0:
            st.set_option(L.OPT_JIT_GREEDY_PLACE, args.greedy)
        if args.merge >= 0:
            st.set_option(L.OPT_FUSE_MERGE_COMMUTING, args.merge)
        if args.merge2q >= 0:
            st.set_option(L.OPT_FUSE_MERGE_2Q, args.merge2q)
        if args.lane_move >= 0:
            st.set_option(L.OPT_JIT_LANE_MOVE, args.lane_move)
        if args.hscale >= 0:
            st.set_option(L.OPT_FUSE_H_SCALE, args.hscale)
        if args.pextract >= 0:
            st.set_option(L.OPT_FUSE_PHASE_EXTRACT, args.pextract)
        if args.perm >= 0:
            st.set_option(L.OPT_FUSE_PERM, args.perm)
        for name in args.circuits.split(","):
            gates, init, meta = circuits[name]
            arr = L.marshal_gates(gates)
            orc = oracle_circuit_prefix(n, gates, args.oracle_s) if args.oracle_s > 0 else None
            for mode in args.modes.split(","):
                flags = {"fused": L.FUSE_LOW, "phase": L.FUSE_LOW | L.FUSE_PHASE,
                         "jit": L.FUSE_LOW | L.FUSE_JIT,
                         "jit+phase": L.FUSE_LOW | L.FUSE_JIT | L.FUSE_PHASE,
                         "unfused": L.FUSE_NONE}[mode]
                compile_s = None
                if flags & L.FUSE_JIT:  # compile outside the timed region (reported)
                    t0 = time.time()
                    L.lfqs_jit_precompile(n, arr, flags, c64=args.c64)
                    compile_s = time.time() - t0
                times, passes = [], 0
                for r in range(args.reps + 1):
                    init(st)
                    x0 = st.exchange_stats()[0]
                    torch.cuda.synchronize()
                    c0 = st.launches()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(s)
                    L.lfqs_run_circuit(st.h, arr, flags)
                    e1.record(s)
                    torch.cuda.synchronize()
                    if r > 0 or args.reps == 0:
                        times.append(e0.elapsed_time(e1))
                    passes = st.launches() - c0
                    x1 = st.exchange_stats()[0]
                res = check(name, n, st, meta)
                t = min(times)
                rec = {"circuit": name, "mode": mode, "n": n, "gates": len(gates), "passes": passes,
                       "ms": t, "gates_per_s": len(gates) / (t / 1e3),
                       "conv_GBps": 2.0 * ab * 2 ** n * len(gates) / (t / 1e3) / 1e9,
                       "pass_GBps": 2.0 * ab * 2 ** n * passes / (t / 1e3) / 1e9,
                       "dtype": "c64" if args.c64 else "c128", "world": args.world,
                       "exchanges": x1 - x0, "lane_move": args.lane_move, "merge": args.merge, "merge2q": args.merge2q, "jit_threads": args.jit_threads, "greedy": args.greedy, "lane_reg2": args.lane_reg2, "pool": args.pool, "partial_rt": args.partial_rt, "phase_split": args.phase_split, "hscale": args.hscale, "pextract": args.pextract, "perm": args.perm,
                       "hbm_peak_GBps": peak, "peak_source": peak_src}
                # fraction of the HBM roofline: per pass actually made, and against the
                # north-star convention of one 2*16*2^n-byte pass per gate
                rec["pass_frac"] = rec["pass_GBps"] / peak
                rec["conv_frac"] = rec["conv_GBps"] / peak
                if compile_s is not None:
                    rec["jit_compile_s"] = round(compile_s, 3)
                rec.update(res)
                if orc is not None:
                    rec["oracle"] = orc
                    if "gates_per_s" in orc:
                        rec["gpu_over_oracle"] = rec["gates_per_s"] / orc["gates_per_s"]
                print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()
