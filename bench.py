#!/usr/bin/env python
"""Benchmark: BASELINE.json metric "gates/s and achieved HBM GB/s (% of B200 peak)".

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl lfqs|reference] [--n 30]

Workload at N = 1 (BASELINE.json configs[1]): the 30-qubit single-gate sweep --
every gate class (diagonal Z/S/T/Rz/Phase/CZ/CPhase, permutation X/Y/CNOT/SWAP/
Toffoli, dense H/Rx/Ry/U3 and 4x4 UNITARY2 on adjacent and distant pairs) on
every target qubit, 18 x 30 = 540 gates, applied in place to a 16 GiB
complex128 state resident in HBM.  One "step" = one pass of the whole sweep.
The state (16 GiB) is >> the 126 MB L2, so no L2 flush is needed.

N > 1 (torchrun, one rank per GPU): weak scaling, 2^30 amplitudes per GPU,
n = 30 + log2 N, the same sweep over all n qubits (gates on the top log2 N
"global" qubits go through the half-shard exchange: by default the in-place
peer-memory swap kernel over NVLink (CUDA IPC, --transport p2p), or staged NCCL
send/recv (--transport nccl)).

--impl reference: the CPU oracle (oracle/, tier B index loop with OpenMP on
all host cores) on a bounded sample of the same sweep, rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

METRIC = "gates/s and achieved HBM GB/s (% of B200 peak) at 30-36 qubits, 1/2/4/8 GPUs"
UNIT = "gates/s"


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


# ----------------------------------------------------------------------------
# clocks sampling during the timed region
# ----------------------------------------------------------------------------
_REASONS = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]


class ClockSampler:
    def __init__(self, device: int):
        self.device = device
        self.proc = None
        self.lines = []

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,utilization.gpu,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={q}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for ln in self.proc.stdout:
            self.lines.append(ln.strip())

    def __exit__(self, *exc):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], [], set()
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                s, m, util = float(f[0]), float(f[1]), float(f[3])
            except ValueError:
                continue
            mx.append(m)
            if util > 50:
                sm.append(s)
            for name, v in zip(_REASONS, f[4:8]):
                if v.lower() == "active":
                    reasons.add(name)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.lines)}


# ----------------------------------------------------------------------------
# CPU oracle timing (cpu_baseline and --impl reference)
# ----------------------------------------------------------------------------

def host_avail_gib():
    try:
        with open("/proc/meminfo") as f:
            for ln in f:
                if ln.startswith("MemAvailable:"):
                    return int(ln.split()[1]) / 2 ** 20
    except Exception:
        pass
    return 0.0


class OracleSweep:
    """The oracle (as it stands) applying the sweep gates to a host state, OpenMP tier B."""

    def __init__(self, n: int, seed: int):
        import oracle
        self.O = oracle
        self.n = n
        avail = host_avail_gib()
        need = 16 * 2 ** n / 2 ** 30
        while need > 0.45 * avail and self.n > 20:
            self.n -= 1
            need /= 2
        self.state = oracle.fill_random(seed, 0, 1 << self.n)
        self.gates = [g for _, g in W.sweep_gates(self.n)]
        self.cores = oracle.omp_max_threads()
        self.pos = 0

    def run(self, n_gates: int) -> float:
        t0 = time.perf_counter()
        for _ in range(n_gates):
            g = self.gates[self.pos % len(self.gates)]
            self.O.apply_gate(self.n, g, self.state, omp=True)
            self.pos += 1
        return time.perf_counter() - t0

    def calibrate(self, budget_s: float) -> int:
        t = self.run(2) / 2
        return max(1, int(budget_s / max(t, 1e-6)))


def cpu_baseline(n: int, budget_s: float = 15.0):
    ow = OracleSweep(n, seed=0xC0FFEE)
    g = ow.calibrate(budget_s / 2)
    t = ow.run(g)
    res = {"value": g / t, "unit": UNIT, "cores": ow.cores, "kind": "oracle",
           "sample": f"first {g} gates of the n={ow.n} sweep (of {len(ow.gates)}), oracle tier B "
                     f"(naive index loop, OpenMP static schedule), host state "
                     f"{16 * 2 ** ow.n / 2 ** 30:.0f} GiB"}
    del ow
    return res


def oracle_circuit_prefix(n: int, gates, budget_s: float) -> dict:
    """cpu_baseline for the macro circuits (tools/bench_circuits.py --oracle-s): the oracle as
    it stands (tier B index loop, OpenMP static schedule on every host core) on the first
    gates of the same circuit at the same n, from a seeded random host state, for about
    budget_s seconds.  Needs 16 * 2^n B of host memory; beyond 45 % of MemAvailable it
    reports why it did not run."""
    import oracle
    cores = oracle.omp_max_threads()
    if 16.0 * 2 ** n > 0.45 * host_avail_gib() * 2 ** 30:
        return {"unavailable": f"16*2^{n} B host state exceeds 45% of MemAvailable "
                               f"({host_avail_gib():.0f} GiB)", "cores": cores}
    st = oracle.fill_random(0x0AC1E, 0, 1 << n)
    done, t0 = 0, time.perf_counter()
    while done < len(gates) and time.perf_counter() - t0 < budget_s:
        oracle.apply_gate(n, gates[done], st, omp=True)
        done += 1
    t = time.perf_counter() - t0
    del st
    return {"gates_per_s": done / t, "gates": done, "of": len(gates), "s": t, "cores": cores,
            "kind": "oracle tier B (OpenMP), circuit prefix"}


def oracle_circuit_time(n: int, gates, psi) -> float:
    """Seconds the oracle (tier B, one host thread) takes for a whole small circuit
    (configs[0], tools/bench_small.py)."""
    import oracle
    oracle.build()
    t0 = time.perf_counter()
    oracle.run_circuit(n, gates, psi.copy())
    return time.perf_counter() - t0


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    ow = OracleSweep(args.n, seed=0xC0FFEE)
    per_step = ow.calibrate(budget_s=args.ref_step_s)
    for _ in range(args.warmup):
        ow.run(per_step)
    times = [ow.run(per_step) for _ in range(args.steps)]
    total = sum(times)
    value = per_step * args.steps / total
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT,
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * total / args.steps, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"configs[1]: {ow.n}-qubit single-gate sweep (bounded sample)",
                   "n_qubits": ow.n, "gates_per_step": per_step},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": ow.cores, "kind": "oracle",
                         "sample": f"{per_step} sweep gates per step, n={ow.n}, oracle tier B "
                                   f"OpenMP on {ow.cores} threads"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ----------------------------------------------------------------------------
# configs[2]: 33-qubit QFT and GHZ on one B200 (macro leg of the N = 1 line)
# ----------------------------------------------------------------------------

def _closed_form_err(name, n, st, meta):
    """Max abs error against the closed form (readings R10/R11) on 64 sampled
    indices plus both ends; GHZ also reports bit-exactness (amplitude M_SQRT1_2 exactly)."""
    rng = np.random.default_rng(1)
    idx = np.unique(np.concatenate([rng.integers(0, 1 << n, 64), [0, (1 << n) - 1]]))
    got = np.array([st.copy_out(int(k), 1)[0] for k in idx])
    if name == "qft":
        x = meta["x"]
        ph = ((x * idx.astype(object)) % (1 << n)).astype(np.float64) / (1 << n)
        ref = np.exp(2j * np.pi * ph) / math.sqrt(2.0 ** n)
        err = float(np.max(np.abs(got - ref)))
        return {"closed_form_max_abs_err": err,
                "closed_form_rel_err": err * math.sqrt(2.0 ** n),  # amplitudes are 2^(-n/2)
                "samples": int(idx.size)}
    ref = np.where((idx == 0) | (idx == (1 << n) - 1), math.sqrt(0.5), 0.0).astype(complex)
    return {"closed_form_max_abs_err": float(np.max(np.abs(got - ref))),
            "bit_exact": bool(np.array_equal(got, ref)), "samples": int(idx.size)}


def run_macro(lfqs, stream, n: int, reps: int, unfused: bool, hbm_peak: float):
    """configs[2]: QFT(n)|x> and GHZ(n) from |0> on one GPU (n = 33: a 128 GiB state), as
    compiled fused passes (LFQS_FUSE_JIT, compile outside the timed region) and, strict,
    one class-kernel pass per gate (LFQS_FUSE_NONE).  CUDA events on the launching stream;
    min and mean over `reps` after one warm-up; closed-form checks on sampled amplitudes."""
    import torch
    x = int(W.SplitMix64(n).next_u64() & ((1 << n) - 1))
    circuits = [("qft", W.qft(n), x, {"x": x}), ("ghz", W.ghz(n), 0, {})]
    modes = [("jit+phase", lfqs.FUSE_LOW | lfqs.FUSE_JIT | lfqs.FUSE_PHASE)]
    if unfused:
        modes.append(("unfused", lfqs.FUSE_NONE))
    out = {}
    with lfqs.State.create(n, 0, stream=stream) as st:
        for name, gates, init, meta in circuits:
            arr = lfqs.marshal_gates(gates)
            for mode, flags in modes:
                compile_s = None
                if flags & lfqs.FUSE_JIT:
                    t0 = time.time()
                    lfqs.lfqs_jit_precompile(n, arr, flags)
                    compile_s = time.time() - t0
                times, passes = [], 0
                nrep = reps if mode != "unfused" or name == "ghz" else 1
                for r in range(nrep + (1 if mode != "unfused" else 0)):
                    st.init_basis(init)
                    torch.cuda.synchronize()
                    c0 = st.launches()
                    e0 = torch.cuda.Event(enable_timing=True)
                    e1 = torch.cuda.Event(enable_timing=True)
                    e0.record(stream)
                    lfqs.lfqs_run_circuit(st.h, arr, flags)
                    e1.record(stream)
                    torch.cuda.synchronize()
                    passes = st.launches() - c0
                    if mode == "unfused" or r > 0:
                        times.append(e0.elapsed_time(e1))
                t = min(times)
                pass_bytes = 2.0 * 16 * 2 ** n
                # bytes the passes must move: a fused pass reads and writes the whole state;
                # a per-gate pass its touched part / its DRAM lines
                if mode == "unfused":
                    need = sum(W.algorithmic_bytes(g, n) for g in gates)
                    need_dram = sum(W.dram_line_bytes(g, n) for g in gates)
                else:
                    need = need_dram = pass_bytes * passes
                rec = {"mode": mode, "gates": len(gates), "passes": int(passes),
                       "ms": round(t, 3), "ms_mean": round(float(np.mean(times)), 3),
                       "reps": len(times), "gates_per_s": len(gates) / (t / 1e3),
                       "hbm_frac": need / (t / 1e3) / 1e9 / hbm_peak,
                       "hbm_frac_dram_model": need_dram / (t / 1e3) / 1e9 / hbm_peak,
                       "conv_frac": pass_bytes * len(gates) / (t / 1e3) / 1e9 / hbm_peak}
                if compile_s is not None:
                    rec["jit_compile_s_untimed"] = round(compile_s, 3)
                rec.update(_closed_form_err(name, n, st, meta))
                out[f"{name}{n}_{mode}"] = rec
    torch.cuda.synchronize()
    return out


# ----------------------------------------------------------------------------
# configs[0]: the 10-qubit micro-benchmark gates (launch-bound regime)
# ----------------------------------------------------------------------------

def cpu_baseline_small(n, gates, psi):
    """configs[0]'s cpu_baseline: the oracle (tier B, one host thread) on the whole
    470-gate circuit; its result is also the reference the GPU runs are checked against."""
    import oracle
    t0 = time.perf_counter()
    ref = oracle.run_circuit(n, gates, psi.copy())
    return ref, {"kind": "oracle", "cores": 1,
                 "us_per_gate": (time.perf_counter() - t0) / len(gates) * 1e6}


def run_small(lfqs, stream, with_oracle: bool, reps: int = 50):
    """configs[0] (n = 10: H and Rz on every qubit, CNOT on every ordered pair, Toffoli on
    every (c1 < c2, t); 470 gates): per-gate class kernels replayed from a CUDA graph, and
    the compiled fused passes replayed from a CUDA graph, CUDA events over `reps` replays;
    each checked against the oracle's result on the same seeded state (cpu_baseline_small)."""
    import torch
    n = 10
    gates = W.micro_gates_10q(n)
    psi = W.random_state(n, 0x1F5)
    arr = lfqs.marshal_gates(gates)
    out = {"config": "configs[0]", "n": n, "gates": len(gates)}
    ref = None
    if with_oracle:
        ref, out["cpu_baseline"] = cpu_baseline_small(n, gates, psi)
    with lfqs.State.create(n, 0, stream=stream) as st:
        lfqs.lfqs_jit_precompile(n, arr, "jit")
        for mode, fuse in (("graph_per_gate", False), ("graph_compiled_passes", "jit")):
            st.copy_in(psi)
            with st.compile(arr, fuse=fuse) as c:
                c.launch()
                err = None if ref is None else float(np.max(np.abs(st.copy_out() - ref)))
                torch.cuda.synchronize()
                a = torch.cuda.Event(enable_timing=True)
                b = torch.cuda.Event(enable_timing=True)
                a.record(stream)
                for _ in range(reps):
                    c.launch()
                b.record(stream)
                torch.cuda.synchronize()
                t = a.elapsed_time(b) / 1e3 / reps
                out[mode] = {"us_per_gate": t / len(gates) * 1e6, "gates_per_s": len(gates) / t,
                             "kernels_per_circuit": int(c.kernels), "max_abs_err_vs_oracle": err}
    return out


# ----------------------------------------------------------------------------
# N > 1: QFT(n_local + log2 N) sharded across the ranks (configs[4] shape)
# ----------------------------------------------------------------------------

NVLINK_GBPS = 900.0  # NVLink 5 per GPU per direction, nominal (no measured peak here)


def run_sharded_circuits(lfqs, st, n, n_loc, world, rank, stream, barrier, dist, device_reduce,
                         hbm_peak, reps):
    """Macro circuits on the sharded state (n = n_loc + log2 world): QFT(n)|x> (8 GPUs x 2^30:
    QFT(33), the configs[4] circuit at this per-GPU size), and the configs[3] shapes Grover(n)
    (2 iterations) and a random layered circuit of depth 20 -- compiled passes + phase
    tables, exchanges overlapped with local passes; the timed region ends after the final
    canonicalisation (relabels are not free).  Device time (CUDA events), max
    over ranks.  Combined roofline (SURVEY §8(d) [4]): T_roof = passes x 32 * 2^n_loc B / HBM
    + exchanges x 16 * 2^(n_loc - 1) B / NVLink, with the north-star form (one pass per gate)
    beside it.  Checks: QFT and Grover closed forms on 64 sampled amplitudes of every rank's
    shard (readings R10, R12), the random circuit's norm."""
    import torch
    x = int(W.SplitMix64(n).next_u64() & ((1 << n) - 1))
    w = int(W.SplitMix64(n + 1).next_u64() & ((1 << n) - 1))
    k_it = 2
    th = math.asin(2.0 ** (-n / 2))

    def qft_ref(idx):
        ph = ((x * idx.astype(object)) % (1 << n)).astype(np.float64) / (1 << n)
        return np.exp(2j * np.pi * ph) / math.sqrt(2.0 ** n), math.sqrt(2.0 ** n)

    def grover_ref(idx):
        ref = np.full(idx.shape, (-1) ** k_it * math.cos((2 * k_it + 1) * th) /
                      math.sqrt(2.0 ** n - 1), dtype=complex)
        ref[idx == w] = (-1) ** k_it * math.sin((2 * k_it + 1) * th)
        return ref, math.sqrt(2.0 ** n)

    circuits = [("qft", W.qft(n), x, qft_ref), ("grover", W.grover(n, w, k_it), 0, grover_ref),
                ("random", W.random_layered(n, 20, seed=7), 0, None)]
    flags = lfqs.FUSE_LOW | lfqs.FUSE_JIT | lfqs.FUSE_PHASE
    out = {}
    for name, gates, init, ref_fn in circuits:
        arr = lfqs.marshal_gates(gates)

        def once():
            st.init_basis(init)
            barrier()
            p0, e0 = st.passes(), st.exchange_stats()
            a = torch.cuda.Event(enable_timing=True)
            b = torch.cuda.Event(enable_timing=True)
            a.record(stream)
            lfqs.lfqs_run_circuit(st.h, arr, flags)
            st.copy_out(0, 0)  # canonicalise the qubit map (collective), in the timed region
            b.record(stream)
            barrier()
            e1 = st.exchange_stats()
            return a.elapsed_time(b), st.passes() - p0, e1[0] - e0[0], e1[1] - e0[1]

        once()  # warm-up: compiles every pass shape
        runs = [once() for _ in range(reps)]
        t = torch.tensor([min(r[0] for r in runs)], device=device_reduce)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
        _, passes, n_ex, ex_bytes = runs[0]
        if ref_fn is not None:  # closed form on this rank's shard (canonical order)
            rng = np.random.default_rng(rank + 1)
            idx = (rank << n_loc) + rng.integers(0, 1 << n_loc, 64)
            if name == "grover" and (w >> n_loc) == rank:
                idx[0] = w
            got = np.array([st.copy_out(int(k), 1)[0] for k in idx])
            ref, scale = ref_fn(idx)
            e = torch.tensor([float(np.max(np.abs(got - ref)))], device=device_reduce,
                             dtype=torch.float64)
            dist.all_reduce(e, op=dist.ReduceOp.MAX)
            check = {"closed_form_max_abs_err": float(e.item()),
                     "closed_form_rel_err": float(e.item()) * scale}
        else:
            check = {"norm2": st.norm2()}  # all ranks (reduction across them)
        pb = 32.0 * 2 ** n_loc
        t_ex = n_ex * 16.0 * 2 ** (n_loc - 1) / (NVLINK_GBPS * 1e9)
        t_roof = passes * pb / (hbm_peak * 1e9) + t_ex
        t_roof_gates = len(gates) * pb / (hbm_peak * 1e9) + t_ex
        out[f"{name}{n}"] = {
            "circuit": f"{name}({n}) on {world} ranks, 2^{n_loc} amplitudes per rank",
            "mode": "jit+phase, exchanges overlapped", "gates": len(gates),
            "ms": round(ms, 3), "gates_per_s": len(gates) / (ms / 1e3),
            "passes_per_rank": int(passes), "exchanges_per_rank": int(n_ex),
            "exchange_bytes_per_rank_per_direction": int(ex_bytes),
            "t_roof_ms": round(t_roof * 1e3, 3), "roof_frac": (t_roof * 1e3) / ms,
            "t_roof_north_star_ms": round(t_roof_gates * 1e3, 3),
            "roof_frac_north_star": (t_roof_gates * 1e3) / ms, **check}
    out["roofline_terms"] = ("passes x 32*2^n_loc B / hbm_peak + exchanges x 16*2^(n_loc-1) B "
                             f"/ {NVLINK_GBPS} GB/s (north star: one pass per gate)")
    return out


# ----------------------------------------------------------------------------
# GPU arm
# ----------------------------------------------------------------------------

def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="lfqs", choices=["lfqs", "reference"])
    ap.add_argument("--n", "--qubits-per-gpu", dest="n", type=int, default=30, help="qubits per GPU")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--ref-step-s", type=float, default=12.0)
    ap.add_argument("--per-gate-json", default="", help="write per-gate timings here")
    ap.add_argument("--macro-n", type=int, default=33,
                    help="configs[2] leg at N = 1: QFT and GHZ at this many qubits after the "
                         "sweep (0: skip)")
    ap.add_argument("--macro-reps", type=int, default=3)
    ap.add_argument("--no-small", action="store_true", help="skip the configs[0] leg")
    ap.add_argument("--no-macro-unfused", action="store_true",
                    help="skip the strict one-pass-per-gate QFT/GHZ runs of the macro leg")
    ap.add_argument("--qft-reps", type=int, default=3,
                    help="N > 1: timed runs of each sharded macro circuit (QFT, Grover, "
                         "random layered; 0: skip)")
    ap.add_argument("--same-device", action="store_true",
                    help="test only: every rank on cuda:0 (exercises the N>1 path on one GPU)")
    ap.add_argument("--transport", default="p2p", choices=["p2p", "nccl"],
                    help="N>1 global-qubit exchange: in-place peer-memory swap kernel (CUDA IPC "
                         "over NVLink) or staged NCCL send/recv")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import paper_conf_cgo_tarabkhahdds25_b200 as lfqs

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    assert world == args.gpus, f"--gpus {args.gpus} but WORLD_SIZE={world}"
    assert args.warmup >= 3 or os.environ.get("LFQS_BENCH_ALLOW_SHORT"), "need >= 3 warm-up steps"
    if args.same_device:
        local_rank = 0
    torch.cuda.set_device(local_rank)
    stream = torch.cuda.Stream()      # the library launches on this stream; events too
    torch.cuda.set_stream(stream)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo" if args.same_device else "nccl",
                                device_id=None if args.same_device
                                else torch.device("cuda", local_rank))
        p = world.bit_length() - 1
        assert 1 << p == world, "world size must be a power of two"
        n = args.n + p
        if args.transport == "p2p":
            st = lfqs.State.p2p(n, rank, world, local_rank, stream=stream)
        else:
            obj = [lfqs.lfqs_dist_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0)
            st = lfqs.State.distributed(n, rank, world, obj[0], local_rank, stream=stream)
    else:
        n = args.n
        st = lfqs.State.create(n, local_rank, stream=stream)

    sweep = W.sweep_gates(n)
    seed = 0xC0FFEE
    st.init_random(seed)

    def barrier():
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()

    ex_marks = np.zeros((max(args.steps, 1), len(sweep)), dtype=np.int64)  # exchanges (N > 1)

    def one_step(evs=None, k=0):
        for i, (_, g) in enumerate(sweep):
            if evs is not None:
                evs[i].record(stream)
            if world > 1:
                e0 = st.exchange_stats()[0]
                st.apply(g)
                ex_marks[k, i] = st.exchange_stats()[0] - e0
            else:
                st.apply(g)
        if evs is not None:
            evs[len(sweep)].record(stream)

    for _ in range(args.warmup):
        one_step()
    barrier()

    launches0 = st.launches()
    ex0 = st.exchange_stats()
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(len(sweep) + 1)]
           for _ in range(args.steps)]
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    with ClockSampler(local_rank) as clk:
        barrier()
        t_start.record(stream)
        for k in range(args.steps):
            one_step(evs[k], k)
        t_end.record(stream)
        barrier()
    launches = st.launches() - launches0
    ex1 = st.exchange_stats()
    elapsed_ms = t_start.elapsed_time(t_end)
    if dist is not None:
        t = torch.tensor([elapsed_ms], device="cpu" if args.same_device else "cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        elapsed_ms = float(t.item())
    ms_per_step = elapsed_ms / args.steps
    gates_per_step = len(sweep)
    value = gates_per_step / (ms_per_step / 1e3)

    # per-gate / per-class durations (CUDA events on the launching stream)
    per_gate = np.zeros((args.steps, len(sweep)))
    for k in range(args.steps):
        for i in range(len(sweep)):
            per_gate[k, i] = evs[k][i].elapsed_time(evs[k][i + 1])
    mean_ms = per_gate.mean(axis=0)
    n_loc = n - (world.bit_length() - 1)
    classes = {}
    for i, (cls, g) in enumerate(sweep):
        c = classes.setdefault(cls, {"gates": 0, "ms": 0.0, "alg_bytes": 0.0, "conv_bytes": 0.0})
        c["gates"] += 1
        c["ms"] += mean_ms[i]
        c["alg_bytes"] += W.algorithmic_bytes(g, n_loc)
        c["conv_bytes"] += 32.0 * 2 ** n_loc
    hbm_peak, peak_src = peaks()
    for c in classes.values():
        c["alg_GBps"] = c["alg_bytes"] / (c["ms"] / 1e3) / 1e9
        c["conv_GBps"] = c["conv_bytes"] / (c["ms"] / 1e3) / 1e9
        c["frac_alg"] = c["alg_GBps"] / hbm_peak
        c["ms_per_gate"] = c["ms"] / c["gates"]
        c["share"] = c["ms"] / mean_ms.sum()
    dom = max(classes, key=lambda k: classes[k]["ms"])
    dc = classes[dom]
    # the gate furthest below its own roofline (SURVEY §8(d) touched bytes / mean time)
    fr = [(W.algorithmic_bytes(g, n_loc) / (mean_ms[i] / 1e3) / 1e9 / hbm_peak, i)
          for i, (_, g) in enumerate(sweep)]
    wf, wi = min(fr)

    def gate_rec(i):
        g = sweep[i][1]
        t = mean_ms[i] / 1e3
        return {"label": g.label(), "class": sweep[i][0], "ms": round(float(mean_ms[i]), 4),
                "alg_bytes": W.algorithmic_bytes(g, n_loc),
                "alg_frac": round(W.algorithmic_bytes(g, n_loc) / t / 1e9 / hbm_peak, 4),
                "dram_model_bytes": W.dram_line_bytes(g, n_loc),
                "dram_model_frac": round(W.dram_line_bytes(g, n_loc) / t / 1e9 / hbm_peak, 4),
                "conv_frac": round(32.0 * 2 ** n_loc / t / 1e9 / hbm_peak, 4)}
    # worst by SURVEY §8(d) touched bytes, and by the DRAM line-granularity model
    # (workloads.dram_line_bytes, from tools/probe_sparse.cu)
    worst_gate = gate_rec(wi)
    dm = min(range(len(sweep)), key=lambda i: W.dram_line_bytes(sweep[i][1], n_loc) / mean_ms[i])
    worst_gate["worst_by_dram_model"] = gate_rec(dm)
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic_per_launch.json")
    if world == 1 and os.path.exists(tp):  # ncu capture of the N = 1 workload
        try:
            traffic = json.load(open(tp)).get(dom)
        except Exception:
            traffic = None
    roofline = {"bound": "hbm",
                "kernel": f"{dom} class per-gate kernels (apply_kernels.cu k_group_x2 / k_group)",
                "achieved": dc["alg_GBps"], "peak": hbm_peak, "unit": "GB/s",
                "frac": dc["alg_GBps"] / hbm_peak,
                "frac_of_nominal_8000GBps": dc["alg_GBps"] / 8000.0, "traffic": traffic,
                "traffic_source": "ncu dram__bytes_read.sum + dram__bytes_write.sum per launch, "
                                  "class mean of the committed capture (profiles/r02_launches.md, "
                                  "profiles/traffic_per_launch.json)" if traffic else None,
                "peak_source": peak_src,
                "bytes_per_launch": dc["alg_bytes"] / dc["gates"],
                "avg_launch_ms": dc["ms"] / dc["gates"]}
    # N > 1: the global-qubit exchanges (half-shard swaps over NVLink).  A gate that
    # issued exchanges costs its local pass plus the exchanges; the local part is
    # estimated by the median of the same class's exchange-free gates.
    nvlink = None
    if world > 1:
        n_ex = (ex1[0] - ex0[0]) / args.steps
        ex_bytes = (ex1[1] - ex0[1]) / args.steps
        t_ex = 0.0
        for k in range(args.steps):
            for i, (cls, g) in enumerate(sweep):
                if ex_marks[k, i] > 0:
                    local = [per_gate[k2, i2] for k2 in range(args.steps)
                             for i2, (c2, _) in enumerate(sweep)
                             if c2 == cls and ex_marks[k2, i2] == 0]
                    t_ex += max(per_gate[k, i] - (float(np.median(local)) if local else 0.0),
                                1e-6)
        t_ex /= args.steps
        link_gbps = ex_bytes / (t_ex / 1e3) / 1e9 if t_ex > 0 else None
        nvlink = {"exchanges_per_step": n_ex, "bytes_per_rank_per_direction_per_step": ex_bytes,
                  "exchange_ms_per_step": t_ex, "achieved": link_gbps, "unit": "GB/s",
                  "peak": 900.0, "peak_source": "nominal NVLink 5, per GPU per direction",
                  "frac": link_gbps / 900.0 if link_gbps else None,
                  "transport": args.transport}

    qft = None
    if world > 1 and args.qft_reps > 0:
        qft = run_sharded_circuits(lfqs, st, n, n_loc, world, rank, stream, barrier, dist,
                                   "cpu" if args.same_device else "cuda", hbm_peak,
                                   args.qft_reps)

    if args.per_gate_json and rank == 0:
        with open(args.per_gate_json, "w") as f:
            json.dump([{"cls": cls, "gate": g.label(), "ms": float(mean_ms[i]),
                        "alg_bytes": W.algorithmic_bytes(g, n_loc)}
                       for i, (cls, g) in enumerate(sweep)], f, indent=0)

    # end to end through the public API: H2D of the input state from pinned host
    # memory, the sweep, and a D2H read of the measured probabilities each step
    e2e = None
    need_gib = 16.0 * 2 ** n_loc / 2 ** 30 * world  # every rank's pinned shard, one host
    if not args.no_e2e and world > 1 and host_avail_gib() < 1.25 * need_gib:
        # every rank pins its own 16 GiB shard: skip (and say so) when the host cannot
        e2e = {"unavailable": f"{world} ranks x {16.0 * 2 ** n_loc / 2 ** 30:.0f} GiB pinned "
                              f"host buffers exceed 80 % of MemAvailable "
                              f"({host_avail_gib():.0f} GiB)"}
    elif not args.no_e2e:
        host = torch.empty(1 << n_loc, dtype=torch.complex128, pin_memory=True)
        hv = host.numpy()
        st.copy_out(rank << n_loc, 1 << n_loc, out=hv)
        mq = list(range(10))
        # lfqs_run_circuit_streamed (every rank: its own shard): the 16 GiB upload in 32
        # pieces on a copy stream, each piece running the sweep prefix that stays below
        # local qubit n_loc - 5 as soon as it has landed (bit-identical to copy_in + the
        # sweep; tests/test_gpu_streamed.py).  Pieces only need their own launches while
        # later pieces are in flight: piece c+1 lands (PCIe, ~55 GB/s) after
        # 16*2^25 B / 55 GB/s = 9.8 ms; q gates on a 1/32 piece take q * 3.65 ms / 32, so
        # q >= 86 keeps the GPU busy; the other gates run on the whole shard.
        marshalled = lfqs.marshal_gates([g for _, g in sweep])
        st.set_option(lfqs.OPT_STREAM_MAX_PREFIX, 96)

        def e2e_step():
            st.run_circuit_streamed(hv, marshalled, fuse=False, chunk_bits=5)
            st.measure_probs(mq)
        e2e_step()
        barrier()
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(stream)
        for _ in range(args.e2e_steps):
            e2e_step()
        b.record(stream)
        barrier()
        e_ms = a.elapsed_time(b)
        if dist is not None:
            t = torch.tensor([e_ms], device="cpu" if args.same_device else "cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e_ms = float(t.item())
        e2e = {"value": gates_per_step / (e_ms / args.e2e_steps / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": 16 * (1 << n_loc) * world,
               "d2h_bytes_per_step": 8 * (1 << len(mq)) * world,
               "api": "lfqs_run_circuit_streamed (upload overlapped with the sweep prefix) + "
                      "lfqs_measure_probs"}
        del host

    small = None
    if world == 1 and not args.no_small:
        small = run_small(lfqs, stream, with_oracle=not args.no_cpu_baseline)

    macro = None
    if world == 1 and args.macro_n > 0:
        st.close()
        torch.cuda.synchronize()
        macro = run_macro(lfqs, stream, args.macro_n, args.macro_reps,
                          not args.no_macro_unfused, hbm_peak)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        st.close()
        torch.cuda.synchronize()
        cpu = cpu_baseline(n)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"configs[1]: {n}-qubit single-gate sweep "
                                   f"(18 gate kinds x {n} targets, all classes)",
                       "n_qubits": n, "qubits_per_gpu": n_loc, "gates_per_step": gates_per_step,
                       "state_bytes_per_gpu": 16 * 2 ** n_loc,
                       "l2": "state >> 126 MB L2 every gate; no flush needed",
                       "parallelism": f"state sharded by top {world.bit_length() - 1} qubits, "
                                      f"{args.transport} exchange"
                       if world > 1 else "single GPU",
                       **({"test_same_device": "all ranks share cuda:0 -- not a scaling number"}
                          if args.same_device else {})},
            "roofline": roofline,
            "worst_gate": worst_gate,
            "macro": macro,
            "small": small,
            "macro_sharded": qft,
            "nvlink": nvlink,
            "classes": {k: {kk: (round(vv, 4) if isinstance(vv, float) else vv)
                            for kk, vv in v.items()} for k, v in classes.items()},
            "gpu_launches": int(launches),
            "clocks": clk.summary(),
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
