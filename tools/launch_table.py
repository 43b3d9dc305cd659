"""Summarises the ncu launch list of one bench step (tools/gpu_evidence.sh: `ncu --metrics
gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum ... bench.py --steps 1
--warmup 3 --no-e2e --no-cpu-baseline --macro-n 0 --no-small`) into profiles/rNN_launches.md and
profiles/traffic_per_launch.json.

The last 540 gate launches of the capture are the timed step; they are matched, in order,
with the configs[1] sweep (workloads.sweep_gates(30)).

    python tools/launch_table.py gpurun_out/r01e_launches.csv TAG
"""
import csv
import json
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402


def main():
    fn, tag = sys.argv[1], sys.argv[2]
    n = 30
    rows = list(csv.DictReader(ln for ln in open(fn) if not ln.startswith("==")))
    k = {}
    for r in rows:
        d = k.setdefault(int(r["ID"]), {"name": r["Kernel Name"]})
        d[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
    launches = [k[i] for i in sorted(k)]
    gate_kernels = [d for d in launches
                    if ("k_group" in d["name"] or "k_lowq" in d["name"] or "k_lanegroup" in d["name"])]
    sweep = W.sweep_gates(n)
    step = gate_kernels[-len(sweep):]
    assert len(step) == len(sweep), (len(step), len(sweep))
    cls = defaultdict(lambda: {"launches": 0, "ms": 0.0, "dram": 0.0, "alg": 0.0})
    lines = []
    for (c, g), d in zip(sweep, step):
        ms = d["gpu__time_duration.sum"] / 1e6
        dram = d["dram__bytes_read.sum"] + d["dram__bytes_write.sum"]
        alg = W.algorithmic_bytes(g, n)
        e = cls[c]
        e["launches"] += 1
        e["ms"] += ms
        e["dram"] += dram
        e["alg"] += alg
        name = d["name"].replace("(anonymous namespace)", "").replace("lfqs::", "")[:60]
        lines.append(f"{c:7s} {g.label():26s} {name:60s} {ms:7.3f} ms  dram {dram / 1e9:7.3f}  "
                     f"alg {alg / 1e9:7.3f}")
    tot = sum(e["ms"] for e in cls.values())
    out = [f"# {tag} — ncu launch list of one bench step (n = 30 sweep, {len(sweep)} launches)", "",
           "Command: `ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
           "--clock-control none --csv python bench.py --steps 1 --warmup 3 --no-e2e "
           "--no-cpu-baseline --macro-n 0 --no-small` (tools/gpu_evidence.sh); table by "
           "`tools/launch_table.py`.",
           "ncu times are cold-cache and serialised: compare shares, not absolutes. Bench (CUDA "
           "events, same kernels): see the bench JSON line.", "",
           "| class | launches | ncu ms | share | DRAM bytes/launch (traffic) | SURVEY §8(d) "
           "bytes/launch | traffic / algorithmic | DRAM GB/s |",
           "|---|---|---|---|---|---|---|---|"]
    traffic = {}
    for c, e in cls.items():
        nl = e["launches"]
        traffic[c] = int(round(e["dram"] / nl))
        out.append(f"| {c} | {nl} | {e['ms']:.1f} | {100 * e['ms'] / tot:.1f}% | "
                   f"{e['dram'] / nl / 1e9:.3f} GB | {e['alg'] / nl / 1e9:.3f} GB | "
                   f"{e['dram'] / e['alg']:.3f} | {e['dram'] / (e['ms'] / 1e3) / 1e9:.0f} |")
    slow = sorted(zip(sweep, step), key=lambda x: -x[1]["gpu__time_duration.sum"])[:8]
    out += ["", "Slowest launches: " + ", ".join(
        f"{g.label()} {d['gpu__time_duration.sum'] / 1e6:.3f} ms" for (_, g), d in slow), "",
        "Per launch (class, gate, kernel, ms, DRAM GB, algorithmic GB):", "", "```"] + lines + ["```"]
    with open(os.path.join(ROOT, "profiles", f"{tag}_launches.md"), "w") as f:
        f.write("\n".join(out) + "\n")
    with open(os.path.join(ROOT, "profiles", "traffic_per_launch.json"), "w") as f:
        json.dump(traffic, f, indent=1)
    print("\n".join(out[:14]))


if __name__ == "__main__":
    main()
