"""Renders tools/bench_circuits.py JSON lines as the markdown table of profiles/rNN_circuits.md.

    python tools/circuits_table.py gpurun_out/r01_circuits_n30.jsonl [more.jsonl ...]
"""
import json
import sys


def fmt_check(d):
    if "max_abs_err" in d:
        return f"err {d['max_abs_err']:.1e}"
    if "norm2" in d:
        return f"norm² {d['norm2']:.15f}"
    return ""


def fmt_oracle(d):
    o = d.get("oracle")
    if o is None:
        return "", ""
    if "unavailable" in o:
        return f"not run: {o['unavailable']}", ""
    return (f"{o['gates_per_s']:.2f} ({o['gates']}/{o['of']} gates, {o['cores']} cores)",
            f"{d['gpu_over_oracle']:.0f}×")


def main():
    print("| n | dtype | circuit | mode | gates | passes | time ms | gates/s | ms/pass | "
          "HBM frac per pass | HBM frac, 1 pass/gate convention | check | compile s | "
          "oracle gates/s | GPU / oracle |")
    print("|" + "---|" * 15)
    for fn in sys.argv[1:]:
        for ln in open(fn):
            if not ln.startswith("{"):
                continue
            d = json.loads(ln)
            o, ratio = fmt_oracle(d)
            comp = d.get("jit_compile_s")
            print(f"| {d['n']} | {d['dtype']} | {d['circuit']} | {d['mode']} | {d['gates']} | "
                  f"{d['passes']} | {d['ms']:.1f} | {d['gates_per_s']:.0f} | "
                  f"{d['ms'] / max(d['passes'], 1):.2f} | {d.get('pass_frac', 0):.2f} | "
                  f"{d.get('conv_frac', 0):.2f} | {fmt_check(d)} | "
                  f"{'' if comp is None else comp} | {o} | {ratio} |")


if __name__ == "__main__":
    main()
