#!/bin/bash
# ncu --set full captures of single fused passes (source-level, -lineinfo build).
#   bash tools/ncu_fused.sh TAG
set -u
cd "$(dirname "$0")/.."
O=gpurun_out; mkdir -p $O
TAG=${1:-nf}
cap() {  # name circuit mode skip
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_fused \
    --launch-skip $4 --launch-count 1 -o $O/${TAG}_$1 \
    python tools/bench_circuits.py --n 28 --reps 0 --circuits $2 --modes $3 > $O/${TAG}_$1.out 2>&1
}
cap qft_fused qft fused 0
cap qft_phase qft phase 0
cap random_fused random fused 1
echo done
