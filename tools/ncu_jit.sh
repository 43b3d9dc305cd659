#!/bin/bash
# ncu captures of compiled fused passes (LFQS_FUSE_JIT): per-launch list for several
# circuits and --set full of single passes.   bash tools/ncu_jit.sh TAG
set -u
cd "$(dirname "$0")/.."
O=gpurun_out; mkdir -p $O
TAG=${1:-nj}
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__inst_executed.sum,smsp__inst_executed_pipe_fp64.sum \
  --clock-control none --csv --log-file $O/${TAG}_launches.csv \
  python tools/bench_circuits.py --n 28 --reps 0 --circuits qft,random,sycamore,grover,vqe --modes jit+phase > $O/${TAG}_ncu.out 2>&1
cap() {  # name circuit mode skip
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:lfqs_jit \
    --launch-skip $4 --launch-count 1 -o $O/${TAG}_$1 \
    python tools/bench_circuits.py --n 28 --reps 0 --circuits $2 --modes $3 > $O/${TAG}_$1.out 2>&1
}
cap qft qft jit+phase 0
cap random random jit+phase 1
cap sycamore sycamore jit+phase 2
echo done
