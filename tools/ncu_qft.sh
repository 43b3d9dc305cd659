#!/bin/bash
# ncu of the compiled QFT passes (jit+phase, n = 28): launch list with FP64 / shared-memory /
# barrier-relevant metrics, and --set full of the slowest pass.   bash tools/ncu_qft.sh TAG SKIP
set -u
cd "$(dirname "$0")/.."
O=gpurun_out; mkdir -p $O
TAG=${1:-qf}; SKIP=${2:-0}
M="gpu__time_duration.sum,sm__inst_executed.sum,smsp__inst_executed_pipe_fp64.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum"
timeout 600 ncu --metrics $M --clock-control none --csv --log-file $O/${TAG}_launches.csv -k regex:lfqs_jit \
  python tools/bench_circuits.py --n 28 --reps 0 --circuits qft,qpe --modes jit+phase > $O/${TAG}_ncu.out 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:lfqs_jit \
  --launch-skip $SKIP --launch-count 1 -o $O/${TAG}_qft_p$SKIP \
  python tools/bench_circuits.py --n 28 --reps 0 --circuits qft --modes jit+phase > $O/${TAG}_full.out 2>&1
echo done
