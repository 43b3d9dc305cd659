#!/bin/bash
# Launch list (time, instructions, FP64 pipe, shared-memory wavefronts, bank conflicts) of
# the compiled passes of the heavy macro circuits, and one --set full capture of the
# heaviest Sycamore-like pass.  Run under gpurun on one B200:  bash tools/ncu_heavy.sh TAG
set -u
cd "$(dirname "$0")/.."
O=gpurun_out; mkdir -p $O
TAG=${1:-hv}
M="gpu__time_duration.sum,sm__inst_executed.sum,smsp__inst_executed_pipe_fp64.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,smsp__inst_executed_op_shfl.sum,dram__bytes_read.sum,dram__bytes_write.sum"
timeout 900 ncu --metrics $M --clock-control none --csv --log-file $O/${TAG}_launches.csv -k regex:lfqs_jit \
  python tools/bench_circuits.py --n 28 --reps 0 --circuits sycamore,random,vqe --modes jit+phase > $O/${TAG}_ncu.out 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:lfqs_jit \
  --launch-skip 0 --launch-count 1 -o $O/${TAG}_sycamore_p0 \
  python tools/bench_circuits.py --n 28 --reps 0 --circuits sycamore --modes jit+phase > $O/${TAG}_full.out 2>&1
echo done
