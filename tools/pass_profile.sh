#!/bin/bash
# Per-launch durations of the fused passes of macro circuits (ncu launch list), and one
# ncu --set full capture of a fused pass.  Run under gpurun on one B200.
#   bash tools/pass_profile.sh TAG N CIRCUITS MODES
set -u
cd "$(dirname "$0")/.."
O=gpurun_out; mkdir -p $O
TAG=${1:-pp}; N=${2:-28}; C=${3:-qft,random,grover}; M=${4:-fused,phase}
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__inst_executed.sum,smsp__inst_executed_pipe_fp64.sum \
  --clock-control none --csv --log-file $O/${TAG}_launches.csv \
  python tools/bench_circuits.py --n $N --reps 0 --circuits $C --modes $M > $O/${TAG}_ncu.out 2>&1
echo rc=$?
