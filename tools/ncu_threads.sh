set -u
cd /root/repo
O=gpurun_out; mkdir -p $O
for t in ${THREADS:-256 128}; do
timeout 600 ncu --metrics gpu__time_duration.sum,sm__inst_executed.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active --clock-control none --csv --log-file $O/r02thr_${t}.csv -k regex:lfqs_jit \
  python tools/bench_circuits.py --n 28 --reps 0 --circuits grover,random,vqe,qft --modes jit+phase --jit-threads $t > $O/r02thr_${t}.out 2>&1
done
echo done
