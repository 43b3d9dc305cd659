#!/bin/bash
# Collects the round's GPU evidence into gpurun_out/ (run under gpurun on one B200):
#   tests, smoke, bench line, reference arm, per-launch ncu list of the bench step (time +
#   DRAM bytes), one ncu --set full capture of the dominant kernel, per-gate timings, macro
#   circuits at n = 30 / 33 (and complex64 at 31), configs[0] small-n timings, sanitizers.
#   bash tools/gpu_evidence.sh TAG
set -u
cd "$(dirname "$0")/.."
O=gpurun_out
mkdir -p $O
TAG=${1:-r02}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/${TAG}_gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > $O/${TAG}_smoke.txt 2>&1
timeout 1800 python -m pytest tests -m gpu -q > $O/${TAG}_pytest_gpu.txt 2>&1
timeout 900 python bench.py > $O/${TAG}_bench.json 2> $O/${TAG}_bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 --ref-step-s 6 > $O/${TAG}_bench_ref.json 2> $O/${TAG}_bench_ref.err
timeout 300 python tools/profile_gates.py --n 30 --reps 5 --time --no-shuffle > $O/${TAG}_pergate_n30.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
  --clock-control none --csv --log-file $O/${TAG}_launches.csv \
  python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --macro-n 0 --no-small > $O/${TAG}_ncu_bench.out 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_group_x2 -c 2 \
  -o $O/${TAG}_full_dense1 python tools/profile_gates.py --n 28 --reps 1 --gates RX:12,H:20 \
  > $O/${TAG}_ncu_full.out 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_group -c 1 \
  -o $O/${TAG}_full_toffoli12 python tools/profile_gates.py --n 28 --reps 1 --gates CCX:1/2/5 \
  > $O/${TAG}_ncu_full_toffoli.out 2>&1
timeout 2400 python tools/bench_circuits.py --n 30 --modes jit+phase,unfused --oracle-s 12 > $O/${TAG}_circuits_n30.jsonl 2>&1
timeout 2400 python tools/bench_circuits.py --n 33 --reps 1 --circuits qft,ghz,qpe,grover,random,sycamore --modes jit+phase > $O/${TAG}_circuits_n33.jsonl 2>&1
timeout 900 python tools/bench_circuits.py --n 31 --c64 --circuits qft,ghz,random --modes jit+phase > $O/${TAG}_circuits_c64_n31.jsonl 2>&1
timeout 600 python tools/bench_small.py > $O/${TAG}_small.jsonl 2>&1
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29517 bench.py --gpus 2 --same-device --qubits-per-gpu 28 --steps 2 --warmup 3 \
  > $O/${TAG}_bench_n2_same_device.json 2> $O/${TAG}_bench_n2.err
timeout 900 python tools/bench_overlap.py --n 32 --world 4 --circuit qft --bits 0,2 > $O/${TAG}_overlap_qft32_w4.jsonl 2>&1
# compute-sanitizer is closed on this GPU pool (round 2); tools/sanitize_run.py is the
# workload the r01/r02 sanitizer passes ran (profiles/r0*_sanitizers.md); run here without
# the sanitizer it still exercises every kernel family once and checks its own results.
timeout 600 python tools/sanitize_run.py > $O/${TAG}_sanitize_workload.txt 2>&1
echo done
