cd $GRAFT_REPO_ROOT
O=gpurun_out; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/c8_gpu.txt
timeout 1500 python tools/bench_circuits.py --n 30 --modes fused,phase,jit,jit+phase,unfused > $O/c8_circ30.jsonl 2>&1
timeout 1500 python tools/bench_circuits.py --n 33 --reps 1 --circuits qft,ghz,qpe,grover,random --modes fused,jit,jit+phase > $O/c8_circ33.jsonl 2>&1
timeout 900 python tools/bench_circuits.py --n 31 --c64 --reps 1 --circuits qft,ghz,random --modes fused,jit,jit+phase > $O/c8_circ31c64.jsonl 2>&1
echo done
