mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r02ag_pytest_gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02ag_smoke.txt 2>&1
timeout 2400 python tools/bench_circuits.py --n 30 --modes jit+phase,unfused --oracle-s 12 > gpurun_out/r02ag_circuits_n30.jsonl 2>&1
timeout 2400 python tools/bench_circuits.py --n 33 --reps 1 --circuits qft,ghz,qpe,grover,random,sycamore --modes jit+phase > gpurun_out/r02ag_circuits_n33.jsonl 2>&1
timeout 900 python tools/bench_circuits.py --n 31 --c64 --circuits qft,ghz,random --modes jit+phase > gpurun_out/r02ag_circuits_c64_n31.jsonl 2>&1
timeout 600 python tools/bench_small.py > gpurun_out/r02ag_small.jsonl 2>&1
tail -2 gpurun_out/r02ag_pytest_gpu.txt; cat gpurun_out/r02ag_smoke.txt
