cd $GRAFT_REPO_ROOT
O=gpurun_out; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_jit.py tests/test_gpu_phase.py tests/test_gpu_fused.py -q -x > $O/c7_pytest.txt 2>&1
timeout 1200 python tools/bench_circuits.py --n 30 --circuits qft,qpe,grover,random,vqe,sycamore,ghz --modes jit,jit+phase > $O/c7_circ.jsonl 2>&1
echo done
