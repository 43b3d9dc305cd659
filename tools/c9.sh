cd $GRAFT_REPO_ROOT
O=gpurun_out; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_jit.py -q -x > $O/c9_pytest.txt 2>&1
timeout 1200 python tools/bench_circuits.py --n 30 --circuits qft,qpe,grover,random,vqe,sycamore,ghz --modes jit,jit+phase > $O/c9_circ.jsonl 2>&1
echo done
