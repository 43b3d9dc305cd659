cd $GRAFT_REPO_ROOT
O=gpurun_out; mkdir -p $O
nproc > $O/c4_nproc.txt
timeout 1200 python -m pytest tests/test_gpu_jit.py -q -x > $O/c4_pytest.txt 2>&1
timeout 1200 python tools/bench_circuits.py --n 30 --circuits qft,qpe,grover,random,vqe,sycamore,ghz --modes fused,phase,jit,jit+phase > $O/c4_circ.jsonl 2>&1
echo done
