cd $GRAFT_REPO_ROOT
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_phase.py tests/test_gpu_fused.py -q -x > $O/c2_pytest.txt 2>&1
timeout 900 python tools/bench_circuits.py --n 30 --circuits qft,qpe,grover,random,vqe,sycamore --modes fused,phase > $O/c2_circ.jsonl 2>&1
bash tools/pass_profile.sh c2 28 qft,random,grover fused,phase
