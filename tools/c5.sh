cd $GRAFT_REPO_ROOT
O=gpurun_out; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_jit.py tests/test_gpu_phase.py tests/test_gpu_fused.py -q > $O/c5_pytest.txt 2>&1
echo done
