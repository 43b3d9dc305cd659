cd $GRAFT_REPO_ROOT
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.smoke()" > $O/c10_smoke.txt 2>&1; echo smoke=$? >> $O/c10_smoke.txt
timeout 1800 python -m pytest tests -m gpu -q > $O/c10_pytest_gpu.txt 2>&1
timeout 600 python bench.py > $O/c10_bench.json 2> $O/c10_bench.err
echo done
