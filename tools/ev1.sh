set -u
cd $GRAFT_REPO_ROOT
O=gpurun_out; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/gpu.txt
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; echo smoke=$? >> $O/smoke.txt
timeout 1200 python -m pytest tests -m gpu -q -x > $O/pytest_gpu.txt 2>&1
timeout 600 python bench.py > $O/bench.json 2> $O/bench.err
timeout 900 python tools/bench_circuits.py --n 30 > $O/circuits_n30.jsonl 2>&1
echo done
