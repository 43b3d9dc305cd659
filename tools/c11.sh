cd $GRAFT_REPO_ROOT
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_soa.py -q -x > $O/c11_pytest.txt 2>&1
G="H:2,H:20,H:29,X:0,X:20,Y:7,RX:12,U3:25,Z:15,Z:0,T:0,S:1,PHASE:6,RZ:0,RZ:20,CZ:0/9,SWAP:1/20,SWAP:0/20,U2:0/7,U2:20/25,CX:1/0,CX:10/11,CCX:20/21/5,U3q:0/4/9,U3q:20/25/28"
timeout 600 python tools/profile_gates.py --n 30 --reps 5 --time --no-shuffle --gates $G > $O/c11_aos.txt 2>&1
timeout 600 python tools/profile_gates.py --n 30 --reps 5 --time --no-shuffle --soa --gates $G > $O/c11_soa.txt 2>&1
echo done
