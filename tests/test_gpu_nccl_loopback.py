"""The NCCL transport (csrc/comm.cu) executed on one GPU: a one-rank communicator exchanging
with itself through the real ncclSend/ncclRecv groups, staging buffers, events and copies,
plus the all-reduce and the polling wait (tests/_nccl_loopback.cu).  Two ranks cannot share
one GPU under NCCL, so the multi-rank exchange itself stays unexercised here."""
import os
import subprocess

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_nccl_transport_loopback(tmp_path):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import nvidia.nccl
    nccl = list(nvidia.nccl.__path__)[0]
    csrc = os.path.join(ROOT, "paper_conf_cgo_tarabkhahdds25_b200", "csrc")
    exe = str(tmp_path / "nccl_loopback")
    cmd = ["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O2",
           "-std=c++17", "-I", os.path.join(ROOT, "include"), "-I", csrc,
           "-I", os.path.join(nccl, "include"), os.path.join(ROOT, "tests", "_nccl_loopback.cu"),
           os.path.join(csrc, "comm.cu"), "-L", os.path.join(nccl, "lib"), "-l:libnccl.so.2",
           "-Xlinker", "-rpath=" + os.path.join(nccl, "lib"), "-o", exe]
    subprocess.run(cmd, check=True, capture_output=True, timeout=600)
    r = subprocess.run([exe], capture_output=True, text=True, timeout=300)
    last = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else ""
    assert r.returncode == 0 and last.startswith("ok"), r.stdout + r.stderr
