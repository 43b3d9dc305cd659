"""Peer-memory sharding (NEXT-3) end to end on the GPU: P processes share cuda:0,
map each other's shards through CUDA IPC, and run the product planner with the
in-place P2P swap kernel, device-flag barriers and the rank-ordered probability
sum.  Every rank checks its slice against the oracle (bit-exact for permutation /
diagonal circuits, <= 1e-12 otherwise)."""
import socket

import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.timeout(600)
@pytest.mark.parametrize("world", [2, 4])
def test_p2p_sharded_circuits(world):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import torch.multiprocessing as mp

    from tests._p2p_worker import worker

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=worker, args=(r, world, port, 12, 40 + world, q))
             for r in range(world)]
    for p in procs:
        p.start()
    results = {}
    try:
        for _ in range(world):
            rank, status, payload = q.get(timeout=540)
            results[rank] = (status, payload)
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    for rank in range(world):
        status, payload = results[rank]
        assert status == "ok", f"rank {rank}:\n{payload}"
        for fuse in (0, 1, 2):  # unfused, fused (interpreted), fused (compiled passes)
            err, perr = payload[f"fuse{fuse}"]
            assert err <= 1e-12 and perr <= 1e-12, (rank, fuse, err, perr)
            assert payload[f"exact{fuse}"], (rank, fuse)
        assert payload["apply"] <= 1e-12
        same, err = payload["overlap"]
        assert same and err <= 1e-12, (rank, same, err)
        same, err, strided = payload["overlap_fused"]
        assert same and err <= 1e-12 and (strided > 0 or world > 2), (rank, same, err, strided)
        same, err = payload["streamed"]
        assert same and err <= 1e-12, (rank, same, err)
