"""Two processes, one per rank, running the partitioned BFS with the exchange
over peer memory (efg_peer_alloc / efg_peer_open with CUDA IPC handles;
SURVEY §8(e)).  On a multi-GPU box each rank would own a GPU and the regions
would be reached over NVLink; here both ranks share cuda:0 (this run has one
GPU), which exercises the same IPC mapping and the same exchange kernels.
Ranks time-sharing one GPU must not run kernels that wait on one another
(nothing schedules two processes' kernels together; B200_PROFILING.md reports
Xid 109 for exactly that), so the exchange runs host-sequenced here
(efg_xchg_peer_phase, a gloo barrier after every phase); the device-barrier
form (efg_xchg_peer, collective efg_bfs) is tested with simulated ranks in one
process (tests/test_gpu_bfs.py, tests/test_gpu_boundary.py).  The handles are
all-gathered over gloo; no data-path collective.  Every rank's depth must
equal the oracle's.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu

WORLD = 2
SOURCES = (0, 3, 9999)


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank: int, port: int, q):
    try:
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        import torch
        import torch.distributed as dist
        import oracle
        import synth
        import paper_conf_ipps_gerak23_b200 as efg
        from paper_conf_ipps_gerak23_b200.dist import peer_setup, partitioned_bfs_peer_hostseq
        dist.init_process_group("gloo", rank=rank, world_size=WORLD)
        torch.cuda.set_device(0)
        n, src, dst = synth.rmat(14, 16, seed=13)
        whole = efg.Graph.build(n, src, dst, device=-1)
        vlist, _, offsets, _ = whole.export()
        bounds = efg.partition(vlist, offsets, WORLD)
        whole.free()
        g = efg.Graph.build(n, src, dst, rows=(int(bounds[rank]), int(bounds[rank + 1])))
        peer_setup(g, rank, bounds)
        ov, oe = oracle.csr_build(n, src, dst)
        bad = []
        for s in SOURCES:
            ref = oracle.bfs(ov, oe, s)
            depth = torch.empty(n, dtype=torch.int32, device="cuda")
            depth.fill_(-7)
            partitioned_bfs_peer_hostseq(g, s, depth, dist.barrier)
            torch.cuda.synchronize()
            if not np.array_equal(depth.cpu().numpy(), ref):
                bad.append(("hostseq", s))
        dist.barrier()
        g.free()
        dist.destroy_process_group()
        q.put((rank, "ok" if not bad else f"depth mismatch for sources {bad}"))
    except Exception as e:  # report, do not hang the parent
        q.put((rank, f"error: {type(e).__name__}: {e}"))


def test_peer_exchange_two_processes_ipc(cuda_ok):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(WORLD)]
    for p in procs:
        p.start()
    results = {}
    try:
        for _ in range(WORLD):
            r, msg = q.get(timeout=300)
            results[r] = msg
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    assert results == {r: "ok" for r in range(WORLD)}, results
