"""Multi-process (world_size 2, gloo, CPU) test of the partitioned-BFS exchange
protocol in paper_conf_ipps_gerak23_b200/dist.py.

The per-rank computations are stood in for by a host model of the stepwise
handle (same slice / OR / unpack rules as efg_xchg_*, expand over the rank's
own CSR rows); the bytes move through torch.distributed exactly as on GPUs
(there over NCCL).  The depths every rank ends with must equal the oracle's.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth


class HostRank:
    """Host model of one rank's stepwise handle (stored ids = input ids)."""

    def __init__(self, vlist, elist, lo, hi):
        self.v, self.e = vlist, elist
        self.n = vlist.size - 1
        self.lo, self.hi = lo, hi
        self.nw = (self.n + 31) // 32

    def xchg_geometry(self, bounds):
        return int(max((int(bounds[r + 1]) + 31) // 32 - int(bounds[r]) // 32
                       for r in range(bounds.size - 1)))

    def _set(self, bm, x):
        bm[x >> 5] |= np.uint32(1 << (int(x) & 31))

    def bfs_begin(self, s, depth):
        self.vis = np.zeros(self.nw, np.uint32)
        self.prev = np.zeros(self.nw, np.uint32)
        self.depth = depth
        self.depth.fill_(-1)
        self.level = 0
        self._set(self.vis, s)
        self._finish()

    def _finish(self):
        new = self.vis & ~self.prev
        self.prev = self.vis.copy()
        ids = np.flatnonzero(np.unpackbits(new.view(np.uint8), bitorder="little"))
        ids = ids[ids < self.n]
        self.depth[torch.from_numpy(ids.astype(np.int64))] = self.level
        self.frontier = ids[(ids >= self.lo) & (ids < self.hi)]
        return ids.size

    def bfs_expand(self):
        for u in self.frontier:
            for x in self.e[self.v[u]:self.v[u + 1]]:
                self._set(self.vis, x)
        self.level += 1

    def xchg_pack(self, bounds, S, send):
        world = bounds.size - 1
        out = np.zeros(world * S, np.uint32)
        new = self.vis & ~self.prev
        for h in range(world):
            w0, w1 = int(bounds[h]) // 32, (int(bounds[h + 1]) + 31) // 32
            out[h * S:h * S + (w1 - w0)] = new[w0:w1]
        send.copy_(torch.from_numpy(out.view(np.int32)))

    def xchg_reduce(self, world, S, recv, mine):
        r = recv.numpy().view(np.uint32).reshape(world, S)
        mine.copy_(torch.from_numpy(np.bitwise_or.reduce(r, axis=0).view(np.int32)))

    def xchg_unpack(self, bounds, S, gathered):
        gd = gathered.numpy().view(np.uint32)
        for h in range(bounds.size - 1):
            w0, w1 = int(bounds[h]) // 32, (int(bounds[h + 1]) + 31) // 32
            self.vis[w0:w1] |= gd[h * S:h * S + (w1 - w0)]

    def bfs_finish_level(self):
        return self._finish()


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_gerak23_b200.dist import TorchTransport, partitioned_bfs
    n, src, dst = synth.rmat(11, 8, seed=3)
    vlist, elist = oracle.csr_build(n, src, dst)
    # byte-balanced-like bounds (multiples of 64), rows of the other rank emptied
    bounds = np.array([0, 640, n], np.uint64)
    lo, hi = int(bounds[rank]), int(bounds[rank + 1])
    deg = np.diff(vlist).copy()
    deg[:lo] = 0
    deg[hi:] = 0
    mine_v = np.concatenate([[0], np.cumsum(deg)]).astype(np.uint64)
    mine_e = np.concatenate([elist[vlist[u]:vlist[u + 1]] for u in range(lo, hi)] or [np.zeros(0, np.uint32)])
    h = HostRank(mine_v, mine_e, lo, hi)
    ok = True
    for s in (0, 5, 700, n - 1):
        depth = torch.empty(n, dtype=torch.int32)
        partitioned_bfs(h, s, depth, bounds, TorchTransport(),
                        lambda k: torch.zeros(k, dtype=torch.int32))
        ok &= bool(np.array_equal(depth.numpy(), oracle.bfs(vlist, elist, s)))
    q.put((rank, ok))
    dist.destroy_process_group()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_partitioned_bfs_protocol_gloo_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {0: True, 1: True}
