"""1-D partitioned BFS across ranks: the per-level exchange.

Every computation (expand, pack, OR-reduce, unpack, frontier compaction) runs
in libefg.so on the rank's GPU; this module only moves bytes between ranks
with torch.distributed (NCCL over NVLink on GPUs; gloo in the CPU tests).

Per level (all ranks in lock step):
    g.bfs_expand()                      decode + visit the rank's own rows
    g.xchg_pack(bounds, S, send)        slice h of the rank's new bits -> send[h]
    all_to_all(send -> recv)            rank h receives every rank's slice h
    g.xchg_reduce(P, S, recv, mine)     OR of the P copies of slice h
    all_gather(mine -> gathered)        every rank gets every owner's slice
    g.xchg_unpack(bounds, S, gathered)  visited |= global new bits
    g.bfs_finish_level()                next frontier = new owned vertices,
                                        depth of all new vertices; global count
The global new-vertex count is identical on every rank (same bitmap), so the
loop ends on all ranks at the same level with no extra collective.
"""
from __future__ import annotations

import numpy as np


class TorchTransport:
    """all_to_all / all_gather of equal slices with torch.distributed.

    stage_on_host=True copies device buffers through host memory (for the gloo
    backend, e.g. several ranks sharing one GPU in a functional test)."""

    def __init__(self, group=None, stage_on_host: bool = False):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.host = stage_on_host

    def all_to_all(self, send, recv):
        if self.host:
            r = recv.cpu()
            self.dist.all_to_all_single(r, send.cpu(), group=self.group)
            recv.copy_(r)
            return
        self.dist.all_to_all_single(recv, send, group=self.group)

    def all_gather(self, mine, gathered):
        if self.host:
            gh = gathered.cpu()
            self._all_gather(mine.cpu(), gh)
            gathered.copy_(gh)
            return
        self._all_gather(mine, gathered)

    def _all_gather(self, mine, gathered):
        try:
            self.dist.all_gather_into_tensor(gathered, mine, group=self.group)
        except (RuntimeError, NotImplementedError):
            world = self.dist.get_world_size(self.group)
            parts = list(gathered.chunk(world))
            self.dist.all_gather(parts, mine, group=self.group)


def partition_bounds(vlist: np.ndarray, offsets: np.ndarray, world: int) -> np.ndarray:
    from . import partition
    return partition(vlist, offsets, world)


def partitioned_bfs(g, source: int, depth, bounds: np.ndarray, transport, make_buffer):
    """Run one BFS over the partitioned handles of all ranks.

    g          this rank's Graph (built with rows=(bounds[r], bounds[r+1]))
    depth      this rank's device int32 buffer (n); receives the full depth array
    bounds     np.uint64[world+1] vertex boundaries (efg_partition)
    transport  object with all_to_all(send, recv) and all_gather(mine, gathered)
    make_buffer(nwords) -> device uint32/int32 tensor
    Returns the list of global new-vertex counts per level.
    """
    world = bounds.size - 1
    S = g.xchg_geometry(bounds)
    send = make_buffer(world * S)
    recv = make_buffer(world * S)
    mine = make_buffer(S)
    gathered = make_buffer(world * S)
    g.bfs_begin(source, depth)
    counts = [1]
    while True:
        g.bfs_expand()
        g.xchg_pack(bounds, S, send)
        transport.all_to_all(send, recv)
        g.xchg_reduce(world, S, recv, mine)
        transport.all_gather(mine, gathered)
        g.xchg_unpack(bounds, S, gathered)
        new = g.bfs_finish_level()
        if new == 0:
            break
        counts.append(new)
    return counts


def simulated_partitioned_bfs(graphs, source: int, depths, bounds: np.ndarray, make_buffer):
    """The same protocol with all `world` rank handles in one process (one GPU):
    the all-to-all and all-gather become buffer copies.  Used by the GPU tests to
    run the partitioned kernels without several GPUs.  The handles may run on
    their own streams: the copies (torch's current stream) are fenced with
    device synchronisations on both sides."""
    import torch
    world = bounds.size - 1
    S = graphs[0].xchg_geometry(bounds)
    send = [make_buffer(world * S) for _ in range(world)]
    recv = [make_buffer(world * S) for _ in range(world)]
    mine = [make_buffer(S) for _ in range(world)]
    gathered = make_buffer(world * S)
    for g, d in zip(graphs, depths):
        g.bfs_begin(source, d)
    counts = [1]
    while True:
        for r, g in enumerate(graphs):
            g.bfs_expand()
            g.xchg_pack(bounds, S, send[r])
        torch.cuda.synchronize()
        for r in range(world):          # all-to-all
            for p in range(world):
                recv[r][p * S:(p + 1) * S].copy_(send[p][r * S:(r + 1) * S])
        torch.cuda.synchronize()
        for r, g in enumerate(graphs):
            g.xchg_reduce(world, S, recv[r], mine[r])
        torch.cuda.synchronize()
        for r in range(world):          # all-gather
            gathered[r * S:(r + 1) * S].copy_(mine[r])
        torch.cuda.synchronize()
        news = []
        for g in graphs:
            g.xchg_unpack(bounds, S, gathered)
            news.append(g.bfs_finish_level())
        assert len(set(news)) == 1, news
        if news[0] == 0:
            break
        counts.append(news[0])
    return counts


# ---------------------------------------------------------------------------
# The same exchange over peer memory (efg.h "exchange over peer memory"): the
# library's kernels read and write the other ranks' HBM over NVLink; this
# module only all-gathers the 64-byte CUDA IPC handles once per partition.
# ---------------------------------------------------------------------------
def peer_setup(g, rank: int, bounds: np.ndarray, group=None) -> None:
    """Collective: allocate this rank's region, all-gather the IPC handles,
    map the other ranks' regions."""
    import torch.distributed as dist
    world = bounds.size - 1
    _, handle = g.peer_alloc(world)
    handles = [None] * world
    dist.all_gather_object(handles, handle, group=group)
    g.peer_open(rank, bounds, handles=handles)


def partitioned_bfs_peer(g, source: int, depth):
    """One partitioned BFS after peer_setup: per level expand, peer exchange,
    level end.  Returns the list of global new-vertex counts per level."""
    g.bfs_begin(source, depth)
    counts = [1]
    while True:
        g.bfs_expand()
        g.xchg_peer()
        new = g.bfs_finish_level()
        if new == 0:
            break
        counts.append(new)
    return counts


def partitioned_bfs_peer_hostseq(g, source: int, depth, host_barrier):
    """The same partitioned BFS over peer memory with host-sequenced exchange
    phases (efg_xchg_peer_phase + `host_barrier()` after each): no kernel waits
    for another rank, so ranks may time-share one GPU."""
    g.bfs_begin(source, depth)
    counts = [1]
    while True:
        g.bfs_expand()
        for phase in (0, 1, 2):
            g.xchg_peer_phase(phase)
            if phase < 2:
                host_barrier()
        new = g.bfs_finish_level()
        host_barrier()  # every rank's unpack read res before the next publish / OR
        if new == 0:
            break
        counts.append(new)
    return counts


def simulated_peer_setup(graphs, bounds: np.ndarray) -> None:
    """All `world` rank handles in one process on one device (tests): the
    regions are mapped by address instead of IPC.  Each handle must have been
    built on its own non-blocking stream."""
    world = bounds.size - 1
    regions = [g.peer_alloc(world)[0] for g in graphs]
    for r, g in enumerate(graphs):
        g.peer_open(r, bounds, regions=regions)


def simulated_partitioned_bfs_peer(graphs, source: int, depths):
    for g, d in zip(graphs, depths):
        g.bfs_begin(source, d)
    counts = [1]
    while True:
        for g in graphs:
            g.bfs_expand()
        for g in graphs:      # every rank's barrier kernels are enqueued before any wait
            g.xchg_peer()
        news = [g.bfs_finish_level() for g in graphs]
        assert len(set(news)) == 1, news
        if news[0] == 0:
            break
        counts.append(news[0])
    return counts
