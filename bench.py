#!/usr/bin/env python
"""bench.py — BFS GTEPS over an Elias-Fano-compressed graph on B200.

Contract (driver): ``python bench.py --gpus N --steps K --warmup W`` prints ONE
JSON line on rank 0.  A "step" is one full BFS (all levels: frontier
materialisation, scan, partition, decode, visit, compaction — SURVEY §8(a)
rows a1-a7) from one seeded source over the BASELINE.json configs[2] graph
(Twitter-shaped power-law graph, the config the 1/2/4/8-GPU metric is quoted
on; ``--config 2`` = RMAT-24/ef16, ``--config 4`` = web-shaped) resident in HBM.

  value      whole-job GTEPS = sum over ranks of traversed edges / max-over-ranks
             device time (traversed edges = sum of degrees of reached vertices,
             DESIGN.md reading C18)
  e2e        the same metric through the C ABI with a pinned HOST depth buffer
             (device->host copy of the depth array inside the timed region)
  roofline   expand+decode kernel: algorithmic bytes (compressed list bytes of the
             frontier + 21 B per frontier vertex) / its
             CUDA-event time, against MEASURED_PEAKS.json hbm_gbs
  cpu_baseline  the oracle (plain single-threaded FIFO BFS over CSR) timed on
             this host on a bounded sample (one BFS of the same graph, pinned to
             one core, in a spawned process that overlaps the GPU work), with a
             bit-exact depth check against the GPU BFS from that source

``--impl reference`` runs the reference arm: the oracle, as it stands, on one
host core, same config/metric; each step is a bounded sample of one BFS (the
oracle's FIFO BFS from that step's source, stopped after 2^28 scanned edges:
or_bfs_bounded), so that the whole run stays within minutes on C3/C4.
With N > 1 (torchrun) the default is the north_star's 1-D row partition: each
rank holds a byte-balanced row range of the EFG, every BFS level exchanges the
new-vertex bitmap ("scaling": "strong"): by default the library's kernels
read every rank's new bits over NVLink peer memory and broadcast the owners'
OR (``--xchg peer``; CUDA IPC handles all-gathered once), or all_to_all + OR +
all_gather with torch.distributed over NCCL (``--xchg nccl``).
``--mode replicas`` runs independent BFS problems per rank on
disjoint sources (no data-path collective, "scaling": "weak").
Also reported on one GPU: PageRank (50 iterations) and SSSP over the same graph.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "BFS GTEPS on EF-compressed graph"
UNIT = "GTEPS"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="efg", choices=["efg", "reference"])
    p.add_argument("--config", type=int, default=3, help="BASELINE.json config index (1-based); "
                   "3 = twitter_like, the config of the 1/2/4/8-GPU metric")
    p.add_argument("--scale", type=int, default=None, help="override RMAT scale (debug only)")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-alt", action="store_true", help="skip the reorder=none comparison run "
                   "(run by default on the configs that name it: C2 and C4 'with and without reordering')")
    p.add_argument("--alt", action="store_true", help="force the reorder=none comparison run")
    p.add_argument("--mode", default="partition", choices=["partition", "replicas"],
                   help="N > 1: 1-D partitioned BFS with a per-level NCCL exchange (SURVEY 8(e)), "
                        "or independent replicas on disjoint sources")
    p.add_argument("--xchg", default="peer", choices=["peer", "hostseq", "nccl"],
                   help="N > 1 partition mode: per-level exchange by the library's kernels over "
                        "NVLink peer memory (CUDA IPC, efg_xchg_peer; collective efg_bfs), the same "
                        "kernels host-sequenced (efg_xchg_peer_phase + a barrier per phase: no kernel "
                        "waits for another rank; used automatically when ranks share a GPU), or "
                        "all_to_all + all_gather with torch.distributed (efg_xchg_pack/reduce/unpack)")
    p.add_argument("--host-resident", action="store_true",
                   help="out-of-core EFG (EFG_HOST_RESIDENT, P:34/P:222): EF data in pinned host memory, "
                        "read by the kernels over the host link")
    p.add_argument("--permute", action="store_true",
                   help="random relabelling of the generator's ids (P:248-258 'random ordering' arm)")
    p.add_argument("--reorder", default=None, choices=["none", "degree"],
                   help="EFG_REORDER_DEGREE relabelling at build time (results stay in input ids); "
                        "default degree, none on C5 (permuted ids, sharded build without global degrees)")
    p.add_argument("--profile-levels", action="store_true", help="print per-level stats to stderr")
    p.add_argument("--no-sssp", action="store_true",
                   help="skip the SSSP (NEXT-1) timing over the same graph built with synthetic weights "
                        "(on by default on C4, BASELINE configs[3] 'BFS and SSSP')")
    p.add_argument("--sssp", action="store_true", help="force the SSSP timing on other configs")
    p.add_argument("--no-pagerank", action="store_true",
                   help="skip the PageRank measurement (on by default on C2, BASELINE configs[1]: "
                        "BFS and PageRank)")
    p.add_argument("--pagerank", action="store_true", help="force the PageRank timing on other configs")
    a = p.parse_args()
    if a.reorder is None:
        a.reorder = "none" if a.config == 5 else "degree"
    a.do_alt = (a.alt or a.config in (2, 4)) and not a.no_alt
    a.do_sssp = (a.sssp or a.config == 4) and not a.no_sssp
    a.do_pagerank = (a.pagerank or a.config == 2) and not a.no_pagerank
    return a


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


class ClockSampler:
    """SM clock and clock-event (throttle) reasons sampled DURING the timed
    region: an NVML thread polling every ~2 ms (ctypes calls release the GIL,
    so it runs while the main thread waits on the device); falls back to
    `nvidia-smi -lms 100` when NVML is unavailable."""

    NAMES = (("hw_slowdown", "nvmlClocksEventReasonHwSlowdown"),
             ("hw_thermal_slowdown", "nvmlClocksEventReasonHwThermalSlowdown"),
             ("sw_thermal_slowdown", "nvmlClocksEventReasonSwThermalSlowdown"),
             ("sw_power_cap", "nvmlClocksEventReasonSwPowerCap"),
             ("hw_power_brake", "nvmlClocksEventReasonHwPowerBrakeSlowdown"))

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.thread = None
        self.samples = []
        self.reasons = set()
        self.smax = None
        self.stop_flag = False
        self.nv = None

    def start(self):
        import threading
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.index)
            self.smax = float(nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM))
            self.nv = nv

            def run():
                while not self.stop_flag:
                    self.samples.append(float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)))
                    r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                    for nm, attr in self.NAMES:
                        if r & getattr(nv, attr):
                            self.reasons.add(nm)
                    time.sleep(0.002)

            self.thread = threading.Thread(target=run, daemon=True)
            self.thread.start()
            while not self.samples:  # the first sample precedes the timed region
                time.sleep(0.001)
            return
        except Exception:  # noqa: BLE001 - NVML missing: nvidia-smi fallback
            self.nv = None
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index),
                 "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
                 "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
                 "clocks_event_reasons.sw_power_cap",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            time.sleep(0.5)
        except OSError:
            self.proc = None

    def stop(self) -> dict:
        if self.thread is not None:
            self.stop_flag = True
            self.thread.join()
            return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                    "sm_max_mhz": self.smax, "reasons": sorted(self.reasons),
                    "samples": len(self.samples), "sampler": "nvml"}
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["clock sampling unavailable"]}
        self.proc.terminate()
        try:
            out, _ = self.proc.communicate(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
            out, _ = self.proc.communicate()
        sm, smax, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                smax = float(f[1])
            except ValueError:
                continue
            for nm, val in zip(names, f[2:6]):
                if val.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": smax,
                "reasons": sorted(reasons), "samples": len(sm), "sampler": "nvidia-smi"}


def load_traffic(workload: str, reorder: str):
    """dram bytes per expand launch from the newest committed ncu capture of
    this workload (profiles/r<NN>_expand_traffic*.json, written by
    tools/expand_traffic.py), or None."""
    import glob
    for path in sorted(glob.glob(os.path.join(ROOT, "profiles", "r*_expand_traffic*.json")), reverse=True):
        with open(path) as f:
            t = json.load(f)
        if t.get("workload") == workload and t.get("reorder") == reorder:
            t["file"] = os.path.relpath(path, ROOT)
            return t
    return None


def load_peak():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            pk = json.load(f)
        return float(pk["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def make_graph_edges(cfg: int, scale: int | None):
    import synth
    t0 = time.time()
    n, src, dst = synth.config_edges(cfg, scale_override=scale)
    return n, src, dst, time.time() - t0


def build_graph(efg, args, *, permute=None, weighted=False, **kw):
    """The config's EFG built from its generator (efg_build_stream: the edge list
    is never materialised in this process, which keeps C4/C5 within host RAM).
    Returns (graph, generator-setup seconds)."""
    import synth
    t0 = time.time()
    sg = synth.config_stream(args.config, scale_override=args.scale, permute=permute)
    gen_s = time.time() - t0
    g = efg.Graph.build_stream(sg.n, sg.m, sg.fn, sg.user, weighted=weighted,
                               n_threads=os.cpu_count() or 1, **kw)
    return g, gen_s


def peak_rss_gb() -> float:
    """Peak resident set of this process (ru_maxrss, KiB on Linux) in GB."""
    import resource
    return resource.getrusage(resource.RUSAGE_SELF).ru_maxrss * 1024 / 1e9


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


REF_STEP_EDGES = 1 << 28  # reference-arm step: FIFO BFS stopped after this many scanned edges


def _cpu_baseline_child(cfg: int, scale, index: int, count: int, out_dir: str, core: int, permute=None,
                        go_parallel=None, timed_lock=None):
    """Spawned process (bench.py cpu_baseline leg): the oracle's CSR of the
    same seeded graph, then ONE plain single-threaded FIFO BFS from the first
    timed source, pinned to `core` (the parent keeps off that core).  Writes
    depth.npy and meta.json to out_dir."""
    import oracle
    import synth
    n, src, dst = synth.config_edges(cfg, scale_override=scale, permute=permute)
    os.sched_setaffinity(0, {core})
    t0 = time.time()
    ov, oe = oracle.csr_build(n, src, dst)
    csr_s = time.time() - t0
    del src, dst
    deg = np.diff(ov)
    s0 = int(synth.sources(n, count, seed=1000 + cfg, nonisolated_mask=deg > 0)[index])
    if timed_lock is not None:
        timed_lock.acquire()  # the parent never pauses this process inside its timed BFS
    t = time.perf_counter()
    d = oracle.bfs(ov, oe, s0)
    cs = time.perf_counter() - t
    if timed_lock is not None:
        timed_lock.release()
    np.save(os.path.join(out_dir, "depth.npy"), d)
    # a second parity source (untimed): the next timed source
    s1 = int(synth.sources(n, count, seed=1000 + cfg, nonisolated_mask=deg > 0)[min(index + 1, count - 1)])
    np.save(os.path.join(out_dir, "depth1.npy"), oracle.bfs(ov, oe, s1))
    meta = {"source": s0, "source1": s1, "bfs_s": cs, "csr_s": csr_s, "edges": int(deg[d >= 0].sum()),
            "core": core, "affinity": sorted(os.sched_getaffinity(0))}
    # the optional all-core baseline (BASELINE.md CPU plan), once the parent's
    # GPU work is over: OpenMP top-down BFS on the same CSR and source
    if go_parallel is not None and go_parallel.wait(timeout=3600):
        import cpu_baseline
        os.sched_setaffinity(0, set(range(os.cpu_count() or 1)))
        threads = len(os.sched_getaffinity(0))
        cpu_baseline.bfs(ov, oe, s0, threads)  # warm-up (page faults of the CSR in every thread)
        t = time.perf_counter()
        dp = cpu_baseline.bfs(ov, oe, s0, threads)
        meta.update(par_s=time.perf_counter() - t, par_threads=threads, par_exact=bool(np.array_equal(dp, d)))
    with open(os.path.join(out_dir, "meta.json"), "w") as f:
        json.dump(meta, f)


def start_cpu_baseline(args, count: int, index: int):
    """Start the cpu_baseline child on the last host core and move this
    process (and every thread it creates from now on) off that core."""
    import multiprocessing as mp
    import tempfile
    cores = sorted(os.sched_getaffinity(0))
    core = cores[-1]
    out_dir = tempfile.mkdtemp(prefix="efg_cpu_baseline_")
    ctx = mp.get_context("spawn")
    go = ctx.Event()
    lock = ctx.Lock()
    proc = ctx.Process(target=_cpu_baseline_child,
                       args=(args.config, args.scale, index, count, out_dir, core, args.permute or None, go, lock))
    proc.start()
    if len(cores) > 1:
        os.sched_setaffinity(0, set(cores[:-1]))
    return proc, out_dir, go, lock


def pause_cpu_baseline(job, stop: bool, was_paused: bool = True) -> bool:
    """SIGSTOP / SIGCONT the cpu_baseline child (None-safe).  Returns whether
    the child was stopped.  Only outside its timed BFS: the parent holds the
    child's timing lock while the child is stopped (if the child is inside
    its timed BFS, nothing is paused)."""
    import signal
    if job is None or not was_paused:
        return False
    proc, lock = job[0], job[3]
    if stop:
        if not proc.is_alive() or not lock.acquire(block=False):
            return False
        try:
            os.kill(proc.pid, signal.SIGSTOP)
        except OSError:
            lock.release()
            return False
        return True
    try:
        os.kill(proc.pid, signal.SIGCONT)
    except OSError:
        pass
    lock.release()
    return True


def finish_cpu_baseline(proc, out_dir: str, go, lock, g, n: int):
    go.set()  # the GPU measurements are over: the child may use every core
    proc.join()
    if proc.exitcode != 0:
        return {"unavailable": f"cpu_baseline process exited with {proc.exitcode}"}
    with open(os.path.join(out_dir, "meta.json")) as f:
        meta = json.load(f)
    dref = np.load(os.path.join(out_dir, "depth.npy"))
    ok = bool(np.array_equal(dref, g.bfs(meta["source"])))
    psrc = [meta["source"]]
    if "source1" in meta:
        ok = ok and bool(np.array_equal(np.load(os.path.join(out_dir, "depth1.npy")), g.bfs(meta["source1"])))
        psrc.append(meta["source1"])
    return {"value": meta["edges"] / meta["bfs_s"] / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"one single-threaded FIFO BFS (source {meta['source']}, {meta['edges']} edges) over "
                      f"the oracle CSR of the same graph ({meta['bfs_s']:.1f} s; CSR build "
                      f"{meta['csr_s']:.1f} s untimed), pinned to host core {meta['core']} "
                      f"(sched_setaffinity = taskset -c {meta['core']}; bench's own threads kept off it)",
            "cpu_model": cpu_model(), "host_cores": os.cpu_count(),
            "parity_bit_exact": ok, "parity_sources": psrc,
            "all_cores": ({"value": meta["edges"] / meta["par_s"] / 1e9, "unit": UNIT,
                           "cores": meta["par_threads"], "kind": "openmp top-down BFS (cpu_baseline/omp_bfs.c)",
                           "sample": "the same source and CSR, after the GPU work", "depth_equal_oracle":
                           meta["par_exact"]} if "par_s" in meta else None)}


def run_reference(args, rank, world):
    """Reference arm: the oracle (plain CPU BFS) on one host core, rank 0 only.
    Each step (warm-up and timed) is a bounded sample of one BFS: the oracle's
    FIFO BFS from that step's source, stopped once REF_STEP_EDGES adjacency
    entries were scanned (or_bfs_bounded); GTEPS = scanned edges / time."""
    if rank != 0:
        return
    import oracle
    import synth
    n, src, dst, gen_s = make_graph_edges(args.config, args.scale)
    core = sorted(os.sched_getaffinity(0))[-1]
    os.sched_setaffinity(0, {core})
    t0 = time.time()
    vlist, elist = oracle.csr_build(n, src, dst)
    csr_s = time.time() - t0
    del src, dst
    deg = np.diff(vlist)
    srcs = synth.sources(n, args.warmup + args.steps, seed=1000 + args.config,
                         nonisolated_mask=deg > 0)
    for s in srcs[:args.warmup]:
        oracle.bfs_bounded(vlist, elist, int(s), REF_STEP_EDGES)
    edges, secs, full = 0, 0.0, 0
    for s in srcs[args.warmup:]:
        t = time.perf_counter()
        d, nv, scanned = oracle.bfs_bounded(vlist, elist, int(s), REF_STEP_EDGES)
        secs += time.perf_counter() - t
        edges += scanned
        full += int(scanned < REF_STEP_EDGES)
    v = edges / secs / 1e9
    cfgname = synth.CONFIGS[args.config]["name"] + (f"_scale{args.scale}" if args.scale else "")
    sample = (f"{args.steps} single-threaded FIFO BFS over the oracle CSR, each stopped after "
              f"{REF_STEP_EDGES} scanned edges ({full} ran to completion); pinned to host core {core}")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": secs / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": cfgname, "n": int(n), "m_directed": int(vlist[-1]),
                       "sources": args.steps, "csr_build_s": round(csr_s, 2),
                       "step_edges_cap": REF_STEP_EDGES},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                             "cpu_model": cpu_model()},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def stream_degree_bounds(sg, world: int, relabel: bool, chunk: int = 1 << 27):
    """1-D partition bounds from ONE counting pass over the generator stream
    (no EFG build): per-vertex degree estimate = endpoint count of the non-loop
    samples (duplicates included), cost per vertex = 29 B + its estimated EF
    list bytes deg * (2 + log2(n / deg)) / 8 (efg_partition's model, SURVEY
    8(e)), in the relabelled order (degree descending, ties by id) when
    `relabel`.  Cut points are 64-aligned (one owner per bitmap word).
    Returns (bounds uint64[world + 1], degree estimate in input ids)."""
    n, m = sg.n, sg.m
    deg = np.zeros(n, np.int64)
    for first in range(0, m, chunk):
        src, dst = sg.range(first, min(chunk, m - first))
        keep = src != dst
        deg += np.bincount(src[keep], minlength=n)
        deg += np.bincount(dst[keep], minlength=n)
    order = np.lexsort((np.arange(n), -deg)) if relabel else np.arange(n)
    d = deg[order].astype(np.float64)
    cost = 29.0 + np.where(d > 0, d * (2.0 + np.log2(np.maximum(n / np.maximum(d, 1.0), 1.0))) / 8.0, 0.0)
    c = np.cumsum(cost)
    b = [0]
    for r in range(1, world):
        v = int(np.searchsorted(c, c[-1] * r / world))
        b.append(min(n, max(b[-1], (v + 63) // 64 * 64)))
    b.append(n)
    return np.array(b, np.uint64), deg


def run_partitioned(args, rank, world, local):
    """N ranks, one collective BFS at a time over the 1-D row partition (strong
    scaling).  Each rank builds only its rows from the generator
    (efg_build_stream); per level the library expands the rank's rows, ORs the
    new bits over peer memory and ends the level on the device (efg_bfs on a
    partitioned handle: no host round trip per level).  --xchg nccl drives the
    same levels step by step with torch.distributed collectives instead."""
    import torch
    import torch.distributed as dist
    import synth
    import paper_conf_ipps_gerak23_b200 as efg
    from paper_conf_ipps_gerak23_b200.dist import (TorchTransport, partitioned_bfs, partitioned_bfs_peer_hostseq,
                                                   peer_setup)
    if args.xchg == "peer" and world > torch.cuda.device_count():
        # ranks time-sharing a GPU must not run kernels that wait on each other
        # (B200_PROFILING.md: Xid 109): host-sequenced exchange instead
        args.xchg = "hostseq"

    dev = torch.device("cuda", local)
    stream = torch.cuda.Stream(device=dev)
    flags = efg.EFG_DEFAULT_FLAGS | (efg.EFG_REORDER_DEGREE if args.reorder == "degree" else 0)
    cdev = dev if dist.get_backend() == "nccl" else torch.device("cpu")
    sg = synth.config_stream(args.config, scale_override=args.scale, permute=args.permute or None)
    n = sg.n
    bounds = torch.zeros(world + 1, dtype=torch.int64, device=cdev)
    srcs_t = torch.zeros(args.warmup + args.steps, dtype=torch.int64, device=cdev)
    nthr = max(1, (os.cpu_count() or 1) // world)
    if rank == 0:
        # bounds from one counting pass over the generator (no whole-graph build
        # on rank 0; every rank then builds only its rows)
        if args.reorder == "degree":
            b, deg = stream_degree_bounds(sg, world, relabel=True)
            s = synth.sources(n, args.warmup + args.steps, seed=1000 + args.config, nonisolated_mask=deg > 0)
        else:
            # generator order (e.g. permuted RMAT, C5): equal vertex ranges, 64-aligned
            b = np.array([min(n, (n * r // world + 63) // 64 * 64) for r in range(world)] + [n], np.uint64)
            s = synth.sources(n, args.warmup + args.steps, seed=1000 + args.config)
        bounds.copy_(torch.from_numpy(b.astype(np.int64)))
        srcs_t.copy_(torch.from_numpy(s.astype(np.int64)))
    dist.broadcast(bounds, 0)
    dist.broadcast(srcs_t, 0)
    b = bounds.cpu().numpy().astype(np.uint64)
    srcs = srcs_t.cpu().numpy()
    t0 = time.time()
    g = efg.Graph.build_stream(n, sg.m, sg.fn, sg.user, device=local, stream=stream.cuda_stream, flags=flags,
                               rows=(int(b[rank]), int(b[rank + 1])), n_threads=nthr)
    build_s = time.time() - t0
    depth = torch.empty(n, dtype=torch.int32, device=dev)
    tr = TorchTransport(stage_on_host=dist.get_backend() != "nccl")
    mk = lambda k: torch.zeros(k, dtype=torch.int32, device=dev)  # noqa: E731
    if args.xchg == "peer":
        peer_setup(g, rank, b)  # IPC handles all-gathered once; no collective per level
        one_bfs = lambda s: g.bfs(s, depth=depth)  # noqa: E731  collective, enqueue-only
    elif args.xchg == "hostseq":
        peer_setup(g, rank, b)
        one_bfs = lambda s: partitioned_bfs_peer_hostseq(g, s, depth, dist.barrier)  # noqa: E731
    else:
        one_bfs = lambda s: partitioned_bfs(g, s, depth, b, tr, mk)  # noqa: E731
    with torch.cuda.stream(stream):
        for s in srcs[:args.warmup]:
            one_bfs(int(s))
    torch.cuda.synchronize()
    dist.barrier()
    torch.cuda.synchronize()
    clk = ClockSampler(local)
    clk.start()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    with torch.cuda.stream(stream):
        for s in srcs[args.warmup:]:
            one_bfs(int(s))
    e1.record(stream)
    torch.cuda.synchronize()
    clocks = clk.stop()
    ms = e0.elapsed_time(e1)
    # traversed edges of this rank's rows (untimed statistics pass; the
    # collective call with statistics synchronises)
    edges, launches = 0, 0
    for s in srcs[args.warmup:]:
        if args.xchg == "peer":
            _, _, st = g.bfs(int(s), depth=depth, stats=True)
        else:
            one_bfs(int(s))
            st = g.bfs_end()
        edges += st["edges_traversed"]
        launches += st["kernel_launches"]
    # e2e: the same collective calls with a pinned host depth array
    hdepth = torch.empty(n, dtype=torch.int32, pin_memory=True)
    dist.barrier()
    t1 = time.perf_counter()
    d2h = 0
    if args.xchg == "peer":
        for s in srcs[args.warmup:]:
            _, _, st_e = g.bfs(int(s), depth=hdepth, stats=True)  # includes the device->host depth copy
            d2h += st_e["d2h_bytes"]
    e2e_s = time.perf_counter() - t1
    t = torch.tensor([ms, e2e_s], dtype=torch.float64, device=cdev)
    e = torch.tensor([edges, d2h], dtype=torch.float64, device=cdev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    dist.all_reduce(e, op=dist.ReduceOp.SUM)
    value = float(e[0].item()) / (float(t[0].item()) * 1e-3) / 1e9
    if rank == 0:
        cfgname = synth.CONFIGS[args.config]["name"] + (f"_scale{args.scale}" if args.scale else "")
        gpus = torch.cuda.device_count()
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": float(t[0].item()) / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": cfgname, "n": int(n), "reorder": args.reorder, "permute": bool(args.permute),
                       "parallelism": f"1-D row partition over {world} ranks on {min(world, gpus)} GPU(s), "
                                      "per-level bitmap "
                                      + ("exchange by the library's kernels over peer memory (owner OR + "
                                         "broadcast, CUDA IPC), collective efg_bfs with the level loop on "
                                         "the device" if args.xchg == "peer" else
                                         "exchange by the library's kernels over peer memory, host-sequenced "
                                         "(a barrier per phase; functional: ranks share a GPU)"
                                         if args.xchg == "hostseq" else
                                         "exchange (all_to_all + OR + all_gather, torch.distributed)"),
                       "ranks_per_gpu": world / max(1, min(world, gpus)),
                       "xchg": args.xchg, "bounds": [int(x) for x in b],
                       "build_s_rank0": round(build_s, 2),
                       "l2_policy": "inputs larger than L2"},
            "clocks": clocks, "gpu_launches": launches,
            "gpu_launches_note": "rank 0's kernels (every rank launches the same number per level)",
            "e2e": ({"value": float(e[0].item()) / float(t[1].item()) / 1e9, "unit": UNIT,
                     "h2d_bytes_per_step": 4 * world,
                     "d2h_bytes_per_step": int(float(e[1].item()) / max(1, args.steps)),
                     "d2h_note": "summed over ranks: every rank receives the full depth array in a pinned "
                                 "host buffer (4-bit codes when the BFS has < 15 levels)"}
                    if args.xchg == "peer" else None),
            "roofline": None,
            "roofline_note": "N > 1: the expand roofline is reported on the N = 1 line (same kernel, a "
                             "1/N row range per rank)",
            "cpu_baseline": None,
            "cpu_baseline_note": "rank 0 at N = 1 only (contract)",
        }
        print(json.dumps(line), flush=True)
    g.free()
    dist.destroy_process_group()


def main():
    args = parse()
    rank, world, local = dist_env()
    if world > 1:
        # torchrun sets OMP_NUM_THREADS=1; the library's host-side OpenMP work
        # (depth widening of the e2e call) gets this rank's share of the cores
        os.environ["OMP_NUM_THREADS"] = str(max(1, (os.cpu_count() or 1) // world))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    # the oracle baseline runs in a spawned process on its own core while this
    # process builds and measures (started before any thread pool exists here)
    cpu_job = None
    # (C4's oracle CSR alone needs ~130 GB of host memory next to this process's
    # build: its parity runs in tests/verify_full.py instead)
    if rank == 0 and world == 1 and not args.no_cpu_baseline and args.config != 4:
        cpu_job = start_cpu_baseline(args, args.warmup + args.steps, args.warmup)

    import torch
    import synth
    import paper_conf_ipps_gerak23_b200 as efg

    if world > 1:
        import torch.distributed as dist
        backend = os.environ.get("EFG_DIST_BACKEND", "nccl")  # gloo: functional runs on 1 GPU
        local = local % torch.cuda.device_count()
        torch.cuda.set_device(local)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
        if args.mode == "partition":
            return run_partitioned(args, rank, world, local)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    stream = torch.cuda.Stream(device=dev)

    flags = efg.EFG_DEFAULT_FLAGS | (efg.EFG_REORDER_DEGREE if args.reorder == "degree" else 0)
    if args.host_resident:
        flags |= efg.EFG_HOST_RESIDENT
    g, gen_s = build_graph(efg, args, device=local, stream=stream.cuda_stream, flags=flags,
                           permute=args.permute or None)
    n = g.n
    info = g.info
    vlist, nlb, offsets, _ = g.export()
    perm = g.perm()  # stored id -> input id
    deg = np.empty(n, np.int64)
    deg[perm] = np.diff(vlist).astype(np.int64)       # input-id order
    sizes = np.empty(n, np.int64)
    sizes[perm] = np.diff(offsets).astype(np.int64)   # input-id order

    nsrc = args.warmup + args.steps
    all_srcs = synth.sources(n, nsrc * world, seed=1000 + args.config, nonisolated_mask=deg > 0)
    my = all_srcs[rank::world][:nsrc]

    depth = torch.empty(n, dtype=torch.int32, device=dev)
    with torch.cuda.stream(stream):
        for s in my[:args.warmup]:
            g.bfs(int(s), depth=depth)
    torch.cuda.synchronize()

    # ---- timed region: device-resident input, device depth output ----
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    clk = ClockSampler(local)
    clk.start()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    # device depth and no statistics: efg_bfs only enqueues (stream order), so
    # the K BFS run back to back with no host round trip in between
    e0.record(stream)
    with torch.cuda.stream(stream):
        for s in my[args.warmup:]:
            g.bfs(int(s), depth=depth)
    e1.record(stream)
    torch.cuda.synchronize()
    clocks = clk.stop()
    ms = e0.elapsed_time(e1)
    # traversed edges per source (deterministic): one untimed pass with statistics
    stats = []
    with torch.cuda.stream(stream):
        for s in my[args.warmup:]:
            _, _, st = g.bfs(int(s), depth=depth, stats=True)
            stats.append((int(s), st))
    torch.cuda.synchronize()
    edges = sum(st["edges_traversed"] for _, st in stats)
    launches = sum(st["kernel_launches"] for _, st in stats)
    t_tot = torch.tensor([ms], dtype=torch.float64, device=dev)
    e_tot = torch.tensor([edges], dtype=torch.float64, device=dev)
    if world > 1:
        import torch.distributed as dist
        dist.all_reduce(t_tot, op=dist.ReduceOp.MAX)
        dist.all_reduce(e_tot, op=dist.ReduceOp.SUM)
    value = float(e_tot.item()) / (float(t_tot.item()) * 1e-3) / 1e9

    # ---- roofline of the expand+decode kernel (per-level algorithmic bytes) ----
    # Timed region 2 (same sources): host-driven level loop so that every expand
    # launch is bracketed by CUDA events on the library's stream.
    g.set_level_loop(True)
    ev_stats = []
    torch.cuda.synchronize()
    with torch.cuda.stream(stream):
        for s, _ in stats:
            _, _, st = g.bfs(s, depth=depth, stats=True)
            ev_stats.append((s, st))
    torch.cuda.synchronize()
    g.set_level_loop(False)
    alg_bytes, exp_ms, exp_launch, exp_ms_gt = 0, 0.0, 0, 0.0
    lvl_rows = []
    for (s, st), (_, stg) in zip(ev_stats, stats):
        d = g.bfs(s)  # host depth to attribute frontier bytes per level (untimed)
        for L in range(st["levels"]):
            fr = d == L
            b = int(sizes[fr].sum()) + 21 * int(fr.sum())
            alg_bytes += b
            lvl_rows.append((s, L, int(fr.sum()), int(st["level_edges"][L]), b,
                             float(st["level_expand_ms"][L]), float(stg["level_expand_ms"][L]),
                             float(st["level_end_ms"][L])))
        exp_ms += st["expand_ms"]
        exp_ms_gt += stg["expand_ms"]
        exp_launch += st["expand_launches"]
    peak, peak_src = load_peak()
    achieved = alg_bytes / (exp_ms * 1e-3) / 1e9 if exp_ms > 0 else 0.0
    if args.profile_levels and rank == 0:
        for r in lvl_rows:
            print("level src=%d L=%d |F|=%d E=%d bytes=%d expand_ms(ev)=%.4f (gt)=%.4f end_ms=%.4f GB/s=%.1f" %
                  (*r, r[4] / max(r[5], 1e-9) / 1e6), file=sys.stderr)

    # ---- e2e: through the C ABI with a pinned host depth buffer ----
    hdepth = torch.empty(n, dtype=torch.int32, pin_memory=True)
    e2e_edges = 0
    # the cpu_baseline child (building its CSR on another core) is paused while
    # the host side of the e2e call is timed: the host memory bandwidth the
    # depth widening needs is not shared with our own background job
    paused = pause_cpu_baseline(cpu_job, True)
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    t0 = time.perf_counter()
    d2h_bytes = []
    for s, st in stats:
        _, _, st_e = g.bfs(s, depth=hdepth, stats=True)  # includes the device->host copy of depth
        e2e_edges += st["edges_traversed"]
        d2h_bytes.append(st_e["d2h_bytes"])
    e2e_s = time.perf_counter() - t0
    e2e_t = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
    e2e_e = torch.tensor([e2e_edges], dtype=torch.float64, device=dev)
    if world > 1:
        import torch.distributed as dist
        dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
        dist.all_reduce(e2e_e, op=dist.ReduceOp.SUM)
    e2e_val = float(e2e_e.item()) / float(e2e_t.item()) / 1e9

    pause_cpu_baseline(cpu_job, False, paused)

    # ---- the same measurement without the degree relabelling (transparency) ----
    alt = None
    if world == 1 and args.reorder == "degree" and args.do_alt:
        g2, _ = build_graph(efg, args, device=local, stream=stream.cuda_stream, permute=args.permute or None)
        with torch.cuda.stream(stream):
            for s in my[:args.warmup]:
                g2.bfs(int(s), depth=depth)
        torch.cuda.synchronize()
        a0 = torch.cuda.Event(enable_timing=True)
        a1 = torch.cuda.Event(enable_timing=True)
        e_alt = sum(st["edges_traversed"] for _, st in stats)  # same graph and sources, other labels
        a0.record(stream)
        with torch.cuda.stream(stream):
            for s in my[args.warmup:]:
                g2.bfs(int(s), depth=depth)
        a1.record(stream)
        torch.cuda.synchronize()
        alt = {"reorder": "none", "value": e_alt / (a0.elapsed_time(a1) * 1e-3) / 1e9, "unit": UNIT,
               "ef_data_bytes_per_edge": g2.info["data_bytes"] / g2.info["m"]}
        g2.free()

    # ---- the same BFS without the visited-prefix skip (EFG_OPT_PREFIX_SKIP = 0):
    # every element decoded and probed, as in the paper's expansion ----
    alt_ns = None
    if world == 1:
        g.set_prefix_skip(False)
        with torch.cuda.stream(stream):
            for s in my[:args.warmup]:
                g.bfs(int(s), depth=depth)
        torch.cuda.synchronize()
        a0 = torch.cuda.Event(enable_timing=True)
        a1 = torch.cuda.Event(enable_timing=True)
        e_ns = sum(st["edges_traversed"] for _, st in stats)  # same graph, same sources
        a0.record(stream)
        with torch.cuda.stream(stream):
            for s, _ in stats:
                g.bfs(s, depth=depth)
        a1.record(stream)
        torch.cuda.synchronize()
        g.set_prefix_skip(True)
        alt_ns = {"prefix_skip": False, "value": e_ns / (a0.elapsed_time(a1) * 1e-3) / 1e9, "unit": UNIT}

    # ---- PageRank over the same EFG (BASELINE configs[1] "BFS and PageRank"):
    # 50 push iterations, fp64 accumulation (reading C21) ----
    pr = None
    if world == 1 and args.do_pagerank:
        rank_d = torch.empty(n, dtype=torch.float64, device=dev)
        with torch.cuda.stream(stream):
            g.pagerank(0.85, 50, rank=rank_d)  # warm-up (builds the all-vertex plan once)
        torch.cuda.synchronize()
        p0 = torch.cuda.Event(enable_timing=True)
        p1 = torch.cuda.Event(enable_timing=True)
        p0.record(stream)
        with torch.cuda.stream(stream):
            g.pagerank(0.85, 50, rank=rank_d)
        p1.record(stream)
        torch.cuda.synchronize()
        pms = p0.elapsed_time(p1)
        rs = float(rank_d.sum().item())
        pr = {"iters": 50, "damping": 0.85, "ms": pms, "ms_per_iter": pms / 50,
              "gteps": 50 * int(info["m"]) / (pms * 1e-3) / 1e9, "unit": "GTEPS (edges pushed / s)",
              "rank_sum": rs, "accumulate": "fp64; symmetric graph: each vertex gathers r(u)/deg(u) over its own list (one atomicAdd per list run; push with an atomic per edge, P:185, for directed graphs)"}

    # ---- SSSP (NEXT-1; BASELINE configs[3] "BFS and SSSP with synthetic
    # weights"): frontier Bellman-Ford over the EFG, fp32 weights (reading C20) ----
    sssp = None
    if world == 1 and args.do_sssp:
        # weighted build in the generator's order (no relabelling: the weighted
        # builder keeps 8-byte adjacency entries; C4's generator order is its
        # locality order, the paper's "with reordering" arm)
        g3, _ = build_graph(efg, args, device=local, stream=stream.cuda_stream, weighted=True,
                            permute=args.permute or None)
        dist_d = torch.empty(n, dtype=torch.float32, device=dev)
        with torch.cuda.stream(stream):
            g3.sssp(int(my[0]), dist=dist_d)  # warm-up
        torch.cuda.synchronize()
        q0 = torch.cuda.Event(enable_timing=True)
        q1 = torch.cuda.Event(enable_timing=True)
        relaxed, iters, nsrc = 0, 0, min(3, len(stats))
        q0.record(stream)
        with torch.cuda.stream(stream):
            for s, _ in stats[:nsrc]:
                _, sst = g3.sssp(s, dist=dist_d, stats=True)
                relaxed += sst["edges_relaxed"]
                iters += sst["iterations"]
        q1.record(stream)
        torch.cuda.synchronize()
        qms = q0.elapsed_time(q1)
        sssp = {"sources": nsrc, "ms_per_source": qms / nsrc, "iterations_per_source": iters / nsrc,
                "edges_relaxed_per_source": relaxed / nsrc,
                "gteps_reached_edges": nsrc * float(np.mean([st["edges_traversed"] for _, st in stats[:nsrc]]))
                / (qms * 1e-3) / 1e9,
                "relax_gteps": relaxed / (qms * 1e-3) / 1e9,
                "note": "frontier Bellman-Ford, fp32 __fadd_rn + int-punned atomicMin; bit-exact vs fp32 "
                        "Dijkstra in tests"}
        g3.free()

    # ---- cpu baseline: the oracle on a bounded sample (rank 0, N=1 only) ----
    cpu = None
    if cpu_job is not None:
        cpu = finish_cpu_baseline(*cpu_job, g, n)
        if "parity_sources" in cpu and cpu["parity_sources"][0] != stats[0][0]:
            cpu["parity_note"] = "source differs from the first timed source"

    if rank == 0:
        cfgname = synth.CONFIGS[args.config]["name"] + (f"_scale{args.scale}" if args.scale else "")
        trf = load_traffic(cfgname, args.reorder)
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": float(t_tot.item()) / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": cfgname, "n": int(n), "m_directed": int(info["m"]),
                       "reorder": args.reorder,
                       "sources_per_rank": args.steps, "fwd_quantum": int(info["fwd_quantum"]),
                       "efg_bytes_per_edge": (info["data_bytes"] + 17 * n) / info["m"],
                       "ef_data_bytes_per_edge": info["data_bytes"] / info["m"],
                       "csr32_over_efg": (4 * info["m"] + 4 * (n + 1)) / (info["data_bytes"] + 17 * n),
                       "l2_policy": "inputs larger than L2 (EF data %.2f GB > 126 MB)" % (info["data_bytes"] / 1e9),
                       "parallelism": f"{world} independent BFS replicas" if world > 1 else "1 GPU",
                       "data_location": "host (pinned, mapped: out-of-core)" if info["data_location"] else "HBM",
                       "build_s": round(info["build_seconds"], 2), "gen_s": round(gen_s, 2),
                       "host_peak_rss_gb": round(peak_rss_gb(), 2)},
            "clocks": clocks,
            "gpu_launches": launches,
            "roofline": {"bound": "hbm", "kernel": "expand_kernel (a4+a5+a6)",
                         "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak,
                         "traffic": (trf or {}).get("dram_bytes_per_launch"),
                         "traffic_source": ((trf or {}).get("source") or "") + (
                             f" ({trf['file']})" if trf else ""),
                         # ncu-measured DRAM bandwidth of the heaviest expand launch
                         # (dram__bytes_read+write / gpu__time_duration, cold cache)
                         "dram_heavy_launch": (trf or {}).get("heavy"),
                         "frac_dram_heavy_launch": ((trf or {}).get("heavy") or {}).get("gbps", 0) / peak
                         if trf and trf.get("heavy") else None,
                         "alg_bytes_per_launch": alg_bytes / max(exp_launch, 1),
                         "peak_source": peak_src,
                         "expand_launches": exp_launch, "expand_ms_total": exp_ms,
                         "expand_ms_total_graph_mode_globaltimer": exp_ms_gt,
                         "expand_share_of_step": exp_ms_gt / ms if ms else None,
                         "timing": "CUDA events around each expand launch (host-driven level "
                                   "loop, same sources, on the library stream)"},
            "e2e": {"value": e2e_val, "unit": UNIT, "h2d_bytes_per_step": 4,
                    "d2h_bytes_per_step": int(np.mean(d2h_bytes)) if d2h_bytes else None,
                    "d2h_note": "depth array into a pinned host buffer; 4 bits per vertex "
                                "over PCIe when the BFS has < 15 levels (1 byte when every "
                                "depth < 127), widened to int32 on the host inside the call"},
            "cpu_baseline": cpu,
            "alt_no_reorder": alt,
            "alt_no_prefix_skip": alt_ns,
            "pagerank": pr,
            "sssp": sssp,
        }
        print(json.dumps(line), flush=True)
    g.free()
    if world > 1:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
