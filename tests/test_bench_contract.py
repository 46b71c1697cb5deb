"""bench.py contract (driver): the reference arm (the oracle on the host, no
GPU) prints one JSON line with the keys the driver reads.  C1 (RMAT-16) keeps
it to a few seconds."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "1",
                          "--steps", "2", "--warmup", "1"], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference"
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["steps"] == 2 and d["warmup"] == 1 and d["unit"] == "GTEPS" and d["value"] > 0
    assert d["config"]["workload"] == "rmat16_ef16"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] == 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]


def test_cpu_baseline_child_pinned_and_checked():
    """bench.py's cpu_baseline leg: a spawned process builds the oracle CSR of
    the same seeded graph, times one FIFO BFS pinned to one core, and the
    parent compares that depth with the traversal it is handed (here a stub
    returning the oracle's own answer, and one returning a wrong answer)."""
    import numpy as np
    import bench
    import oracle
    import synth

    class Args:
        config, scale, permute = 1, None, False

    n, src, dst = synth.config_edges(1)
    ov, oe = oracle.csr_build(n, src, dst)

    class Stub:
        def __init__(self, wrong):
            self.wrong = wrong

        def bfs(self, s):
            d = oracle.bfs(ov, oe, s)
            if self.wrong:
                d[np.flatnonzero(d > 0)[0]] += 1
            return d

    before = os.sched_getaffinity(0)
    try:
        for wrong in (False, True):
            job = bench.start_cpu_baseline(Args, 4, 1)
            if not wrong:  # the e2e pause: stopped outside its timed BFS, then resumed
                import time
                time.sleep(0.5)
                if bench.pause_cpu_baseline(job, True):
                    time.sleep(0.2)
                    with open(f"/proc/{job[0].pid}/stat") as f:
                        assert f.read().split(") ")[1][0] == "T"
                    assert bench.pause_cpu_baseline(job, False, True)
            cpu = bench.finish_cpu_baseline(*job, Stub(wrong), n)
            os.sched_setaffinity(0, before)
            assert cpu["kind"] == "oracle" and cpu["cores"] == 1 and cpu["value"] > 0
            assert cpu["parity_bit_exact"] is (not wrong)
            srcs = synth.sources(n, 4, seed=1001, nonisolated_mask=np.diff(ov) > 0)
            assert cpu["parity_sources"] == [int(srcs[1]), int(srcs[2])]
            assert "taskset -c" in cpu["sample"] and cpu["cpu_model"]
            assert cpu["all_cores"]["depth_equal_oracle"] and cpu["all_cores"]["value"] > 0
    finally:
        os.sched_setaffinity(0, before)


def test_stream_degree_bounds_partition():
    """N > 1 bench: rank 0's partition bounds come from one counting pass over
    the generator (no whole-graph build).  Bounds are monotone, 64-aligned,
    cover [0, n], and balance the EF bytes + 29 B per vertex of the real build
    (efg_partition's model) within 10 % per rank; the degree estimate marks
    exactly the non-isolated vertices."""
    import numpy as np
    import bench
    import synth
    import paper_conf_ipps_gerak23_b200 as efg
    sg = synth.config_stream(1)
    for world in (2, 3, 4, 8):
        b, deg = bench.stream_degree_bounds(sg, world, relabel=True, chunk=1 << 18)
        assert b[0] == 0 and b[-1] == sg.n and np.all(np.diff(b.astype(np.int64)) >= 0)
        assert np.all(b[1:-1] % 64 == 0)
        g = efg.Graph.build_stream(sg.n, sg.m, sg.fn, sg.user, device=-1,
                                   flags=efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE)
        vl, _, of, _ = g.export()
        true_deg = np.empty(sg.n, np.int64)
        true_deg[g.perm()] = np.diff(vl).astype(np.int64)
        cost = np.diff(of).astype(np.float64) + 29.0
        g.free()
        per = np.array([cost[int(b[r]):int(b[r + 1])].sum() for r in range(world)])
        assert per.max() / per.mean() < 1.10, (world, per)
        assert np.array_equal(deg > 0, true_deg > 0)
