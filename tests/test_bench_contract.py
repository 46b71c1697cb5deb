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
