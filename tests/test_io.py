"""On-disk EFG (efg_save / efg_load, include/efg.h): a saved graph loads back
equal — the P:113 arrays, the relabelling, the statistics — and the oracle
still decodes it (the arrays are checked against the oracle's own encoder, not
against the handle that wrote them).  Malformed files fail with EFG_EIO.  The
GPU tests traverse a loaded graph against the oracle's BFS / SSSP."""
import os

import numpy as np
import pytest

import oracle
import synth


@pytest.fixture(scope="module")
def efg():
    import paper_conf_ipps_gerak23_b200 as m
    return m


def _same_info(a, b):
    for k in ("n", "m", "m_input", "fwd_quantum", "data_bytes", "fwd_bytes", "lower_bytes", "upper_bytes",
              "apriori_bits", "row_lo", "row_hi"):
        assert a[k] == b[k], k


def test_save_load_roundtrip_host(efg, tmp_path):
    n, src, dst = synth.rmat(12, 8, seed=7)
    w = synth.weights(src, dst, seed=2007)
    for flags, k, rows in ((efg.EFG_DEFAULT_FLAGS, 512, None),
                           (efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE, 64, None),
                           (efg.EFG_DEFAULT_FLAGS, 8, (1024, 2048))):
        g = efg.Graph.build(n, src, dst, k=k, flags=flags, device=-1, weights=w, rows=rows)
        path = str(tmp_path / f"g_{flags}_{k}.efg")
        g.save(path)
        h = efg.Graph.load(path, device=-1)
        _same_info(g.info, h.info)
        for x, y in zip(g.export(), h.export()):
            assert np.array_equal(x, y)
        assert np.array_equal(g.perm(), h.perm())
        if rows is None and not flags & efg.EFG_REORDER_DEGREE:
            # independent check: the oracle's encoder gives the same bytes for every list
            vl, nlb, of, data = h.export()
            ov, oe = oracle.csr_build(n, src, dst)
            oof, onlb, odata = oracle.efg_encode(ov, oe, k)
            assert np.array_equal(vl, ov) and np.array_equal(nlb, onlb)
            assert np.array_equal(of, oof) and np.array_equal(data, odata)
        g.free()
        h.free()


def test_load_errors(efg, tmp_path):
    n, src, dst = synth.rmat(10, 8, seed=3)
    g = efg.Graph.build(n, src, dst, device=-1)
    good = str(tmp_path / "good.efg")
    g.save(good)
    g.free()
    with pytest.raises(efg.EFGError, match="EFG_EIO"):
        efg.Graph.load(str(tmp_path / "missing.efg"), device=-1)
    bad = str(tmp_path / "bad.efg")
    with open(bad, "wb") as f:
        f.write(b"NOTANEFG" + bytes(200))
    with pytest.raises(efg.EFGError, match="EFG_EIO"):
        efg.Graph.load(bad, device=-1)
    blob = open(good, "rb").read()
    trunc = str(tmp_path / "trunc.efg")
    with open(trunc, "wb") as f:
        f.write(blob[: len(blob) - 100])
    with pytest.raises(efg.EFGError, match="EFG_EIO"):
        efg.Graph.load(trunc, device=-1)
    h = efg.Graph.build(n, src, dst, device=-1)
    with pytest.raises(efg.EFGError, match="EFG_EIO"):
        h.save(str(tmp_path / "no_such_dir" / "x.efg"))
    h.free()


@pytest.mark.gpu
def test_loaded_graph_traverses(efg, tmp_path, cuda_ok):
    n, src, dst = synth.rmat(14, 16, seed=9)
    w_in = synth.weights(src, dst, seed=2009)
    ov, oe = oracle.csr_build(n, src, dst)
    u = np.repeat(np.arange(n, dtype=np.uint32), np.diff(ov).astype(np.int64))
    w_csr = synth.weights(u, oe, seed=2009)
    g = efg.Graph.build(n, src, dst, flags=efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE, weights=w_in,
                        device=-1)
    path = str(tmp_path / "g.efg")
    g.save(path)
    g.free()
    for flags in (0, efg.EFG_HOST_RESIDENT):
        h = efg.Graph.load(path, flags=flags, device=0)
        assert h.info["data_location"] == (1 if flags else 0)
        for s in (0, 5, 4321):
            assert np.array_equal(h.bfs(s), oracle.bfs(ov, oe, s))
        d = h.sssp(5)
        assert np.array_equal(d.view(np.uint32), oracle.sssp(ov, oe, w_csr, 5).view(np.uint32))
        h.free()
