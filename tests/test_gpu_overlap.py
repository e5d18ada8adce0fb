"""Overlapped passes (row a5) against the
oracle and against the one-launch-per-pass barrier mode (Fig. 5).

Default runs draw shard tickets across pass boundaries inside one launch
(at most W passes in flight, W = 2, or 4 on graphs of average degree < 4; a
shard's passes in order); convergence is concluded when W consecutive passes
committed nothing (L189; the argument is in csrc/kernels.cu).  The
integer fixed points are unique, so both modes must match the oracle bit for
bit; PR stays within R10.  Small |S| (down to one shard) exercises the
per-shard pass order, where a CTA's next ticket is the shard it is still
processing.
"""
import numpy as np
import pytest

import graphgen
import oracle
from gpu_common import gpu_run, pr_check
from paper_conf_hpdc_khorasanivgb14_b200 import cusha

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def c1():
    wl = graphgen.workload("C1")
    return wl.V, wl.src, wl.dst, wl.edge_u32


@pytest.mark.parametrize("barrier", [False, True])
@pytest.mark.parametrize("repr", ["gs", "cw"])
@pytest.mark.parametrize("alg", ["bfs", "sssp", "sswp", "cc"])
def test_integer_both_modes(c1, alg, repr, barrier):
    V, s, d, w = c1
    want = {"bfs": lambda: oracle.bfs(V, s, d, 0), "sssp": lambda: oracle.sssp(V, s, d, w, 0),
            "sswp": lambda: oracle.sswp(V, s, d, w, 0), "cc": lambda: oracle.cc(V, s, d)}[alg]()
    got, st = gpu_run(alg, V, s, d, ev=w if alg in ("sssp", "sswp") else None, repr=repr, N=128,
                      pass_barrier=barrier)
    np.testing.assert_array_equal(got, want)
    assert st["converged"] == 1
    assert st["device_loop"] == (1 if barrier else 2)


@pytest.mark.parametrize("N", [4096, 2048, 1366, 64, 7])
def test_small_shard_counts(c1, N):
    """|S| = 1, 2, 3 (fewer shards than CTAs: tickets of consecutive passes hit
    the same shard), and many tiny shards."""
    V, s, d, w = c1
    want = oracle.sssp(V, s, d, w, 0)
    for repr in ("gs", "cw"):
        got, st = gpu_run("sssp", V, s, d, ev=w, repr=repr, N=N)
        np.testing.assert_array_equal(got, want)
        assert st["converged"] == 1


def test_mesh_many_passes():
    """A high-diameter mesh: hundreds of overlapped passes, then a confirming one."""
    wl = graphgen.workload("mesh:60000:120:80000:41")
    want = oracle.sssp(wl.V, wl.src, wl.dst, wl.edge_u32, 0)
    for barrier in (False, True):
        got, st = gpu_run("sssp", wl.V, wl.src, wl.dst, ev=wl.edge_u32, repr="cw", N=512, pass_barrier=barrier)
        np.testing.assert_array_equal(got, want)
        assert st["iterations"] > 50


@pytest.mark.parametrize("barrier", [False, True])
def test_pagerank_both_modes(barrier):
    V = 1 << 15
    s, d = graphgen.rmat(V, 1 << 19, seed=31)
    x_star, _ = oracle.pagerank(V, s, d, tol=1e-9)
    for repr in ("gs", "cw"):
        got, st = gpu_run("pr", V, s, d, repr=repr, pass_barrier=barrier)
        pr_check(got, x_star)
        assert st["converged"] == 1


def test_max_iters_stops_exactly(c1):
    """max_iters = k: NOT_CONVERGED after exactly k passes in both modes (R23)."""
    from paper_conf_hpdc_khorasanivgb14_b200 import cusha
    wl = graphgen.workload("mesh:20000:100:26000:43")
    for barrier in (False, True):
        for k in (1, 3, 10):
            with cusha.build_graph(wl.V, wl.src, wl.dst, edge_values=wl.edge_u32, repr="cw", vertices_per_shard=256,
                                   pass_barrier=barrier) as g:
                rc = cusha.run("sssp", g, source=0, max_iters=k)
                st = cusha.get_stats(g)
                assert rc == cusha.NOT_CONVERGED and st["iterations"] == k and st["converged"] == 0
                vals = cusha.get_values(g)
                # committed values are upper bounds of the exact distances, source exact
                exact = oracle.sssp(wl.V, wl.src, wl.dst, wl.edge_u32, 0)
                assert vals[0] == 0 and np.all(vals >= exact)


def test_trace_cap_fallback(c1):
    """max_iters above the per-pass trace capacity (2^20) uses the one-launch-per-pass loop."""
    V, s, d, _ = c1
    got, st = gpu_run("bfs", V, s, d, repr="cw", N=128, max_iters=(1 << 20) + 1)
    np.testing.assert_array_equal(got, oracle.bfs(V, s, d, 0))
    assert st["device_loop"] == 1


def test_skip_clean_with_overlap():
    wl = graphgen.workload("mesh:40000:200:52000:33")
    want = oracle.sssp(wl.V, wl.src, wl.dst, wl.edge_u32, 0)
    for repr in ("gs", "cw"):
        got, st = gpu_run("sssp", wl.V, wl.src, wl.dst, ev=wl.edge_u32, repr=repr, N=400, skip=True)
        np.testing.assert_array_equal(got, want)


@pytest.mark.parametrize("mode", [0, 2])
@pytest.mark.parametrize("alg", ["bfs", "sssp"])
def test_automatic_mode_many_small_shards(alg, mode):
    """pass_barrier = 0 (automatic) picks one launch per pass when there are
    >= 16 shards per resident CTA of <= 16K entries each (include/cusha.h);
    2 forces overlapped passes.  Both reach the oracle's fixed point."""
    V = 400_000
    s, d = graphgen.rmat(V, 2_000_000, seed=91)
    w = graphgen.edge_u32(s, d, seed=91, lo=1, hi=255)
    want = oracle.bfs(V, s, d, 0) if alg == "bfs" else oracle.sssp(V, s, d, w, 0)
    got, st = gpu_run(alg, V, s, d, ev=w if alg == "sssp" else None, repr="cw", N=64, pass_barrier=mode)
    np.testing.assert_array_equal(got, want)
    assert st["num_shards"] == 6250
    assert st["device_loop"] == (1 if mode == 0 else 2)


@pytest.mark.parametrize("repr", ["gs", "cw"])
def test_pass_barrier_graph_reuse(c1, repr):
    """pass_barrier = 1: the instantiated CUDA graph (one per algorithm) is
    reused across runs on one handle, with changing sources and algorithms
    interleaved; every run must still reach the oracle's fixed point (L189)."""
    from paper_conf_hpdc_khorasanivgb14_b200 import cusha
    V, s, d, w = c1
    with cusha.build_graph(V, s, d, edge_values=w, repr=repr, vertices_per_shard=128, pass_barrier=1) as g:
        for source in (0, 17, V - 1, 0):
            for alg in ("bfs", "sssp", "cc", "sswp"):
                rc = cusha.run(alg, g, source=source)
                assert rc == cusha.OK
                got = cusha.get_values(g)
                if alg == "bfs":
                    want = oracle.bfs(V, s, d, source)
                elif alg == "sssp":
                    want = oracle.sssp(V, s, d, w, source)
                elif alg == "sswp":
                    want = oracle.sswp(V, s, d, w, source)
                else:
                    want = oracle.cc(V, s, d)
                np.testing.assert_array_equal(got, want, err_msg=f"{alg} source {source}")
                assert cusha.get_stats(g)["device_loop"] == 1


def test_wide_window_on_low_degree_graph():
    """A mesh (average degree < 4) runs with 4 passes in flight: bit-exact, and
    the run ends with 4 consecutive clean passes (the last trace records)."""
    wl = graphgen.workload("mesh:40000:200:52000:33")
    got, st = gpu_run("sssp", wl.V, wl.src, wl.dst, ev=wl.edge_u32, repr="cw")
    np.testing.assert_array_equal(got, oracle.sssp(wl.V, wl.src, wl.dst, wl.edge_u32, 0))
    assert st["device_loop"] == 2
    with cusha.build_graph(wl.V, wl.src, wl.dst, edge_values=wl.edge_u32, repr="cw") as g:
        cusha.run("sssp", g)
        upd, _ = cusha.get_trace(g)
    assert len(upd) >= 5 and (upd[-4:] == 0).all() and upd[-5] > 0
