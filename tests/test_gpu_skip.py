"""GPU parity of the opt-in clean-shard skipping (include/cusha.h
skip_clean_shards).  Skipping a shard none
of whose windows changed since its last pass is exact, so every algorithm must
meet the same bar as the full passes: bit-exact integer results, R10 for PR,
the contraction tolerance (R16) for NN/HS/CS — on both representations, in
both loop modes and with the partitioned mode.  edges_processed must count
the edges actually streamed (fewer than iterations x |E| on a high-diameter
mesh in natural vertex order, where shards outside the wave sit idle)."""
import numpy as np
import pytest

import graphgen
import oracle
from paper_conf_hpdc_khorasanivgb14_b200 import cusha
from gpu_common import EPS, cs_inputs, float_tol, gpu_run, hs_inputs, nn_inputs, pr_check

pytestmark = pytest.mark.gpu

REPRS = ["gs", "cw"]


@pytest.fixture(scope="module")
def c1():
    wl = graphgen.workload("C1")
    return wl.V, wl.src, wl.dst, wl.edge_u32


class _Mesh:
    """A mesh in its natural (row-major) vertex order: shards are bands of
    rows, so the SSSP wave touches few of them per pass.  (The C3 recipe
    permutes vertex ids, which puts wave-front vertices in every shard.)"""

    def __init__(self, V, width, pairs, seed):
        self.V = V
        self.src, self.dst = graphgen.mesh(V, width, pairs, seed=seed, permute=False)
        self.E = len(self.src)
        self.edge_u32 = graphgen.edge_u32(self.src, self.dst, seed=seed, lo=1, hi=255, symmetric=True)
        # natural order: vertex 0 is a corner that may have lost its bonds; start
        # from the grid centre (the C3 recipe maps the centre to id 0 instead)
        self.source = V // 2 + width // 2


@pytest.fixture(scope="module")
def mesh():
    return _Mesh(40000, 200, 52000, 33)


@pytest.mark.parametrize("repr", REPRS)
@pytest.mark.parametrize("host_loop", [False, True])
def test_skip_integer_algorithms_bit_exact(c1, repr, host_loop):
    V, s, d, w = c1
    for alg, want, ev in (("bfs", oracle.bfs(V, s, d, 0), None), ("sssp", oracle.sssp(V, s, d, w, 0), w),
                          ("sswp", oracle.sswp(V, s, d, w, 0), w), ("cc", oracle.cc(V, s, d), None)):
        got, st = gpu_run(alg, V, s, d, ev=ev, repr=repr, N=128, skip=True, host_loop=host_loop)
        np.testing.assert_array_equal(got, want, err_msg=alg)
        assert 0 < st["edges_processed"] <= st["iterations"] * len(s)


@pytest.mark.parametrize("repr", REPRS)
def test_skip_mesh_sssp_saves_work(mesh, repr):
    wl = mesh
    want = oracle.sssp(wl.V, wl.src, wl.dst, wl.edge_u32, wl.source)
    assert (want != cusha.INF).sum() > wl.V // 2                       # a non-trivial wave
    full, st_full = gpu_run("sssp", wl.V, wl.src, wl.dst, ev=wl.edge_u32, repr=repr, N=500, source=wl.source)
    got, st = gpu_run("sssp", wl.V, wl.src, wl.dst, ev=wl.edge_u32, repr=repr, N=500, skip=True, source=wl.source)
    np.testing.assert_array_equal(full, want)
    np.testing.assert_array_equal(got, want)
    assert st_full["edges_processed"] == st_full["iterations"] * wl.E   # the paper's full passes
    # the diagonal SSSP wave spans many row bands, so only part of each pass is skipped
    assert st["edges_processed"] < 0.9 * st["iterations"] * wl.E


def test_skip_pagerank(c1):
    V = 20000
    s, d = graphgen.rmat(V, 200000, seed=24)
    x_star, _ = oracle.pagerank(V, s, d, tol=1e-9)
    for repr in REPRS:
        got, st = gpu_run("pr", V, s, d, repr=repr, N=500, skip=True)
        pr_check(got, x_star)
        assert st["converged"] == 1


@pytest.mark.parametrize("repr", REPRS)
def test_skip_nn_hs_cs(repr):
    V = 4096
    s, d, w, x0 = nn_inputs()
    _, n1 = oracle.nn(V, s, d, w, x0, tol=EPS)
    x_star, n2 = oracle.nn(V, s, d, w, x0, tol=1e-9)
    got, _ = gpu_run("nn", V, s, d, ev=w, repr=repr, N=256, init=x0, skip=True)
    np.testing.assert_allclose(got, x_star, rtol=0, atol=float_tol(n1, n2) * np.maximum(1, np.abs(x_star)).max())

    s, d, c, q0 = hs_inputs()
    _, n1 = oracle.hs(V, s, d, c, q0, tol=EPS)
    q_star, n2 = oracle.hs(V, s, d, c, q0, tol=1e-9)
    got, _ = gpu_run("hs", V, s, d, ev=c, repr=repr, N=256, init=np.stack([q0, q0], 1), skip=True)
    np.testing.assert_allclose(got[:, 0], q_star, rtol=0, atol=float_tol(n1, n2) + 4e-6 * 100)

    s, d, G, v0, a0 = cs_inputs()
    _, n1 = oracle.cs(V, s, d, G, v0, a0, tol=EPS)
    v_star, n2 = oracle.cs(V, s, d, G, v0, a0, tol=1e-9)
    got, _ = gpu_run("cs", V, s, d, ev=G, repr=repr, N=256, init=np.stack([v0, a0], 1), skip=True)
    np.testing.assert_allclose(got[:, 0], v_star, rtol=0, atol=float_tol(n1, n2))


@pytest.mark.parametrize("G", [2, 4])
def test_skip_partitioned(mesh, G):
    wl = mesh
    want = oracle.sssp(wl.V, wl.src, wl.dst, wl.edge_u32, wl.source)
    got, st = gpu_run("sssp", wl.V, wl.src, wl.dst, ev=wl.edge_u32, repr="cw", N=500, skip=True, world_size=G,
                      source=wl.source)
    np.testing.assert_array_equal(got, want)
    assert st["edges_processed"] < st["iterations"] * wl.E
    V = 20000
    s, d = graphgen.rmat(V, 200000, seed=61)
    got, _ = gpu_run("bfs", V, s, d, repr="cw", N=300, skip=True, world_size=G)
    np.testing.assert_array_equal(got, oracle.bfs(V, s, d, 0))
