"""Pins for the floating-point oracle functions (PR, NN, HS, CS) — CPU only.

Pins are computations other than the oracle's Jacobi sweep: dense linear
solves (numpy.linalg.solve) of the fixed-point equations, networkx.pagerank
(library) on dangling-free graphs, scalar root finding (scipy brentq) on
graphs whose fixed point collapses to one equation, closed forms on cycles,
complete graphs and stars, and the PageRank mass identity of DESIGN.md R6.
"""
import networkx as nx
import numpy as np
import pytest
from scipy.optimize import brentq

import graphgen
import oracle
from helpers import random_simple_graph

D = 0.85


def dense_pr(V, s, d, damping=D):
    """x* = (1-d) (I - d M)^-1 1 with M[v,u] = (#edges u->v) / outdeg(u)."""
    out = np.bincount(s, minlength=V).astype(np.float64)
    M = np.zeros((V, V))
    np.add.at(M, (d, s), 1.0 / out[s])
    return np.linalg.solve(np.eye(V) - damping * M, np.full(V, 1.0 - damping))


def test_pr_dense_solve_random():
    rng = np.random.default_rng(7)
    for V, E in [(10, 30), (60, 400), (300, 2500)]:
        s, d = random_simple_graph(rng, V, E) if V <= 60 else graphgen.uniform(V, E, seed=V)
        x, it = oracle.pagerank(V, s, d, tol=1e-13)
        np.testing.assert_allclose(x, dense_pr(V, s, d), rtol=0, atol=1e-10)


def test_pr_dense_solve_rmat_with_duplicates():
    rng = np.random.default_rng(8)
    s, d = random_simple_graph(rng, 40, 300, allow_dups=True)   # R22: duplicates count in NbrsNum
    x, _ = oracle.pagerank(40, s, d, tol=1e-13)
    np.testing.assert_allclose(x, dense_pr(40, s, d), atol=1e-10)


def test_pr_vs_networkx_dangling_free():
    # symmetric graph: no dangling vertices once isolated ones are excluded
    V = 2000
    s, d = graphgen.rmat(V, 8000, seed=21, symmetric=True)
    deg = np.bincount(s, minlength=V)
    keep = np.nonzero(deg > 0)[0]
    remap = -np.ones(V, np.int64)
    remap[keep] = np.arange(len(keep))
    s2, d2 = remap[s].astype(np.uint32), remap[d].astype(np.uint32)
    n = len(keep)
    x, _ = oracle.pagerank(n, s2, d2, tol=1e-13)
    G = nx.DiGraph()
    G.add_nodes_from(range(n))
    G.add_edges_from(zip(s2.tolist(), d2.tolist()))
    p = nx.pagerank(G, alpha=D, tol=1e-14, max_iter=10000)
    ref = np.array([p[i] for i in range(n)]) * n
    np.testing.assert_allclose(x, ref, atol=1e-8)
    assert abs(x.sum() / n - 1.0) < 1e-6          # north_star mass invariant (dangling-free form)


def test_pr_mass_identity_rmat():
    """R6: sum x* = |V| - d/(1-d) * sum_{outdeg=0} x*_u (exact for the paper's formula)."""
    V = 4096
    s, d = graphgen.rmat(V, 32768, seed=22)
    x, _ = oracle.pagerank(V, s, d, tol=1e-12)
    dangling = np.bincount(s, minlength=V) == 0
    assert dangling.any()
    assert abs(x.sum() - (V - D / (1 - D) * x[dangling].sum())) / V < 1e-9
    assert (x >= 1 - D - 1e-12).all()


def test_pr_closed_forms():
    n = 17
    cyc_s = np.arange(n, dtype=np.uint32)
    cyc_d = (cyc_s + 1) % n
    x, _ = oracle.pagerank(n, cyc_s, cyc_d, tol=1e-13)
    np.testing.assert_allclose(x, 1.0, atol=1e-11)
    ks = np.array([u for u in range(n) for v in range(n) if u != v], np.uint32)
    kd = np.array([v for u in range(n) for v in range(n) if u != v], np.uint32)
    x, _ = oracle.pagerank(n, ks, kd, tol=1e-13)
    np.testing.assert_allclose(x, 1.0, atol=1e-11)
    # in-star: leaves -> 0; leaves have no in-edges so x_leaf = 1-d
    s = np.arange(1, n, dtype=np.uint32)
    d = np.zeros(n - 1, np.uint32)
    x, it = oracle.pagerank(n, s, d, tol=1e-13)
    np.testing.assert_allclose(x[1:], 1 - D, atol=1e-12)
    np.testing.assert_allclose(x[0], (1 - D) + D * (n - 1) * (1 - D), atol=1e-12)


def test_pr_not_converged_flag():
    s, d = graphgen.rmat(256, 2048, seed=3)
    with pytest.raises(RuntimeError):
        oracle.pagerank(256, s, d, tol=1e-12, max_iters=3)


# ------------------------------------------------------------------- NN
def test_nn_contractive_goes_to_zero():
    """R12: with |sum of in-weights| < 1 the only fixed point is x = 0."""
    V = 4096
    s, d = graphgen.rmat(V, 32768, seed=31)
    indeg = np.bincount(d, minlength=V).astype(np.float32)
    w = graphgen.edge_f32(s, d, seed=31, lo=-1.0, hi=1.0) * 0.9 / indeg[d]
    x0 = graphgen.vertex_f32(V, seed=31, stream=0, lo=-1.0, hi=1.0)
    x, _ = oracle.nn(V, s, d, w, x0, tol=1e-12)
    assert np.abs(x).max() < 1e-11


def test_nn_complete_graph_scalar_root():
    n, gain = 9, 2.0
    ks = np.array([u for u in range(n) for v in range(n) if u != v], np.uint32)
    kd = np.array([v for u in range(n) for v in range(n) if u != v], np.uint32)
    w = np.full(len(ks), gain / (n - 1), np.float32)
    x0 = np.linspace(0.2, 0.9, n).astype(np.float32)
    x, _ = oracle.nn(n, ks, kd, w, x0, tol=1e-14)
    root = brentq(lambda t: np.tanh(np.float64(np.float32(gain / (n - 1))) * (n - 1) * t) - t, 0.1, 1.0, xtol=1e-15)
    np.testing.assert_allclose(x, root, atol=1e-12)


def test_nn_weighted_cycle_scalar_root():
    """Directed cycle i -> i+1 with distinct weights: x_{i+1} = tanh(w_i x_i);
    the fixed point solves one scalar equation (catches a weight/edge mix-up)."""
    n = 5
    s = np.arange(n, dtype=np.uint32)
    d = (s + 1) % n
    w = np.array([1.7, 2.3, 1.4, 3.1, 1.9], np.float32)
    x0 = np.full(n, 0.8, np.float32)
    x, _ = oracle.nn(n, s, d, w, x0, tol=1e-14)
    wd = w.astype(np.float64)

    def around(t):
        for i in range(n):
            t = np.tanh(wd[i] * t)
        return t

    x_at0 = brentq(lambda t: around(t) - t, 0.05, 1.0, xtol=1e-15)
    want = [x_at0]
    for i in range(n - 1):
        want.append(np.tanh(wd[i] * want[-1]))
    np.testing.assert_allclose(x, want, atol=1e-12)


# ------------------------------------------------------------------- HS
def dagify(V, s, d, seed):
    """Keep u->v only if rank(u) < rank(v) for a seeded random rank: a DAG, so
    the only source SCCs are in-degree-0 vertices (R14 boundary)."""
    rank = graphgen.permute_vertices(V, seed, 0, np.arange(V, dtype=np.uint32))
    keep = rank[s] < rank[d]
    return s[keep], d[keep]


def test_hs_dense_harmonic_solve():
    V = 300
    s, d = graphgen.uniform(V, 2400, seed=41)
    s, d = dagify(V, s, d, 41)
    indeg = np.bincount(d, minlength=V).astype(np.float32)
    c = (np.float32(0.5) / indeg[d]).astype(np.float32)
    q0 = graphgen.vertex_f32(V, seed=41, stream=0, lo=0.0, hi=100.0)
    q, _ = oracle.hs(V, s, d, c, q0, tol=1e-13)
    # fixed point: for indeg>0, sum_e c_e (Q_u - Q_v) = 0 ; boundary keeps Q0
    A = np.zeros((V, V))
    b = np.zeros(V)
    for v in range(V):
        if indeg[v] == 0:
            A[v, v] = 1.0
            b[v] = q0[v]
    np.add.at(A, (d, s), c.astype(np.float64))
    np.add.at(A, (d, d), -c.astype(np.float64))
    want = np.linalg.solve(A, b)
    np.testing.assert_allclose(q, want, atol=1e-9)


def test_hs_two_vertex_closed_form():
    # 0 -> 1 with coefficient c: Q1 -> Q0 (boundary), Q0 fixed
    q, _ = oracle.hs(2, np.array([0], np.uint32), np.array([1], np.uint32), np.array([0.25], np.float32),
                     np.array([10.0, 50.0], np.float32), tol=1e-13)
    np.testing.assert_allclose(q, [10.0, 10.0], atol=1e-11)


# ------------------------------------------------------------------- CS
def test_cs_dense_dirichlet_solve():
    V = 400
    s, d = graphgen.rmat(V, 1500, seed=51, symmetric=True)
    G = graphgen.edge_f32(s, d, seed=51, lo=0.1, hi=1.0, symmetric=True)
    anchor = graphgen.vertex_f32(V, seed=51, stream=1, lo=0.0, hi=1.0) < 0.05
    anchor[0] = True
    v0 = np.where(anchor, (graphgen.vertex_f32(V, seed=51, stream=2, lo=0, hi=1) < 0.5).astype(np.float32), 0).astype(np.float32)
    a0 = anchor.astype(np.float32)
    v, _ = oracle.cs(V, s, d, G, v0, a0, tol=1e-14, max_iters=10**6)
    indeg = np.bincount(d, minlength=V)
    A = np.zeros((V, V))
    b = np.zeros(V)
    fixed = anchor | (indeg == 0)
    A[fixed, fixed] = 1.0
    b[fixed] = v0[fixed]
    free = ~fixed
    g = G.astype(np.float64)
    m = free[d]
    np.add.at(A, (d[m], s[m]), g[m])
    np.add.at(A, (d[m], d[m]), -g[m])
    # components with no anchor are singular for the dense solve: they stay at 0
    # under the iteration from V = 0 (R15); pin them separately
    import scipy.sparse as sp
    from scipy.sparse import csgraph
    _, comp = csgraph.connected_components(sp.csr_matrix((np.ones(len(s)), (s, d)), shape=(V, V)), directed=False)
    has_anchor = np.zeros(comp.max() + 1, bool)
    has_anchor[comp[anchor]] = True
    floating = ~has_anchor[comp]
    A[floating] = 0.0
    A[floating, floating] = 1.0
    b[floating] = 0.0
    want = np.linalg.solve(A, b)
    np.testing.assert_allclose(v, want, atol=1e-9)
    np.testing.assert_array_equal(v[anchor], v0[anchor])


def test_cs_divider_closed_form():
    # anchors 0 (V=0) and 2 (V=1), middle vertex 1; conductances g01, g21 into 1
    s = np.array([0, 1, 2, 1], np.uint32)
    d = np.array([1, 0, 1, 2], np.uint32)
    G = np.array([0.3, 0.3, 0.7, 0.7], np.float32)
    v, _ = oracle.cs(3, s, d, G, np.array([0, 0, 1], np.float32), np.array([1, 0, 1], np.float32), tol=1e-14)
    np.testing.assert_allclose(v, [0.0, np.float32(0.7) / (np.float64(np.float32(0.3)) + np.float32(0.7)), 1.0], atol=1e-12)


def test_pr_residual_vs_dense_and_fixed_point():
    """or_pagerank_residual: x - ((1-d) + d M x) equals the dense formula for
    any x, and vanishes (to float32 rounding) at the oracle's fixed point."""
    rng = np.random.default_rng(71)
    V = 200
    s, d = random_simple_graph(rng, V, 1500)
    x = rng.uniform(0.1, 3.0, V).astype(np.float32)
    out = np.bincount(s, minlength=V).astype(np.float64)
    M = np.zeros((V, V))
    np.add.at(M, (d, s), 1.0 / out[s])
    want = x.astype(np.float64) - ((1 - D) + D * (M @ x.astype(np.float64)))
    np.testing.assert_allclose(oracle.pagerank_residual(V, s, d, x), want, atol=1e-12)
    xs, _ = oracle.pagerank(V, s, d, tol=1e-13)
    assert np.abs(oracle.pagerank_residual(V, s, d, xs.astype(np.float32))).max() < 1e-5


def test_c5_golden_sample_is_consistent():
    """The committed C5 PageRank sample (tools/golden_c5_pr.py: oracle.pagerank to
    1e-9 on graphgen C5) is internally consistent: the config's sizes, a sorted
    sample that contains the 16 first vertices, every x* >= 1 - d (R6: x = (1-d)
    + d * a non-negative sum), and the mass below |V| (R6: sum x* = |V| minus the
    dangling leak).  With the git-ignored full vector (float32) present, the
    sample equals its entries."""
    import os
    z = np.load(os.path.join(os.path.dirname(__file__), "golden", "c5_pr_sample.npz"))
    V = int(z["V"])
    assert V == 1 << 26 and int(z["E"]) == 1 << 30 and float(z["tol"]) == 1e-9
    idx = z["idx"].astype(np.int64)
    assert (np.diff(idx) > 0).all() and idx[0] == 0 and (idx[:16] == np.arange(16)).all() and idx[-1] < V
    assert (z["xstar"] >= 0.15 - 1e-12).all()
    assert 0 < float(z["mass"]) < V
    full = os.path.join(os.path.dirname(__file__), "golden_cache", "c5_pr_xstar.f32")
    if os.path.exists(full):
        xs = np.fromfile(full, np.float32)
        np.testing.assert_array_equal(xs[idx], z["xstar"].astype(np.float32))
