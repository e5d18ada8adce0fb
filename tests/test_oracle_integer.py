"""Pins for the integer oracle functions (BFS, SSSP, SSWP, CC) — CPU only.

Each oracle function is checked against something other than itself:
brute-force enumeration of simple paths / reachability on tiny graphs,
scipy's csgraph routines (library), closed forms on path / star / cycle
graphs, and the invariants of DESIGN.md "Pins" (triangle inequality and
tightness on every edge, north_star).
"""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse import csgraph

import graphgen
import oracle
from helpers import INF, random_simple_graph, reach_matrix, simple_paths


def tiny_graphs(n=40, seed=0):
    rng = np.random.default_rng(seed)
    for _ in range(n):
        V = int(rng.integers(2, 8))
        E = int(rng.integers(0, V * (V - 1) + 1))
        s, d = random_simple_graph(rng, V, E)
        w = rng.integers(1, 20, len(s)).astype(np.uint32)
        yield V, s, d, w, int(rng.integers(0, V))


# ----------------------------------------------------------------- BFS
def test_bfs_bruteforce_paths():
    for V, s, d, _, src in tiny_graphs():
        want = np.full(V, INF, np.uint32)
        for v, path in simple_paths(V, s, d, src):
            want[v] = min(int(want[v]), len(path))
        np.testing.assert_array_equal(oracle.bfs(V, s, d, src), want)


def test_bfs_closed_forms():
    n = 50
    s = np.arange(n - 1, dtype=np.uint32)
    d = s + 1
    np.testing.assert_array_equal(oracle.bfs(n, s, d, 0), np.arange(n))
    # direction matters: from the far end nothing is reachable
    lv = oracle.bfs(n, s, d, n - 1)
    assert lv[n - 1] == 0 and (lv[:-1] == INF).all()
    # star out of 0
    s = np.zeros(n - 1, np.uint32)
    d = np.arange(1, n, dtype=np.uint32)
    lv = oracle.bfs(n, s, d, 0)
    assert lv[0] == 0 and (lv[1:] == 1).all()
    # no edges
    lv = oracle.bfs(5, np.zeros(0, np.uint32), np.zeros(0, np.uint32), 3)
    assert lv[3] == 0 and (np.delete(lv, 3) == INF).all()


def test_bfs_vs_scipy_unweighted_rmat():
    V = 4096
    s, d = graphgen.rmat(V, 32768, seed=11)
    lv = oracle.bfs(V, s, d, 0)
    A = sp.csr_matrix((np.ones(len(s)), (s, d)), shape=(V, V))
    ref = csgraph.shortest_path(A, method="D", unweighted=True, directed=True, indices=0)
    reach = np.isfinite(ref)
    assert ((lv != INF) == reach).all()
    np.testing.assert_array_equal(lv[reach], ref[reach].astype(np.int64))


def test_bfs_rejects_bad_source():
    with pytest.raises(RuntimeError):
        oracle.bfs(4, np.array([0], np.uint32), np.array([1], np.uint32), 4)


# ----------------------------------------------------------------- SSSP
def test_sssp_bruteforce_paths():
    for V, s, d, w, src in tiny_graphs(seed=1):
        want = np.full(V, INF, np.uint64)
        for v, path in simple_paths(V, s, d, src):
            want[v] = min(int(want[v]), int(w[path].sum()) if path else 0)
        np.testing.assert_array_equal(oracle.sssp(V, s, d, w, src), want.astype(np.uint32))


def test_sssp_vs_scipy_dijkstra():
    V = 4096
    s, d = graphgen.rmat(V, 32768, seed=12)     # simple graph: scipy would sum duplicates
    w = graphgen.edge_u32(s, d, seed=12, lo=1, hi=255)
    dist = oracle.sssp(V, s, d, w, 0)
    A = sp.csr_matrix((w.astype(np.float64), (s, d)), shape=(V, V))
    ref = csgraph.dijkstra(A, directed=True, indices=0)
    reach = np.isfinite(ref)
    assert ((dist != INF) == reach).all()
    np.testing.assert_array_equal(dist[reach], ref[reach].astype(np.int64))


def test_sssp_invariants_mesh():
    """north_star: triangle inequality on every edge; plus tightness."""
    V = 20000
    s, d = graphgen.mesh(V, 141, 27000, seed=5)
    w = graphgen.edge_u32(s, d, seed=5, lo=1, hi=255, symmetric=True)
    dist = oracle.sssp(V, s, d, w, 0).astype(np.int64)
    assert dist[0] == 0
    reached = dist != INF
    ok = reached[s]
    assert (dist[d[ok]] <= dist[s[ok]] + w[ok]).all()                 # triangle inequality
    tight = np.zeros(V, bool)
    tight[d[ok][dist[d[ok]] == dist[s[ok]] + w[ok]]] = True
    assert tight[reached & (np.arange(V) != 0)].all()                  # every reached v has a tight in-edge
    # reachability agrees with the oracle's BFS (different routine)
    np.testing.assert_array_equal(reached, oracle.bfs(V, s, d, 0) != INF)


# ----------------------------------------------------------------- SSWP
def test_sswp_bruteforce_paths():
    for V, s, d, w, src in tiny_graphs(seed=2):
        want = np.zeros(V, np.uint64)
        for v, path in simple_paths(V, s, d, src):
            width = int(w[path].min()) if path else INF
            want[v] = max(int(want[v]), width)
        np.testing.assert_array_equal(oracle.sswp(V, s, d, w, src), want.astype(np.uint32))


def test_sswp_invariants_rmat():
    V = 4096
    s, d = graphgen.rmat(V, 32768, seed=13)
    w = graphgen.edge_u32(s, d, seed=13, lo=1, hi=255)
    bw = oracle.sswp(V, s, d, w, 0).astype(np.int64)
    assert bw[0] == INF
    assert (bw[d] >= np.minimum(bw[s], w)).all()                       # no edge can widen further
    tight = np.zeros(V, bool)
    tight[d[bw[d] == np.minimum(bw[s], w)]] = True
    assert tight[(bw > 0) & (np.arange(V) != 0)].all()
    # unreachable <=> 0
    lv = oracle.bfs(V, s, d, 0)
    np.testing.assert_array_equal(bw == 0, lv == INF)


# ------------------------------------------------------------------- CC
def test_cc_bruteforce_min_ancestor():
    for V, s, d, _, _ in tiny_graphs(seed=3):
        R = reach_matrix(V, s, d)                  # R[u, v]: u reaches v
        want = np.array([np.nonzero(R[:, v])[0].min() for v in range(V)], np.uint32)
        np.testing.assert_array_equal(oracle.cc(V, s, d), want)


def test_cc_vs_scipy_components_symmetric():
    V = 20000
    s, d = graphgen.rmat(V, 30000, seed=14, symmetric=True)
    lab = oracle.cc(V, s, d)
    A = sp.csr_matrix((np.ones(len(s)), (s, d)), shape=(V, V))
    n, comp = csgraph.connected_components(A, directed=False)
    minid = np.full(n, V, np.int64)
    np.minimum.at(minid, comp, np.arange(V))
    np.testing.assert_array_equal(lab, minid[comp])
    # invariants: equal labels across every edge, label <= v, idempotent
    assert (lab[s] == lab[d]).all() and (lab <= np.arange(V)).all() and (lab[lab] == lab).all()


def test_cc_closed_forms():
    # directed path 0 -> 1 -> 2 -> 3: vertex 0 reaches everything
    s = np.array([0, 1, 2], np.uint32)
    d = np.array([1, 2, 3], np.uint32)
    np.testing.assert_array_equal(oracle.cc(4, s, d), [0, 0, 0, 0])
    # reversed path 3 -> 2 -> 1 -> 0: ancestors of v are {v..3}, min is v itself
    np.testing.assert_array_equal(oracle.cc(4, d, s), [0, 1, 2, 3])
    # isolated vertices keep their own id
    np.testing.assert_array_equal(oracle.cc(3, np.zeros(0, np.uint32), np.zeros(0, np.uint32)), [0, 1, 2])
