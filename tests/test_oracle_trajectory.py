"""Pins of the oracle's mode T (oracle.c or_trajectory: Fig. 5 L193-265 pass by
pass, two-phase BSP) against what the mathematics fixes
independently of it:

- BFS under BSP commits exactly the vertices of level k in pass k, so it runs
  eccentricity + 1 passes (the last one clean), for every shard size |N|;
- SSSP / SSWP / CC under BSP are hop-limited Jacobi relaxations: the value of
  v after pass k is the best over paths of at most k edges (k-hop dynamic
  programming with numpy, a textbook Bellman-Ford round, not the oracle's
  shard-by-shard code), so per-pass update counts and the pass count follow;
- PR / NN / HS / CS with one shard (|N| = |V|): while the shard stays active
  the write-back values are the plain Jacobi iterates of the Table-3 update
  (dense numpy), so the committed values after k passes are within TOL of
  the k-th iterate;
- the fixed points of the integer algorithms equal mode X (or_bfs, or_sssp,
  or_sswp, or_cc), which are pinned in test_oracle_integer.py.
No GPU."""
import numpy as np
import pytest

import graphgen
import oracle

INF = 0xFFFFFFFF
TOL = 1e-5


def small_graph(V=300, E=2000, seed=11, symmetric=False):
    s, d = graphgen.rmat(V, E // 2 if symmetric else E, seed=seed, symmetric=symmetric)
    w = graphgen.edge_u32(s, d, seed=seed, lo=1, hi=255, symmetric=symmetric)
    return V, s.astype(np.int64), d.astype(np.int64), w.astype(np.int64)


def khop(V, s, d, w, init, relax, better, k_max=10_000):
    """values after k Jacobi rounds: x_k[v] = better(x_{k-1}[v], relax over in-edges of x_{k-1}[u])."""
    xs = [init.copy()]
    x = init.copy()
    for _ in range(k_max):
        cand = relax(x[s], w)
        nxt = x.copy()
        ok = cand >= 0
        for v, c in zip(d[ok], cand[ok]):
            nxt[v] = better(nxt[v], c)
        xs.append(nxt)
        if np.array_equal(nxt, x):
            return xs
        x = nxt
    raise AssertionError("no convergence")


@pytest.mark.parametrize("N", [1, 7, 64, 300])
def test_bfs_passes_are_levels(N):
    V, s, d, _ = small_graph()
    lvl = oracle.bfs(V, s, d, 0)
    ecc = int(lvl[lvl != INF].max())
    t = oracle.trajectory("bfs", V, s, d, N)
    assert t["converged"] and t["passes"] == ecc + 1
    np.testing.assert_array_equal(t["values"], lvl)
    want = [int((lvl == k).sum()) for k in range(1, ecc + 1)] + [0]
    np.testing.assert_array_equal(t["updated"], want)


def test_bfs_path_graph_closed_form():
    n = 50
    s = np.arange(n - 1, dtype=np.uint32)
    d = s + 1
    for N in (1, 5, n):
        t = oracle.trajectory("bfs", n, s, d, N)
        assert t["passes"] == n and (t["updated"][:-1] == 1).all() and t["updated"][-1] == 0
    t = oracle.trajectory("bfs", 10, np.zeros(0, np.uint32), np.zeros(0, np.uint32), 3)
    assert t["passes"] == 1 and t["converged"]


@pytest.mark.parametrize("N", [1, 16, 300])
def test_sssp_passes_are_bellman_ford_rounds(N):
    V, s, d, w = small_graph()
    init = np.full(V, INF, np.int64)
    init[0] = 0
    rounds = khop(V, s, d, w, init, lambda xu, ww: np.where(xu != INF, xu + ww, -1), min)
    t = oracle.trajectory("sssp", V, s, d, N, ev=w.astype(np.uint32))
    assert t["passes"] == len(rounds) - 1
    np.testing.assert_array_equal(t["values"], rounds[-1].astype(np.uint32))
    np.testing.assert_array_equal(t["values"], oracle.sssp(V, s, d, w, 0))
    want = [int((rounds[k] != rounds[k - 1]).sum()) for k in range(1, len(rounds))]
    np.testing.assert_array_equal(t["updated"], want)


@pytest.mark.parametrize("N", [1, 32])
def test_sswp_and_cc_passes(N):
    V, s, d, w = small_graph()
    init = np.zeros(V, np.int64)
    init[0] = INF
    rounds = khop(V, s, d, w, init, lambda xu, ww: np.where(xu != 0, np.minimum(xu, ww), -1), max)
    t = oracle.trajectory("sswp", V, s, d, N, ev=w.astype(np.uint32))
    assert t["passes"] == len(rounds) - 1
    np.testing.assert_array_equal(t["values"], oracle.sswp(V, s, d, w, 0))
    V, s, d, w = small_graph(symmetric=True, seed=12)
    rounds = khop(V, s, d, w, np.arange(V, dtype=np.int64), lambda xu, ww: xu, min)
    t = oracle.trajectory("cc", V, s, d, N)
    assert t["passes"] == len(rounds) - 1
    np.testing.assert_array_equal(t["values"], oracle.cc(V, s, d))
    want = [int((rounds[k] != rounds[k - 1]).sum()) for k in range(1, len(rounds))]
    np.testing.assert_array_equal(t["updated"], want)


def dense_in(V, s, d, vals):
    A = np.zeros((V, V))
    np.add.at(A, (d, s), vals)
    return A


def test_pagerank_k_passes_are_jacobi_iterates():
    V, s, d, _ = small_graph(V=200, E=1500, seed=13)
    out = np.bincount(s, minlength=V).astype(np.float64)
    M = dense_in(V, s, d, 1.0 / out[s])          # x -> A^T D^-1 x
    x = np.ones(V)
    for k in range(1, 8):
        x = 0.15 + 0.85 * (M @ x)
        t = oracle.trajectory("pr", V, s, d, V, max_passes=k)
        assert t["passes"] == k
        np.testing.assert_allclose(t["values"], x, rtol=0, atol=TOL + 1e-12)
    # run to the end: within the R10 bound of the exact fixed point
    t = oracle.trajectory("pr", V, s, d, V)
    xs = np.linalg.solve(np.eye(V) - 0.85 * M, np.full(V, 0.15))
    assert t["converged"]
    assert (np.abs(t["values"] - xs) <= 2 * TOL / 0.15 * np.maximum(1, xs)).all()


def test_nn_hs_cs_k_passes_are_jacobi_iterates():
    V, s, d, _ = small_graph(V=200, E=1500, seed=14)
    w = graphgen.edge_f32(s.astype(np.uint32), d.astype(np.uint32), seed=14, lo=-0.5, hi=0.5)
    x0 = graphgen.vertex_f32(V, seed=14, stream=0, lo=-1, hi=1)
    W = dense_in(V, s, d, w.astype(np.float64))
    x = x0.astype(np.float64)
    for k in range(1, 5):
        x = np.tanh(W @ x)
        t = oracle.trajectory("nn", V, s, d, V, ev=w, init=x0, max_passes=k)
        np.testing.assert_allclose(t["values"], x, rtol=0, atol=TOL + 1e-12)
    # HS: Q_new = Q + sum c (Q_u - Q)
    c = (np.float32(0.3) / np.maximum(np.bincount(d, minlength=V), 1)[d]).astype(np.float32)
    q0 = graphgen.vertex_f32(V, seed=14, stream=1, lo=0, hi=100)
    C = dense_in(V, s, d, c.astype(np.float64))
    q = q0.astype(np.float64)
    for k in range(1, 5):
        q = q + C @ q - C.sum(1) * q
        t = oracle.trajectory("hs", V, s, d, V, ev=c, init=q0, max_passes=k)
        np.testing.assert_allclose(t["values"], q, rtol=0, atol=TOL + 1e-9)
    # CS: anchors keep V, others take the conductance-weighted mean of their in-neighbours
    G = graphgen.edge_f32(s.astype(np.uint32), d.astype(np.uint32), seed=14, lo=0.1, hi=1.0)
    anc = np.zeros(V, bool)
    anc[::10] = True
    v0 = np.where(anc, (np.arange(V) % 20 == 0).astype(np.float32), 0).astype(np.float32)
    init = np.stack([v0, anc.astype(np.float32)], 1)
    Gm = dense_in(V, s, d, G.astype(np.float64))
    den = Gm.sum(1)
    v = v0.astype(np.float64)
    for k in range(1, 5):
        num = Gm @ v
        v = np.where(anc, v0, np.where(den > 0, num / np.where(den > 0, den, 1), 0.0))
        t = oracle.trajectory("cs", V, s, d, V, ev=G, init=init, max_passes=k)
        np.testing.assert_allclose(t["values"], v, rtol=0, atol=TOL + 1e-9)


def test_trajectory_rejects_bad_arguments():
    s = np.zeros(1, np.uint32)
    with pytest.raises(RuntimeError):
        oracle.trajectory("sssp", 4, s, s, 2)            # SSSP without EdgeValue
    with pytest.raises(RuntimeError):
        oracle.trajectory("bfs", 4, s, s, 2, source=9)   # source out of range
    with pytest.raises(RuntimeError):
        oracle.trajectory("nn", 4, s, s, 2, ev=np.zeros(1, np.float32))   # NN without x0
