"""Pins for the oracle's G-Shards / CW layout (or_build_shards) — CPU only.

Pinned by: the counts PAPER.md prints for its Fig. 2-4 example
(tests/golden/fig2_toy_counts.txt), Python's sorted() applied to the
definition's key (a different computation), and the representation's
invariants (Partitioned L128, Ordered L129, windows L155, CW/Mapper L175-179).
"""
import numpy as np

import graphgen
import oracle
from helpers import read_golden

# Hand-built 14-edge graph meeting every count recoverable from the paper
# (the figure images are lost; R25).
TOY_SRC = np.array([1, 7, 2, 4, 5, 6, 6, 0, 1, 3, 2, 4, 5, 7], np.uint32)
TOY_DST = np.array([2, 2, 0, 0, 1, 1, 3, 4, 5, 6, 7, 5, 6, 4], np.uint32)


def test_fig2_toy_counts():
    g = read_golden("fig2_toy_counts.txt")
    V, N = g["num_vertices"], g["vertices_per_shard"]
    r = oracle.build_shards(V, TOY_SRC, TOY_DST, N)
    assert r["S"] == g["num_shards"]
    so = r["shard_off"]
    assert so[1] - so[0] == g["shard0_size"] and so[2] - so[1] == g["shard1_size"]
    W = np.diff(r["win"], axis=0)                 # W[i, j] = |W_ij|
    assert W[0, 0] == g["W00"] and W[0, 1] == g["W01"] and W[1, 0] == g["W10"] and W[1, 1] == g["W11"]
    cw = np.diff(r["cw_off"])
    assert cw[0] == g["CW0"] and cw[1] == g["CW1"]
    # CSR view of L86: in-neighbours of vertex 2 and where they start
    order = np.lexsort((TOY_SRC, TOY_DST))
    assert sorted(TOY_SRC[TOY_DST == 2].tolist()) == g["in_neighbours_of_2"]
    assert int(np.searchsorted(TOY_DST[order], 2)) == g["csr_first_in_edge_of_2"]
    # L155: "the windows W0j are ... first two elements of shard-0 and first four elements of shard-1"
    assert (r["gs_src"][0:2] < N).all() and (r["gs_src"][7:11] < N).all()
    # L179: CW1's first five entries come from W10, the rest from W11
    m = r["mapper"]
    assert (m[6:11] < 7).all() and (m[11:14] >= 7).all()


def by_definition(V, src, dst, N):
    E = len(src)
    S = (V + N - 1) // N
    order = sorted(range(E), key=lambda e: (int(dst[e]) // N, int(src[e]), int(dst[e]), e))
    pos = {e: p for p, e in enumerate(order)}
    shard_of_pos = [int(dst[e]) // N for e in order]
    cw = sorted(range(E), key=lambda p: (int(src[order[p]]) // N, shard_of_pos[p], p))
    return order, [pos[order[p]] for p in cw], S


def test_layout_matches_sorted_definition():
    rng = np.random.default_rng(5)
    for V, E, N in [(9, 40, 2), (37, 300, 5), (64, 500, 64), (100, 900, 7), (50, 0, 3), (33, 200, 33), (40, 300, 1)]:
        src = rng.integers(0, V, E).astype(np.uint32)    # duplicates and self-loops allowed here (R22)
        dst = rng.integers(0, V, E).astype(np.uint32)
        r = oracle.build_shards(V, src, dst, N)
        order, mapper, S = by_definition(V, src, dst, N)
        assert r["S"] == S
        np.testing.assert_array_equal(r["gs_eid"], order)
        np.testing.assert_array_equal(r["mapper"], mapper)
        np.testing.assert_array_equal(r["cw_src"], r["gs_src"][np.array(mapper, np.int64)] if E else [])


def test_layout_invariants_rmat():
    V, N = 4096, 128
    src, dst = graphgen.rmat(V, 32768, seed=1)
    r = oracle.build_shards(V, src, dst, N)
    S, so, gs_src, gs_dst = r["S"], r["shard_off"].astype(np.int64), r["gs_src"], r["gs_dst"]
    assert S == 32 and so[0] == 0 and so[-1] == len(src)
    for s in range(S):
        a, b = so[s], so[s + 1]
        assert ((gs_dst[a:b] // N) == s).all()                       # Partitioned
        assert (np.diff(gs_src[a:b].astype(np.int64)) >= 0).all()    # Ordered
    win = r["win"].astype(np.int64)
    for i in range(S):
        for j in range(S):
            w = slice(win[i, j], win[i + 1, j])
            assert ((gs_src[w] // N) == i).all()                     # W_ij: sources in range i
    assert (win[0] == so[:-1]).all() and (win[S] == so[1:]).all()
    m = r["mapper"].astype(np.int64)
    assert np.array_equal(np.sort(m), np.arange(len(src)))            # Mapper is a bijection
    np.testing.assert_array_equal(r["cw_src"], gs_src[m])
    outdeg = np.bincount(src, minlength=S * N)
    np.testing.assert_array_equal(np.diff(r["cw_off"]), outdeg.reshape(S, N).sum(1))   # |CW_i| = sum outdeg


def test_window_size_model_uniform():
    """L161/L173: average window |E|/|S|^2 ~= |E||N|^2/|V|^2."""
    V, E, N = 20000, 200000, 700
    src, dst = graphgen.uniform(V, E, seed=9)
    r = oracle.build_shards(V, src, dst, N)
    S = r["S"]
    W = np.diff(r["win"].astype(np.int64), axis=0)
    assert W.sum() == E
    assert abs(W.mean() - E / S**2) < 1e-9
    assert abs(W.mean() / (E * N * N / V**2) - 1) < 0.1
