"""Seeded input generators: determinism and the shape properties of the recipe."""
import numpy as np

import graphgen


def test_rmat_exact_simple_and_deterministic():
    s1, d1 = graphgen.rmat(4096, 32768, seed=1)
    s2, d2 = graphgen.rmat(4096, 32768, seed=1)
    assert len(s1) == 32768
    assert np.array_equal(s1, s2) and np.array_equal(d1, d2)
    assert (s1 != d1).all() and s1.max() < 4096 and d1.max() < 4096
    k = s1.astype(np.uint64) << np.uint64(32) | d1
    assert len(np.unique(k)) == len(k)
    s3, _ = graphgen.rmat(4096, 32768, seed=2)
    assert not np.array_equal(s1, s3)


def test_rmat_vertex0_is_top_hub():
    s, d = graphgen.rmat(1 << 14, 1 << 17, seed=3)
    deg = np.bincount(s, minlength=1 << 14) + np.bincount(d, minlength=1 << 14)
    assert deg.argmax() == 0            # pi(0) = 0 keeps the R-MAT top hub at id 0
    # permutation spreads the other hubs: top-100 by degree are not all low ids
    top = np.argsort(-deg)[1:100]
    assert np.median(top) > 1000


def test_symmetric_rmat_both_directions():
    s, d = graphgen.rmat(5000, 20000, seed=4, symmetric=True)
    assert len(s) == 40000
    fwd = set(zip(s.tolist(), d.tolist()))
    assert all((v, u) in fwd for u, v in fwd)


def test_mesh_shape():
    V, W, P = 10000, 100, 13000
    s, d = graphgen.mesh(V, W, P, seed=5, permute=False)
    assert len(s) == 2 * P
    diff = np.abs(s.astype(np.int64) - d.astype(np.int64))
    assert set(np.unique(diff).tolist()) <= {1, W}
    deg = np.bincount(s, minlength=V)
    assert deg.max() <= 4
    sp_, dp = graphgen.mesh(V, W, P, seed=5, permute=True)
    assert len(sp_) == 2 * P


def test_permutation_is_bijection_with_anchor():
    n = 100003
    v = np.arange(n, dtype=np.uint32)
    p = graphgen.permute_vertices(n, 77, 123, v)
    assert p[123] == 0
    assert np.array_equal(np.sort(p), v)


def test_edge_values_symmetric_and_ranged():
    s, d = graphgen.rmat(3000, 9000, seed=6, symmetric=True)
    w = graphgen.edge_u32(s, d, seed=6, lo=1, hi=255, symmetric=True)
    assert w.min() >= 1 and w.max() <= 255
    m = dict(zip(zip(s.tolist(), d.tolist()), w.tolist()))
    assert all(m[(v, u)] == x for (u, v), x in m.items())
    f = graphgen.edge_f32(s, d, seed=6, lo=0.1, hi=1.0)
    assert f.min() >= 0.1 and f.max() < 1.0
