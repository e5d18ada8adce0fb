"""Shared helpers for the -m gpu parity tests: seeded inputs (graphgen), the
CUDA path through the C-ABI binding, and tolerance rules."""
from __future__ import annotations

import numpy as np

import graphgen
import oracle
from paper_conf_hpdc_khorasanivgb14_b200 import cusha

EPS = 1e-5      # TOLERANCE of Table 3 (R9)
D = 0.85


def gpu_run(alg, V, src, dst, ev=None, repr="gs", N=0, source=0, init=None, max_iters=1 << 20, expect_converged=True,
            host_loop=False, skip=False, world_size=1, pass_barrier=False):
    with cusha.build_graph(V, src, dst, edge_values=ev, repr=repr, vertices_per_shard=N, host_loop=host_loop,
                           skip_clean_shards=skip, world_size=world_size, pass_barrier=pass_barrier) as g:
        if init is not None:
            cusha.set_vertex_values(g, alg, init)
        rc = cusha.run(alg, g, source=source, max_iters=max_iters)
        if expect_converged:
            assert rc == cusha.OK
        vals = cusha.get_values(g)
        st = cusha.get_stats(g)
    return vals, st


def pr_check(x_gpu, x_star):
    """R10: |g - x*| <= 1e-4 * max(1, x*) for every vertex; returns strict-abs stats."""
    err = np.abs(x_gpu.astype(np.float64) - x_star)
    bound = 1e-4 * np.maximum(1.0, x_star)
    bad = np.nonzero(err > bound)[0]
    assert bad.size == 0, f"{bad.size} vertices over the R10 bound; worst {err[bad].max()} at x*={x_star[bad[np.argmax(err[bad])]]}"
    return float(err.max()), int((err > 1e-4).sum())


def float_tol(iters_eps, iters_tight, tight=1e-9, eps=EPS):
    """Tolerance derived from the iteration's contraction (R16): the oracle's
    sweep counts to eps and to `tight` give rho ~ (tight/eps)^(1/(n2-n1));
    a run stopped at per-vertex change <= eps is within eps/(1-rho) of the
    fixed point; the GPU's asynchronous staleness can double it (R10)."""
    n = max(iters_tight - iters_eps, 1)
    rho = (tight / eps) ** (1.0 / n)
    return 2.0 * eps / max(1.0 - rho, 1e-3) + 1e-6


# ------------------------------------------------------------------ recipes
def nn_inputs(V=4096, E=32768, seed=6):
    """R12 reading: positive weights w = U(0.5,1.5) * 2 / indeg(dest) (gain ~2, so
    the fixed point is non-trivial), x0 = U(0.1, 1)."""
    s, d = graphgen.rmat(V, E, seed=seed)
    indeg = np.bincount(d, minlength=V).astype(np.float32)
    w = (graphgen.edge_f32(s, d, seed=seed, lo=0.5, hi=1.5) * np.float32(2.0) / indeg[d]).astype(np.float32)
    x0 = graphgen.vertex_f32(V, seed=seed, stream=0, lo=0.1, hi=1.0)
    return s, d, w, x0


def hs_inputs(V=4096, E=32768, seed=7):
    """R13/R14: R-MAT made acyclic by a seeded rank (only in-degree-0 vertices
    are source SCCs, so the fixed point is unique); coeff = 0.5/indeg(dest);
    Q0 = U(0, 100)."""
    s, d = graphgen.rmat(V, E, seed=seed)
    rank = graphgen.permute_vertices(V, seed, 0, np.arange(V, dtype=np.uint32))
    keep = rank[s] < rank[d]
    s, d = s[keep], d[keep]
    indeg = np.bincount(d, minlength=V).astype(np.float32)
    c = (np.float32(0.5) / indeg[d]).astype(np.float32)
    q0 = graphgen.vertex_f32(V, seed=seed, stream=0, lo=0.0, hi=100.0)
    return s, d, c, q0


def cs_inputs(V=4096, P=16384, seed=8, anchor_frac=0.2):
    """R15: symmetric R-MAT circuit, conductance G = U(0.1, 1) (symmetric),
    anchors = vertex 0 plus a seeded fraction, anchor V in {0, 1}, others 0."""
    s, d = graphgen.rmat(V, P, seed=seed, symmetric=True)
    G = graphgen.edge_f32(s, d, seed=seed, lo=0.1, hi=1.0, symmetric=True)
    anc = graphgen.vertex_f32(V, seed=seed, stream=1, lo=0.0, hi=1.0) < anchor_frac
    anc[0] = True
    v0 = np.where(anc, (graphgen.vertex_f32(V, seed=seed, stream=2, lo=0, hi=1) < 0.5), 0).astype(np.float32)
    a0 = anc.astype(np.float32)
    return s, d, G, v0, a0


def as_bits(a):
    return np.ascontiguousarray(a, np.float32).view(np.uint32)
