"""NN, HS and CS at a size where the shard pass takes the paths a full-size
run takes (VERDICT r1 "Parity coverage gaps"): more than 1 M edges, so a pass
streams more than twice the L2 and the producer prefetches stage-2 tiles into
L2 ahead of the ring; CW_i lists longer than one stage-4 tile; both
representations.  Compared with the oracle converged to 1e-9 under the
tolerance derived from the iteration's contraction (gpu_common.float_tol, R16).
The inputs are the R12-R15 recipes of the small parity tests at 2^20 vertices."""
import numpy as np
import pytest

import oracle
from gpu_common import EPS, cs_inputs, float_tol, hs_inputs, nn_inputs
from paper_conf_hpdc_khorasanivgb14_b200 import cusha

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
V = 1 << 20


def run(alg, s, d, ev, init, repr, N=0):
    with cusha.build_graph(V, s, d, edge_values=ev, repr=repr, vertices_per_shard=N) as g:
        cusha.set_vertex_values(g, alg, init)
        assert cusha.run(alg, g) == cusha.OK
        st = cusha.get_stats(g)
        cw = cusha.get_layout(g, "cw_sizes")
        return cusha.get_values(g), st, cw


def paths_taken(st, cw, repr):
    assert st["l2_read_ahead"] == 1                  # the pass streams from HBM
    assert st["num_edges"] > 1_000_000
    if repr == "cw":
        assert cw.max() > 5120                       # a CW_i spans several stage-4 tiles


@pytest.fixture(scope="module")
def nn_case():
    s, d, w, x0 = nn_inputs(V, 24 << 20, seed=6)
    _, n1 = oracle.nn(V, s, d, w, x0, tol=EPS)
    x_star, n2 = oracle.nn(V, s, d, w, x0, tol=1e-9)
    return s, d, w, x0, x_star, float_tol(n1, n2)


# |N| = 0: the L310 rule; a large |N| puts one CTA on an SM, where the ring takes a 4th slot
CASES = [("gs", 0), ("cw", 0), ("cw", "big")]
BIG_N = {"nn": 16000, "hs": 10000, "cs": 8000}


@pytest.mark.parametrize("repr,N", CASES)
def test_nn_at_size(nn_case, repr, N):
    s, d, w, x0, x_star, tol = nn_case
    got, st, cw = run("nn", s, d, w.view(np.uint32), x0, repr, BIG_N["nn"] if N else 0)
    paths_taken(st, cw, repr)
    assert st["ring_slots"] >= (4 if N else 3)
    np.testing.assert_allclose(got, x_star, rtol=0, atol=tol * max(1.0, np.abs(x_star).max()))


@pytest.fixture(scope="module")
def hs_case():
    s, d, c, q0 = hs_inputs(V, 48 << 20, seed=7)
    _, n1 = oracle.hs(V, s, d, c, q0, tol=EPS)
    q_star, n2 = oracle.hs(V, s, d, c, q0, tol=1e-9)
    return s, d, c, q0, q_star, float_tol(n1, n2) + 4e-6 * 100


@pytest.mark.parametrize("repr,N", CASES)
def test_hs_at_size(hs_case, repr, N):
    s, d, c, q0, q_star, tol = hs_case
    got, st, cw = run("hs", s, d, c.view(np.uint32), np.stack([q0, q0], 1), repr, BIG_N["hs"] if N else 0)
    paths_taken(st, cw, repr)
    assert st["ring_slots"] >= (4 if N else 3)
    np.testing.assert_allclose(got[:, 0], q_star, rtol=0, atol=tol)


@pytest.fixture(scope="module")
def cs_case():
    s, d, G, v0, a0 = cs_inputs(V, 12 << 20, seed=8)
    _, n1 = oracle.cs(V, s, d, G, v0, a0, tol=EPS)
    v_star, n2 = oracle.cs(V, s, d, G, v0, a0, tol=1e-9)
    return s, d, G, v0, a0, v_star, float_tol(n1, n2)


@pytest.mark.parametrize("repr,N", CASES)
def test_cs_at_size(cs_case, repr, N):
    s, d, G, v0, a0, v_star, tol = cs_case
    got, st, cw = run("cs", s, d, G.view(np.uint32), np.stack([v0, a0], 1), repr, BIG_N["cs"] if N else 0)
    paths_taken(st, cw, repr)
    assert st["ring_slots"] >= (4 if N else 3)
    np.testing.assert_allclose(got[:, 0], v_star, rtol=0, atol=tol)
    anc = a0 != 0
    np.testing.assert_array_equal(got[anc, 0], v0[anc])
