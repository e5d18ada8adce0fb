"""The GPU's two-phase BSP mode (include/cusha.h cusha_build_opts.mode) against
the oracle's mode T (oracle.trajectory: Fig. 5 literally, pass by pass).

Integer algorithms: the pass count, the committed updates per pass and the
updating shards per pass are equal EXACTLY, in both representations and at
several shard sizes; the final values equal mode X (bit-exact).  This catches
a stage bug that only delays convergence, which the fixed-point comparisons
of test_gpu_parity.py cannot see.  Float algorithms: the committed values
after k passes agree within TOL plus float32 rounding (a vertex whose change
sits at the threshold may commit on one side only, which moves its committed
value by at most TOL; the write-back value is the same either way)."""
import numpy as np
import pytest

import graphgen
import oracle
from gpu_common import as_bits, cs_inputs, hs_inputs, nn_inputs
from paper_conf_hpdc_khorasanivgb14_b200 import cusha

pytestmark = pytest.mark.gpu
TOL = 1e-5


def bsp_run(alg, V, s, d, N, repr, ev=None, init=None, max_iters=1 << 20, source=0):
    with cusha.build_graph(V, s, d, edge_values=ev, repr=repr, vertices_per_shard=N, mode="bsp") as g:
        if init is not None:
            cusha.set_vertex_values(g, alg, init)
        rc = cusha.run(alg, g, source=source, max_iters=max_iters)
        vals = cusha.get_values(g)
        st = cusha.get_stats(g)
        upd, act = cusha.get_trace(g)
    return rc, vals, st, upd, act


GRAPHS = {
    "c1": lambda: graphgen.workload("C1"),
    "mesh": lambda: graphgen.workload("mesh:40000:200:52000:33"),
    "rmat": lambda: graphgen.workload("rmat:20000:200000:61"),
}


@pytest.mark.parametrize("gname", sorted(GRAPHS))
@pytest.mark.parametrize("repr", ["gs", "cw"])
@pytest.mark.parametrize("alg", ["bfs", "sssp", "sswp", "cc"])
def test_bsp_integer_trajectory_matches_mode_t(gname, repr, alg):
    wl = GRAPHS[gname]()
    ev = wl.edge_u32 if alg in ("sssp", "sswp") else None
    for N in (128, 1000):
        if N >= wl.V:
            continue
        rc, got, st, upd, act = bsp_run(alg, wl.V, wl.src, wl.dst, N, repr, ev=ev)
        t = oracle.trajectory(alg, wl.V, wl.src, wl.dst, N, ev=ev)
        assert rc == cusha.OK and t["converged"]
        assert st["iterations"] == t["passes"], (N, st["iterations"], t["passes"])
        np.testing.assert_array_equal(upd, t["updated"])
        np.testing.assert_array_equal(act, t["active_shards"])
        np.testing.assert_array_equal(got, t["values"])
        assert st["device_loop"] == 0


def test_bsp_max_iters_prefix():
    wl = graphgen.workload("mesh:40000:200:52000:33")
    t = oracle.trajectory("sssp", wl.V, wl.src, wl.dst, 500, ev=wl.edge_u32, max_passes=37)
    rc, got, st, upd, _ = bsp_run("sssp", wl.V, wl.src, wl.dst, 500, "cw", ev=wl.edge_u32, max_iters=37)
    assert rc == cusha.NOT_CONVERGED and st["iterations"] == 37 == t["passes"]
    np.testing.assert_array_equal(got, t["values"])        # the state after exactly 37 BSP passes
    np.testing.assert_array_equal(upd, t["updated"])


def close(got, want, extra=0.0):
    err = np.abs(got.astype(np.float64) - want)
    bound = TOL + 4e-6 * np.maximum(1.0, np.abs(want)) + extra
    bad = err > bound
    assert not bad.any(), f"{bad.sum()} vertices off; worst {err.max()}"


@pytest.mark.parametrize("repr", ["gs", "cw"])
def test_bsp_float_k_pass_states(repr):
    wl = graphgen.workload("rmat:20000:200000:61")
    V, s, d = wl.V, wl.src, wl.dst
    for k in (1, 2, 3, 5):
        _, got, st, _, _ = bsp_run("pr", V, s, d, 2000, repr, max_iters=k)
        t = oracle.trajectory("pr", V, s, d, 2000, max_passes=k)
        assert st["iterations"] == k
        close(got, t["values"])
    s2, d2, w, x0 = nn_inputs()
    for k in (1, 3):
        _, got, _, _, _ = bsp_run("nn", 4096, s2, d2, 512, repr, ev=as_bits(w), init=x0, max_iters=k)
        close(got, oracle.trajectory("nn", 4096, s2, d2, 512, ev=w, init=x0, max_passes=k)["values"])
    s3, d3, c, q0 = hs_inputs()
    for k in (1, 3):
        _, got, _, _, _ = bsp_run("hs", 4096, s3, d3, 512, repr, ev=as_bits(c), init=np.stack([q0, q0], 1),
                                  max_iters=k)
        close(got[:, 0], oracle.trajectory("hs", 4096, s3, d3, 512, ev=c, init=q0, max_passes=k)["values"],
              extra=1e-5 * 100)
    s4, d4, G, v0, a0 = cs_inputs()
    init = np.stack([v0, a0], 1).astype(np.float32)
    for k in (1, 3):
        _, got, _, _, _ = bsp_run("cs", 4096, s4, d4, 512, repr, ev=as_bits(G), init=init, max_iters=k)
        close(got[:, 0], oracle.trajectory("cs", 4096, s4, d4, 512, ev=G, init=init, max_passes=k)["values"])


def test_bsp_mode_argument_checks():
    wl = graphgen.workload("C1")
    with pytest.raises(cusha.CushaError) as e:
        cusha.build_graph(wl.V, wl.src, wl.dst, repr="cw", vertices_per_shard=128, mode="bsp", world_size=2)
    assert e.value.code == cusha.EUNSUPPORTED
    with pytest.raises(cusha.CushaError) as e:
        cusha.build_graph(wl.V, wl.src, wl.dst, repr="cw", vertices_per_shard=128, mode=7)
    assert e.value.code == cusha.EINVAL
