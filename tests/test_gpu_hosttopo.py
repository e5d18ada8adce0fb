"""GPU parity of the host-streamed topology mode (row f3, include/cusha.h
device_topology_budget): shards past the HBM budget
keep their per-entry arrays in pinned host memory and the shard pass streams
them over the host link.  The layout must be identical to the all-HBM build
(bit-exact, every array), results must meet the usual parity bars, for both
representations, with the split anywhere (all on the host, half, none)."""
import numpy as np
import pytest

import graphgen
import oracle
from gpu_common import pr_check
from paper_conf_hpdc_khorasanivgb14_b200 import cusha

pytestmark = pytest.mark.gpu

REPRS = ["gs", "cw"]
PARTS = {"gs": ["shard_offsets", "shard_sizes", "src_index", "dest_local", "edge_id", "windows"],
         "cw": ["shard_offsets", "shard_sizes", "dest_local", "edge_id", "windows", "cw_offsets", "cw_sizes",
                "cw_src_local", "mapper"]}


@pytest.fixture(scope="module")
def rm():
    V = 20000
    s, d = graphgen.rmat(V, 200000, seed=71)
    w = graphgen.edge_u32(s, d, seed=71, lo=1, hi=255)
    return V, s, d, w


def _layout(g, repr):
    return {k: cusha.get_layout(g, k) for k in PARTS[repr]}


@pytest.mark.parametrize("repr", REPRS)
@pytest.mark.parametrize("budget_frac", [1e-9, 0.5])
def test_host_topology_layout_and_results(rm, repr, budget_frac):
    V, s, d, w = rm
    with cusha.build_graph(V, s, d, edge_values=w, repr=repr, vertices_per_shard=500, keep_layout=True) as g0:
        want_layout = _layout(g0, repr)
        st0 = cusha.get_stats(g0)
    # topology bytes per entry of the all-HBM build, to place the split
    budget = max(1, int(budget_frac * st0["entries_padded"] * (14 if repr == "gs" else 16)))
    with cusha.build_graph(V, s, d, edge_values=w, repr=repr, vertices_per_shard=500,
                           device_topology_budget=budget, keep_layout=True) as g:
        st = cusha.get_stats(g)
        assert st["host_bytes"] > 0 and st["host_shard"] < st["num_shards"]
        if budget_frac < 1e-6:
            assert st["host_shard"] == 0
        else:
            assert 0 < st["host_shard"]
        assert st["device_bytes"] < st0["device_bytes"]
        got_layout = _layout(g, repr)
        for k in want_layout:
            np.testing.assert_array_equal(got_layout[k], want_layout[k], err_msg=k)
        for alg, want, ev in (("bfs", oracle.bfs(V, s, d, 0), None), ("sssp", oracle.sssp(V, s, d, w, 0), w),
                              ("cc", oracle.cc(V, s, d), None)):
            assert cusha.run(alg, g) == cusha.OK
            np.testing.assert_array_equal(cusha.get_values(g), want, err_msg=alg)
        x_star, _ = oracle.pagerank(V, s, d, tol=1e-9)
        assert cusha.run("pr", g) == cusha.OK
        pr_check(cusha.get_values(g), x_star)


def test_host_topology_zero_budget_is_all_hbm(rm):
    V, s, d, w = rm
    with cusha.build_graph(V, s, d, repr="cw", vertices_per_shard=500, device_topology_budget=0) as g:
        st = cusha.get_stats(g)
        assert st["host_bytes"] == 0 and st["host_shard"] == st["num_shards"]


def test_host_topology_partitioned(rm):
    """Row f3 with the destination-range partition: every partition keeps its
    per-entry topology in pinned host memory (budget 1 byte per partition) and
    only SrcValue / VertexValues in HBM; the stage-4 stores still reach the
    sibling partitions.  Results stay bit-exact."""
    V, s, d, w = rm
    with cusha.build_graph(V, s, d, edge_values=w, repr="cw", vertices_per_shard=500, world_size=4,
                           device_topology_budget=1) as g:
        st = cusha.get_stats(g)
        assert st["partitions"] == 4 and st["host_bytes"] > 0
        for q in range(4):
            assert cusha.get_part_stats(g, q)["device_bytes"] < 16 * V
        assert cusha.run("sssp", g) == cusha.OK
        np.testing.assert_array_equal(cusha.get_values(g), oracle.sssp(V, s, d, w, 0))
        assert cusha.run("bfs", g) == cusha.OK
        np.testing.assert_array_equal(cusha.get_values(g), oracle.bfs(V, s, d, 0))


def test_host_topology_mesh_many_passes():
    wl = graphgen.workload("mesh:40000:200:52000:33")
    with cusha.build_graph(wl.V, wl.src, wl.dst, edge_values=wl.edge_u32, repr="gs",
                           device_topology_budget=1) as g:
        assert cusha.run("sssp", g) == cusha.OK
        np.testing.assert_array_equal(cusha.get_values(g), oracle.sssp(wl.V, wl.src, wl.dst, wl.edge_u32, 0))
        assert cusha.get_stats(g)["iterations"] > 50
