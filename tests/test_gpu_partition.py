"""GPU parity of the destination-range partitioned mode (row e) on one device:
world_size = G partitions simulated in one process (the same pass, exchange
payload and refresh kernels as the NCCL mode; only the transport differs).
Integer algorithms stay bit-exact for every G; PR stays within R10."""
import numpy as np
import pytest

import graphgen
import oracle
from gpu_common import pr_check
from paper_conf_hpdc_khorasanivgb14_b200 import cusha

pytestmark = pytest.mark.gpu

GS = [2, 3, 4, 8]


def run_part(alg, V, s, d, G, ev=None, N=0, source=0, max_iters=1 << 20):
    with cusha.build_graph(V, s, d, edge_values=ev, repr="cw", vertices_per_shard=N, world_size=G) as g:
        rc = cusha.run(alg, g, source=source, max_iters=max_iters)
        vals = cusha.get_values(g)
        st = cusha.get_stats(g)
        bounds = cusha.get_partition(g)
    return rc, vals, st, bounds


@pytest.fixture(scope="module")
def rm():
    V = 20000
    s, d = graphgen.rmat(V, 200000, seed=61)
    w = graphgen.edge_u32(s, d, seed=61, lo=1, hi=255)
    return V, s, d, w


@pytest.mark.parametrize("G", GS)
def test_partition_bfs_sssp_sswp_bit_exact(rm, G):
    V, s, d, w = rm
    rc, got, st, b = run_part("bfs", V, s, d, G, N=300)
    assert rc == cusha.OK and len(b) == G + 1 and b[-1] == st["num_shards"]
    np.testing.assert_array_equal(got, oracle.bfs(V, s, d, 0))
    _, got, _, _ = run_part("sssp", V, s, d, G, ev=w, N=300)
    np.testing.assert_array_equal(got, oracle.sssp(V, s, d, w, 0))
    _, got, _, _ = run_part("sswp", V, s, d, G, ev=w, N=300)
    np.testing.assert_array_equal(got, oracle.sswp(V, s, d, w, 0))


@pytest.mark.parametrize("G", GS)
def test_partition_cc_symmetric_bit_exact(G):
    wl = graphgen.workload("rmatsym:30000:60000:62")
    _, got, _, _ = run_part("cc", wl.V, wl.src, wl.dst, G, N=500)
    np.testing.assert_array_equal(got, oracle.cc(wl.V, wl.src, wl.dst))


@pytest.mark.parametrize("G", [2, 8])
def test_partition_pagerank(rm, G):
    V, s, d, _ = rm
    x_star, _ = oracle.pagerank(V, s, d, tol=1e-9)
    rc, got, st, _ = run_part("pr", V, s, d, G, N=300)
    assert rc == cusha.OK
    pr_check(got, x_star)


def test_partition_mesh_sssp_many_iterations():
    wl = graphgen.workload("mesh:40000:200:52000:33")
    _, got, st, _ = run_part("sssp", wl.V, wl.src, wl.dst, 4, ev=wl.edge_u32)
    np.testing.assert_array_equal(got, oracle.sssp(wl.V, wl.src, wl.dst, wl.edge_u32, 0))
    assert st["iterations"] > 50 and st["world_size"] == 4


def test_partition_more_parts_than_shards():
    V = 300
    s, d = graphgen.rmat(V, 2000, seed=63)
    _, got, st, b = run_part("bfs", V, s, d, 8, N=100)   # 3 shards -> 3 partitions
    assert len(b) == 4
    np.testing.assert_array_equal(got, oracle.bfs(V, s, d, 0))


def test_partition_max_iters(rm):
    V, s, d, _ = rm
    rc, got, st, _ = run_part("bfs", V, s, d, 4, N=300, max_iters=2)
    assert rc == cusha.NOT_CONVERGED and st["iterations"] == 2
