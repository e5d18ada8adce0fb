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


# ------------------------------------------------ per-partition layout (row e)
@pytest.mark.parametrize("G", [2, 3, 8])
def test_partition_layout_is_the_global_layout_sliced(rm, G):
    """Each partition holds exactly its shards' entries (the global layout's
    slice, positions rebased) and the CW of its source shards, whose Mapper
    points into the OWNING partition's SrcValue: target + that partition's
    first position = the global Mapper, and the segment of CW_i aimed at
    partition q holds exactly the entries whose target shard q owns."""
    V, s, d, w = rm
    N = 300
    with cusha.build_graph(V, s, d, edge_values=w, repr="cw", vertices_per_shard=N, keep_layout=True) as g1:
        off = cusha.get_layout(g1, "shard_offsets").astype(np.int64)
        cnt = cusha.get_layout(g1, "shard_sizes").astype(np.int64)
        dest = cusha.get_layout(g1, "dest_local")
        coff = cusha.get_layout(g1, "cw_offsets").astype(np.int64)
        ccnt = cusha.get_layout(g1, "cw_sizes").astype(np.int64)
        csrc = cusha.get_layout(g1, "cw_src_local")
        mapper = cusha.get_layout(g1, "mapper").astype(np.int64)
        cwin = cusha.get_layout(g1, "cw_window").astype(np.int64)
        outdeg = cusha.get_layout(g1, "out_degree")
        single = cusha.get_stats(g1)
    S = single["num_shards"]
    with cusha.build_graph(V, s, d, edge_values=w, repr="cw", vertices_per_shard=N, world_size=G,
                           keep_layout=True) as g:
        b = cusha.get_partition(g).astype(np.int64)
        assert len(b) == G + 1 and b[0] == 0 and b[-1] == S
        pb = off[b]                                           # first global position of each partition
        owner = np.repeat(np.arange(G), np.diff(b))
        total_bytes = 0
        for q in range(G):
            s0, s1 = b[q], b[q + 1]
            lo = cusha.get_layout(g, "shard_offsets", partition=q).astype(np.int64)
            np.testing.assert_array_equal(lo, off[s0:s1 + 1] - off[s0])
            np.testing.assert_array_equal(cusha.get_layout(g, "shard_sizes", partition=q), cnt[s0:s1])
            np.testing.assert_array_equal(cusha.get_layout(g, "dest_local", partition=q), dest[off[s0]:off[s1]])
            lc = cusha.get_layout(g, "cw_offsets", partition=q).astype(np.int64)
            np.testing.assert_array_equal(lc, coff[s0:s1 + 1] - coff[s0])
            np.testing.assert_array_equal(cusha.get_layout(g, "cw_src_local", partition=q), csrc[coff[s0]:coff[s1]])
            np.testing.assert_array_equal(cusha.get_layout(g, "out_degree", partition=q),
                                          outdeg[s0 * N:min(V, s1 * N)])
            lm = cusha.get_layout(g, "mapper", partition=q).astype(np.int64)
            cwp = cusha.get_layout(g, "cw_partition_offsets", partition=q).astype(np.int64).reshape(s1 - s0, G + 1)
            for il in range(s1 - s0):
                i = s0 + il
                assert cwp[il, 0] == lc[il] and cwp[il, G] == lc[il] + ccnt[i]
                assert (np.diff(cwp[il]) >= 0).all()
                for t in range(G):
                    seg = np.arange(cwp[il, t], cwp[il, t + 1])
                    glob_k = seg + coff[s0]
                    assert (owner[cwin[glob_k]] == t).all()                     # aimed at partition t
                    np.testing.assert_array_equal(lm[seg] + pb[t], mapper[glob_k])
            st = cusha.get_part_stats(g, q)
            total_bytes += st["device_bytes"]
        assert cusha.get_stats(g)["partitions"] == G
    # per-partition memory is the global layout split, not replicated
    assert total_bytes < 1.25 * single["device_bytes"] + G * 4 * (S + 1) * S


def test_partition_device_bytes_shrink_with_G():
    wl = graphgen.workload("rmat:200000:3200000:64")
    sizes = {}
    for G in (1, 2, 4, 8):
        with cusha.build_graph(wl.V, wl.src, wl.dst, repr="cw", world_size=G) as g:
            sizes[G] = cusha.get_stats(g)["max_part_device_bytes"]
    for G in (2, 4, 8):
        assert sizes[G] < 1.6 * sizes[1] / G, sizes


def test_partition_edge_cases():
    """The partitioned build straight from the edge list on degenerate inputs:
    no edges, a partial last shard, more partitions than shards, duplicate
    edges and self-loops (R22), and an empty partition-to-be (one huge shard)."""
    # no edges at all
    z = np.zeros(0, np.uint32)
    _, got, st, b = run_part("bfs", 1000, z, z, 4, N=100, source=7)
    assert got[7] == 0 and (np.delete(got, 7) == 0xFFFFFFFF).all() and len(b) == 5
    # partial last shard (V not a multiple of N), duplicates and self-loops
    V = 1003
    s, d = graphgen.rmat(1024, 9000, seed=95)
    keep = (s < V) & (d < V)
    s, d = s[keep], d[keep]
    rng = np.random.default_rng(95)
    dup = rng.integers(0, len(s), 500)
    loops = rng.integers(0, V, 50).astype(np.uint32)
    s = np.concatenate([s, s[dup], loops]).astype(np.uint32)
    d = np.concatenate([d, d[dup], loops]).astype(np.uint32)
    w = graphgen.edge_u32(s, d, seed=95, lo=1, hi=255)
    for G in (2, 5):
        _, got, _, _ = run_part("sssp", V, s, d, G, ev=w, N=97)
        np.testing.assert_array_equal(got, oracle.sssp(V, s, d, w, 0))
        _, got, _, _ = run_part("cc", V, s, d, G, N=97)
        np.testing.assert_array_equal(got, oracle.cc(V, s, d))
    # one shard holds almost all the work: the greedy split leaves a partition thin
    V = 4000
    hub_s = np.arange(1, 3000, dtype=np.uint32)
    s2 = np.concatenate([hub_s, np.array([3500, 3600], np.uint32)])
    d2 = np.concatenate([np.zeros(len(hub_s), np.uint32), np.array([3600, 3700], np.uint32)])
    for G in (2, 4):
        _, got, st, b = run_part("bfs", V, s2, d2, G, N=500, source=3500)
        np.testing.assert_array_equal(got, oracle.bfs(V, s2, d2, 3500))
