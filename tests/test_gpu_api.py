"""GPU tests of the C-ABI contract around the hot path (include/cusha.h):
argument checks of the Python binding for device tensors, the fixed-point
range check of the float algorithms, the keep_layout option, the private
memory pool, and the automatic iteration-boundary mode."""
import numpy as np
import pytest
import torch

import graphgen
import oracle
from gpu_common import gpu_run, nn_inputs, as_bits
from paper_conf_hpdc_khorasanivgb14_b200 import cusha

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def c1():
    wl = graphgen.workload("C1")
    return wl.V, wl.src, wl.dst, wl.edge_u32


def test_device_tensor_checks(c1):
    V, s, d, _ = c1
    st = torch.from_numpy(s.astype(np.int64)).cuda()
    dt = torch.from_numpy(d.astype(np.int64)).cuda()
    with pytest.raises(TypeError):
        cusha.build_graph(V, st, dt, repr="cw", vertices_per_shard=128)          # int64 is not packed u32
    pair = torch.from_numpy(np.stack([s, d], 1).view(np.int32)).cuda()
    with pytest.raises(ValueError):
        cusha.build_graph(V, pair[:, 0], pair[:, 1], repr="cw", vertices_per_shard=128)  # strided column
    with pytest.raises(ValueError):
        cusha.build_graph(V, torch.from_numpy(s.view(np.int32)).cuda(), d, vertices_per_shard=128)  # mixed
    # int32 device tensors on torch's current stream: same result as host arrays
    with cusha.build_graph(V, torch.from_numpy(s.view(np.int32)).cuda(), torch.from_numpy(d.view(np.int32)).cuda(),
                           repr="cw", vertices_per_shard=128) as g:
        assert cusha.run("bfs", g) == cusha.OK
        np.testing.assert_array_equal(cusha.get_values(g), oracle.bfs(V, s, d, 0))


def test_fixed_point_range_check(c1):
    """NN/HS/CS whose |value| x |edge value| x in-degree reaches 2^31 are refused
    (include/cusha.h "Fixed-point range"); in range they run."""
    V, s, d, _ = c1
    s2, d2, w, x0 = nn_inputs()
    with cusha.build_graph(V, s2, d2, edge_values=as_bits(w * np.float32(1e9)), repr="cw", vertices_per_shard=128) as g:
        cusha.set_vertex_values(g, "nn", x0)
        with pytest.raises(cusha.CushaError) as e:
            cusha.run("nn", g)
        assert e.value.code == cusha.EINVAL and b"fixed-point" in cusha.lib().cusha_last_error()
    with cusha.build_graph(V, s2, d2, edge_values=as_bits(w), repr="cw", vertices_per_shard=128) as g:
        cusha.set_vertex_values(g, "nn", x0)
        assert cusha.run("nn", g) == cusha.OK
        inf_x = x0.copy()
        inf_x[5] = np.inf
        cusha.set_vertex_values(g, "nn", inf_x)
        with pytest.raises(cusha.CushaError):
            cusha.run("nn", g)


def test_keep_layout_releases_inspection_arrays(c1):
    V, s, d, _ = c1
    with cusha.build_graph(V, s, d, repr="cw", vertices_per_shard=128) as g:
        for part in ("edge_id", "windows"):
            with pytest.raises(cusha.CushaError) as e:
                cusha.get_layout(g, part)
            assert e.value.code == cusha.EUNSUPPORTED
        plain = cusha.get_stats(g)["device_bytes"]
    with cusha.build_graph(V, s, d, repr="cw", vertices_per_shard=128, keep_layout=True) as g:
        assert len(cusha.get_layout(g, "edge_id")) == cusha.get_stats(g)["entries_padded"]
        assert cusha.get_stats(g)["device_bytes"] > plain


def test_private_pool_trim(c1):
    V, s, d, _ = c1
    free0 = torch.cuda.mem_get_info()[0]
    wl = graphgen.workload("rmat:200000:3200000:64")
    g = cusha.build_graph(wl.V, wl.src, wl.dst, repr="cw")
    cusha.run("pr", g)
    g.close()
    cusha.trim_memory(0)
    free1 = torch.cuda.mem_get_info()[0]
    assert free1 > free0 - (64 << 20)   # the freed graph's memory went back to the device


def test_per_pass_mode_uses_fixed_graph_chunks(c1):
    """pass_barrier = 1 runs passes in fixed-count CUDA graphs (16 per host
    check; no conditional node): results bit-exact, iteration count exact even
    when it is not a multiple of 16, max_iters honoured exactly."""
    V, s, d, w = c1
    for N in (64, 128, 1000):
        got, st = gpu_run("sssp", V, s, d, ev=w, repr="cw", N=N, pass_barrier=True)
        np.testing.assert_array_equal(got, oracle.sssp(V, s, d, w, 0))
        assert st["device_loop"] == 1
    for k in (1, 5, 16, 17):
        got, st = gpu_run("bfs", V, s, d, repr="gs", N=128, pass_barrier=True, max_iters=k,
                          expect_converged=False)
        assert st["iterations"] == min(k, st["iterations"]) and st["iterations"] <= k


def test_run_host_path_reuse_and_long_trace(c1):
    """cusha_run's host path: the pass
    configuration is cached per graph and algorithm, so one handle running
    different algorithms in turn must give each one's own result; a run of
    more than 256 passes reads its trace beyond the head copied with the Ctl
    block, and the trace must account for every committed update."""
    V, s, d, _ = c1
    with cusha.build_graph(V, s, d, repr="cw", vertices_per_shard=128) as g:
        want_bfs = oracle.bfs(V, s, d, 0)
        want_cc = oracle.cc(V, s, d)
        for alg in ("bfs", "cc", "bfs", "pr", "cc"):
            assert cusha.run(alg, g) == cusha.OK
            got = cusha.get_values(g)
            if alg == "bfs":
                np.testing.assert_array_equal(got, want_bfs)
            elif alg == "cc":
                np.testing.assert_array_equal(got, want_cc)
    # a path against the shard order: edges (i+1 -> i), source V-1, |N| = 8.
    # Shards run in id order, so each pass carries the wave about one shard
    # further: several hundred passes
    n = 4000
    ps = np.arange(1, n, dtype=np.uint32)
    pd = ps - 1
    with cusha.build_graph(n, ps, pd, repr="cw", vertices_per_shard=8) as g:
        assert cusha.run("bfs", g, source=n - 1, max_iters=1 << 16) == cusha.OK
        np.testing.assert_array_equal(cusha.get_values(g), oracle.bfs(n, ps, pd, n - 1))
        st = cusha.get_stats(g)
        assert st["iterations"] > 256
        upd, act = cusha.get_trace(g)
        assert len(upd) == st["iterations"]
        assert int(upd.sum()) == n - 1 == st["updated_total"]  # every vertex but the source commits once
