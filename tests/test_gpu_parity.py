"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by
element, on seeded inputs that span several shards and a ragged last shard.

Integer algorithms (BFS, SSSP, SSWP, CC) and every layout array: bit-exact.
PR: R10 bound.  NN / HS / CS: tolerance derived from the contraction (R16).
"""
import numpy as np
import pytest

import graphgen
import oracle
from gpu_common import (EPS, cs_inputs, float_tol, gpu_run, hs_inputs, nn_inputs, pr_check)
from paper_conf_hpdc_khorasanivgb14_b200 import cusha

pytestmark = pytest.mark.gpu

REPRS = ["gs", "cw"]


@pytest.fixture(scope="module")
def c1():
    wl = graphgen.workload("C1")
    return wl.V, wl.src, wl.dst, wl.edge_u32


# ------------------------------------------------------------------ BFS
@pytest.mark.parametrize("repr", REPRS)
@pytest.mark.parametrize("N", [0, 7, 32, 128, 1000, 1568, 4096])
def test_bfs_c1_shard_sweep(c1, repr, N):
    """C1 (BFS from 0, R-MAT 4096/32768) with the |N| sweep of SURVEY §8(d)
    (odd, non-multiple-of-32, partial last shard, single shard)."""
    V, s, d, _ = c1
    want = oracle.bfs(V, s, d, 0)
    got, st = gpu_run("bfs", V, s, d, repr=repr, N=N)
    np.testing.assert_array_equal(got, want)
    assert st["converged"] == 1 and st["iterations"] >= 2


@pytest.mark.parametrize("repr", REPRS)
def test_bfs_sources_and_unreachable(repr):
    V = 3000
    s, d = graphgen.rmat(V, 9000, seed=21)
    for src in (0, 1, 2999, 1234):
        want = oracle.bfs(V, s, d, src)
        got, _ = gpu_run("bfs", V, s, d, repr=repr, N=100, source=src)
        np.testing.assert_array_equal(got, want)


# ----------------------------------------------------------------- SSSP
@pytest.mark.parametrize("repr", REPRS)
def test_sssp_rmat(c1, repr):
    V, s, d, w = c1
    want = oracle.sssp(V, s, d, w, 0)
    got, _ = gpu_run("sssp", V, s, d, ev=w, repr=repr, N=128)
    np.testing.assert_array_equal(got, want)


@pytest.mark.parametrize("repr", REPRS)
def test_sssp_mesh(repr):
    wl = graphgen.workload("mesh:40000:200:52000:33")
    want = oracle.sssp(wl.V, wl.src, wl.dst, wl.edge_u32, 0)
    got, st = gpu_run("sssp", wl.V, wl.src, wl.dst, ev=wl.edge_u32, repr=repr)
    np.testing.assert_array_equal(got, want)


# ----------------------------------------------------------------- SSWP
@pytest.mark.parametrize("repr", REPRS)
def test_sswp(c1, repr):
    V, s, d, w = c1
    want = oracle.sswp(V, s, d, w, 0)
    got, _ = gpu_run("sswp", V, s, d, ev=w, repr=repr, N=300)
    np.testing.assert_array_equal(got, want)


@pytest.mark.parametrize("repr", REPRS)
def test_sources_on_one_graph(c1, repr):
    """SSSP and SSWP from several sources on one graph, alternating with BFS.
    Their start state is uniform except at the source, so a run initialises
    SrcValue by a fill of every entry and a patch of the source's out-edges
    (DESIGN.md "Host path of a run"); nothing of the previous run may survive."""
    V, s, d, w = c1
    with cusha.build_graph(V, s, d, edge_values=w, repr=repr, vertices_per_shard=128) as g:
        for src in (0, 777, V - 1, 129):
            for alg, want in (("sssp", oracle.sssp(V, s, d, w, src)), ("sswp", oracle.sswp(V, s, d, w, src)),
                              ("bfs", oracle.bfs(V, s, d, src))):
                assert cusha.run(alg, g, source=src) == cusha.OK
                np.testing.assert_array_equal(cusha.get_values(g), want)


# ------------------------------------------------------------------- CC
@pytest.mark.parametrize("repr", REPRS)
def test_cc_symmetric(repr):
    wl = graphgen.workload("rmatsym:20000:30000:14")
    want = oracle.cc(wl.V, wl.src, wl.dst)
    got, _ = gpu_run("cc", wl.V, wl.src, wl.dst, repr=repr, N=700)
    np.testing.assert_array_equal(got, want)


@pytest.mark.parametrize("repr", REPRS)
def test_cc_directed_min_ancestor(c1, repr):
    V, s, d, _ = c1
    want = oracle.cc(V, s, d)
    got, _ = gpu_run("cc", V, s, d, repr=repr, N=128)
    np.testing.assert_array_equal(got, want)


# ------------------------------------------------------------------- PR
@pytest.mark.parametrize("repr", REPRS)
def test_pr_rmat(repr):
    V = 1 << 16
    s, d = graphgen.rmat(V, 1 << 20, seed=23)
    x_star, _ = oracle.pagerank(V, s, d, tol=1e-9)
    got, st = gpu_run("pr", V, s, d, repr=repr)
    maxerr, n_abs = pr_check(got, x_star)
    assert st["converged"] == 1


def test_pr_deterministic_sum():
    """Fixed-point accumulation: the same run twice gives identical bits."""
    V = 20000
    s, d = graphgen.rmat(V, 200000, seed=24)
    a, _ = gpu_run("pr", V, s, d, repr="cw", N=500)
    b, _ = gpu_run("pr", V, s, d, repr="cw", N=500)
    # asynchronous visibility can differ between runs, so only check parity for both
    x_star, _ = oracle.pagerank(V, s, d, tol=1e-9)
    pr_check(a, x_star)
    pr_check(b, x_star)


# ------------------------------------------------------------- NN/HS/CS
@pytest.mark.parametrize("repr", REPRS)
def test_nn(repr):
    s, d, w, x0 = nn_inputs()
    V = 4096
    x_eps, n1 = oracle.nn(V, s, d, w, x0, tol=EPS)
    x_star, n2 = oracle.nn(V, s, d, w, x0, tol=1e-9)
    got, _ = gpu_run("nn", V, s, d, ev=w, repr=repr, N=256, init=x0)
    tol = float_tol(n1, n2)
    np.testing.assert_allclose(got, x_star, rtol=0, atol=tol * np.maximum(1, np.abs(x_star)).max())


@pytest.mark.parametrize("repr", REPRS)
def test_hs(repr):
    s, d, c, q0 = hs_inputs()
    V = 4096
    _, n1 = oracle.hs(V, s, d, c, q0, tol=EPS)
    q_star, n2 = oracle.hs(V, s, d, c, q0, tol=1e-9)
    got, _ = gpu_run("hs", V, s, d, ev=c, repr=repr, N=256, init=np.stack([q0, q0], 1))
    tol = float_tol(n1, n2) + 4e-6 * 100  # plus float32 rounding at |Q| <= 100
    np.testing.assert_allclose(got[:, 0], q_star, rtol=0, atol=tol)


@pytest.mark.parametrize("repr", REPRS)
def test_cs(repr):
    s, d, G, v0, a0 = cs_inputs()
    V = 4096
    _, n1 = oracle.cs(V, s, d, G, v0, a0, tol=EPS)
    v_star, n2 = oracle.cs(V, s, d, G, v0, a0, tol=1e-9)
    got, _ = gpu_run("cs", V, s, d, ev=G, repr=repr, N=256, init=np.stack([v0, a0], 1))
    tol = float_tol(n1, n2)
    np.testing.assert_allclose(got[:, 0], v_star, rtol=0, atol=tol)
    anc = a0 != 0
    np.testing.assert_array_equal(got[anc, 0], v0[anc])      # anchors keep V exactly
    np.testing.assert_array_equal(got[anc, 1], a0[anc])


# ------------------------------------------------------- layout (row a0)
@pytest.mark.parametrize("repr", REPRS)
@pytest.mark.parametrize("V,E,N", [(4096, 32768, 128), (1000, 7000, 37), (500, 3000, 500), (777, 0, 50)])
def test_layout_matches_oracle(repr, V, E, N):
    if E:
        s, d = graphgen.rmat(V, E, seed=V + E)
    else:
        s = d = np.zeros(0, np.uint32)
    ev = np.arange(len(s), dtype=np.uint32) * 7 + 3
    ref = oracle.build_shards(V, s, d, N)
    S = ref["S"]
    with cusha.build_graph(V, s, d, edge_values=ev, repr=repr, vertices_per_shard=N, keep_layout=True) as g:
        off = cusha.get_layout(g, "shard_offsets").astype(np.int64)
        cnt = cusha.get_layout(g, "shard_sizes").astype(np.int64)
        dest = cusha.get_layout(g, "dest_local")
        eid = cusha.get_layout(g, "edge_id")
        win = cusha.get_layout(g, "windows").astype(np.int64).reshape(S + 1, S)
        outdeg = cusha.get_layout(g, "out_degree")
        cw_cnt = cusha.get_layout(g, "cw_sizes")
        st = cusha.get_stats(g)
        if repr == "gs":
            srcidx = cusha.get_layout(g, "src_index")
        else:
            cw_off = cusha.get_layout(g, "cw_offsets").astype(np.int64)
            cw_src = cusha.get_layout(g, "cw_src_local")
            mapper = cusha.get_layout(g, "mapper").astype(np.int64)
            cw_win = cusha.get_layout(g, "cw_window").astype(np.int64)
            cw_delta = cusha.get_layout(g, "cw_delta").astype(np.int64).reshape(S, S)
    assert st["num_shards"] == S and st["vertices_per_shard"] == N
    assert st["max_in_degree"] == (np.bincount(d, minlength=V).max() if E else 0)
    np.testing.assert_array_equal(cnt, np.diff(ref["shard_off"].astype(np.int64)))
    assert (off % 8 == 0).all()
    # unpadded view: real entries of each shard in order
    real = np.concatenate([np.arange(off[j], off[j] + cnt[j]) for j in range(S)]) if E else np.zeros(0, np.int64)
    np.testing.assert_array_equal(eid[real], ref["gs_eid"])
    shard_of_real = np.repeat(np.arange(S), cnt)
    np.testing.assert_array_equal(dest[real].astype(np.int64) + shard_of_real * N, ref["gs_dst"])
    fill = np.setdiff1d(np.arange(len(dest)), real)
    assert (dest[fill] == N).all() and (eid[fill] == 0xFFFFFFFF).all()
    # windows: padded -> unpadded position
    ref_off = ref["shard_off"].astype(np.int64)
    np.testing.assert_array_equal(win - off[:-1][None, :] + ref_off[:-1][None, :], ref["win"].astype(np.int64))
    np.testing.assert_array_equal(outdeg, np.bincount(s, minlength=V))
    np.testing.assert_array_equal(cw_cnt, np.diff(ref["cw_off"].astype(np.int64)))
    # padded position -> unpadded index
    to_unpadded = np.full(int(off[-1]) + 1, -1, np.int64)
    to_unpadded[real] = np.arange(len(real))
    if repr == "gs":
        np.testing.assert_array_equal(srcidx[real].astype(np.int64), ref["gs_src"].astype(np.int64) % N)
    else:
        creal = np.concatenate([np.arange(cw_off[i], cw_off[i] + cw_cnt[i]) for i in range(S)]) if E else np.zeros(0, np.int64)
        np.testing.assert_array_equal(to_unpadded[mapper[creal]], ref["mapper"].astype(np.int64))
        src_shard = np.repeat(np.arange(S), cw_cnt)
        np.testing.assert_array_equal(cw_src[creal].astype(np.int64) + src_shard * N, ref["cw_src"])
        cfill = np.setdiff1d(np.arange(len(mapper)), creal)
        assert (mapper[cfill] == off[-1]).all()
        # Mapper in window form: j = the shard the oracle's Mapper target lies in, and
        # delta[i][j] + k reproduces Mapper exactly; filler entries carry j = 0xFFFF
        tgt_shard = np.searchsorted(ref_off, ref["mapper"].astype(np.int64), side="right") - 1
        np.testing.assert_array_equal(cw_win[creal], tgt_shard)
        np.testing.assert_array_equal((cw_delta[src_shard, cw_win[creal]] + creal) % (1 << 32), mapper[creal])
        assert (cw_win[cfill] == 0xFFFF).all()


# ----------------------------------------------------------- edge cases
@pytest.mark.parametrize("repr", REPRS)
def test_edge_cases(repr):
    # empty graph: nothing changes; the barrier mode stops after one clean pass,
    # overlapped passes after W consecutive clean ones, W = 4 passes in flight on
    # a graph of average degree < 4
    for barrier, passes in ((True, 1), (False, 4)):
        got, st = gpu_run("bfs", 10, np.zeros(0, np.uint32), np.zeros(0, np.uint32), repr=repr, source=3,
                          pass_barrier=barrier)
        assert got[3] == 0 and (np.delete(got, 3) == cusha.INF).all() and st["iterations"] == passes
    # single vertex
    got, _ = gpu_run("cc", 1, np.zeros(0, np.uint32), np.zeros(0, np.uint32), repr=repr)
    assert got.tolist() == [0]
    # self-loops and duplicates are separate edges (R22)
    s = np.array([0, 0, 1, 1, 2, 2], np.uint32)
    d = np.array([1, 1, 1, 2, 2, 0], np.uint32)
    np.testing.assert_array_equal(gpu_run("bfs", 3, s, d, repr=repr)[0], oracle.bfs(3, s, d, 0))
    x, _ = oracle.pagerank(3, s, d, tol=1e-10)
    pr_check(gpu_run("pr", 3, s, d, repr=repr)[0], x)


def test_max_iters_and_errors():
    V = 4096
    s, d = graphgen.rmat(V, 32768, seed=1)
    with cusha.build_graph(V, s, d, vertices_per_shard=128) as g:
        assert cusha.run("bfs", g, 0, max_iters=1) == cusha.NOT_CONVERGED
        st = cusha.get_stats(g)
        assert st["iterations"] == 1 and st["converged"] == 0
        lv = cusha.get_values(g)
        assert lv[0] == 0
        assert cusha.run("bfs", g, 0, max_iters=0) == cusha.NOT_CONVERGED
        with pytest.raises(cusha.CushaError):
            cusha.run("bfs", g, V, 10)            # source out of range
        with pytest.raises(cusha.CushaError):
            cusha.run("sssp", g, 0, 10)           # needs edge values
        with pytest.raises(cusha.CushaError):
            cusha.run("nn", g, 0, 10)             # needs initial values
        with pytest.raises(cusha.CushaError):
            cusha.set_vertex_values(g, "nn", np.zeros(V - 1, np.float32))
        assert cusha.run("bfs", g, 0) == cusha.OK
        small = np.zeros(3, np.uint32)
        assert cusha.lib().cusha_get_values(g.handle, cusha._ptr(small), small.nbytes) == cusha.EINVAL
    with pytest.raises(cusha.CushaError):
        cusha.build_graph(10, np.array([0, 11], np.uint32), np.array([1, 2], np.uint32))   # endpoint >= |V|


def test_trace_matches_bfs_levels():
    """Fig. 7 analogue (L433): per-iteration committed updates; every reached
    vertex is committed at least once, so the total >= reached - 1."""
    V = 4096
    s, d = graphgen.rmat(V, 32768, seed=1)
    with cusha.build_graph(V, s, d, vertices_per_shard=128) as g:
        cusha.run("bfs", g, 0)
        upd, act = cusha.get_trace(g)
        st = cusha.get_stats(g)
    lv = oracle.bfs(V, s, d, 0)
    assert len(upd) == st["iterations"] and upd[-1] == 0 and act[-1] == 0
    assert upd.sum() >= (lv != cusha.INF).sum() - 1


@pytest.mark.parametrize("repr", REPRS)
def test_host_loop_mode_same_results(c1, repr):
    """host_loop=1 (profiler mode: host-launched passes that early-exit once
    converged) reaches the same values and the same pass count semantics."""
    V, s, d, w = c1
    got, st = gpu_run("sssp", V, s, d, ev=w, repr=repr, N=128, host_loop=True)
    np.testing.assert_array_equal(got, oracle.sssp(V, s, d, w, 0))
    assert st["device_loop"] == 0 and st["converged"] == 1
    x_star, _ = oracle.pagerank(V, s, d, tol=1e-9)
    got, st = gpu_run("pr", V, s, d, repr=repr, N=128, host_loop=True)
    pr_check(got, x_star)
    got, st = gpu_run("bfs", V, s, d, repr=repr, N=128, host_loop=True, max_iters=3, expect_converged=False)
    assert st["iterations"] == 3 and st["converged"] == 0


# -------------------------------------- layout of unsorted input with duplicates
@pytest.mark.parametrize("repr", REPRS)
def test_layout_shuffled_duplicates_self_loops(repr):
    """The builder's order is the definition's (shard(dst), src, dst, INPUT
    ORDER) (L129, R17) on an edge list that is shuffled and carries duplicate
    edges and self-loops (kept as separate edges, R22): every array bit-exact
    against oracle.build_shards, and the integer fixed points still exact."""
    V = 3000
    s, d = graphgen.rmat(V, 30000, seed=81)
    rng = np.random.default_rng(81)
    dup = rng.integers(0, len(s), 4000)
    loops = rng.integers(0, V, 500).astype(np.uint32)
    s = np.concatenate([s, s[dup], loops])
    d = np.concatenate([d, d[dup], loops])
    perm = rng.permutation(len(s))
    s, d = s[perm].astype(np.uint32), d[perm].astype(np.uint32)
    w = graphgen.edge_u32(s, d, seed=81, lo=1, hi=255)
    for N in (97, 512):
        ref = oracle.build_shards(V, s, d, N)
        S = ref["S"]
        with cusha.build_graph(V, s, d, edge_values=w, repr=repr, vertices_per_shard=N, keep_layout=True) as g:
            off = cusha.get_layout(g, "shard_offsets").astype(np.int64)
            cnt = cusha.get_layout(g, "shard_sizes").astype(np.int64)
            eid = cusha.get_layout(g, "edge_id")
            dest = cusha.get_layout(g, "dest_local").astype(np.int64)
            real = np.concatenate([np.arange(off[j], off[j] + cnt[j]) for j in range(S)])
            np.testing.assert_array_equal(eid[real], ref["gs_eid"])          # includes the tie-break order
            np.testing.assert_array_equal(dest[real] + np.repeat(np.arange(S), cnt) * N, ref["gs_dst"])
            if repr == "cw":
                coff = cusha.get_layout(g, "cw_offsets").astype(np.int64)
                ccnt = cusha.get_layout(g, "cw_sizes").astype(np.int64)
                mapper = cusha.get_layout(g, "mapper").astype(np.int64)
                to_unpadded = np.full(int(off[-1]) + 1, -1, np.int64)
                to_unpadded[real] = np.arange(len(real))
                creal = np.concatenate([np.arange(coff[i], coff[i] + ccnt[i]) for i in range(S)])
                np.testing.assert_array_equal(to_unpadded[mapper[creal]], ref["mapper"].astype(np.int64))
            for alg, want, ev in (("bfs", oracle.bfs(V, s, d, 0), None), ("sssp", oracle.sssp(V, s, d, w, 0), w),
                                  ("cc", oracle.cc(V, s, d), None)):
                assert cusha.run(alg, g) == cusha.OK
                np.testing.assert_array_equal(cusha.get_values(g), want, err_msg=f"{alg} N={N}")


# ------------------------------ chunked sort of a host edge list (row f2)
@pytest.mark.parametrize("repr", REPRS)
def test_layout_chunked_host_sort(repr, monkeypatch):
    """A host edge list of >= 2^22 edges crosses in 8 chunks, each radix-sorted
    as it lands and merged into the sorted prefix (builder.cu k_merge).  On a
    shuffled list with many duplicate edges spread over every chunk (ties
    across chunk boundaries, R17) the layout is bit-exact against
    oracle.build_shards and identical to the single-sort build."""
    V = 1500
    s, d = graphgen.rmat(V, 300000, seed=83)
    rng = np.random.default_rng(83)
    pick = rng.integers(0, len(s), (1 << 22) + 12345 - len(s))
    s = np.concatenate([s, s[pick]])
    d = np.concatenate([d, d[pick]])
    perm = rng.permutation(len(s))
    s, d = s[perm].astype(np.uint32), d[perm].astype(np.uint32)
    N = 200
    ref = oracle.build_shards(V, s, d, N)
    S = ref["S"]
    parts = ("edge_id", "dest_local") + (("mapper", "cw_src_local") if repr == "cw" else ("src_index",))
    got = {}
    for chunked in (True, False):
        if chunked:
            monkeypatch.delenv("CUSHA_NO_CHUNK_SORT", raising=False)
        else:
            monkeypatch.setenv("CUSHA_NO_CHUNK_SORT", "1")
        with cusha.build_graph(V, s, d, repr=repr, vertices_per_shard=N, keep_layout=True) as g:
            got[chunked] = {p: cusha.get_layout(g, p) for p in parts + ("shard_offsets", "shard_sizes")}
            if chunked:
                max_indeg = cusha.get_stats(g)["max_in_degree"]
                assert cusha.run("bfs", g) == cusha.OK
                np.testing.assert_array_equal(cusha.get_values(g), oracle.bfs(V, s, d, 0))
    for p in got[True]:
        np.testing.assert_array_equal(got[True][p], got[False][p], err_msg=p)
    off = got[True]["shard_offsets"].astype(np.int64)
    cnt = got[True]["shard_sizes"].astype(np.int64)
    real = np.concatenate([np.arange(off[j], off[j] + cnt[j]) for j in range(S)])
    np.testing.assert_array_equal(got[True]["edge_id"][real], ref["gs_eid"])
    assert max_indeg == np.bincount(d, minlength=V).max()
    np.testing.assert_array_equal(got[True]["dest_local"][real].astype(np.int64) + np.repeat(np.arange(S), cnt) * N,
                                  ref["gs_dst"])


def test_max_in_degree_both_counting_paths():
    """The largest in-degree (fixed-point range check) is counted per shard in
    shared memory for N <= 24576 and by global atomics during ingest above."""
    V = 70000
    s, d = graphgen.rmat(V, 400000, seed=84)
    want = np.bincount(d, minlength=V).max()
    for N in (1000, 30000):
        with cusha.build_graph(V, s, d, repr="cw", vertices_per_shard=N) as g:
            assert cusha.get_stats(g)["max_in_degree"] == want
