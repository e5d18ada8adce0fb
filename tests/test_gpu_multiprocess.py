"""Row e with one process per partition, on the one GPU a test box has: two
processes (ranks) build their own partitions (include/cusha.h transport IPC),
exchange their CUDA IPC handles over a gloo process group (the caller's
bootstrap), and run.  Everything the multi-GPU mode does after the bootstrap
runs here across process boundaries: stage-4 stores into the other rank's
SrcValue through an IPC mapping, the per-pass barrier and convergence vote
through the ranks' barrier blocks, and cusha_get_values reading the other
rank's slice.  Only NCCL itself (the bootstrap the NCCL transport uses
instead of gloo) needs a second GPU.  Results must be bit-exact against the
oracle for the integer algorithms and within R10 for PR."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import graphgen
import oracle
from gpu_common import pr_check

pytestmark = [pytest.mark.gpu, pytest.mark.timeout(600)]


def _free_port():
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def _rank(rank, world, port, q, V, s, d, w, N):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    from paper_conf_hpdc_khorasanivgb14_b200 import cusha
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        g = cusha.build_graph(V, s, d, edge_values=w, repr="cw", vertices_per_shard=N, world_size=world, rank=rank,
                              transport="ipc", comm_timeout_ms=120000)
        blobs = [None] * world
        dist.all_gather_object(blobs, cusha.ipc_export(g))
        cusha.ipc_connect(g, blobs)
        out = {}
        for alg in ("bfs", "sssp", "cc", "pr"):
            rc = cusha.run(alg, g, source=0)
            st = cusha.get_stats(g)
            out[alg] = (rc, cusha.get_values(g), st["iterations"], st["edges_processed"], st["partitions"])
        part = cusha.get_part_stats(g, 0)["device_bytes"]
        dist.barrier()
        g.close()
        q.put((rank, out, part, None))
    except Exception as e:  # report instead of hanging the parent
        q.put((rank, repr(e), 0, None))
    finally:
        dist.destroy_process_group()


def test_two_processes_one_gpu_ipc_transport():
    V = 20000
    s, d = graphgen.rmat(V, 200000, seed=91)
    w = graphgen.edge_u32(s, d, seed=91, lo=1, hi=255)
    N = 300
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank, args=(r, 2, port, q, V, s, d, w, N)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict((r, (o, b)) for r, o, b, _ in (q.get(timeout=500) for _ in range(2)))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in (0, 1):
        assert not isinstance(res[r][0], str), res[r][0]
    want = {"bfs": oracle.bfs(V, s, d, 0), "sssp": oracle.sssp(V, s, d, w, 0), "cc": oracle.cc(V, s, d)}
    x_star, _ = oracle.pagerank(V, s, d, tol=1e-9)
    for r in (0, 1):
        out, part_bytes = res[r]
        for alg, ref in want.items():
            rc, vals, iters, edges, parts = out[alg]
            assert rc == 0 and parts == 2
            np.testing.assert_array_equal(vals, ref, err_msg=f"rank {r} {alg}")
        rc, vals, iters, edges, parts = out["pr"]
        assert rc == 0
        pr_check(vals, x_star)
    # both ranks ran the same passes; each streamed its own partition's edges
    for alg in want:
        assert res[0][0][alg][2] == res[1][0][alg][2]
        assert res[0][0][alg][3] + res[1][0][alg][3] == res[0][0][alg][2] * len(s)
    assert res[0][1] > 0 and res[1][1] > 0


def _rank_c4(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    from paper_conf_hpdc_khorasanivgb14_b200 import cusha
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        wl = graphgen.workload("C4")
        g = cusha.build_graph(wl.V, wl.src, wl.dst, edge_values=wl.edge_u32, repr="cw", world_size=world, rank=rank,
                              transport="ipc", comm_timeout_ms=120000)
        blobs = [None] * world
        dist.all_gather_object(blobs, cusha.ipc_export(g))
        cusha.ipc_connect(g, blobs)
        out = {}
        for alg in ("cc", "sswp"):
            rc = cusha.run(alg, g, source=0)
            out[alg] = (rc, cusha.get_values(g))
        dist.barrier()
        g.close()
        q.put((rank, out))
    except Exception as e:
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_c4_cc_sswp_ranks_as_processes(world):
    """BASELINE.json configs[3] (C4, HiggsTwitter-shaped, CC and SSWP "at 1 and
    2 GPUs") with each partition in its own process (2 and 4 ranks, one GPU):
    bit-exact against the oracle on every rank."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_c4, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=500) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    wl = graphgen.workload("C4")
    want = {"cc": oracle.cc(wl.V, wl.src, wl.dst), "sswp": oracle.sswp(wl.V, wl.src, wl.dst, wl.edge_u32, 0)}
    for r in range(world):
        assert not isinstance(res[r], str), res[r]
        for alg, ref in want.items():
            rc, vals = res[r][alg]
            assert rc == 0
            np.testing.assert_array_equal(vals, ref, err_msg=f"rank {r} {alg}")


def test_bench_two_ranks_on_one_gpu(tmp_path):
    """bench.py's multi-rank path (torchrun launch, IPC bootstrap over
    torch.distributed, max-over-ranks timing, one JSON line from rank 0) with
    both ranks sharing cuda:0 (--share-gpu; the numbers are not a scaling
    result, the code path is the driver's N>1 one)."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                          "--master-addr", "127.0.0.1", "--master-port", str(_free_port()),
                          os.path.join(root, "bench.py"), "--gpus", "2", "--share-gpu", "--workload", "C4cc",
                          "--steps", "2", "--warmup", "3", "--e2e-steps", "1", "--no-cpu-baseline",
                          "--cache-dir", str(tmp_path)],
                         capture_output=True, text=True, timeout=500, cwd=root)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["run"]["partitions"] == 2
    assert d["e2e"]["value"] > 0
