"""Host logic of the destination-range partition (row e) without a GPU:
the balanced split, its determinism across ranks, and the rank-0 id broadcast
over a world_size-2 gloo process group (the plumbing bench.py uses with NCCL)."""
import ctypes
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_hpdc_khorasanivgb14_b200 import cusha


def test_partition_bounds_properties():
    rng = np.random.default_rng(0)
    for S, G in [(1430, 2), (1430, 8), (5878, 4), (7, 7), (3, 5), (100, 1)]:
        work = rng.pareto(1.5, S).astype(np.float64) * 1000 + 1
        work = work.astype(np.uint64)
        b = cusha.partition_shards(work, G)
        assert b[0] == 0 and b[-1] == S and len(b) == G + 1
        assert (np.diff(b.astype(np.int64)) >= 0).all()
        parts = [int(work[b[q]:b[q + 1]].sum()) for q in range(G)]
        assert sum(parts) == int(work.sum())
        # greedy split: each part within one shard's work of the ideal share
        ideal = work.sum() / G
        assert max(parts) <= ideal + work.max() + 1
        np.testing.assert_array_equal(b, cusha.partition_shards(work, G))   # deterministic


def test_partition_uniform_work_is_even():
    b = cusha.partition_shards(np.full(800, 10, np.uint64), 8)
    np.testing.assert_array_equal(b, np.arange(0, 801, 100))


def test_partition_rejects_bad_args():
    assert cusha.lib().cusha_partition_shards(4, None, 2, None) == cusha.EINVAL


def test_multi_rank_argument_validation():
    L = cusha.lib()
    s = np.zeros(1, np.uint32)
    h = ctypes.c_void_p()
    idb = ctypes.create_string_buffer(128)
    o = cusha.BuildOpts()
    o.repr = cusha.REPR_CW
    o.world_size = 2
    o.rank = 5                                  # out of range
    o.nccl_unique_id = ctypes.cast(idb, ctypes.c_void_p)
    assert L.cusha_build_graph(8, 1, cusha._ptr(s), cusha._ptr(s), None, ctypes.byref(o), ctypes.byref(h)) == cusha.EINVAL
    o.rank = 0
    o.repr = cusha.REPR_GSHARDS                 # partitioned mode is CW only
    assert L.cusha_build_graph(8, 1, cusha._ptr(s), cusha._ptr(s), None, ctypes.byref(o), ctypes.byref(h)) == cusha.EUNSUPPORTED


def _free_port():
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # every rank partitions the same (seeded) shard work independently
        work = np.random.default_rng(42).integers(1, 10000, 1430).astype(np.uint64)
        b = torch.from_numpy(cusha.partition_shards(work, world).astype(np.int64))
        allb = [torch.zeros_like(b) for _ in range(world)]
        dist.all_gather(allb, b)
        same = all(torch.equal(allb[0], x) for x in allb)
        # rank 0's 128-byte NCCL id reaches every rank unchanged (as in bench.py)
        idt = torch.zeros(128, dtype=torch.uint8)
        if rank == 0:
            try:
                raw = cusha.nccl_unique_id()
            except Exception:
                raw = bytes(range(128))      # no NCCL bootstrap possible here: any 128 bytes
            idt = torch.frombuffer(bytearray(raw), dtype=torch.uint8).clone()
        dist.broadcast(idt, 0)
        ids = [torch.zeros(128, dtype=torch.uint8) for _ in range(world)]
        dist.all_gather(ids, idt)
        q.put((rank, same, all(torch.equal(ids[0], x) for x in ids), int(b[-1])))
    finally:
        dist.destroy_process_group()


def test_gloo_two_ranks_agree_on_partition_and_id():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(same and ids_same and last == 1430 for _, same, ids_same, last in res)
