#!/usr/bin/env python
"""Benchmark of the CuSha shard-processing path on B200 (BASELINE.json metric:
edges processed/s (GTEPS) and time to convergence; shard-pass HBM GB/s vs peak).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C2] [--impl cusha|reference]

A step = one full run of the hot path to convergence (every row of SURVEY
§8(a): init, then shard passes — stages 1-4 + convergence flag — until a pass
commits nothing) on the workload's synthetic graph, already resident in HBM.
`e2e` times the same metric through the C ABI from pinned HOST buffers: build
(H2D + layout) + run + D2H of the values.  Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

# workload -> (algorithm, representation, source, description)
WORKLOADS = {
    "C1": ("bfs", "gs", 0, "BFS from 0 on R-MAT 4,096 V / 32,768 E, |N| = 128 (SURVEY §8(a) override)"),
    "C2": ("pr", "cw", 0, "PageRank (d=0.85, eps=1e-5) on LiveJournal-shaped R-MAT 4,847,571 V / 68,993,773 E, CW"),
    "C3": ("sssp", "cw", 0, "SSSP on RoadNet-CA-shaped mesh 1,971,281 V / 5,533,214 E, CW"),
    "C3gs": ("sssp", "gs", 0, "SSSP on RoadNet-CA-shaped mesh 1,971,281 V / 5,533,214 E, G-Shards"),
    "C3o": ("sssp", "cw", 0, "SSSP on the C3 mesh in natural (row-major) vertex order, CW"),
    "C4cc": ("cc", "cw", 0, "CC on HiggsTwitter-shaped symmetric R-MAT 456,631 V / 14,855,874 E"),
    "C4sswp": ("sswp", "cw", 0, "SSWP on HiggsTwitter-shaped symmetric R-MAT 456,631 V / 14,855,874 E"),
    "C5pr": ("pr", "cw", 0, "PageRank on R-MAT scale 26 (67,108,864 V / 1,073,741,824 E)"),
    "C5bfs": ("bfs", "cw", 0, "BFS on R-MAT scale 26 (67,108,864 V / 1,073,741,824 E)"),
}
METRIC = "edges processed/sec (GTEPS) and time-to-convergence; shard-kernel HBM GB/s vs peak"  # BASELINE.json
GRAPH_OF = {"C1": "C1", "C2": "C2", "C3": "C3", "C3gs": "C3", "C3o": "C3o", "C4cc": "C4", "C4sswp": "C4", "C5pr": "C5", "C5bfs": "C5"}
L2_BYTES = 126 * 1024 * 1024


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def measured_peak_gbs():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            return float(json.load(f)["hbm_gbs"]), "measured"
    return 6650.0, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except FileNotFoundError:
            self.proc = None
        time.sleep(0.25)
        return self

    def __exit__(self, *a):
        time.sleep(0.15)

    def result(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        out, _ = self.proc.communicate(timeout=10)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for n, v in zip(names, f[2:6]):
                if v.lower() == "active":
                    reasons.add(n)
        busy = [x for x in sm if x > 500] or sm
        return {"sm_mhz": statistics.median(busy) if busy else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def load_graph(name, cache):
    import graphgen
    t = time.time()
    wl = graphgen.workload(GRAPH_OF[name], cache_dir=cache)
    log(f"[bench] graph {GRAPH_OF[name]}: V={wl.V} E={wl.E} ({time.time() - t:.1f}s)")
    return wl


def traffic_for(workload, overlapped, passes):
    """DRAM bytes (read + write) of one shard_pass launch from the committed ncu
    --set full capture (profiles/traffic.json), for the launch shape this run
    used, and where that capture came from.  A captured whole-run launch is
    scaled by passes (this launch's over the captured one's): the pass count of
    a PR run varies by a few between runs.  It is NOT measured in this run (ncu
    replays each kernel ~40 times; a number taken under a profiler is never a
    bench value), hence the label."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if not os.path.exists(p):
        return None, None
    with open(p) as f:
        t = json.load(f).get(f"{workload}:{'run' if overlapped else 'pass'}")
    if not t:
        return None, None
    src = {"file": "profiles/traffic.json", "capture": t.get("file"), "commit": t.get("commit"),
           "captured_passes": t.get("passes"), "kind": "committed ncu --set full capture, scaled per launch"}
    return int(t["bytes"] * (passes / t["passes"] if overlapped else 1)), src


def oracle_pr_sweeps(wl, k):
    """Wall time of k fp64 Jacobi sweeps of oracle.pagerank over the full edge
    list, CSR build excluded: the difference of a (k+1)-sweep and a 1-sweep
    call (each call builds its own CSR)."""
    import oracle
    t0 = time.perf_counter()
    oracle.pagerank(wl.V, wl.src, wl.dst, tol=0.0, max_iters=1, allow_notconv=True)
    t1 = time.perf_counter() - t0
    t0 = time.perf_counter()
    oracle.pagerank(wl.V, wl.src, wl.dst, tol=0.0, max_iters=k + 1, allow_notconv=True)
    tk = time.perf_counter() - t0
    return max(tk - t1, 1e-9), t1


def pr_sample_text(wl, k):
    return (f"{k} fp64 Jacobi sweeps of oracle.pagerank over the full {wl.name} edge list ({wl.E} edges each); "
            "CSR build excluded (difference of a (k+1)-sweep and a 1-sweep call)")


def cpu_baseline(wl, alg, source, budget_s=15.0):
    """The oracle as it stands, single-threaded on this host, on a bounded sample."""
    import oracle
    V, s, d = wl.V, wl.src, wl.dst
    if alg == "pr":
        _, t1 = oracle_pr_sweeps(wl, 1)          # ~ CSR build + 2 sweeps: sizes the sample
        k = max(2, int(budget_s / max(t1, 1e-3)))
        el, _ = oracle_pr_sweeps(wl, k)
        val = k * wl.E / el / 1e9
        sample = pr_sample_text(wl, k)
    else:
        fn = {"bfs": lambda: oracle.bfs(V, s, d, source), "cc": lambda: oracle.cc(V, s, d),
              "sssp": lambda: oracle.sssp(V, s, d, wl.edge_u32, source),
              "sswp": lambda: oracle.sswp(V, s, d, wl.edge_u32, source)}[alg]
        t0 = time.perf_counter()
        n = 0
        while True:
            fn()
            n += 1
            if time.perf_counter() - t0 > budget_s / 3:
                break
        el = time.perf_counter() - t0
        val = n * wl.E / el / 1e9
        sample = f"{n} full oracle.{alg} runs (textbook definition; each edge relaxed once) on {wl.name}"
    return {"value": round(val, 6), "unit": "GTEPS", "cores": 1, "kind": "oracle", "sample": sample,
            "host_cores_available": os.cpu_count()}


def static_config(workload, wl, alg, repr_):
    """`config` of both arms (identical): the workload, and whether a pass's
    inputs exceed L2 (no flush is needed then).  Per-run facts go to `run`."""
    desc = WORKLOADS[workload][3]
    evb = 4 if alg in ("sssp", "sswp", "nn", "hs", "cs") else 0
    per_pass = wl.E * (6 + evb)                # stage-2 stream of one pass (compressed layout)
    l2 = (f"inputs larger than L2: {per_pass / 1e9:.3f} GB streamed by stage 2 per pass vs 0.126 GB L2"
          if per_pass > L2_BYTES else f"L2-resident workload ({per_pass / 1e6:.1f} MB per pass); no flush")
    return {"workload": workload, "description": desc, "V": wl.V, "E": wl.E, "algorithm": alg, "repr": repr_,
            "l2": l2}


def bench_reference(args):
    """--impl reference: the oracle (test infrastructure) timed on the host."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    alg, repr_, source, desc = WORKLOADS[args.workload]
    if args.repr:
        repr_ = args.repr
    if args.gpus > 1:
        repr_ = "cw"  # as the cusha arm: the partitioned mode uses CW
    wl = load_graph(args.workload, args.cache_dir)
    import oracle
    V, s, d = wl.V, wl.src, wl.dst

    def step():
        if alg == "pr":
            oracle.pagerank(V, s, d, tol=0.0, max_iters=1, allow_notconv=True)
        elif alg == "bfs":
            oracle.bfs(V, s, d, source)
        elif alg == "cc":
            oracle.cc(V, s, d)
        elif alg == "sssp":
            oracle.sssp(V, s, d, wl.edge_u32, source)
        else:
            oracle.sswp(V, s, d, wl.edge_u32, source)

    if alg == "pr":
        # the same measurement as the cusha arm's cpu_baseline: a step = one
        # fp64 sweep over the whole graph, the CSR build excluded
        if args.warmup:
            oracle.pagerank(V, s, d, tol=0.0, max_iters=args.warmup, allow_notconv=True)
        el, _ = oracle_pr_sweeps(wl, args.steps)
        sample = pr_sample_text(wl, args.steps)
    else:
        for _ in range(args.warmup):
            step()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            step()
        el = time.perf_counter() - t0
        sample = f"{args.steps} full oracle.{alg} runs (textbook definition; each edge relaxed once) on {wl.name}"
    val = args.steps * wl.E / el / 1e9
    line = {"impl": "reference", "metric": METRIC,
            "value": round(val, 6), "unit": "GTEPS", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(el / args.steps * 1e3, 3), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64" if alg == "pr" else "u32", "data": "synthetic",
            "config": static_config(args.workload, wl, alg, repr_),
            "cpu_baseline": {"value": round(val, 6), "unit": "GTEPS", "cores": 1, "kind": "oracle", "sample": sample,
                             "host_cores_available": os.cpu_count()},
            "e2e": {"value": round(val, 6), "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def kernel_launches(st, world_local_parts):
    """Our kernels in one cusha_run: reset_ctl,
    init_vertex_values and init_srcvalue per partition, then the passes: one
    launch (overlapped passes, device_loop 2) or chunks of 16 per-pass launches
    per partition (+ one close_parts per pass slot when partitioned)."""
    parts = world_local_parts
    n = 3 * parts
    if st["device_loop"] == 2:
        return n + 1
    chunks = max(1, -(-st["iterations"] // 16))
    return n + 16 * chunks * (parts + (1 if st["partitions"] > 1 else 0))


def bench_cusha(args):
    import torch
    from paper_conf_hpdc_khorasanivgb14_b200 import cusha
    if args.lib:  # tuning experiments: a variant build of libcusha.so
        cusha.LIB_PATH = os.path.abspath(args.lib)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # --share-gpu (tests only): every rank on cuda:0 over a gloo group, to run
    # this multi-rank path on a one-GPU box; its numbers are not a scaling result
    dev = 0 if args.share_gpu else local
    torch.cuda.set_device(dev)
    dist = None
    nccl_id = None
    if world > 1:
        # one process per GPU; libcusha's stage 4 stores into the other ranks'
        # SrcValue over NVLink and the pass barrier / convergence vote run in
        # peer memory (CUDA IPC; destination-range partition).
        # torch.distributed carries the ranks' IPC handles (transport IPC), the
        # barriers and the max-over-ranks time
        import torch.distributed as dist
        if args.share_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device(f"cuda:{dev}"))
    cdev = "cpu" if args.share_gpu else f"cuda:{dev}"  # device of the small collectives
    alg, repr_, source, desc = WORKLOADS[args.workload]
    if args.N == 0 and args.workload == "C1":
        args.N = 128  # the L310 rule gives 3 shards at this size
    if args.repr:
        repr_ = args.repr
    if world > 1 or args.sim_parts > 1:
        repr_ = "cw"  # the partitioned mode uses CW
    wl = load_graph(args.workload, args.cache_dir)
    stream = torch.cuda.current_stream()
    if world > 1:
        part = dict(world_size=world, rank=rank, transport="ipc")
    else:
        part = dict(world_size=max(1, args.sim_parts))  # > 1: one-process partition simulation (tests/tools)

    def barrier():
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(x):
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=cdev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sum_over_ranks(x):
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=cdev)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return float(t.item())

    src_d = torch.from_numpy(wl.src.view(np.int32)).to(f"cuda:{dev}")
    dst_d = torch.from_numpy(wl.dst.view(np.int32)).to(f"cuda:{dev}")
    ev = None
    if alg in ("sssp", "sswp"):
        ev = torch.from_numpy(wl.edge_u32.view(np.int32)).to(f"cuda:{dev}")
    torch.cuda.synchronize()
    def connect(gh):
        if world > 1:  # the caller's bootstrap of the IPC transport
            blobs = [None] * world
            dist.all_gather_object(blobs, cusha.ipc_export(gh))
            cusha.ipc_connect(gh, blobs)
        return gh

    g = connect(cusha.build_graph(wl.V, src_d, dst_d, edge_values=ev, repr=repr_, vertices_per_shard=args.N,
                                  device=dev, stream=stream.cuda_stream, host_loop=args.host_loop,
                                  skip_clean_shards=args.skip_clean, pass_barrier=args.pass_barrier, **part))
    st0 = cusha.get_stats(g)
    log(f"[bench] rank {rank}/{world} built {repr_} |N|={st0['vertices_per_shard']} |S|={st0['num_shards']} "
        f"partitions={st0['partitions']} in {st0['build_ms']:.1f} ms; device bytes {st0['device_bytes'] / 1e9:.3f} GB "
        f"(largest partition {st0['max_part_device_bytes'] / 1e9:.3f} GB)")
    del src_d, dst_d, ev
    local_parts = st0["partitions"] if world == 1 else 1

    for _ in range(args.warmup):
        cusha.run(alg, g, source=source)
    barrier()
    steps = []
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    with ClockSampler(dev) as clk:
        e0.record(stream)
        for _ in range(args.steps):
            rc = cusha.run(alg, g, source=source)
            steps.append(cusha.get_stats(g))
        e1.record(stream)
        torch.cuda.synchronize()
    barrier()
    clocks = clk.result()
    total_ms = max_over_ranks(e0.elapsed_time(e1))  # device time, max over ranks
    edges = sum_over_ranks(sum(s["edges_processed"] for s in steps))  # each rank streams its partition's edges
    iters = [s["iterations"] for s in steps]
    loop_ms = max_over_ranks(sum(s["loop_ms"] for s in steps))
    alg_bytes = sum_over_ranks(sum(s["algorithmic_bytes"] for s in steps))
    paper_bytes = sum_over_ranks(sum(s["paper_bytes"] for s in steps))
    value = edges / (total_ms / 1e3) / 1e9
    launches = int(sum_over_ranks(sum(kernel_launches(s, local_parts) for s in steps)))
    overlapped = steps[-1]["device_loop"] == 2
    n_pass_launches = len(steps) if overlapped else sum(iters)
    peak, peak_kind = measured_peak_gbs()
    # one GPU's bandwidth is the roofline of its shard passes: bytes per GPU per second
    achieved = alg_bytes / world / (loop_ms / 1e3) / 1e9
    achieved_paper = paper_bytes / world / (loop_ms / 1e3) / 1e9
    st = cusha.get_stats(g)
    g.close()

    # ---- e2e through the public API from pinned host buffers
    e2e = None
    if not args.no_e2e:
        pin_s = torch.from_numpy(wl.src.view(np.int32)).pin_memory()
        pin_d = torch.from_numpy(wl.dst.view(np.int32)).pin_memory()
        pin_w = torch.from_numpy(wl.edge_u32.view(np.int32)).pin_memory() if alg in ("sssp", "sswp") else None
        vb = cusha.value_bytes(alg)
        out = torch.empty(wl.V * vb // 4, dtype=torch.int32).pin_memory()
        n_e2e = max(1, min(args.steps, args.e2e_steps))
        h2d = 4 * wl.E * (3 if pin_w is not None else 2)

        def e2e_step():
            # the user's call sequence: build from host buffers (H2D inside), run, read the result (D2H)
            gh = connect(cusha.build_graph(wl.V, pin_s.numpy().view(np.uint32), pin_d.numpy().view(np.uint32),
                                           edge_values=None if pin_w is None else pin_w.numpy().view(np.uint32),
                                           repr=repr_, vertices_per_shard=args.N, device=dev,
                                           stream=stream.cuda_stream, skip_clean_shards=args.skip_clean,
                                           pass_barrier=args.pass_barrier, **part))
            cusha.run(alg, gh, source=source)
            n = cusha.get_stats(gh)["edges_processed"]
            rc = cusha.lib().cusha_get_values(gh.handle, cusha._ptr(out), wl.V * vb)
            assert rc == 0
            gh.close()
            return n

        e2e_step()  # untimed warm-up (module loading, memory pool growth)
        e2e_edges = 0
        barrier()
        t0 = time.perf_counter()
        for _ in range(n_e2e):
            ts = time.perf_counter()
            e2e_edges += e2e_step()
            log(f"[bench] e2e step {1e3 * (time.perf_counter() - ts):.1f} ms")
        torch.cuda.synchronize()
        el = max_over_ranks(time.perf_counter() - t0)
        e2e_edges = sum_over_ranks(e2e_edges)
        e2e = {"value": round(e2e_edges / el / 1e9, 4), "unit": "GTEPS", "h2d_bytes_per_step": h2d * world,
               "d2h_bytes_per_step": wl.V * vb * world, "ms_per_step": round(el / n_e2e * 1e3, 3),
               "steps": n_e2e, "warmup": 1}

    traffic, traffic_src = traffic_for(args.workload, overlapped, sum(iters) / len(iters)) \
        if world == 1 and local_parts == 1 else (None, None)
    line = {
        "metric": METRIC,
        "value": round(value, 4),
        "unit": "GTEPS",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(total_ms / args.steps, 4),
        "higher_is_better": True,
        "scaling": "strong",
        "vs_baseline": None,
        "dtype": "f32" if alg in ("pr", "nn", "hs", "cs") else "u32",
        "data": "synthetic",
        "config": static_config(args.workload, wl, alg, repr_),
        "run": {"vertices_per_shard": st0["vertices_per_shard"], "num_shards": st0["num_shards"],
                "iterations": iters[-1], "time_to_convergence_ms": round(total_ms / args.steps, 4),
                "build_ms": round(st0["build_ms"], 3), "skip_clean_shards": bool(args.skip_clean),
                "passes": "one launch per pass, device-wide barrier between passes" if not overlapped
                else "overlapped passes in one launch (DESIGN.md \"Overlapped passes\")",
                "parallelism": (f"destination-range partition x{world}: stage-4 stores over NVLink (CUDA IPC), "
                                "pass barrier and convergence vote in peer memory") if world > 1 else
                               (f"1 GPU, {local_parts} simulated partitions" if local_parts > 1 else "1 GPU"),
                "partitions": st0["partitions"], "device_bytes_per_gpu": st0["max_part_device_bytes"]},
        "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                     "frac": round(achieved / peak, 4),
                     "traffic": traffic, "traffic_source": traffic_src,
                     "launch": "one shard_pass launch per run (overlapped passes)" if overlapped
                     else "one shard_pass launch per pass",
                     "passes_per_step": round(sum(iters) / len(iters), 2),
                     "avg_pass_us": round(loop_ms / max(sum(iters), 1) * 1e3, 3),
                     "kernel": f"shard_pass<{alg},{repr_}>", "peak_kind": peak_kind,
                     "bytes": "compressed layout actually streamed (u16 indices, pre-divided PR, window-form Mapper; "
                              "DESIGN.md §7)",
                     "algorithmic_bytes_per_launch": int(alg_bytes / world / max(n_pass_launches, 1)),
                     "avg_launch_us": round(loop_ms / max(n_pass_launches, 1) * 1e3, 3),
                     "paper_layout": {"bytes": "SURVEY §8(d) per-unit figures (4-byte fields: stage 2 12 B/edge for PR, "
                                               "stage 4 12 B per active CW edge, 8 B/vertex); not physical here",
                                      "algorithmic_bytes_per_launch": int(paper_bytes / world / max(n_pass_launches, 1)),
                                      "achieved": round(achieved_paper, 1),
                                      "frac": round(achieved_paper / peak, 4)}},
        "clocks": clocks,
        "gpu_launches": launches,
        "e2e": e2e,
        "paper_context": {"hardware": "GTX 780 (Kepler), PCIe 3.0, CUDA 5.5 (L379)",
                          "table4_livejournal_pr_ms": {"CuSha-CW": 709, "CuSha-GS": 885, "VWC-CSR": "2814-3503"},
                          "avg_speedup_over_vwc": {"GS": "1.72-4.05x", "CW": "1.89-4.89x"}},
    }
    if rank == 0 and not args.no_cpu_baseline and world == 1:
        line["cpu_baseline"] = cpu_baseline(wl, alg, source, budget_s=args.cpu_budget)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def relaunch_under_torchrun(args) -> int:
    """`python bench.py --gpus N` (N > 1) without torchrun: start N ranks on
    this node (the contract's launch line), or refuse when fewer GPUs exist."""
    import socket
    import torch
    have = torch.cuda.device_count()
    if have < args.gpus:
        log(f"[bench] --gpus {args.gpus} but only {have} CUDA device(s) visible; refusing to report a "
            f"{args.gpus}-GPU number")
        return 2
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")          # NCCL's init log (rank count) stays visible
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    log("[bench] launching " + " ".join(cmd[2:7]))
    return subprocess.call(cmd, env=env)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="cusha", choices=["cusha", "reference"])
    ap.add_argument("--workload", default="C2", choices=sorted(WORKLOADS))
    ap.add_argument("--repr", default=None, choices=[None, "gs", "cw"])
    ap.add_argument("--N", type=int, default=0, help="vertices per shard (0 = L310 rule)")
    ap.add_argument("--cache-dir", default=None)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--host-loop", action="store_true", help="host-launched passes (for ncu); default: device loop")
    ap.add_argument("--lib", default=None, help="alternative libcusha.so (tuning variants)")
    ap.add_argument("--skip-clean", action="store_true",
                    help="opt-in exact clean-shard skipping (not the paper's full passes; off by default)")
    ap.add_argument("--pass-barrier", action="store_true",
                    help="one launch per pass with a device-wide barrier between passes (Fig. 5) instead of "
                         "the default overlapped passes")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--share-gpu", action="store_true",
                    help="tests only: all ranks on cuda:0 over gloo (exercises the multi-rank path on one GPU)")
    ap.add_argument("--sim-parts", type=int, default=1,
                    help="one process: simulate this many destination-range partitions on one GPU (tools/tests)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    args = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "0"))
    if world and world != args.gpus:
        log(f"[bench] WORLD_SIZE={world} but --gpus {args.gpus}")
        return 2
    if args.gpus > 1 and not world and args.impl == "cusha" and not args.share_gpu:
        return relaunch_under_torchrun(args)
    if world > 1:
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    if args.warmup < 3 and args.impl == "cusha":
        log("[bench] warmup raised to 3 (timing rules)")
        args.warmup = 3
    if args.impl == "reference":
        return bench_reference(args)
    return bench_cusha(args)


if __name__ == "__main__":
    sys.exit(main())
