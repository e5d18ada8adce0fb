"""Row f3 measurement: the shard pass with host-streamed topology.

For a workload, builds the graph with device_topology_budget = all / half /
none of the per-entry topology in HBM, runs the algorithm to convergence, and
reports per-pass time and the host-link rate: bytes the pass streams from
pinned host memory per pass (host shards' DestIndex [+EdgeValue] for stage 2,
their CW arrays for stage 4 of active shards) / pass time, against the
measured pinned H2D copy bandwidth (torch copy of a 1 GiB pinned buffer).
usage: python tools/ooc_probe.py [workload] [out.json]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen  # noqa: E402
from paper_conf_hpdc_khorasanivgb14_b200 import cusha  # noqa: E402

wname = sys.argv[1] if len(sys.argv) > 1 else "C2"
out_path = sys.argv[2] if len(sys.argv) > 2 else "gpurun_out/ooc_probe.json"
ALG = {"C2": ("pr", "cw"), "C3": ("sssp", "cw"), "C4": ("cc", "cw"), "C5": ("pr", "cw")}
alg, repr_ = ALG.get(wname, ("pr", "cw"))


def h2d_gbs(nbytes=1 << 30, reps=5):
    h = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        d.copy_(h, non_blocking=True)
    e1.record()
    torch.cuda.synchronize()
    return nbytes * reps / (e0.elapsed_time(e1) / 1e3) / 1e9


link = h2d_gbs()
print(f"pinned H2D copy: {link:.1f} GB/s", flush=True)
wl = graphgen.workload(wname, cache_dir="/tmp/gg")
ev = wl.edge_u32 if alg in ("sssp", "sswp") else None
src = torch.from_numpy(wl.src.view(np.int32)).cuda()
dst = torch.from_numpy(wl.dst.view(np.int32)).cuda()
evd = torch.from_numpy(ev.view(np.int32)).cuda() if ev is not None else None
rows = []
with cusha.build_graph(wl.V, src, dst, edge_values=evd, repr=repr_) as g0:
    st0 = cusha.get_stats(g0)
    P = st0["entries_padded"]
    cw_off = cusha.get_layout(g0, "cw_offsets").astype(np.int64)
    sh_off = cusha.get_layout(g0, "shard_offsets").astype(np.int64)
bP = 2 + 4 + (4 if ev is not None else 0)        # DestIndex, edge id, EdgeValue per shard position
bQ = 6                                           # SrcIndexCW + Mapper per CW position
full = int(sh_off[-1] * bP + cw_off[-1] * bQ)
for frac in (None, 0.5, 0.0):
    budget = 0 if frac is None else max(1, int(full * frac))
    with cusha.build_graph(wl.V, src, dst, edge_values=evd, repr=repr_, device_topology_budget=budget) as g:
        cusha.run(alg, g)  # warm-up
        ts = []
        for _ in range(3):
            cusha.run(alg, g)
            st = cusha.get_stats(g)
            ts.append(st["loop_ms"])
        ms = float(np.median(ts))
        h = st["host_shard"]
        upd, act = cusha.get_trace(g)
        it = st["iterations"]
        # host-streamed bytes: stage 2 of host shards every pass + stage 4 of host shards when active
        # (active shard counts are per pass over all shards; scaled by the host shards' CW share)
        s2 = (sh_off[-1] - sh_off[h]) * (2 + (4 if ev is not None else 0))
        cw_host_share = (cw_off[-1] - cw_off[h]) / max(cw_off[-1], 1)
        s4 = float(np.sum(act[:it])) / st["num_shards"] * cw_off[-1] * cw_host_share * bQ
        host_bytes_run = s2 * it + s4
        row = {"budget_frac": frac, "host_shard": h, "num_shards": st["num_shards"], "host_bytes": st["host_bytes"],
               "device_bytes": st["device_bytes"], "iterations": it, "loop_ms": round(ms, 3),
               "us_per_pass": round(ms / it * 1e3, 1), "host_stream_gb_per_pass": round(host_bytes_run / it / 1e9, 4),
               "host_link_gbs": round(host_bytes_run / (ms / 1e3) / 1e9, 2) if h < st["num_shards"] else None,
               "gteps": round(st["edges_processed"] / (ms / 1e3) / 1e9, 3)}
        rows.append(row)
        print(json.dumps(row), flush=True)
res = {"workload": wname, "algorithm": alg, "repr": repr_, "pinned_h2d_gbs": round(link, 2), "rows": rows}
os.makedirs(os.path.dirname(out_path) or ".", exist_ok=True)
with open(out_path, "w") as f:
    json.dump(res, f, indent=1)
print("wrote", out_path)
