"""Per-ticket latency breakdown of the overlapped shard pass (diagnostic).

Needs a library built with -DCUSHA_TIMELINE=1 (tools/tune.sh build
"TL:-DCUSHA_TIMELINE=1").  Runs the workload's algorithm to convergence twice
(the second run's stamps are kept), then prints, over the tickets of the
steady-state passes, the median duration of each step of a ticket and of the
waits between tickets (csrc/kernels.cu, kTlSlots).
usage: python tools/timeline.py <workload> <lib.so> [out.json]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402  (workload table)
import graphgen  # noqa: E402
from paper_conf_hpdc_khorasanivgb14_b200 import cusha  # noqa: E402

wname, lib = sys.argv[1], sys.argv[2]
out_path = sys.argv[3] if len(sys.argv) > 3 else None
alg, repr_, source, desc = bench.WORKLOADS[wname][:4]
cusha._lib = None
cusha.LIB_PATH = os.path.abspath(lib)
wl = graphgen.workload(bench.GRAPH_OF[wname], cache_dir="/tmp/gg")
src = torch.from_numpy(wl.src.view(np.int32)).cuda()
dst = torch.from_numpy(wl.dst.view(np.int32)).cuda()
ev = torch.from_numpy(wl.edge_u32.view(np.int32)).cuda() if alg in ("sssp", "sswp") else None
N = 128 if wname == "C1" else 0
with cusha.build_graph(wl.V, src, dst, edge_values=ev, repr=repr_, vertices_per_shard=N) as g:
    cusha.run(alg, g, source=source)
    cusha.run(alg, g, source=source)
    st = cusha.get_stats(g)
    S = st["num_shards"]
    buf = np.zeros((1 << 18) * 13, dtype=np.uint32)
    n = cusha.lib().cusha_diag_timeline(buf.ctypes.data, buf.nbytes)
    assert n > 0, cusha.lib().cusha_last_error()
    shard_cnt, cw_cnt = cusha.get_layout(g, "shard_sizes"), cusha.get_layout(g, "cw_sizes")
iters = st["iterations"]
T = buf.reshape(-1, 13)[: min(n, (iters + 1) * S)].astype(np.int64)
if out_path:  # raw stamps (row = ticket pass * S + shard) for per-shard analysis
    np.savez_compressed(out_path.rsplit(".", 1)[0] + "_raw.npz", T=T, S=S, iters=iters,
                        shard_cnt=shard_cnt, cw_cnt=cw_cnt)
# steady state: skip the first 2 and the last 2 passes
lo, hi = 2 * S, max(2 * S, (iters - 2) * S)
T = T[lo:hi]
T = T[T[:, 7] != 0]
def d(a, b):
    x = (T[:, b] - T[:, a]) % (1 << 32)
    return x.astype(np.float64) / 1e3  # us
names = {"draw->waited": (0, 1), "waited->first tile": (1, 2), "stage1": (2, 3), "stage2": (3, 4),
         "stage3": (4, 5), "stage4": (5, 6), "done": (6, 7), "ticket total (first tile->done)": (2, 7),
         "draw->done": (0, 7)}
res = {k: {"median_us": round(float(np.median(d(*v))), 3), "mean_us": round(float(np.mean(d(*v))), 3),
           "p90_us": round(float(np.percentile(d(*v), 90)), 3)} for k, v in names.items()}
# consumer idle between two tickets of one CTA: done of one -> first tile of the next
T2 = T[np.argsort(T[:, 2])]
gaps = []
for c in np.unique(T2[:, 8]):
    t = T2[T2[:, 8] == c]
    if len(t) > 1:
        gaps.extend(((t[1:, 2] - t[:-1, 7]) % (1 << 32)) / 1e3)
res["cta idle between tickets"] = {"median_us": round(float(np.median(gaps)), 3),
                                   "mean_us": round(float(np.mean(gaps)), 3)}
res["prefetched_stage4_frac"] = round(float(T[:, 9].mean()), 3)
res["tickets"] = int(len(T))
res["passes"] = iters
res["us_per_pass"] = round(st["loop_ms"] / max(iters, 1) * 1e3, 2)
res["S"] = S
print(json.dumps({"workload": wname, "timeline": res}, indent=1))
if out_path:
    with open(out_path, "w") as f:
        json.dump({"workload": wname, "timeline": res}, f, indent=1)
