"""Row f1 (§5.2, Fig. 11-12) and f4 (Fig. 7) on B200.

f1: SSSP on R-MAT graphs "i_j" (about i M edges, j M vertices), G-Shards vs CW,
    for several |N|; reports time to convergence, passes, and the window-size
    histogram (windows of 0..128 entries, Fig. 11) read from the window table.
f4: per-pass committed updates / active shards of BFS and PageRank (Fig. 7's
    observable: CuSha needs more passes than a CSR method, each cheaper).
Writes JSON to the path given (default gpurun_out/sensitivity.json).
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen  # noqa: E402
from paper_conf_hpdc_khorasanivgb14_b200 import cusha  # noqa: E402

out_path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/sensitivity.json"
M = 1 << 20
GRAPHS = [("67_4", 67, 4), ("67_8", 67, 8), ("67_16", 67, 16), ("134_16", 134, 16)]
NS = [1536, 3072, 6144, 12288]
res = {"f1": [], "f4": {}}


def timed_run(g, alg, source=0, reps=3):
    cusha.run(alg, g, source=source)
    ts, its = [], []
    for _ in range(reps):
        cusha.run(alg, g, source=source)
        st = cusha.get_stats(g)
        ts.append(st["run_ms"])
        its.append(st["iterations"])
    return float(np.median(ts)), int(np.median(its))


for name, ei, vj in GRAPHS:
    V, E = vj * M, ei * M
    t = time.time()
    s, d = graphgen.rmat(V, E, seed=100 + ei + vj)
    w = graphgen.edge_u32(s, d, seed=100 + ei + vj, lo=1, hi=255)
    sd = torch.from_numpy(s.view(np.int32)).cuda()
    dd = torch.from_numpy(d.view(np.int32)).cuda()
    wd = torch.from_numpy(w.view(np.int32)).cuda()
    print(f"{name}: V={V} E={E} gen {time.time() - t:.1f}s", flush=True)
    for N in NS:
        row = {"graph": name, "V": V, "E": E, "N": N}
        for repr_ in ("gs", "cw"):
            with cusha.build_graph(V, sd, dd, edge_values=wd, repr=repr_, vertices_per_shard=N) as g:
                ms, it = timed_run(g, "sssp")
                row[f"{repr_}_ms"] = round(ms, 3)
                row[f"{repr_}_passes"] = it
                if repr_ == "cw":
                    S = cusha.get_stats(g)["num_shards"]
                    win = cusha.get_layout(g, "windows").astype(np.int64).reshape(S + 1, S)
                    sizes = np.diff(win, axis=0).ravel()
                    row["S"] = S
                    row["avg_window"] = round(float(sizes.mean()), 2)
                    row["model_avg_window"] = round(E * N * N / V / V, 2)   # L173
                    row["window_hist_0_128"] = np.bincount(np.minimum(sizes, 128), minlength=129).tolist()
        print(json.dumps({k: v for k, v in row.items() if k != "window_hist_0_128"}), flush=True)
        res["f1"].append(row)
    del sd, dd, wd

# f4: per-pass traces on C2 (BFS and PR) and C4 (CC)
for wname, alg in (("C2", "bfs"), ("C2", "pr"), ("C4", "cc")):
    wl = graphgen.workload(wname, cache_dir="/tmp/gg")
    with cusha.build_graph(wl.V, wl.src, wl.dst, repr="cw") as g:
        cusha.run(alg, g)
        upd, act = cusha.get_trace(g)
        st = cusha.get_stats(g)
    res["f4"][f"{wname}_{alg}"] = {"passes": st["iterations"], "updated_vertices": upd.tolist(),
                                   "active_shards": act.tolist(), "num_shards": st["num_shards"],
                                   "run_ms": st["run_ms"]}
    print(wname, alg, "passes", st["iterations"], "updated", upd[:12].tolist(), flush=True)

os.makedirs(os.path.dirname(out_path) or ".", exist_ok=True)
with open(out_path, "w") as f:
    json.dump(res, f)
print("wrote", out_path)
