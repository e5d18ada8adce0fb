"""Row f3 (L455, "a multi-streamed procedure ... if graphs do not fit in the
GPU RAM"): BFS on R-MAT scale 28 (2^28 V / 4.03 G E) on one B200 whose free
HBM is first cut to AVAIL_GB by a ballast allocation, so that the graph's
layout does not fit in the HBM the run may use.  The graph is built as G
destination-range partitions straight from the host edge list (partition.cu:
one partition's sort at a time, streamed in chunks), each partition's per-entry
topology kept in pinned host memory (device_topology_budget = 1 byte), and
every pass streams it over the host link through the shard pass's TMA ring.
BFS is compared bit for bit with the oracle's textbook BFS.
    python tools/ooc_probe_r28.py [R28] [G] [AVAIL_GB]      (one JSON line)"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_hpdc_khorasanivgb14_b200 import cusha  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "R28"
G = int(sys.argv[2]) if len(sys.argv) > 2 else 4
avail_gb = float(sys.argv[3]) if len(sys.argv) > 3 else 40.0
t = time.time()
wl = graphgen.workload(name)
gen_s = time.time() - t
print(f"[ooc] {name}: V={wl.V} E={wl.E} generated in {gen_s:.0f}s", file=sys.stderr, flush=True)
free0, total = torch.cuda.mem_get_info()
ballast = None
if free0 > avail_gb * 1e9:
    ballast = torch.empty(int(free0 - avail_gb * 1e9), dtype=torch.uint8, device="cuda")
free1 = torch.cuda.mem_get_info()[0]
t = time.time()
g = cusha.build_graph(wl.V, wl.src, wl.dst, repr="cw", world_size=G, device_topology_budget=1)
build_s = time.time() - t
st = cusha.get_stats(g)
rec = {"workload": name, "V": wl.V, "E": wl.E, "partitions": st["partitions"], "N": st["vertices_per_shard"],
       "S": st["num_shards"], "hbm_total_GB": round(total / 1e9, 1), "hbm_free_for_run_GB": round(free1 / 1e9, 1),
       "layout_device_GB": round(st["device_bytes"] / 1e9, 2), "layout_host_GB": round(st["host_bytes"] / 1e9, 2),
       "layout_total_GB": round((st["device_bytes"] + st["host_bytes"]) / 1e9, 2), "build_s": round(build_s, 1),
       "h2d_bytes_build": st["h2d_bytes"]}
runs = []
for k in range(2):
    rc = cusha.run("bfs", g)
    s2 = cusha.get_stats(g)
    runs.append({"rc": rc, "passes": s2["iterations"], "run_ms": round(s2["run_ms"], 1),
                 "gteps": round(s2["edges_processed"] / s2["run_ms"] / 1e6, 3),
                 "host_topology_GBps_if_all_streamed": round(st["host_bytes"] * s2["iterations"] / s2["loop_ms"] / 1e6, 1)})
rec["bfs"] = runs
vals = cusha.get_values(g)
g.close()
del ballast
t = time.time()
ref = oracle.bfs(wl.V, wl.src, wl.dst, 0)
rec["oracle_bfs_s"] = round(time.time() - t, 1)
rec["bit_exact"] = bool(np.array_equal(vals, ref))
rec["reached"] = int((ref != 0xFFFFFFFF).sum())
print(json.dumps(rec), flush=True)
