"""Row f3 probe: R-MAT scale 27 (2^27 V / 2^31 E) BFS on one B200, bit-exact
against the oracle's textbook BFS; optional host-streamed topology budget.
    python tools/r27_probe.py [R27] [budget_GB]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import graphgen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_hpdc_khorasanivgb14_b200 import cusha  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "R27"
budget = int(float(sys.argv[2]) * 1e9) if len(sys.argv) > 2 else 0
t = time.time()
wl = graphgen.workload(name)
gen_s = time.time() - t
print(f"[probe] {name}: V={wl.V} E={wl.E} generated in {gen_s:.0f}s", file=sys.stderr, flush=True)
t = time.time()
g = cusha.build_graph(wl.V, wl.src, wl.dst, repr="cw", device_topology_budget=budget)
st = cusha.get_stats(g)
build_s = time.time() - t
rec = {"workload": name, "V": wl.V, "E": wl.E, "build_s": round(build_s, 1), "build_ms_device": round(st["build_ms"], 1),
       "h2d_ms": round(st["h2d_ms"], 1), "N": st["vertices_per_shard"], "S": st["num_shards"],
       "device_bytes": st["device_bytes"], "host_bytes": st["host_bytes"], "host_shard": st["host_shard"]}
runs = []
for k in range(2):
    rc = cusha.run("bfs", g)
    s2 = cusha.get_stats(g)
    runs.append({"rc": rc, "passes": s2["iterations"], "run_ms": round(s2["run_ms"], 2),
                 "gteps": round(s2["edges_processed"] / s2["run_ms"] / 1e6, 2),
                 "paper_teps_G": round(wl.E / s2["loop_ms"] / 1e6, 2)})
rec["bfs"] = runs
vals = cusha.get_values(g)
g.close()
t = time.time()
ref = oracle.bfs(wl.V, wl.src, wl.dst, 0)
rec["oracle_bfs_s"] = round(time.time() - t, 1)
rec["bit_exact"] = bool(np.array_equal(vals, ref))
rec["reached"] = int((ref != 0xFFFFFFFF).sum())
print(json.dumps(rec), flush=True)
