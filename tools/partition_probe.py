"""Row e on one GPU: the destination-range partition of a workload simulated
with G partitions in one process (the per-rank layout, kernels and stage-4
stores into the sibling partitions' SrcValue; include/cusha.h world_size with
no NCCL id).  For each G: per-partition device bytes (what one GPU would hold),
bit-exactness of BFS against the oracle, PR passes, and the run time - the
partitions' passes run one after another on this GPU, so the time is the
single-GPU work plus the per-pass overheads, NOT a multi-GPU number.

    python tools/partition_probe.py [C5] [G ...]      (prints one JSON line per G)"""
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

name = sys.argv[1] if len(sys.argv) > 1 else "C5"
Gs = [int(x) for x in sys.argv[2:]] or [1, 2, 4, 8]
t = time.time()
wl = graphgen.workload(name)
print(f"[probe] {name}: V={wl.V} E={wl.E} generated in {time.time() - t:.0f}s", file=sys.stderr, flush=True)
s_d = torch.from_numpy(wl.src.view(np.int32)).cuda()
d_d = torch.from_numpy(wl.dst.view(np.int32)).cuda()
torch.cuda.synchronize()
ref = None
for G in Gs:
    t = time.time()
    g = cusha.build_graph(wl.V, s_d, d_d, repr="cw", world_size=G)
    st = cusha.get_stats(g)
    parts = [cusha.get_part_stats(g, q)["device_bytes"] for q in range(st["partitions"])]
    rec = {"workload": name, "G": G, "partitions": st["partitions"], "build_s": round(time.time() - t, 1),
           "device_bytes_total": st["device_bytes"], "device_bytes_per_partition": parts,
           "max_over_single": None}
    for alg in ("bfs", "pr"):
        cusha.run(alg, g)  # warm-up
        rc = cusha.run(alg, g)
        s2 = cusha.get_stats(g)
        rec[alg] = {"rc": rc, "passes": s2["iterations"], "run_ms": round(s2["run_ms"], 2),
                    "edges_processed": s2["edges_processed"],
                    "wb_entries": s2["wb_entries"]}
        if alg == "bfs":
            vals = cusha.get_values(g)
            if ref is None:
                ref = oracle.bfs(wl.V, wl.src, wl.dst, 0)
            rec["bfs"]["bit_exact_vs_oracle"] = bool(np.array_equal(vals, ref))
    g.close()
    cusha.trim_memory(0)
    print(json.dumps(rec), flush=True)
