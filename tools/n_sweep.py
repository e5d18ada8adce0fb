"""|N| sweep (L310 rule vs alternatives) on one B200: time to convergence,
passes, per-pass time and fraction of the copy peak per (workload, |N|).
    python tools/n_sweep.py C2:pr:cw:3392,4700 C5:pr:cw:11417,14500 ...   (one JSON line per point)"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen  # noqa: E402
from paper_conf_hpdc_khorasanivgb14_b200 import cusha  # noqa: E402

PEAK = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")))["hbm_gbs"] \
    if os.path.exists("MEASURED_PEAKS.json") else 6528.4
cache = {}
for spec in sys.argv[1:]:
    wname, alg, repr_, Ns = spec.split(":")
    gname = {"C4cc": "C4", "C4sswp": "C4"}.get(wname, wname)
    if gname not in cache:
        cache.clear()
        torch.cuda.empty_cache()
        wl = graphgen.workload(gname, cache_dir="/tmp/gg")
        s = torch.from_numpy(wl.src.view(np.int32)).cuda()
        d = torch.from_numpy(wl.dst.view(np.int32)).cuda()
        w = torch.from_numpy(wl.edge_u32.view(np.int32)).cuda() if wl.edge_u32 is not None else None
        cache[gname] = (wl, s, d, w)
    wl, s, d, w = cache[gname]
    for N in [int(x) for x in Ns.split(",")]:
        ev = w if alg in ("sssp", "sswp") else None
        g = cusha.build_graph(wl.V, s, d, edge_values=ev, repr=repr_, vertices_per_shard=N)
        for _ in range(2):
            cusha.run(alg, g)
        ts, its, fr = [], [], []
        for _ in range(5):
            cusha.run(alg, g)
            st = cusha.get_stats(g)
            ts.append(st["run_ms"])
            its.append(st["iterations"])
            fr.append(st["algorithmic_bytes"] / st["loop_ms"] / 1e6 / PEAK)
        st = cusha.get_stats(g)
        print(json.dumps({"workload": wname, "alg": alg, "repr": repr_, "N": st["vertices_per_shard"],
                          "S": st["num_shards"], "ms": round(float(np.median(ts)), 3), "passes": its,
                          "us_per_pass": round(float(np.median(ts)) / float(np.median(its)) * 1e3, 2),
                          "frac": round(float(np.median(fr)), 4), "ring_slots": st["ring_slots"],
                          "mapper_form": st["mapper_form"]}), flush=True)
        g.close()
