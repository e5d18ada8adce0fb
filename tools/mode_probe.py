"""Overlapped passes vs per-pass barrier on an R-MAT "i_j" graph at a given |N| (SSSP, CW).
usage: python tools/mode_probe.py <i> <j> <N> [repr]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen  # noqa: E402
from paper_conf_hpdc_khorasanivgb14_b200 import cusha  # noqa: E402

i, j, N = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
repr_ = sys.argv[4] if len(sys.argv) > 4 else "cw"
M = 1 << 20
V, E = j * M, i * M
s, d = graphgen.rmat(V, E, seed=11)
w = graphgen.edge_u32(s, d, seed=11, lo=1, hi=255)
S_, D_, W_ = (torch.from_numpy(x.view(np.int32)).cuda() for x in (s, d, w))
for barrier in (False, True):
    with cusha.build_graph(V, S_, D_, edge_values=W_, repr=repr_, vertices_per_shard=N, pass_barrier=barrier) as g:
        t = []
        for _ in range(4):
            cusha.run("sssp", g, source=0)
            st = cusha.get_stats(g)
            t.append((st["run_ms"], st["iterations"], st["loop_ms"] / max(st["iterations"], 1) * 1e3))
        t = t[1:]
        print(f"{i}_{j} N={N} S={st['num_shards']} barrier={barrier}: run_ms {np.median([x[0] for x in t]):.3f} "
              f"passes {[x[1] for x in t]} us/pass {np.median([x[2] for x in t]):.1f}", flush=True)
