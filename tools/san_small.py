import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np
import graphgen, oracle
from paper_conf_hpdc_khorasanivgb14_b200 import cusha
V = 20000
s, d = graphgen.rmat(V, 200000, seed=71)
w = graphgen.edge_u32(s, d, seed=71, lo=1, hi=255)
for repr_ in ("gs", "cw"):
    for alg in ("bfs", "sssp", "pr", "cc"):
        with cusha.build_graph(V, s, d, edge_values=w if alg == "sssp" else None, repr=repr_, vertices_per_shard=500) as g:
            cusha.run(alg, g, source=0)
            x = cusha.get_values(g)
        print(repr_, alg, "ok", flush=True)
