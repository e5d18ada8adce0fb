"""Generate C5 (R-MAT scale 26) and time it; then run BFS and PR once on the GPU and
check BFS bit-exact against the oracle (textbook O(V+E) BFS)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import graphgen, oracle
from paper_conf_hpdc_khorasanivgb14_b200 import cusha
t = time.time(); wl = graphgen.workload("C5"); print(f"gen {time.time()-t:.1f}s V={wl.V} E={wl.E}", flush=True)
s_d = torch.from_numpy(wl.src.view(np.int32)).cuda(); d_d = torch.from_numpy(wl.dst.view(np.int32)).cuda()
N = int(sys.argv[1]) if len(sys.argv) > 1 else 0
for alg in ("bfs", "pr"):
    t = time.time()
    g = cusha.build_graph(wl.V, s_d, d_d, repr="cw", vertices_per_shard=N)
    st = cusha.get_stats(g); print(f"build {time.time()-t:.1f}s N={st['vertices_per_shard']} S={st['num_shards']} dev_bytes={st['device_bytes']/1e9:.1f}GB", flush=True)
    for k in range(2):
        rc = cusha.run(alg, g)
        st = cusha.get_stats(g)
        print(f"{alg} rc={rc} it={st['iterations']} run_ms={st['run_ms']:.1f} pass_us={st['loop_ms']/max(st['iterations'],1)*1e3:.0f} GB/s={st['algorithmic_bytes']/st['loop_ms']/1e6:.0f} GTEPS={st['edges_processed']/st['run_ms']/1e6:.1f}", flush=True)
    vals = cusha.get_values(g); g.close()
    if alg == "bfs":
        t = time.time(); ref = oracle.bfs(wl.V, wl.src, wl.dst, 0); print(f"oracle bfs {time.time()-t:.1f}s equal={np.array_equal(vals, ref)}", flush=True)
