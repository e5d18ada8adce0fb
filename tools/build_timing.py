"""Time cusha_build_graph phases (CUSHA_DEBUG_BUILD=1) for a workload, host and device inputs."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if "--quiet" not in sys.argv:
    os.environ["CUSHA_DEBUG_BUILD"] = "1"
sys.argv = [a for a in sys.argv if a != "--quiet"]
import numpy as np, torch
import graphgen
from paper_conf_hpdc_khorasanivgb14_b200 import cusha
wl = graphgen.workload(sys.argv[1] if len(sys.argv) > 1 else "C2", cache_dir="/tmp/gg")
repr_ = sys.argv[2] if len(sys.argv) > 2 else "cw"
ps = torch.from_numpy(wl.src.view(np.int32)).pin_memory()
pd = torch.from_numpy(wl.dst.view(np.int32)).pin_memory()
for k in range(int(os.environ.get("BT_REPS", "3"))):
    torch.cuda.synchronize()
    t = time.perf_counter()
    g = cusha.build_graph(wl.V, ps.numpy().view(np.uint32), pd.numpy().view(np.uint32), repr=repr_)
    t1 = time.perf_counter()
    st = cusha.get_stats(g)
    print(f"build {k}: wall {1e3*(t1-t):.1f} ms  build_ms {st['build_ms']:.1f}  h2d_ms {st['h2d_ms']:.1f}", flush=True)
    t = time.perf_counter(); g.close(); print(f"free {1e3*(time.perf_counter()-t):.1f} ms", flush=True)
