"""Break an e2e step (build from pinned host buffers, run, D2H values, free) into parts."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import graphgen
from paper_conf_hpdc_khorasanivgb14_b200 import cusha
wl = graphgen.workload(sys.argv[1] if len(sys.argv) > 1 else "C2", cache_dir="/tmp/gg")
alg = sys.argv[2] if len(sys.argv) > 2 else "pr"
ps = torch.from_numpy(wl.src.view(np.int32)).pin_memory()
pd = torch.from_numpy(wl.dst.view(np.int32)).pin_memory()
out = torch.empty(wl.V * 2, dtype=torch.int32).pin_memory()
stream = torch.cuda.current_stream().cuda_stream
for k in range(4):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    g = cusha.build_graph(wl.V, ps.numpy().view(np.uint32), pd.numpy().view(np.uint32), repr="cw", stream=stream)
    t1 = time.perf_counter()
    cusha.run(alg, g)
    t2 = time.perf_counter()
    rc = cusha.lib().cusha_get_values(g.handle, cusha._ptr(out), wl.V * 4)
    t3 = time.perf_counter()
    st = cusha.get_stats(g)
    g.close()
    t4 = time.perf_counter()
    print(f"step {k}: build {1e3*(t1-t0):.1f} run {1e3*(t2-t1):.1f} (run_ms {st['run_ms']:.1f}, it {st['iterations']}) get {1e3*(t3-t2):.1f} free {1e3*(t4-t3):.1f} ms", flush=True)
