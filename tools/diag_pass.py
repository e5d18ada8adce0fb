"""Per-stage cost split of the shard pass (diagnostic, not a benchmark).

Times PR passes on a workload with diagnostic builds of libcusha.so
(CUSHA_DIAG bits, csrc/kernels.cu): every shard forced active, then with the
stage-2 reduction and/or the stage-4 stores removed.  Results of these builds
are wrong by design; only the per-pass time is read.
usage: python tools/diag_pass.py <workload> <alg> lib1.so [lib2.so ...]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen  # noqa: E402
from paper_conf_hpdc_khorasanivgb14_b200 import cusha  # noqa: E402

wname, alg, libs = sys.argv[1], sys.argv[2], sys.argv[3:]
wl = graphgen.workload(wname, cache_dir="/tmp/gg")
src = torch.from_numpy(wl.src.view(np.int32)).cuda()
dst = torch.from_numpy(wl.dst.view(np.int32)).cuda()
ev = torch.from_numpy(wl.edge_u32.view(np.int32)).cuda() if alg in ("sssp", "sswp") else None
for path in libs:
    # a fresh process would be cleaner; ctypes can load several copies side by side
    cusha._lib = None
    cusha.LIB_PATH = os.path.abspath(path)
    with cusha.build_graph(wl.V, src, dst, edge_values=ev, repr="cw") as g:
        cusha.run(alg, g, max_iters=30)
        t = []
        for _ in range(3):
            cusha.run(alg, g, max_iters=30)
            st = cusha.get_stats(g)
            t.append(st["loop_ms"] / max(st["iterations"], 1) * 1e3)
        print(f"{os.path.basename(path)}: {np.median(t):.1f} us/pass over {st['iterations']} passes", flush=True)
