#!/usr/bin/env python
"""Expected values for the C5 PageRank parity test, written by the ORACLE only.

    python tools/golden_c5_pr.py            (~40 min single-threaded on the dev host)

C5 = R-MAT scale 26 (BASELINE.json configs[4]; graphgen.workload("C5")).  Runs
oracle.pagerank (fp64 Jacobi of Table 3, R6-R8) to max |dx| <= 1e-9
(north_star) and writes
  tests/golden/c5_pr_sample.npz      committed: a seeded sample of 200,000
                                     vertices plus the 2,000 largest x*, their
                                     x* (fp64), the sweep count, the mass sum,
                                     and the SHA-256 of the full fp64 vector;
  tests/golden_cache/c5_pr_xstar.f32 git-ignored: the full x* vector rounded
                                     to float32 (268 MB; relative rounding
                                     6e-8, far inside the 1e-4 bound) for the
                                     element-by-element leg of
                                     tests/test_gpu_fullsize.py, when present.
Nothing here reads the CUDA path."""
import hashlib
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import graphgen  # noqa: E402
import oracle  # noqa: E402


def main():
    t = time.time()
    wl = graphgen.workload("C5")
    print(f"C5 generated: V={wl.V} E={wl.E} in {time.time() - t:.0f}s", flush=True)
    t = time.time()
    x, sweeps = oracle.pagerank(wl.V, wl.src, wl.dst, tol=1e-9)
    print(f"oracle.pagerank: {sweeps} sweeps in {time.time() - t:.0f}s", flush=True)
    digest = hashlib.sha256(x.tobytes()).hexdigest()
    rng = np.random.default_rng(20261017)
    idx = np.unique(np.concatenate([rng.choice(wl.V, 200_000, replace=False),
                                    np.argsort(x)[-2000:], np.arange(16)])).astype(np.uint32)
    np.savez_compressed(os.path.join(ROOT, "tests", "golden", "c5_pr_sample.npz"), idx=idx, xstar=x[idx],
                        sweeps=np.int64(sweeps), V=np.int64(wl.V), E=np.int64(wl.E), mass=np.float64(x.sum()),
                        sha256=np.array(digest), tol=np.float64(1e-9))
    os.makedirs(os.path.join(ROOT, "tests", "golden_cache"), exist_ok=True)
    x.astype(np.float32).tofile(os.path.join(ROOT, "tests", "golden_cache", "c5_pr_xstar.f32"))
    print(f"wrote sample ({idx.size} vertices) and full vector; sha256 {digest}", flush=True)


if __name__ == "__main__":
    main()
