"""Small test-side helpers: brute force on tiny graphs, golden-file parsing.

Nothing here is used by the product path.  The brute-force routines are
deliberately naive (path enumeration, boolean matrix closure, dense solves) so
that they pin the oracle through a different computation.
"""
from __future__ import annotations

import itertools
import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
INF = 0xFFFFFFFF


def read_golden(name):
    out = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            k, v = [t.strip() for t in line.split("=", 1)]
            out[k] = [int(x) for x in v.split(",")] if "," in v else int(v)
    return out


def random_simple_graph(rng, V, E, allow_dups=False):
    """Random directed graph without self-loops (and without duplicates unless
    allow_dups)."""
    if allow_dups:
        s = rng.integers(0, V, E)
        d = rng.integers(0, V, E)
        keep = s != d
        return s[keep].astype(np.uint32), d[keep].astype(np.uint32)
    pairs = [(u, v) for u in range(V) for v in range(V) if u != v]
    idx = rng.choice(len(pairs), size=min(E, len(pairs)), replace=False)
    s = np.array([pairs[i][0] for i in idx], np.uint32)
    d = np.array([pairs[i][1] for i in idx], np.uint32)
    return s, d


def simple_paths(V, src, dst, source):
    """Yield every simple path from source as a list of edge indices (tiny graphs)."""
    out = [[] for _ in range(V)]
    for e, (u, v) in enumerate(zip(src.tolist(), dst.tolist())):
        out[u].append((v, e))

    def rec(u, seen, path):
        yield u, path
        for v, e in out[u]:
            if v not in seen:
                seen.add(v)
                yield from rec(v, seen, path + [e])
                seen.discard(v)

    yield from rec(source, {source}, [])


def reach_matrix(V, src, dst):
    """Boolean reflexive-transitive closure by repeated squaring."""
    R = np.eye(V, dtype=bool)
    R[src, dst] = True
    while True:
        R2 = R | ((R.astype(np.int64) @ R.astype(np.int64)) > 0)
        if (R2 == R).all():
            return R
        R = R2
