"""CPU oracle for CuSha's shard-processing path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product package
(``paper_conf_hpdc_khorasanivgb14_b200``) never imports it and shares no code
with it.  The arithmetic lives in ``oracle.c`` (plain single-threaded C, fp64
for floating point); this file only marshals numpy arrays through ctypes.

Parity pins for every function are in ``tests/test_oracle_*.py`` (no GPU).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")
_lib = None

INF = 0xFFFFFFFF
OK, NOTCONV = 0, 1


def build(force: bool = False) -> str:
    """Compile liboracle.so: plain C11, single-threaded, -O2."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-std=c11", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _SO)
    return _SO


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        u64, u32, dbl, P = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_double, ctypes.c_void_p
        sig = {
            "or_bfs": [u64, u64, P, P, u32, P],
            "or_sssp": [u64, u64, P, P, P, u32, P],
            "or_sswp": [u64, u64, P, P, P, u32, P],
            "or_cc": [u64, u64, P, P, P],
            "or_pagerank": [u64, u64, P, P, dbl, dbl, u64, P, P],
            "or_nn": [u64, u64, P, P, P, P, dbl, u64, P, P],
            "or_hs": [u64, u64, P, P, P, P, dbl, u64, P, P],
            "or_cs": [u64, u64, P, P, P, P, P, dbl, u64, P, P],
            "or_build_shards": [u64, u64, P, P, u32, P, P, P, P, P, P, P, P],
            "or_pagerank_residual": [u64, u64, P, P, dbl, P, P],
            "or_trajectory": [ctypes.c_int, u64, u64, P, P, P, u32, u32, P, u64, dbl, P, P, P, P, P],
        }
        for name, args in sig.items():
            f = getattr(lib, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        _lib = lib
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _u32(a):
    return np.ascontiguousarray(a, dtype=np.uint32)


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _chk(rc, name, allow_notconv=False):
    if rc < 0 or (rc == NOTCONV and not allow_notconv):
        raise RuntimeError(f"oracle.{name} rc={rc}")
    return rc


def bfs(V, src, dst, source=0):
    src, dst = _u32(src), _u32(dst)
    out = np.empty(V, np.uint32)
    _chk(_L().or_bfs(V, len(src), _p(src), _p(dst), source, _p(out)), "bfs")
    return out


def sssp(V, src, dst, weight, source=0):
    src, dst, weight = _u32(src), _u32(dst), _u32(weight)
    out = np.empty(V, np.uint32)
    _chk(_L().or_sssp(V, len(src), _p(src), _p(dst), _p(weight), source, _p(out)), "sssp")
    return out


def sswp(V, src, dst, width, source=0):
    src, dst, width = _u32(src), _u32(dst), _u32(width)
    out = np.empty(V, np.uint32)
    _chk(_L().or_sswp(V, len(src), _p(src), _p(dst), _p(width), source, _p(out)), "sswp")
    return out


def cc(V, src, dst):
    src, dst = _u32(src), _u32(dst)
    out = np.empty(V, np.uint32)
    _chk(_L().or_cc(V, len(src), _p(src), _p(dst), _p(out)), "cc")
    return out


def pagerank(V, src, dst, damping=0.85, tol=1e-9, max_iters=100000, allow_notconv=False):
    """Returns (rank float64[V], sweeps).  allow_notconv: stopping at max_iters
    is not an error (used to time a bounded number of sweeps)."""
    src, dst = _u32(src), _u32(dst)
    out = np.empty(V, np.float64)
    it = ctypes.c_uint64(0)
    _chk(_L().or_pagerank(V, len(src), _p(src), _p(dst), damping, tol, max_iters, _p(out), ctypes.byref(it)),
         "pagerank", allow_notconv=allow_notconv)
    return out, it.value


def pagerank_residual(V, src, dst, x, damping=0.85):
    """x_v - ((1-d) + d * sum_{u->v} x_u / outdeg(u)) for a given float32 rank vector."""
    src, dst, x = _u32(src), _u32(dst), _f32(x)
    out = np.empty(V, np.float64)
    _chk(_L().or_pagerank_residual(V, len(src), _p(src), _p(dst), damping, _p(x), _p(out)), "pagerank_residual")
    return out


def nn(V, src, dst, weight, x0, tol=1e-9, max_iters=100000):
    src, dst, weight, x0 = _u32(src), _u32(dst), _f32(weight), _f32(x0)
    out = np.empty(V, np.float64)
    it = ctypes.c_uint64(0)
    _chk(_L().or_nn(V, len(src), _p(src), _p(dst), _p(weight), _p(x0), tol, max_iters, _p(out), ctypes.byref(it)), "nn")
    return out, it.value


def hs(V, src, dst, coeff, q0, tol=1e-9, max_iters=100000):
    src, dst, coeff, q0 = _u32(src), _u32(dst), _f32(coeff), _f32(q0)
    out = np.empty(V, np.float64)
    it = ctypes.c_uint64(0)
    _chk(_L().or_hs(V, len(src), _p(src), _p(dst), _p(coeff), _p(q0), tol, max_iters, _p(out), ctypes.byref(it)), "hs")
    return out, it.value


def cs(V, src, dst, G, v0, a0, tol=1e-9, max_iters=100000):
    src, dst, G, v0, a0 = _u32(src), _u32(dst), _f32(G), _f32(v0), _f32(a0)
    out = np.empty(V, np.float64)
    it = ctypes.c_uint64(0)
    _chk(_L().or_cs(V, len(src), _p(src), _p(dst), _p(G), _p(v0), _p(a0), tol, max_iters, _p(out), ctypes.byref(it)),
         "cs")
    return out, it.value


def build_shards(V, src, dst, N):
    """G-Shards + CW layout by definition. Returns a dict of numpy arrays."""
    src, dst = _u32(src), _u32(dst)
    E = len(src)
    S = (V + N - 1) // N
    r = dict(
        S=S,
        shard_off=np.empty(S + 1, np.uint64),
        gs_src=np.empty(E, np.uint32),
        gs_dst=np.empty(E, np.uint32),
        gs_eid=np.empty(E, np.uint64),
        win=np.empty((S + 1) * S, np.uint64),
        cw_off=np.empty(S + 1, np.uint64),
        cw_src=np.empty(E, np.uint32),
        mapper=np.empty(E, np.uint64),
    )
    _chk(_L().or_build_shards(V, E, _p(src), _p(dst), N, _p(r["shard_off"]), _p(r["gs_src"]), _p(r["gs_dst"]),
                              _p(r["gs_eid"]), _p(r["win"]), _p(r["cw_off"]), _p(r["cw_src"]), _p(r["mapper"])),
         "build_shards")
    r["win"] = r["win"].reshape(S + 1, S)
    return r


ALGS = {"bfs": 0, "sssp": 1, "pr": 2, "cc": 3, "sswp": 4, "nn": 5, "hs": 6, "cs": 7}


def trajectory(alg, V, src, dst, N, ev=None, source=0, init=None, max_passes=100000, tol=1e-5):
    """Mode T (oracle.c or_trajectory): the paper's Fig. 5 pass, shard by shard
    with |N| = N, under the two-phase BSP schedule.  ev: raw 4-byte EdgeValue
    per input edge (u32 or f32 array); init: NN x0 / HS Q0 (f32[V]) or CS
    {V0, GsumOrA0} (f32[V, 2]).  Returns dict(values, passes, updated,
    active_shards, converged): values u32[V] (integer algorithms) or f64[V]
    (PR Rank, NN x, HS Q, CS V)."""
    a = ALGS[alg] if isinstance(alg, str) else int(alg)
    src, dst = _u32(src), _u32(dst)
    evb = None if ev is None else np.ascontiguousarray(ev).view(np.uint32)
    ini = None if init is None else np.ascontiguousarray(init, dtype=np.float32).reshape(-1)
    integer = a in (0, 1, 3, 4)
    ou = np.empty(V, np.uint32) if integer else None
    of = None if integer else np.empty(V, np.float64)
    cap = int(max_passes)
    upd = np.zeros(cap, np.uint32)
    act = np.zeros(cap, np.uint32)
    n = ctypes.c_uint64(0)
    rc = _L().or_trajectory(a, V, len(src), _p(src), _p(dst), _p(evb), N, source, _p(ini), cap, tol, _p(ou), _p(of),
                            _p(upd), _p(act), ctypes.byref(n))
    _chk(rc, "trajectory", allow_notconv=True)
    k = int(n.value)
    return {"values": ou if integer else of, "passes": k, "updated": upd[:k], "active_shards": act[:k],
            "converged": rc == OK}
