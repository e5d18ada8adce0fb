"""Seeded synthetic inputs shared by the oracle (``oracle/``) and the CUDA path.

This package holds none of CuSha's arithmetic: it only draws edge lists and
random per-edge / per-vertex values (counter-based, thread-count invariant),
following the input recipe in DESIGN.md ("Input recipe").

The C implementation lives in ``graphgen.c`` and is compiled to
``libgraphgen.so`` next to it (``build()`` / on first use).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libgraphgen.so")
_SRC = os.path.join(_HERE, "graphgen.c")
_lib = None

INF = 0xFFFFFFFF


def build(force: bool = False) -> str:
    """Compile libgraphgen.so (plain C, OpenMP)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-shared", "-fPIC", "-std=c11", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _SO)
    return _SO


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        u64, u32, i32, dbl, flt = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int, ctypes.c_double, ctypes.c_float
        P = ctypes.c_void_p
        lib.gg_rmat.argtypes = [u64, u64, u64, dbl, dbl, dbl, i32, i32, P, P]
        lib.gg_mesh.argtypes = [u64, u64, u64, u64, i32, P, P]
        lib.gg_uniform.argtypes = [u64, u64, u64, P, P]
        lib.gg_edge_u32.argtypes = [u64, P, P, u64, u32, u32, i32, P]
        lib.gg_edge_f32.argtypes = [u64, P, P, u64, flt, flt, i32, P]
        lib.gg_vertex_f32.argtypes = [u64, u64, u64, flt, flt, P]
        lib.gg_permute_vertex.argtypes = [u64, u64, u64, P, P, u64]
        lib.gg_hash.argtypes = [u64, u64, u64]
        lib.gg_hash.restype = u64
        for f in ("gg_rmat", "gg_mesh", "gg_uniform", "gg_edge_u32", "gg_edge_f32", "gg_vertex_f32", "gg_permute_vertex"):
            getattr(lib, f).restype = i32
        _lib = lib
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _chk(rc: int, what: str):
    if rc != 0:
        raise RuntimeError(f"graphgen.{what} failed rc={rc}")


def rmat(V: int, E: int, seed: int, a=0.57, b=0.19, c=0.19, symmetric=False, permute=True):
    """R-MAT edge list with exactly E unique directed edges (or E undirected
    pairs stored both ways when symmetric). Returns (src, dst) uint32, sorted."""
    n = 2 * E if symmetric else E
    src = np.empty(n, np.uint32)
    dst = np.empty(n, np.uint32)
    _chk(_L().gg_rmat(V, E, seed, a, b, c, int(symmetric), int(permute), _p(src), _p(dst)), "rmat")
    return src, dst


def mesh(V: int, width: int, pairs: int, seed: int, permute=True):
    src = np.empty(2 * pairs, np.uint32)
    dst = np.empty(2 * pairs, np.uint32)
    _chk(_L().gg_mesh(V, width, pairs, seed, int(permute), _p(src), _p(dst)), "mesh")
    return src, dst


def uniform(V: int, E: int, seed: int):
    src = np.empty(E, np.uint32)
    dst = np.empty(E, np.uint32)
    _chk(_L().gg_uniform(V, E, seed, _p(src), _p(dst)), "uniform")
    return src, dst


def edge_u32(src, dst, seed: int, lo: int, hi: int, symmetric=False):
    src = np.ascontiguousarray(src, np.uint32)
    dst = np.ascontiguousarray(dst, np.uint32)
    out = np.empty(len(src), np.uint32)
    _chk(_L().gg_edge_u32(len(src), _p(src), _p(dst), seed, lo, hi, int(symmetric), _p(out)), "edge_u32")
    return out


def edge_f32(src, dst, seed: int, lo: float, hi: float, symmetric=False):
    src = np.ascontiguousarray(src, np.uint32)
    dst = np.ascontiguousarray(dst, np.uint32)
    out = np.empty(len(src), np.float32)
    _chk(_L().gg_edge_f32(len(src), _p(src), _p(dst), seed, lo, hi, int(symmetric), _p(out)), "edge_f32")
    return out


def vertex_f32(V: int, seed: int, stream: int, lo: float, hi: float):
    out = np.empty(V, np.float32)
    _chk(_L().gg_vertex_f32(V, seed, stream, lo, hi, _p(out)), "vertex_f32")
    return out


def hash64(seed: int, stream: int, k: int) -> int:
    return int(_L().gg_hash(seed, stream, k))


def permute_vertices(n: int, seed: int, anchor: int, v) -> np.ndarray:
    v = np.ascontiguousarray(v, np.uint32)
    out = np.empty_like(v)
    _chk(_L().gg_permute_vertex(n, seed, anchor, _p(v), _p(out), len(v)), "permute")
    return out


# --------------------------------------------------------------------------
# Workload recipes (BASELINE.json configs)
# --------------------------------------------------------------------------

@dataclass
class Workload:
    name: str
    V: int
    src: np.ndarray
    dst: np.ndarray
    edge_u32: Optional[np.ndarray] = None     # SSSP weight / SSWP width
    meta: dict = field(default_factory=dict)

    @property
    def E(self) -> int:
        return int(len(self.src))


def workload(name: str, cache_dir: Optional[str] = None) -> Workload:
    """The synthetic graphs of BASELINE.json configs (C1..C5) and small extras.

    C1: R-MAT scale 12, V=4096, E=32768, seed 1 (BFS from 0).
    C2: LiveJournal-shaped R-MAT, V=4,847,571, E=68,993,773, seed 2 (PR).
    C3: RoadNet-CA-shaped mesh, V=1,971,281, width 1404, 2,766,607 bonds both
        ways (E=5,533,214), weights U[1,255] symmetric, seed 3 (SSSP).
    C4: HiggsTwitter-shaped symmetric R-MAT, V=456,631, 7,427,937 pairs
        (E=14,855,874), widths U[1,255] symmetric, seed 4 (CC, SSWP).
    C5: R-MAT scale 26, V=2^26, E=2^30, seed 5 (PR, BFS).
    R27 / R28: R-MAT scale 27 / 28, edge factor 16 / 15, seeds 9 / 10 (row f3,
        graphs near / beyond one GPU's HBM).
    """
    if cache_dir:
        path = os.path.join(cache_dir, f"graphgen_{name}.npz")
        if os.path.exists(path):
            z = np.load(path, allow_pickle=False)
            return Workload(name, int(z["V"]), z["src"], z["dst"], z["w"] if z["w"].size else None)
    w = None
    if name == "C1":
        V = 4096
        src, dst = rmat(V, 32768, seed=1)
        w = edge_u32(src, dst, seed=1, lo=1, hi=255)
    elif name == "C2":
        V = 4_847_571
        src, dst = rmat(V, 68_993_773, seed=2)
    elif name == "C3":
        V = 1_971_281
        src, dst = mesh(V, 1404, 2_766_607, seed=3)
        w = edge_u32(src, dst, seed=3, lo=1, hi=255, symmetric=True)
    elif name == "C3o":
        # C3 in the mesh's natural row-major vertex order (no id permutation):
        # shards are bands of rows, as in a road network numbered by locality
        V = 1_971_281
        src, dst = mesh(V, 1404, 2_766_607, seed=3, permute=False)
        w = edge_u32(src, dst, seed=3, lo=1, hi=255, symmetric=True)
    elif name == "C4":
        V = 456_631
        src, dst = rmat(V, 7_427_937, seed=4, symmetric=True)
        w = edge_u32(src, dst, seed=4, lo=1, hi=255, symmetric=True)
    elif name == "C5":
        V = 1 << 26
        src, dst = rmat(V, 1 << 30, seed=5)
    elif name in ("R27", "R28"):
        # row f3 (L455): R-MAT scale 27 (edge factor 16) / 28 (edge factor 15:
        # 4.03 G edges, below the ABI's 2^32 - 2^26 limit), seeds 9 / 10
        k = 27 if name == "R27" else 28
        V = 1 << k
        src, dst = rmat(V, (16 if k == 27 else 15) << k, seed=k - 18)
    elif name.startswith("rmat:"):
        # rmat:V:E:seed  (parity-test sizes)
        _, V, E, seed = name.split(":")
        V, E, seed = int(V), int(E), int(seed)
        src, dst = rmat(V, E, seed=seed)
        w = edge_u32(src, dst, seed=seed, lo=1, hi=255)
    elif name.startswith("rmatsym:"):
        _, V, P, seed = name.split(":")
        V, P, seed = int(V), int(P), int(seed)
        src, dst = rmat(V, P, seed=seed, symmetric=True)
        w = edge_u32(src, dst, seed=seed, lo=1, hi=255, symmetric=True)
    elif name.startswith("mesh:"):
        _, V, width, P, seed = name.split(":")
        V, width, P, seed = int(V), int(width), int(P), int(seed)
        src, dst = mesh(V, width, P, seed=seed)
        w = edge_u32(src, dst, seed=seed, lo=1, hi=255, symmetric=True)
    else:
        raise KeyError(name)
    wl = Workload(name, V, src, dst, w)
    if cache_dir and wl.E < (1 << 28):  # scale-26 lists (8.6 GB) are regenerated rather than cached
        os.makedirs(cache_dir, exist_ok=True)
        tmp = path + ".tmp%d.npz" % os.getpid()
        np.savez(tmp, V=np.int64(V), src=src, dst=dst, w=w if w is not None else np.zeros(0, np.uint32))
        os.replace(tmp, path)
    return wl
