"""Thin ctypes binding of include/cusha.h — argument marshalling only.

Every step of the path (build, iteration, convergence) runs inside
libcusha.so (hand-written sm_100a kernels); this module converts numpy arrays
/ torch CUDA tensors to pointers and return codes to exceptions.  There is no
CPU fallback: if libcusha.so is missing the import fails loudly.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libcusha.so")

# --- enums (include/cusha.h) ---
BFS, SSSP, PR, CC, SSWP, NN, HS, CS = range(8)
ALGORITHMS = {"bfs": BFS, "sssp": SSSP, "pr": PR, "cc": CC, "sswp": SSWP, "nn": NN, "hs": HS, "cs": CS}
REPR_GSHARDS, REPR_CW = 0, 1
REPRS = {"gs": REPR_GSHARDS, "gshards": REPR_GSHARDS, "cw": REPR_CW}
INPUT_HOST, INPUT_DEVICE = 0, 1
OK, NOT_CONVERGED = 0, 1
EINVAL, ENOMEM, ECUDA, ENCCL, EUNSUPPORTED, ESTATE = -1, -2, -3, -4, -5, -6
INF = 0xFFFFFFFF

LAYOUT = {
    "shard_offsets": (0, np.uint32), "shard_sizes": (1, np.uint32), "src_index": (2, np.uint16),
    "dest_local": (3, np.uint16), "edge_id": (4, np.uint32), "windows": (5, np.uint32),
    "cw_offsets": (6, np.uint32), "cw_sizes": (7, np.uint32), "cw_src_local": (8, np.uint16),
    "mapper": (9, np.uint32), "out_degree": (10, np.uint32), "run_k": (11, np.uint32), "run_t": (12, np.uint32),
    "cw_window": (13, np.uint16), "cw_delta": (14, np.uint32), "cw_partition_offsets": (15, np.uint32),
}


class BuildOpts(ctypes.Structure):
    _fields_ = [
        ("repr", ctypes.c_int),
        ("vertices_per_shard", ctypes.c_uint32),
        ("smem_bytes_per_vertex", ctypes.c_uint32),
        ("device", ctypes.c_int),
        ("stream", ctypes.c_void_p),
        ("input_location", ctypes.c_int),
        ("host_loop", ctypes.c_int),
        ("world_size", ctypes.c_int),
        ("rank", ctypes.c_int),
        ("nccl_unique_id", ctypes.c_void_p),
        ("skip_clean_shards", ctypes.c_int),
        ("device_topology_budget", ctypes.c_uint64),
        ("pass_barrier", ctypes.c_int),
        ("keep_layout", ctypes.c_int),
        ("mode", ctypes.c_int),
        ("comm_timeout_ms", ctypes.c_uint32),
        ("transport", ctypes.c_int),
    ]


class Stats(ctypes.Structure):
    _fields_ = [
        ("num_vertices", ctypes.c_uint32),
        ("num_edges", ctypes.c_uint64),
        ("vertices_per_shard", ctypes.c_uint32),
        ("num_shards", ctypes.c_uint32),
        ("repr", ctypes.c_uint32),
        ("last_algorithm", ctypes.c_int32),
        ("iterations", ctypes.c_uint32),
        ("converged", ctypes.c_uint32),
        ("build_ms", ctypes.c_double),
        ("h2d_ms", ctypes.c_double),
        ("run_ms", ctypes.c_double),
        ("loop_ms", ctypes.c_double),
        ("h2d_bytes", ctypes.c_uint64),
        ("device_bytes", ctypes.c_uint64),
        ("entries_padded", ctypes.c_uint64),
        ("stage2_bytes_per_iter", ctypes.c_uint64),
        ("wb_bytes_all_active", ctypes.c_uint64),
        ("algorithmic_bytes", ctypes.c_uint64),
        ("edges_processed", ctypes.c_uint64),
        ("device_loop", ctypes.c_uint32),
        ("world_size", ctypes.c_int),
        ("rank", ctypes.c_int),
        ("host_bytes", ctypes.c_uint64),
        ("host_shard", ctypes.c_uint32),
        ("mapper_form", ctypes.c_uint32),
        ("paper_bytes", ctypes.c_uint64),
        ("wb_entries", ctypes.c_uint64),
        ("vertices_processed", ctypes.c_uint64),
        ("updated_total", ctypes.c_uint64),
        ("partitions", ctypes.c_uint32),
        ("max_in_degree", ctypes.c_uint32),
        ("max_part_device_bytes", ctypes.c_uint64),
        ("ring_slots", ctypes.c_uint32),
        ("l2_read_ahead", ctypes.c_uint32),
    ]


_lib = None


def lib():
    """Load libcusha.so (raises if it was not built: no fallback exists)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: build it with "
                              "`python -m paper_conf_hpdc_khorasanivgb14_b200.build` (nvcc, sm_100a)")
        L = ctypes.CDLL(LIB_PATH)
        P, u32, u64, i32, sz = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, ctypes.c_size_t
        sigs = {
            "cusha_build_graph": (i32, [u32, u64, P, P, P, ctypes.POINTER(BuildOpts), ctypes.POINTER(P)]),
            "cusha_free_graph": (None, [P]),
            "cusha_set_vertex_values": (i32, [P, i32, P, sz]),
            "cusha_run": (i32, [i32, P, u32, u32]),
            "cusha_get_values": (i32, [P, P, sz]),
            "cusha_get_values_device": (i32, [P, P, sz]),
            "cusha_get_stats": (i32, [P, ctypes.POINTER(Stats)]),
            "cusha_get_trace": (i32, [P, P, P, u32]),
            "cusha_get_layout": (i32, [P, i32, P, sz, ctypes.POINTER(u64)]),
            "cusha_get_part_layout": (i32, [P, u32, i32, P, sz, ctypes.POINTER(u64)]),
            "cusha_get_part_stats": (i32, [P, u32, ctypes.POINTER(Stats)]),
            "cusha_trim_memory": (i32, [i32]),
            "cusha_ipc_export": (i32, [P, P, sz]),
            "cusha_ipc_connect": (i32, [P, P, sz]),
            "cusha_shard_size": (u32, [u32, u64, u32, u32, u32]),
            "cusha_value_bytes": (sz, [i32]),
            "cusha_last_error": (ctypes.c_char_p, []),
            "cusha_abi_version": (i32, []),
            "cusha_nccl_unique_id": (i32, [P]),
            "cusha_partition_shards": (i32, [u32, P, u32, P]),
            "cusha_get_partition": (i32, [P, P, u32]),
            "cusha_diag_timeline": (i32, [P, sz]),
        }
        for name, (res, args) in sigs.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


class CushaError(RuntimeError):
    def __init__(self, code: int, where: str):
        msg = lib().cusha_last_error().decode(errors="replace")
        super().__init__(f"{where} failed ({code}): {msg}")
        self.code = code


def _check(rc: int, where: str, ok=(OK,)):
    if rc not in ok:
        raise CushaError(rc, where)
    return rc


def _alg(a) -> int:
    return ALGORITHMS[a.lower()] if isinstance(a, str) else int(a)


def _ptr(x):
    """numpy array -> host pointer; torch tensor -> data_ptr; None -> None."""
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        return x.ctypes.data_as(ctypes.c_void_p)
    if hasattr(x, "data_ptr"):
        return ctypes.c_void_p(x.data_ptr())
    raise TypeError(type(x))


def _is_device(x) -> bool:
    return hasattr(x, "is_cuda") and bool(x.is_cuda)


def _check_device_tensor(name, t, device, float_ok=False):
    """A CUDA tensor passed to the C ABI is read as packed 4-byte values on
    `device`: int32 / uint32 (float32 too for edge values), contiguous."""
    import torch
    ok = (torch.int32, torch.uint32) + ((torch.float32,) if float_ok else ())
    if t.dtype not in ok:
        raise TypeError(f"{name}: dtype {t.dtype} is not one of {ok} (the C ABI reads packed 4-byte values)")
    if not t.is_contiguous():
        raise ValueError(f"{name}: tensor must be contiguous")
    if t.device.index != device:
        raise ValueError(f"{name}: tensor is on cuda:{t.device.index}, the graph is built on cuda:{device}")


class Graph:
    """Owning handle of a cusha_graph (freed on close / garbage collection)."""

    def __init__(self, handle: int, V: int, E: int):
        self.handle = ctypes.c_void_p(handle)
        self.V, self.E = V, E

    def close(self):
        if self.handle:
            lib().cusha_free_graph(self.handle)
            self.handle = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def _preload_nccl():
    """libcusha dlopen()s libnccl.so.2; make torch's copy resolvable by that name."""
    try:
        import nvidia.nccl
        p = os.path.join(list(nvidia.nccl.__path__)[0], "lib", "libnccl.so.2")
        if os.path.exists(p):
            ctypes.CDLL(p, mode=ctypes.RTLD_GLOBAL)
    except Exception:
        pass


def nccl_unique_id() -> bytes:
    """cusha_nccl_unique_id: 128 bytes for rank 0 to broadcast."""
    _preload_nccl()
    buf = ctypes.create_string_buffer(128)
    _check(lib().cusha_nccl_unique_id(buf), "cusha_nccl_unique_id")
    return buf.raw


def partition_shards(work, parts: int) -> np.ndarray:
    """cusha_partition_shards (host logic): G+1 shard bounds of near-equal work."""
    work = np.ascontiguousarray(work, dtype=np.uint64)
    out = np.zeros(parts + 1, np.uint32)
    _check(lib().cusha_partition_shards(len(work), _ptr(work), parts, _ptr(out)), "cusha_partition_shards")
    return out


def get_partition(g: "Graph") -> np.ndarray:
    out = np.zeros(65, np.uint32)
    k = lib().cusha_get_partition(g.handle, _ptr(out), 65)
    if k < 0:
        raise CushaError(k, "cusha_get_partition")
    return out[:k + 1]


def build_graph(num_vertices: int, src, dst, edge_values=None, repr="gs", vertices_per_shard: int = 0,
                smem_bytes_per_vertex: int = 0, device: int = 0, stream: Optional[int] = None,
                host_loop: bool = False, world_size: int = 1, rank: int = 0,
                nccl_id: Optional[bytes] = None, skip_clean_shards: bool = False,
                device_topology_budget: int = 0, pass_barrier: int = 0, keep_layout: bool = False,
                mode="async", transport: str = "nccl", comm_timeout_ms: int = 0) -> Graph:
    """cusha_build_graph.  src/dst/edge_values: numpy (host, copied in) or CUDA tensors (device).
    world_size > 1: destination-range partition; nccl_id = None simulates all
    partitions on this device, else one process per GPU over NCCL.
    skip_clean_shards: opt-in exact skipping of shards whose inputs did not change.
    device_topology_budget: HBM bytes for per-entry topology; the rest is streamed from pinned host memory.
    pass_barrier: True / 1 = one launch per pass with a device-wide barrier between passes (Fig. 5);
    2 = always overlapped passes (one launch per run); False / 0 = automatic (overlapped unless the
    graph has many small shards per CTA, include/cusha.h).
    keep_layout: keep the arrays only get_layout reads (input edge index per entry, CW window table).
    mode: "async" (the paper's schedule) or "bsp" (two-phase: each pass reads the previous pass's SrcValues).
    CUDA tensors must be int32/uint32 (edge_values also float32), contiguous and on `device`; with
    stream=None they are read on torch's current stream."""
    on_dev = _is_device(src)
    if on_dev:
        import torch
        if not (_is_device(dst) and (edge_values is None or _is_device(edge_values))):
            raise ValueError("src, dst and edge_values must all be CUDA tensors or all host arrays")
        _check_device_tensor("src", src, device)
        _check_device_tensor("dst", dst, device)
        if edge_values is not None:
            _check_device_tensor("edge_values", edge_values, device, float_ok=True)
        if stream is None:
            # build (and run) on torch's current stream: stream order covers the
            # kernels that produced the tensors
            stream = torch.cuda.current_stream(device).cuda_stream
    else:
        src = np.ascontiguousarray(src, dtype=np.uint32)
        dst = np.ascontiguousarray(dst, dtype=np.uint32)
        if edge_values is not None:
            edge_values = np.ascontiguousarray(edge_values)
            if edge_values.dtype not in (np.uint32, np.float32):
                raise TypeError("edge_values must be uint32 or float32")
    if len(src) != len(dst) or (edge_values is not None and len(edge_values) != len(src)):
        raise ValueError("src/dst/edge_values lengths differ")
    o = BuildOpts()
    o.repr = REPRS[repr] if isinstance(repr, str) else int(repr)
    o.vertices_per_shard = vertices_per_shard
    o.smem_bytes_per_vertex = smem_bytes_per_vertex
    o.device = device
    o.stream = stream
    o.input_location = INPUT_DEVICE if on_dev else INPUT_HOST
    o.host_loop = int(host_loop)
    o.world_size = world_size
    o.rank = rank
    o.skip_clean_shards = int(skip_clean_shards)
    o.device_topology_budget = int(device_topology_budget)
    o.pass_barrier = int(pass_barrier)
    o.keep_layout = int(keep_layout)
    o.mode = {"async": 0, "bsp": 1}[mode] if isinstance(mode, str) else int(mode)
    o.transport = {"nccl": 0, "ipc": 1}[transport] if isinstance(transport, str) else int(transport)
    o.comm_timeout_ms = int(comm_timeout_ms)
    idbuf = None
    if nccl_id is not None:
        if len(nccl_id) != 128:
            raise ValueError("nccl_id must be 128 bytes")
        _preload_nccl()
        idbuf = ctypes.create_string_buffer(bytes(nccl_id), 128)
        o.nccl_unique_id = ctypes.cast(idbuf, ctypes.c_void_p)
    h = ctypes.c_void_p()
    _check(lib().cusha_build_graph(num_vertices, len(src), _ptr(src), _ptr(dst), _ptr(edge_values),
                                   ctypes.byref(o), ctypes.byref(h)), "cusha_build_graph")
    return Graph(h.value, num_vertices, len(src))


IPC_BLOB_BYTES = 256


def ipc_export(g: Graph) -> bytes:
    """cusha_ipc_export: this rank's CUDA IPC handles (one process per GPU)."""
    buf = ctypes.create_string_buffer(IPC_BLOB_BYTES)
    _check(lib().cusha_ipc_export(g.handle, buf, IPC_BLOB_BYTES), "cusha_ipc_export")
    return buf.raw


def ipc_connect(g: Graph, blobs) -> None:
    """cusha_ipc_connect: every rank's ipc_export blob, in rank order."""
    allb = b"".join(bytes(b) for b in blobs)
    buf = ctypes.create_string_buffer(allb, len(allb))
    _check(lib().cusha_ipc_connect(g.handle, buf, len(allb)), "cusha_ipc_connect")


def set_vertex_values(g: Graph, alg, values: np.ndarray):
    values = np.ascontiguousarray(values)
    _check(lib().cusha_set_vertex_values(g.handle, _alg(alg), _ptr(values), values.nbytes), "cusha_set_vertex_values")


def run(alg, g: Graph, source: int = 0, max_iters: int = 1 << 20) -> int:
    """cusha_run; returns OK (0) or NOT_CONVERGED (1)."""
    return _check(lib().cusha_run(_alg(alg), g.handle, source, max_iters), "cusha_run", ok=(OK, NOT_CONVERGED))


def value_dtype(alg):
    a = _alg(alg)
    if a in (BFS, SSSP, CC, SSWP):
        return np.dtype(np.uint32), 1
    if a in (PR, NN):
        return np.dtype(np.float32), 1
    return np.dtype(np.float32), 2


def get_values(g: Graph, alg=None) -> np.ndarray:
    """cusha_get_values into a new host array (|V| or |V|x2 for HS/CS)."""
    st = get_stats(g)
    a = st["last_algorithm"] if alg is None else _alg(alg)
    dt, k = value_dtype(a)
    out = np.empty((g.V, k) if k > 1 else g.V, dt)
    _check(lib().cusha_get_values(g.handle, _ptr(out), out.nbytes), "cusha_get_values")
    return out


def get_values_device(g: Graph, tensor):
    _check(lib().cusha_get_values_device(g.handle, _ptr(tensor), tensor.numel() * tensor.element_size()),
           "cusha_get_values_device")
    return tensor


def get_stats(g: Graph) -> dict:
    s = Stats()
    _check(lib().cusha_get_stats(g.handle, ctypes.byref(s)), "cusha_get_stats")
    return {name: getattr(s, name) for name, _ in Stats._fields_}


def get_trace(g: Graph):
    n = get_stats(g)["iterations"]
    upd = np.zeros(n, np.uint32)
    act = np.zeros(n, np.uint32)
    k = lib().cusha_get_trace(g.handle, _ptr(upd), _ptr(act), n)
    if k < 0:
        raise CushaError(k, "cusha_get_trace")
    return upd[:k], act[:k]


def get_layout(g: Graph, part: str, partition: Optional[int] = None) -> np.ndarray:
    """cusha_get_layout, or cusha_get_part_layout for partition p of a partitioned graph."""
    code, dt = LAYOUT[part]
    cnt = ctypes.c_uint64(0)
    if partition is None:
        call = lambda out, n: lib().cusha_get_layout(g.handle, code, out, n, ctypes.byref(cnt))  # noqa: E731
    else:
        call = lambda out, n: lib().cusha_get_part_layout(g.handle, partition, code, out, n, ctypes.byref(cnt))  # noqa: E731
    _check(call(None, 0), "cusha_get_layout")
    out = np.empty(cnt.value, dt)
    _check(call(_ptr(out), out.nbytes), "cusha_get_layout")
    return out


def get_part_stats(g: Graph, partition: int) -> dict:
    s = Stats()
    _check(lib().cusha_get_part_stats(g.handle, partition, ctypes.byref(s)), "cusha_get_part_stats")
    return {name: getattr(s, name) for name, _ in Stats._fields_}


def trim_memory(device: int = 0):
    _check(lib().cusha_trim_memory(device), "cusha_trim_memory")


def shard_size(num_vertices: int, num_edges: int, vertex_bytes: int = 4, smem_per_sm: int = 0,
               reserved_per_block: int = 0) -> int:
    return int(lib().cusha_shard_size(num_vertices, num_edges, vertex_bytes, smem_per_sm, reserved_per_block))


def value_bytes(alg) -> int:
    return int(lib().cusha_value_bytes(_alg(alg)))


def abi_version() -> int:
    return int(lib().cusha_abi_version())
