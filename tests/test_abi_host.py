"""The C-ABI library without a GPU: it loads, exports every symbol include/*.h
declares, its structs match the binding, and its pure host logic (the L310
shard-size rule, argument validation) behaves.  No compute calls."""
import ctypes
import glob
import os
import re
import subprocess

import numpy as np
import pytest

from paper_conf_hpdc_khorasanivgb14_b200 import cusha

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    names = set()
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        txt = open(h).read()
        names |= set(re.findall(r"CUSHA_API\s+[\w\s\*]*?\b(cusha_\w+)\s*\(", txt))
    return names


def test_library_exports_every_declared_symbol():
    names = declared_symbols()
    assert len(names) >= 14
    L = ctypes.CDLL(cusha.LIB_PATH)
    missing = [n for n in sorted(names) if not hasattr(L, n)]
    assert not missing, missing
    out = subprocess.run(["nm", "-D", "--defined-only", cusha.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\b(cusha_\w+)\b", out))
    assert names <= exported
    assert cusha.abi_version() == 5


def test_struct_layout_matches_header(tmp_path):
    prog = tmp_path / "sizes.c"
    prog.write_text(
        '#include <stdio.h>\n#include <stddef.h>\n#include "cusha.h"\n'
        "int main(void){\n"
        'printf("%zu %zu %zu %zu\\n", sizeof(cusha_build_opts), offsetof(cusha_build_opts, nccl_unique_id),'
        " sizeof(cusha_stats), offsetof(cusha_stats, device_loop));\n"
        "return 0;}\n")
    exe = tmp_path / "sizes"
    subprocess.check_call(["gcc", "-std=c11", "-I", os.path.join(ROOT, "include"), str(prog), "-o", str(exe)])
    a, b, c, d = map(int, subprocess.check_output([str(exe)]).split())
    assert a == ctypes.sizeof(cusha.BuildOpts)
    assert b == cusha.BuildOpts.nccl_unique_id.offset
    assert c == ctypes.sizeof(cusha.Stats)
    assert d == cusha.Stats.device_loop.offset


def test_shard_size_rule_livejournal():
    """L310 + L173 on LiveJournal's counts (Table 1): |N|0 = |V| sqrt(32/|E|) = 3301,
    the "3k" of §5.2 (L473); snapped to B200's 228 KB/SM with 16 CTAs -> 3392."""
    V, E = 4_847_571, 68_993_773
    assert round(V * (32 / E) ** 0.5) == 3301
    assert cusha.shard_size(V, E) == 3392
    # average window at the chosen |N| stays near 32 (warp size)
    N = cusha.shard_size(V, E)
    S = -(-V // N)
    assert 25 < E / S**2 < 40


def test_shard_size_rule_paper_kepler_examples():
    """L310: 48 KB SM, 4-byte vertices: 2 blocks -> |N| <= 6K, 4 blocks -> 3K."""
    V = 10_000_000
    E6k = int(32 * V * V / 6144**2)
    assert cusha.shard_size(V, E6k, 4, 49152, 0) == 6144
    E3k = int(32 * V * V / 3072**2)
    assert cusha.shard_size(V, E3k, 4, 49152, 0) == 3072
    # 8-byte vertices halve the candidates
    assert cusha.shard_size(V, E3k, 8, 49152, 0) == 3072
    assert cusha.shard_size(V, E6k, 8, 49152, 0) == 6144   # one block of 48 KB


def test_shard_size_rule_edges():
    # tiny graph: capped at |V|
    assert cusha.shard_size(100, 50) == 100
    # C1 (4096 / 32768): |N|0 = 128, smallest B200 candidate (32 CTAs/SM) is 1568 -> capped to |V|
    assert cusha.shard_size(4096, 32768) == 1568
    # never above the 16-bit local-index limit
    assert cusha.shard_size(2**30, 2**31, 1) <= 65534
    assert cusha.shard_size(1, 0) == 1


def test_value_bytes():
    assert [cusha.value_bytes(a) for a in range(8)] == [4, 4, 4, 4, 4, 4, 8, 8]
    assert cusha.value_bytes(8) == 0


def test_build_graph_argument_errors():
    L = cusha.lib()
    h = ctypes.c_void_p()
    s = np.zeros(1, np.uint32)
    # null out
    assert L.cusha_build_graph(4, 1, cusha._ptr(s), cusha._ptr(s), None, None, None) == cusha.EINVAL
    # |V| = 0
    assert L.cusha_build_graph(0, 1, cusha._ptr(s), cusha._ptr(s), None, None, ctypes.byref(h)) == cusha.EINVAL
    assert b"num_vertices" in L.cusha_last_error()
    # null src with edges
    assert L.cusha_build_graph(4, 1, None, None, None, None, ctypes.byref(h)) == cusha.EINVAL
    # |N| over the 16-bit limit
    o = cusha.BuildOpts()
    o.vertices_per_shard = 70000
    assert L.cusha_build_graph(100000, 1, cusha._ptr(s), cusha._ptr(s), None, ctypes.byref(o), ctypes.byref(h)) == cusha.EINVAL
    # iteration-boundary mode outside {0 auto, 1 barrier, 2 overlapped}
    o = cusha.BuildOpts()
    o.pass_barrier = 3
    assert L.cusha_build_graph(4, 1, cusha._ptr(s), cusha._ptr(s), None, ctypes.byref(o), ctypes.byref(h)) == cusha.EINVAL
    assert b"pass_barrier" in L.cusha_last_error()
    # multi-GPU through the single-GPU entry point
    o = cusha.BuildOpts()
    o.world_size = 2
    assert L.cusha_build_graph(4, 1, cusha._ptr(s), cusha._ptr(s), None, ctypes.byref(o), ctypes.byref(h)) != cusha.OK
    # null graph handles
    assert L.cusha_run(0, None, 0, 10) == cusha.EINVAL
    assert L.cusha_get_values(None, None, 0) == cusha.EINVAL
    L.cusha_free_graph(None)


def test_no_cpu_fallback_without_gpu():
    """Without a device the product path errors out; it never computes on the CPU."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(cusha.CushaError) as ei:
        cusha.build_graph(4, np.array([0, 1], np.uint32), np.array([1, 2], np.uint32))
    assert ei.value.code == cusha.ECUDA


def test_diag_timeline_absent_from_product_build():
    """The per-ticket timeline exists only in -DCUSHA_TIMELINE=1 diagnostic
    builds (tools/timeline.py); the product library refuses the call."""
    buf = np.zeros(40, dtype=np.uint32)
    assert cusha.lib().cusha_diag_timeline(buf.ctypes.data, buf.nbytes) == cusha.EUNSUPPORTED
    assert cusha.lib().cusha_diag_timeline(None, 0) == cusha.EINVAL
