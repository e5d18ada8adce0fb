"""Small runs of every launch mode for compute-sanitizer (profiles/r1/sanitizer/).
usage: compute-sanitizer --tool memcheck python tools/san_small.py [all | mode ...]  (SAN_REPR=gs|cw, SAN_N=500, SAN_LIB=variant .so)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import graphgen  # noqa: E402
from paper_conf_hpdc_khorasanivgb14_b200 import cusha  # noqa: E402

if os.environ.get("SAN_LIB"):  # a variant library (tools/tune.sh build)
    cusha.LIB_PATH = os.path.abspath(os.environ["SAN_LIB"])

V = 20000
s, d = graphgen.rmat(V, 200000, seed=71)
w = graphgen.edge_u32(s, d, seed=71, lo=1, hi=255)
ALL = {"default": {}, "pass_barrier": {"pass_barrier": True}, "host_loop": {"host_loop": True},
       "partition3": {"world_size": 3}, "skip": {"skip_clean_shards": True},
       "host_topology": {"device_topology_budget": 600000}, "bsp": {"mode": "bsp"},
       "partition3_host": {"world_size": 3, "device_topology_budget": 1}}
names = sys.argv[1:] or ["default"]
if names == ["all"]:
    names = list(ALL)
reprs = [r for r in ("gs", "cw") if os.environ.get("SAN_REPR", r) == r]
NPS = int(os.environ.get("SAN_N", "500"))  # vertices per shard
for mname in names:
    kw = ALL[mname]
    for repr_ in reprs:
        if mname.startswith("partition3") and repr_ == "gs":
            continue  # the partitioned mode uses CW (include/cusha.h)
        for alg in ("bfs", "sssp", "pr", "cc"):
            with cusha.build_graph(V, s, d, edge_values=w if alg == "sssp" else None, repr=repr_,
                                   vertices_per_shard=NPS, **kw) as g:
                cusha.run(alg, g, source=0)
                cusha.get_values(g)
            print(mname, repr_, alg, "ok", flush=True)
