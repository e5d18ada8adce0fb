timeout 900 python -m pytest tests/test_gpu_partition.py tests/test_gpu_bsp.py tests/test_gpu_skip.py tests/test_gpu_hosttopo.py tests/test_gpu_parity.py -q -p no:cacheprovider 2>&1 | tail -2
timeout 1200 python tools/partition_probe.py C5 1 8 > gpurun_out/partition_C5_graph.jsonl 2> /dev/null; cut -c1-120 gpurun_out/partition_C5_graph.jsonl; python -c "
import json
for l in open('gpurun_out/partition_C5_graph.jsonl'):
    d=json.loads(l); print(d['G'], d['bfs']['run_ms'], d['bfs']['bit_exact_vs_oracle'], d['pr']['run_ms'], d['pr']['passes'])"
timeout 600 python bench.py --workload C2 --sim-parts 8 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --cache-dir /tmp/gg 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C2 sim8', d['value'], d['ms_per_step'], d['run']['iterations'])"
