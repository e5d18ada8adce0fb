#!/bin/bash
# one GPU iteration: parity tests, C2 bench, ncu launch list + full capture of the shard pass
# usage (under gpurun): bash tools/gpu_cycle.sh <tag> [workload]
TAG=${1:-x}; WL=${2:-C2}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 600 python bench.py --workload $WL --steps 10 --warmup 3 --cache-dir /tmp/gg --cpu-budget 5 2>gpurun_out/bench_${TAG}.err | tee gpurun_out/bench_${TAG}.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('VALUE', d['value'], d['unit'], 'ms/step', d['ms_per_step'], 'iters', d['config']['iterations'], 'roofline', d['roofline']['achieved'], d['roofline']['frac'], 'pass_us', d['roofline']['avg_pass_us'], 'e2e', (d.get('e2e') or {}).get('value'))"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:shard_pass -s 20 -c 1 -o gpurun_out/prof_${TAG} python bench.py --workload $WL --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --host-loop --cache-dir /tmp/gg > gpurun_out/ncu_${TAG}.log 2>&1; tail -1 gpurun_out/ncu_${TAG}.log
