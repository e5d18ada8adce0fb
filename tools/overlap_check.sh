#!/bin/bash
# overlapped passes: parity tests, then bench lines in both iteration modes
TAG=${1:-ov}
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_overlap.py -x -q -p no:cacheprovider > gpurun_out/${TAG}_overlap.log 2>&1; echo "overlap rc=$?"; tail -3 gpurun_out/${TAG}_overlap.log
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/${TAG}_gpu.log 2>&1; echo "gpu rc=$?"; tail -3 gpurun_out/${TAG}_gpu.log
for w in C2 C3 C3gs C4cc C4sswp C1; do
  for m in "" "--pass-barrier"; do
    timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --cache-dir /tmp/gg --no-e2e --no-cpu-baseline $m 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); c=d['config']; r=d['roofline']; print('$w', '$m', 'GTEPS', d['value'], 'ms', d['ms_per_step'], 'it', c['iterations'], 'us/pass', r['avg_pass_us'], 'frac', r['frac'])"
  done
done
