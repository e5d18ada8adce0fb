#!/bin/bash
# quick status pass on one B200: GPU parity suite, default bench line, other workloads, C5 probe
TAG=${1:-s2}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_gpu.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/${TAG}_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"
timeout 600 python bench.py --cache-dir /tmp/gg > gpurun_out/${TAG}_bench_C2.json 2> gpurun_out/${TAG}_bench_C2.err; echo "bench rc=$?"
for w in C1 C3 C3gs C4cc C4sswp; do timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --cache-dir /tmp/gg --cpu-budget 5 > gpurun_out/${TAG}_bench_$w.json 2>gpurun_out/${TAG}_bench_$w.err; done; echo "others done"
timeout 900 python tools/c5_probe.py > gpurun_out/${TAG}_c5.log 2>&1; echo "c5 rc=$?"
