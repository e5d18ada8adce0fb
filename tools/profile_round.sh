#!/bin/bash
# Evidence for profiles/: ncu launch list of a whole C2 run and full captures of the shard pass
TAG=${1:-r1}
mkdir -p gpurun_out
# every launch of one bench step (host-loop mode: kernels visible to ncu), device time only
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_C2.csv python bench.py --workload C2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --host-loop --cache-dir /tmp/gg > gpurun_out/${TAG}_launches_C2.log 2>&1; echo "list $?"
# full set, early pass (all shards active), default cache control (flush)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:shard_pass -s 10 -c 1 -o gpurun_out/${TAG}_full_C2 python bench.py --workload C2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --host-loop --cache-dir /tmp/gg > gpurun_out/${TAG}_full_C2.log 2>&1; echo "full $?"
# full set, warm caches (steady state as in the timed loop)
timeout 900 ncu --set full --cache-control none --clock-control none --import-source on -k regex:shard_pass -s 30 -c 1 -o gpurun_out/${TAG}_fullwarm_C2 python bench.py --workload C2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --host-loop --cache-dir /tmp/gg > gpurun_out/${TAG}_fullwarm_C2.log 2>&1; echo "warm $?"
# the timed bench line itself
timeout 600 python bench.py --workload C2 --steps 10 --warmup 3 --cache-dir /tmp/gg > gpurun_out/${TAG}_bench_C2.json 2> gpurun_out/${TAG}_bench_C2.err; echo "bench $?"
for w in C3 C3gs C4cc C4sswp C1; do timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --cache-dir /tmp/gg --cpu-budget 5 > gpurun_out/${TAG}_bench_$w.json 2>/dev/null; done; echo "others $?"
