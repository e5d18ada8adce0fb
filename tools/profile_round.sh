#!/bin/bash
# Evidence for profiles/<tag>/: ncu launch list of the default bench command,
# ncu --set full of its shard_pass launch (one launch per run: overlapped
# passes) and of one per-pass launch (host-loop mode), and bench lines.
TAG=${1:-r2final}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
# every launch of one bench step (default mode), device time and DRAM bytes
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/ncu_launches_C2.csv python bench.py --workload C2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --cache-dir /tmp/gg > $O/ncu_launches_C2.log 2>&1; echo "list $?"
# full set of the timed run's shard_pass launch (default cache control: flushed before the launch)
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:shard_pass -s 3 -c 1 -o $O/ncu_full_C2_run python bench.py --workload C2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --cache-dir /tmp/gg > $O/ncu_full_C2_run.log 2>&1; echo "full-run $?"
# full set of one steady-state pass (host-loop mode, warm caches)
timeout 900 ncu --set full --cache-control none --clock-control none --import-source on -k regex:shard_pass -s 30 -c 1 -o $O/ncu_fullwarm_C2_pass python bench.py --workload C2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --host-loop --cache-dir /tmp/gg > $O/ncu_fullwarm_C2_pass.log 2>&1; echo "full-pass $?"
# the bench lines
timeout 900 python bench.py --cache-dir /tmp/gg > $O/bench_C2.json 2> $O/bench_C2.err; echo "bench $?"
for w in C1 C3 C3gs C4cc C4sswp; do timeout 600 python bench.py --workload $w --steps 5 --warmup 3 --cache-dir /tmp/gg --cpu-budget 5 > $O/bench_$w.json 2>$O/bench_$w.err; done; echo "others $?"
timeout 300 python bench.py --workload C2 --steps 5 --warmup 3 --pass-barrier --no-e2e --no-cpu-baseline --cache-dir /tmp/gg > $O/bench_C2_passbarrier.json 2>/dev/null; echo "barrier $?"
for w in C5pr C5bfs; do timeout 900 python bench.py --workload $w --steps 3 --warmup 3 --no-e2e --cache-dir /tmp/gg --cpu-budget 5 > $O/bench_$w.json 2>$O/bench_$w.err; done; echo "c5 $?"
# one warm C5 PageRank pass (host-loop mode), and the timed run's launch of the latency-bound workloads
timeout 1500 ncu --set full --cache-control none --clock-control none --import-source on -k regex:shard_pass -s 20 -c 1 -o $O/ncu_fullwarm_C5pr_pass python bench.py --workload C5pr --steps 1 --warmup 2 --no-e2e --no-cpu-baseline --host-loop --cache-dir /tmp/gg > $O/ncu_fullwarm_C5pr_pass.log 2>&1; echo "c5-pass $?"
for w in C4cc C3; do timeout 900 ncu --set full --clock-control none --import-source on -k regex:shard_pass -s 3 -c 1 -o $O/ncu_full_${w}_run python bench.py --workload $w --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --cache-dir /tmp/gg > $O/ncu_full_${w}_run.log 2>&1; echo "run $w $?"; done
