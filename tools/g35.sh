mkdir -p gpurun_out/c5prof
timeout 1500 ncu --set full --cache-control none --clock-control none --import-source on -k regex:shard_pass -s 20 -c 1 -o gpurun_out/c5prof/c5pr_pass python bench.py --workload C5pr --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --host-loop > gpurun_out/c5prof/log.txt 2>&1; echo "ncu rc=$?"
