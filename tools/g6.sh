mkdir -p gpurun_out
timeout 2400 python tools/partition_probe.py C5 1 2 4 8 > gpurun_out/partition_C5.jsonl 2> gpurun_out/partition_C5.err; echo "probe rc=$?"
cat gpurun_out/partition_C5.jsonl; tail -3 gpurun_out/partition_C5.err
