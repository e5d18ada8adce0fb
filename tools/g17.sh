mkdir -p gpurun_out
timeout 1200 python tools/partition_probe.py C5 1 2 8 > gpurun_out/partition_C5_direct.jsonl 2> gpurun_out/partition_C5_direct.err; echo "probe rc=$?"; cat gpurun_out/partition_C5_direct.jsonl | cut -c1-400
timeout 900 python tools/ooc_probe_r28.py R27 4 24 > gpurun_out/ooc_R27.json 2> gpurun_out/ooc_R27.err; echo "r27 rc=$?"; cat gpurun_out/ooc_R27.json; tail -3 gpurun_out/ooc_R27.err
