mkdir -p gpurun_out
free -g | head -2
timeout 2400 python tools/ooc_probe_r28.py R28 4 40 > gpurun_out/ooc_R28.json 2> gpurun_out/ooc_R28.err; echo "r28 rc=$?"; cat gpurun_out/ooc_R28.json; tail -3 gpurun_out/ooc_R28.err
