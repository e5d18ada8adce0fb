mkdir -p gpurun_out/g37
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/g37/launches.csv python tools/build_timing.py C2 > gpurun_out/g37/log.txt 2>&1; echo rc=$?
