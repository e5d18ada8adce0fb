mkdir -p gpurun_out
timeout 2400 python tools/n_sweep.py C2:pr:cw:3392,4096,4700,5500 C2:bfs:cw:3392,4700,8000 C3:sssp:cw:4608,6600,9000 C4cc:cc:cw:1568,3000 C4sswp:sswp:cw:1568,3000 C5:pr:cw:11417,14500,17500 C5:bfs:cw:11417,17500,24000,31000 > gpurun_out/n_sweep.jsonl 2> gpurun_out/n_sweep.err; echo "sweep rc=$?"
cat gpurun_out/n_sweep.jsonl; tail -3 gpurun_out/n_sweep.err
free -g; nproc
timeout 1800 python tools/r27_probe.py R27 > gpurun_out/r27.json 2> gpurun_out/r27.err; echo "r27 rc=$?"; cat gpurun_out/r27.json; tail -5 gpurun_out/r27.err
