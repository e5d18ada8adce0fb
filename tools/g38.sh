mkdir -p gpurun_out/g38
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_api.py -x -q > gpurun_out/g38/pytest.txt 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/g38/pytest.txt
timeout 300 python tools/build_timing.py C2 > gpurun_out/g38/bt_chunk.txt 2>&1
grep -v "^\[cusha" gpurun_out/g38/bt_chunk.txt | tail -4
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/g38/launches.csv python tools/build_timing.py C2 > gpurun_out/g38/log.txt 2>&1; echo rc=$?
timeout 600 python bench.py > gpurun_out/g38/bench_C2.json 2> gpurun_out/g38/bench_C2.err; tail -c 300 gpurun_out/g38/bench_C2.json
