mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_api.py tests/test_gpu_parity.py tests/test_gpu_hosttopo.py -q -p no:cacheprovider -x > gpurun_out/g8_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/g8_pytest.log
timeout 600 python tools/build_timing.py C2 cw > gpurun_out/g8_build.txt 2>&1; tail -40 gpurun_out/g8_build.txt
timeout 600 python bench.py --steps 10 --warmup 3 --cache-dir /tmp/gg --cpu-budget 2 > gpurun_out/g8_bench.json 2> gpurun_out/g8_bench.err; echo "bench rc=$?"; python -c "import json; d=json.load(open('gpurun_out/g8_bench.json')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['e2e'])"
