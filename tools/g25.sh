timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_partition.py tests/test_gpu_hosttopo.py tests/test_gpu_api.py -q -p no:cacheprovider 2>&1 | tail -2
timeout 600 python tools/build_timing.py C2 cw 2>&1 | tail -12
timeout 600 python bench.py --steps 10 --warmup 3 --cache-dir /tmp/gg --cpu-budget 2 > gpurun_out/g25_bench.json 2> gpurun_out/g25_bench.err; python -c "import json; d=json.load(open('gpurun_out/g25_bench.json')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['e2e'])"
