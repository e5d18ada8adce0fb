# chunked host sort: parity + build timing + C2 bench
mkdir -p gpurun_out/g36
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "layout or chunked" > gpurun_out/g36/pytest.txt 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/g36/pytest.txt
timeout 300 python tools/build_timing.py C2 > gpurun_out/g36/bt_chunk.txt 2>&1
CUSHA_NO_CHUNK_SORT=1 timeout 300 python tools/build_timing.py C2 > gpurun_out/g36/bt_single.txt 2>&1
grep -v "^\[cusha" gpurun_out/g36/bt_chunk.txt | tail -4; grep -v "^\[cusha" gpurun_out/g36/bt_single.txt | tail -4
timeout 600 python bench.py > gpurun_out/g36/bench_C2.json 2> gpurun_out/g36/bench_C2.err; tail -c 600 gpurun_out/g36/bench_C2.json
