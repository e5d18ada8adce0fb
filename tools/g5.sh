mkdir -p gpurun_out
TAG=${1:-g5}
timeout 1200 python -m pytest tests/test_gpu_float_size.py tests/test_gpu_parity.py -q -p no:cacheprovider -k "size or shuffled" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"
tail -30 gpurun_out/${TAG}_pytest.log
