mkdir -p gpurun_out
TAG=${1:-g4}
timeout 900 python -m pytest tests/test_gpu_bsp.py tests/test_gpu_api.py -q -p no:cacheprovider > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"
tail -30 gpurun_out/${TAG}_pytest.log
