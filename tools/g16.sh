timeout 900 python -m pytest tests/test_gpu_partition.py tests/test_gpu_hosttopo.py tests/test_gpu_skip.py tests/test_gpu_api.py -q -p no:cacheprovider 2>&1 | tail -25
