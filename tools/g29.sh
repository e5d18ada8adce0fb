timeout 700 python -m pytest tests/test_gpu_multiprocess.py -q -p no:cacheprovider -x 2>&1 | tail -25
timeout 900 python -m pytest tests/test_gpu_partition.py tests/test_gpu_parity.py tests/test_gpu_api.py -q -p no:cacheprovider 2>&1 | tail -2
