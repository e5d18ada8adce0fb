timeout 600 python -m pytest tests/test_gpu_overlap.py tests/test_gpu_parity.py tests/test_gpu_bsp.py tests/test_gpu_skip.py tests/test_gpu_partition.py -q -p no:cacheprovider 2>&1 | tail -4
export TUNE_TIMEOUT=90
for r in 1 2; do for v in base ww2 ww6; do bash tools/tune.sh run C3 $v; bash tools/tune.sh run C3gs $v; done; done
for v in base ww2; do bash tools/tune.sh run C4cc $v; bash tools/tune.sh run C2 $v; done
