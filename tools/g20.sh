export TUNE_TIMEOUT=90
for r in 1 2; do for v in base prev; do bash tools/tune.sh run C2 $v; bash tools/tune.sh run C3 $v; bash tools/tune.sh run C4cc $v; bash tools/tune.sh run C5pr $v; done; done
timeout 600 python -m pytest tests/test_gpu_overlap.py tests/test_gpu_parity.py tests/test_gpu_partition.py -q -p no:cacheprovider 2>&1 | tail -2
