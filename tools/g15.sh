timeout 600 python -m pytest tests/test_gpu_overlap.py tests/test_gpu_parity.py tests/test_gpu_skip.py -q -p no:cacheprovider 2>&1 | tail -2
export TUNE_TIMEOUT=90
for r in 1 2; do for v in base es0 s4u2 s4u4; do bash tools/tune.sh run C3 $v; bash tools/tune.sh run C4cc $v; done; done
for v in base es0 s4u4; do bash tools/tune.sh run C2 $v; bash tools/tune.sh run C4sswp $v; bash tools/tune.sh run C3gs $v; done
