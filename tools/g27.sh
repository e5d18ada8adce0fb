export TUNE_TIMEOUT=120
for r in 1 2; do for v in base bf0; do for w in C4cc C4sswp C3 C3gs C1; do bash tools/tune.sh run $w $v; done; done; done
timeout 900 python -m pytest tests/test_gpu_overlap.py tests/test_gpu_parity.py tests/test_gpu_bsp.py -q -p no:cacheprovider 2>&1 | tail -2
