timeout 300 python -m pytest tests/test_gpu_overlap.py tests/test_gpu_parity.py -q -p no:cacheprovider -x 2>&1 | tail -4
export TUNE_TIMEOUT=90
for wl in C3 C4cc C4sswp C2 C1; do for v in w2 w3 w4; do bash tools/tune.sh run $wl $v; done; done
for v in w2 w4; do TUNE_TIMEOUT=200 bash tools/tune.sh run C5pr $v; bash tools/tune.sh run C3gs $v; done
