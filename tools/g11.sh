for wl in C3 C4cc C4sswp C2; do for v in base w3 w4; do bash tools/tune.sh run $wl $v; done; done
for v in base w3 w4; do bash tools/tune.sh run C3 $v; done
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_overlap.py -q -p no:cacheprovider -x 2>&1 | tail -2
