for r in 1 2; do for v in base d0; do bash tools/tune.sh run C2 $v; done; done
for r in 1; do for v in base d0; do bash tools/tune.sh run C3 $v; bash tools/tune.sh run C5pr $v; done; done
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bsp.py -q -p no:cacheprovider -x 2>&1 | tail -2
