timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_overlap.py tests/test_gpu_bsp.py tests/test_gpu_skip.py -q -p no:cacheprovider 2>&1 | tail -3
export TUNE_TIMEOUT=120
for r in 1 2; do for v in base v0; do for w in C3 C4cc C4sswp C5bfs C1; do bash tools/tune.sh run $w $v; done; done; done
timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -p no:cacheprovider -k "c3 or c4 or c5_bfs or bfs_cc" 2>&1 | tail -2
