export TUNE_TIMEOUT=120
for w in C4cc C4sswp C3 C3gs C2 C1; do bash tools/tune.sh run $w base; done
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x 2>&1 | tail -3
