export TUNE_TIMEOUT=120
for v in base cw24 cw30; do bash tools/tune.sh run C5pr $v; bash tools/tune.sh run C5bfs $v; bash tools/tune.sh run C2 $v; bash tools/tune.sh run C3 $v; done
