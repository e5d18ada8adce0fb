export TUNE_TIMEOUT=150
for r in 1 2; do for v in base dg; do bash tools/tune.sh run C5pr $v; bash tools/tune.sh run C5bfs $v; bash tools/tune.sh run C2 $v; done; done
for v in base dg; do bash tools/tune.sh run C3 $v; bash tools/tune.sh run C4cc $v; done
