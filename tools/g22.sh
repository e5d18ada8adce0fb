export TUNE_TIMEOUT=120
for v in base one8 one6 one8w24; do bash tools/tune.sh run C2 $v; bash tools/tune.sh run C3 $v; bash tools/tune.sh run C4cc $v; bash tools/tune.sh run C5pr $v; bash tools/tune.sh run C5bfs $v; done
