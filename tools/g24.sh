export TUNE_TIMEOUT=120
for r in 1 2; do for v in base ah2 vb16 spa ept8; do bash tools/tune.sh run C2 $v; done; done
for v in base ah2 vb16 spa; do bash tools/tune.sh run C5pr $v; bash tools/tune.sh run C3 $v; done
