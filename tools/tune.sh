#!/bin/bash
# build variants of libcusha.so (run here) and time each on C2 (run under gpurun)
# usage: bash tools/tune.sh build "A:-DCUSHA_STAGES=4 -DCUSHA_CONSUMER_WARPS=8" "B:..."
#        bash tools/tune.sh run C2 A B
mode=$1; shift
if [ "$mode" = build ]; then
  for spec in "$@"; do name=${spec%%:*}; defs=${spec#*:}
    python -m paper_conf_hpdc_khorasanivgb14_b200.build $defs --out=$PWD/paper_conf_hpdc_khorasanivgb14_b200/variant_$name.so >/dev/null && echo "built $name ($defs)"
  done
else
  wl=$1; shift
  for name in "$@"; do
    lib=paper_conf_hpdc_khorasanivgb14_b200/variant_$name.so; [ "$name" = base ] && lib=paper_conf_hpdc_khorasanivgb14_b200/libcusha.so
    timeout ${TUNE_TIMEOUT:-300} python bench.py --workload $wl --steps 10 --warmup 3 --cache-dir /tmp/gg --no-e2e --no-cpu-baseline --lib $lib $BENCH_EXTRA 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$name', 'GTEPS', d['value'], 'ms', d['ms_per_step'], 'it', d['run']['iterations'], 'pass_us', d['roofline']['avg_pass_us'], 'frac', d['roofline']['frac'])"
  done
fi
