#!/bin/bash
# per-launch device time of every shard pass (ncu, host-loop mode) for library variants
# usage: bash tools/launch_list.sh WORKLOAD name...   (name=base -> libcusha.so)
wl=$1; shift
for v in "$@"; do
  lib=paper_conf_hpdc_khorasanivgb14_b200/variant_$v.so; [ "$v" = base ] && lib=paper_conf_hpdc_khorasanivgb14_b200/libcusha.so
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:shard_pass --csv --log-file gpurun_out/launches_${wl}_$v.csv python bench.py --workload $wl --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --host-loop --cache-dir /tmp/gg --lib $lib > /dev/null 2>&1; echo "list $v $?"
done
