#!/bin/bash
# full ncu capture of one steady-state shard pass with warm caches (no flush), per variant
for v in "$@"; do
  lib=paper_conf_hpdc_khorasanivgb14_b200/variant_$v.so; [ "$v" = base ] && lib=paper_conf_hpdc_khorasanivgb14_b200/libcusha.so
  timeout 600 ncu --set full --cache-control none --clock-control none --import-source on -k regex:shard_pass -s 60 -c 1 -o gpurun_out/profw_$v python bench.py --workload C2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --host-loop --cache-dir /tmp/gg --lib $lib > /dev/null 2>&1; echo "profw $v $?"
done
