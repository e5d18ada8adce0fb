for v in "$@"; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:shard_pass -s 20 -c 1 -o gpurun_out/prof_$v python bench.py --workload C2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --host-loop --cache-dir /tmp/gg --lib paper_conf_hpdc_khorasanivgb14_b200/variant_$v.so > /dev/null 2>&1; echo "prof $v $?"
done
