# full GPU test suite + compute-sanitizer memcheck over every launch mode (small graphs)
mkdir -p gpurun_out/san
TAG=${1:-g3}
timeout 1700 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"
tail -8 gpurun_out/${TAG}_pytest.log
for m in default pass_barrier host_loop partition3 skip host_topology; do
  for r in gs cw; do
    SAN_REPR=$r timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python tools/san_small.py $m > gpurun_out/san/memcheck_${r}_${m}.txt 2>&1
    echo "memcheck $m $r rc=$? $(grep -c 'ok$' gpurun_out/san/memcheck_${r}_${m}.txt) runs; $(grep 'ERROR SUMMARY' gpurun_out/san/memcheck_${r}_${m}.txt)"
  done
done
