mkdir -p gpurun_out/san2
for m in default pass_barrier partition3 partition3_host bsp skip; do
  for r in gs cw; do
    if [[ "$m" == partition3* && "$r" == gs ]]; then continue; fi
    SAN_REPR=$r timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python tools/san_small.py $m > gpurun_out/san2/memcheck_${r}_${m}.txt 2>&1
    echo "memcheck $m $r rc=$? $(grep -c 'ok$' gpurun_out/san2/memcheck_${r}_${m}.txt) runs; $(grep 'ERROR SUMMARY' gpurun_out/san2/memcheck_${r}_${m}.txt)"
  done
done
for t in synccheck initcheck; do
  SAN_REPR=cw timeout 900 compute-sanitizer --tool $t --print-limit 20 python tools/san_small.py default > gpurun_out/san2/${t}_cw_default.txt 2>&1
  echo "$t rc=$? $(grep 'ERROR SUMMARY' gpurun_out/san2/${t}_cw_default.txt)"
done
