mkdir -p gpurun_out/g40
for n in 8 12 16; do echo "chunks $n"; CUSHA_H2D_CHUNKS=$n BT_REPS=8 timeout 300 python tools/build_timing.py C2 --quiet 2>&1 | grep "^build" | awk "{print \$7}" | tr '\n' ' '; echo; done
echo "single sort"; CUSHA_NO_CHUNK_SORT=1 BT_REPS=8 timeout 300 python tools/build_timing.py C2 --quiet 2>&1 | grep "^build" | awk "{print \$7}" | tr '\n' ' '; echo
