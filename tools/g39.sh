mkdir -p gpurun_out/g39
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "layout or degree" > gpurun_out/g39/pytest.txt 2>&1; echo "pytest rc=$?"
tail -2 gpurun_out/g39/pytest.txt
for n in 4 8 12 16; do CUSHA_H2D_CHUNKS=$n timeout 300 python tools/build_timing.py C2 > gpurun_out/g39/bt_$n.txt 2>&1; echo "chunks $n"; grep -v "^\[cusha" gpurun_out/g39/bt_$n.txt | grep "build 2"; grep "keys + degrees" gpurun_out/g39/bt_$n.txt | tail -1; done
