mkdir -p gpurun_out
ls -la tests/golden_cache/
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -q -p no:cacheprovider -s -k "c5" > gpurun_out/g9_pytest.log 2>&1; echo "pytest rc=$?"; grep -i "C5 PR\|passed\|failed\|Error" gpurun_out/g9_pytest.log | head
