mkdir -p gpurun_out/v1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/v1/pytest.txt 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/v1/pytest.txt
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 600 python bench.py > gpurun_out/v1/bench.json 2> gpurun_out/v1/bench.err; echo "bench rc=$?"; cat gpurun_out/v1/bench.json
