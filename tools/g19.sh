mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/g19_build.log 2>&1; echo "build rc=$?"
timeout 1700 python -m pytest tests -m gpu -q -p no:cacheprovider --durations=15 > gpurun_out/g19_pytest.log 2>&1; echo "pytest rc=$?"
tail -30 gpurun_out/g19_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
