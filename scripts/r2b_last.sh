timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/last_gpu_tests.log 2>&1; tail -1 gpurun_out/last_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 600 python bench.py 2>/dev/null | tail -1 | cut -c1-330
