timeout 1500 python -m pytest tests -m gpu -q -x --durations=8 > gpurun_out/r2_gpu_tests.log 2>&1
tail -25 gpurun_out/r2_gpu_tests.log
timeout 300 python bench.py > gpurun_out/r2_bench.log 2>&1
tail -1 gpurun_out/r2_bench.log | cut -c1-1500
