timeout 900 python -m pytest tests -m gpu -q -x -k "unet or alexnet" 2>&1 | tail -4
timeout 300 python bench.py --config unet --no-cpu-baseline > gpurun_out/r2_bench_unet.log 2>&1; tail -1 gpurun_out/r2_bench_unet.log | cut -c1-400
timeout 120 python scripts/step_profile.py unet 12 2>&1 | head -14
