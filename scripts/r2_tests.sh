timeout 1500 python -m pytest tests -m gpu -q -x --durations=5 > gpurun_out/r2_gpu_tests.log 2>&1
tail -12 gpurun_out/r2_gpu_tests.log
for c in resnet50 vgg16_cp alexnet; do timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/r2_bench_$c.log 2>&1; tail -1 gpurun_out/r2_bench_$c.log | cut -c1-260; done
timeout 120 python scripts/step_profile.py vgg16_cp 12 2>&1 | head -14
