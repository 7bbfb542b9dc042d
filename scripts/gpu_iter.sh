# quick GPU iteration: parity tests, per-step profile, benches (used with gpurun)
set -x
timeout 400 python -m pytest tests -m gpu -x -q --timeout 120 > gpurun_out/gpu_tests_all.log 2>&1 || exit 1
timeout 120 python scripts/step_profile.py resnet50 60 > gpurun_out/step_resnet50.log 2>&1
timeout 120 python scripts/step_profile.py densenet121 40 > gpurun_out/step_densenet121.log 2>&1
for c in resnet50 densenet121; do timeout 200 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
