# R37/R38 check: GPU parity (merged groups step by step), benches of the ResNet configs, step profile
set -x
timeout 1200 python -m pytest tests -m gpu -q -x -k "merge or every_step or full_config or bf16_mode or fp32_mode" > gpurun_out/r2b_cse_tests.log 2>&1; tail -4 gpurun_out/r2b_cse_tests.log
for c in resnet50 resnet18_cifar resnet18_tt; do timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/r2b_cse_bench_$c.log 2>&1; tail -1 gpurun_out/r2b_cse_bench_$c.log | cut -c1-200; done
TEMCO_PLAN_FLAGS=4096 timeout 200 python scripts/step_profile.py resnet50 30 > gpurun_out/r2b_cse_step_bound.log 2>&1
timeout 200 python scripts/step_profile.py resnet50 30 > gpurun_out/r2b_cse_step.log 2>&1
head -12 gpurun_out/r2b_cse_step.log gpurun_out/r2b_cse_step_bound.log
