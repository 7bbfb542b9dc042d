TEMCO_WIDE_ASHARE=1 timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for c in resnet50 densenet121; do
for v in "" "TEMCO_WIDE_ASHARE=1"; do
  echo "=== $c $v"; env $v timeout 120 python scripts/step_profile.py $c 400 | grep "tc_chain\|total"
done; done > gpurun_out/exp_ash.log 2>&1
