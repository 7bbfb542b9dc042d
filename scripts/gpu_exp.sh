TEMCO_WIDE_PAIRSTAGE=1 timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for v in "" "TEMCO_WIDE_PAIRSTAGE=1"; do
  echo "=== resnet50 $v"; env $v timeout 120 python scripts/step_profile.py resnet50 400 | grep "tc_chain\|total"
done > gpurun_out/exp_ps.log 2>&1
