timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for c in resnet50 vgg16_cp densenet121; do
  echo "=== $c default"; python scripts/step_profile.py $c 200
done > gpurun_out/exp_lean.log 2>&1
