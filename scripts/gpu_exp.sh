timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for c in densenet121 resnet50 vgg16_cp; do
  echo "=== $c"; python scripts/step_profile.py $c 400 | grep "poolcat\|total"
done > gpurun_out/exp_pc2.log 2>&1
