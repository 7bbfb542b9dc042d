timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for c in resnet50 densenet121 resnet18_cifar; do
  echo "=== $c"; python scripts/step_profile.py $c 400 | grep "conv_rank\|total"
done > gpurun_out/exp_at2.log 2>&1
