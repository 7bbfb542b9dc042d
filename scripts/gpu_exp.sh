timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for c in densenet121 resnet50 vgg16_cp resnet18_cifar; do
for v in "" "TEMCO_NO_CATP=1"; do
  echo "=== $c $v"; env $v python scripts/step_profile.py $c 400
done; done > gpurun_out/exp_catp.log 2>&1
