timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for c in resnet50 densenet121 vgg16_cp resnet18_cifar; do timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
python scripts/step_profile.py resnet50 300 > gpurun_out/step_resnet50.log 2>&1
