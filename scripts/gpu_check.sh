set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for c in resnet50 densenet121 vgg16_cp resnet18_cifar; do timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
timeout 300 python bench.py > gpurun_out/bench_default.log 2>&1
