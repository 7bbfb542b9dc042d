# re-entry check: full GPU suite, smoke, every bench config (N=1)
set -x
timeout 1500 python -m pytest tests -m gpu -q -x --durations=8 > gpurun_out/r2b_gpu_tests.log 2>&1
tail -14 gpurun_out/r2b_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2b_smoke.log 2>&1; tail -3 gpurun_out/r2b_smoke.log
timeout 600 python bench.py > gpurun_out/r2b_bench_resnet50.log 2>&1; tail -1 gpurun_out/r2b_bench_resnet50.log | cut -c1-400
for c in densenet121 vgg16_cp resnet18_cifar alexnet unet resnet18_tt; do timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/r2b_bench_$c.log 2>&1; tail -1 gpurun_out/r2b_bench_$c.log | cut -c1-300; done
