set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python scripts/step_profile.py resnet50 60 > gpurun_out/r2_step_resnet50.log 2>&1
python scripts/step_profile.py densenet121 60 > gpurun_out/r2_step_densenet121.log 2>&1
python scripts/step_profile.py resnet18_cifar 40 > gpurun_out/r2_step_resnet18.log 2>&1
python scripts/step_profile.py vgg16_cp 40 > gpurun_out/r2_step_vgg.log 2>&1
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/r2_bench_base.log 2>&1
