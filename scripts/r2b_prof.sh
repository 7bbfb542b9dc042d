# per-group step profile (ResNet-50, DenseNet-121) + ncu launch lists with DRAM bytes of every config
set -x
timeout 200 python scripts/step_profile.py resnet50 80 > gpurun_out/r2b_step_resnet50.log 2>&1
timeout 200 python scripts/step_profile.py densenet121 60 > gpurun_out/r2b_step_densenet121.log 2>&1
for c in resnet50 densenet121 vgg16_cp resnet18_cifar alexnet unet resnet18_tt; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r2b_launches_$c.csv python scripts/ncu_target.py $c > /dev/null 2>&1
done
ls -la gpurun_out | grep r2b
