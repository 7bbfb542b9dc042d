set -x
python scripts/step_profile.py resnet50 45 > gpurun_out/step_resnet50.log 2>&1
python scripts/step_profile.py densenet121 40 > gpurun_out/step_densenet121.log 2>&1
python scripts/step_profile.py vgg16_cp 20 > gpurun_out/step_vgg16.log 2>&1
python scripts/step_profile.py resnet18_cifar 20 > gpurun_out/step_resnet18.log 2>&1
