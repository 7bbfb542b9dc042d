set -x
./scripts/tmem_bw > gpurun_out/tmem_bw.log 2>&1
python scripts/step_profile.py resnet50 40 > gpurun_out/step_resnet50.log 2>&1
python scripts/step_profile.py densenet121 30 > gpurun_out/step_densenet121.log 2>&1
python scripts/step_profile.py vgg16_cp 30 > gpurun_out/step_vgg16.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_chain -s 1 -c 3 -o gpurun_out/prof_chain python scripts/ncu_target.py resnet50 > gpurun_out/ncu.log 2>&1
