timeout 300 ncu --set full --clock-control none --import-source on -k regex:conv_stem -c 1 -o gpurun_out/ncu_stem python scripts/ncu_target.py resnet50 > gpurun_out/ncu_stem.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_chain -c 1 -o gpurun_out/ncu_vgg_g6 python scripts/ncu_target.py vgg16_cp > gpurun_out/ncu_vgg_g6.log 2>&1
TEMCO_PLAN_FLAGS=128 timeout 300 ncu --set full --clock-control none --import-source on -k regex:mma_chain -c 1 -o gpurun_out/ncu_vgg_mma6 python scripts/ncu_target.py vgg16_cp > gpurun_out/ncu_vgg_mma6.log 2>&1
