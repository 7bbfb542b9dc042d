# ncu --set full of one tc_pair launch (ResNet-50 group 226 = 15th pair launch; group 58 = 3rd)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pair_chain -s 14 -c 1 -o gpurun_out/r2_pair226 python scripts/ncu_target.py resnet50 > gpurun_out/r2_ncu226.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pair_chain -s 2 -c 1 -o gpurun_out/r2_pair58 python scripts/ncu_target.py resnet50 > gpurun_out/r2_ncu58.log 2>&1
tail -3 gpurun_out/r2_ncu226.log
