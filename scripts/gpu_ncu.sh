set -x
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_chain -s 10 -c 1 -o gpurun_out/v2_chain58 python scripts/ncu_target.py resnet50 > gpurun_out/ncu1.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_chain -s 1 -c 1 -o gpurun_out/v2_chain11 python scripts/ncu_target.py resnet50 > gpurun_out/ncu2.log 2>&1
