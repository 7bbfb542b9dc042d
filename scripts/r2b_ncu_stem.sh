timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_stem -c 1 -o gpurun_out/r2b_ncu_stem2 python scripts/ncu_target.py resnet50 > /dev/null 2>&1
