timeout 600 ncu --set full --clock-control none --import-source on -k regex:pair_chain -s 2 -c 1 -o gpurun_out/r2b_pair58 python scripts/ncu_target.py resnet50 > gpurun_out/r2b_ncu58.log 2>&1
tail -2 gpurun_out/r2b_ncu58.log
