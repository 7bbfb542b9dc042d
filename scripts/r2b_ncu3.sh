timeout 600 ncu --set full --clock-control none --import-source on -k regex:mma_poolcat -s 2 -c 1 -o gpurun_out/r2b_ncu_pc3 python scripts/ncu_target.py densenet121 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mma_lean_kernel -s 0 -c 1 -o gpurun_out/r2b_ncu_lean3 python scripts/ncu_target.py densenet121 > /dev/null 2>&1
