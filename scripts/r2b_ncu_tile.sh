timeout 600 ncu --set full --clock-control none --import-source on -k regex:tile_conv -s 1 -c 1 -o gpurun_out/r2b_ncu_tile_dn python scripts/ncu_target.py densenet121 > gpurun_out/r2b_ncu_t1.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tile_conv -s 0 -c 1 -o gpurun_out/r2b_ncu_tile_rn python scripts/ncu_target.py resnet50 > gpurun_out/r2b_ncu_t2.log 2>&1
