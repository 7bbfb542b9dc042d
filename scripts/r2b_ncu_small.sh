# ncu --set full of the HBM-bound small-kernel families: DenseNet block-1 mma_poolcat, ResNet-50 stem, 3x3/8ch core
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mma_poolcat -s 2 -c 1 -o gpurun_out/r2b_ncu_poolcat_dn python scripts/ncu_target.py densenet121 > gpurun_out/r2b_ncu1.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_stem -c 1 -o gpurun_out/r2b_ncu_stem python scripts/ncu_target.py resnet50 > gpurun_out/r2b_ncu2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_rank_kernel -c 1 -o gpurun_out/r2b_ncu_rank python scripts/ncu_target.py resnet50 > gpurun_out/r2b_ncu3.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_rank_mma -s 3 -c 1 -o gpurun_out/r2b_ncu_rankmma python scripts/ncu_target.py resnet50 > gpurun_out/r2b_ncu4.log 2>&1
ls -la gpurun_out/*.ncu-rep
