# usage: gpu_ncu_group.sh <config> <out id> <tag>
i=$(python scripts/ncu_group.py $1 $2)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_chain -s $i -c 1 -o gpurun_out/ncu_$3 python scripts/ncu_target.py $1 > gpurun_out/ncu_$3.log 2>&1
