timeout 120 python scripts/step_profile.py resnet50 60 2>&1 | grep tc_pair | sort -k4 | head -30 > gpurun_out/a.txt
TEMCO_LIB=build/exp/libtemco_spin.so timeout 120 python scripts/step_profile.py resnet50 60 2>&1 | grep tc_pair | sort -k4 | head -30 > gpurun_out/b.txt
paste gpurun_out/a.txt gpurun_out/b.txt | awk '{print $4, $1, $(NF/2+1)}'
