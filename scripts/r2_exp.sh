run() { env $1 timeout 120 python scripts/step_profile.py resnet50 60 2>&1 | grep tc_pair | sort -k4 | awk '{print $4, $1}' > gpurun_out/$2.txt; }
run "X=1" a; run "TEMCO_PAIR_NO_OUTITEM=1" b; run "TEMCO_PAIR_NO_BIASMMA=1" c; run "TEMCO_PAIR_NO_OUTITEM=1 TEMCO_PAIR_NO_BIASMMA=1" d
echo "group outitem noout nobias noout+nobias"
paste gpurun_out/a.txt gpurun_out/b.txt gpurun_out/c.txt gpurun_out/d.txt | awk '{print $1, $2, $4, $6, $8}'
