for v in "" "TEMCO_TC_GRID=74" "TEMCO_TC_GRID=37"; do
  echo "=== resnet50 $v"; env $v python scripts/step_profile.py resnet50 400 | grep "tc_chain\|total"
done > gpurun_out/exp_grid.log 2>&1
