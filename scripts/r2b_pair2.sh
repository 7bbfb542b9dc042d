export TEMCO_PAIR_BIASMMA_ALL=1
for lag in 0 1 2 3; do
  TEMCO_PAIR_FCONV_LAG=$lag timeout 600 python -m pytest tests -m gpu -q -x -k "full_config or bf16_mode" > gpurun_out/r2b_lag_tests_$lag.log 2>&1; echo "lag $lag $(tail -1 gpurun_out/r2b_lag_tests_$lag.log)"
  for c in resnet50 densenet121 resnet18_cifar unet; do
    echo "=== lag $lag $c $(TEMCO_PAIR_FCONV_LAG=$lag timeout 300 python bench.py --config $c --no-cpu-baseline 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]), round(d["ms_per_step"],4), round(d["roofline"]["frac"],3))')"
  done
done
