TEMCO_PAIR_USPLIT=1 timeout 900 python -m pytest tests -m gpu -q -x -k "full_config or bf16_mode or every_step or merge or silu" > gpurun_out/r2b_us_tests.log 2>&1; echo "tests usplit $(tail -1 gpurun_out/r2b_us_tests.log)"
for v in "TEMCO_PAIR_USPLIT=1" "" ; do
for c in resnet50 densenet121 resnet18_cifar unet; do
  echo "=== [$v] $c $(env $v timeout 300 python bench.py --config $c --no-cpu-baseline 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]), round(d["ms_per_step"],4), round(d["roofline"]["frac"],3))')"
done; done
