# tile conv: parity, benches with / without it (same box)
set -x
timeout 1200 python -m pytest tests -m gpu -q -x -k "every_step or full_config or bf16_mode or merge" > gpurun_out/r2b_tile_tests.log 2>&1; tail -4 gpurun_out/r2b_tile_tests.log
for v in "" "TEMCO_NO_TILECONV=1"; do
  for c in resnet50 densenet121 resnet18_cifar unet alexnet resnet18_tt; do
    echo "=== $c $v $(env $v timeout 300 python bench.py --config $c --no-cpu-baseline 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]), round(d["ms_per_step"],4))')"
  done
done > gpurun_out/r2b_tile_ab.log 2>&1
cat gpurun_out/r2b_tile_ab.log
timeout 200 python scripts/step_profile.py densenet121 400 2>&1 | grep -E "total|conv_tile" | head -12
