for v in "" "TEMCO_LIB=build/exp/libtemco_spin.so" "TEMCO_LIB=build/exp/libtemco_h200.so"; do
env $v timeout 600 python -m pytest tests -m gpu -q -x -k "full_config" > gpurun_out/r2b_spin_tests.log 2>&1; echo "tests [$v] $(tail -1 gpurun_out/r2b_spin_tests.log)"
for c in resnet50 densenet121 resnet18_cifar unet; do
  echo "=== [$v] $c $(env $v timeout 300 python bench.py --config $c --no-cpu-baseline 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]), round(d["ms_per_step"],4))')"
done; done
