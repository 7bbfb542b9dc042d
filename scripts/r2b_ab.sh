# kernel-selection A/B on ResNet-50 / DenseNet-121 (same box): env switches of capi.cu lowering
for v in "" "TEMCO_NO_LEAN=1" "TEMCO_NO_RKMMA=1" "TEMCO_CONV_TC=1" "TEMCO_NO_CATP=1"; do
  for c in resnet50 densenet121 resnet18_cifar; do
    echo "=== $c $v $(env $v timeout 300 python bench.py --config $c --no-cpu-baseline 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]), round(d["ms_per_step"],4))')"
  done
done > gpurun_out/r2b_ab.log 2>&1
TEMCO_NO_LEAN=1 timeout 200 python scripts/step_profile.py resnet50 40 > gpurun_out/r2b_ab_nolean.log 2>&1
