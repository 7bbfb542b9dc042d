timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for v in "" "TEMCO_WIDE_NOK2=1"; do
  echo "=== bench $v"; env $v timeout 300 python bench.py --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['fused_group_roofline']['frac'])"
done > gpurun_out/exp_k2b.log 2>&1
for c in densenet121 resnet18_cifar vgg16_cp; do echo "=== $c"; timeout 300 python bench.py --config $c --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'])"; done >> gpurun_out/exp_k2b.log 2>&1
