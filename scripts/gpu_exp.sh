timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
for c in resnet50 densenet121 vgg16_cp resnet18_cifar; do
  for v in "" "TEMCO_NO_PDL=1"; do
    echo "=== $c $v"; env $v timeout 300 python bench.py --config $c --no-cpu-baseline --steps 30 | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], d['e2e']['value'])"
  done
done > gpurun_out/exp_pdl.log 2>&1
