timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
timeout 120 python scripts/step_profile.py resnet50 6 > gpurun_out/exp_f3.log 2>&1
for v in "" "TEMCO_WIDE_NOK2=1"; do env $v timeout 300 python bench.py --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$v', d['value'], d['ms_per_step'], d['roofline']['frac'])"; done >> gpurun_out/exp_f3.log 2>&1
