timeout 900 python -m pytest tests -m gpu -q -x -k "full_config or bf16_mode or every_step or merge or fp32" > gpurun_out/r2b_pc_tests.log 2>&1; echo "tests $(tail -1 gpurun_out/r2b_pc_tests.log)"
for c in densenet121 resnet50 vgg16_cp alexnet resnet18_cifar; do
  echo "=== $c $(timeout 300 python bench.py --config $c --no-cpu-baseline 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]), round(d["ms_per_step"],4), round(d["roofline"]["frac"],3))')"
done
timeout 300 ncu --metrics gpu__time_duration.sum -k regex:poolcat -c 8 --csv python scripts/ncu_target.py densenet121 2>/dev/null | grep gpu__time | awk -F'","' '{print "poolcat dn", $NF}'
for c in resnet50 alexnet densenet121; do timeout 300 ncu --metrics gpu__time_duration.sum -k regex:conv_stem -c 1 --csv python scripts/ncu_target.py $c 2>/dev/null | grep gpu__time | awk -F'","' '{print "stem '$c'", $NF}'; done
