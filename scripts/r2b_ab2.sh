for r in 1 2; do for v in "" "TEMCO_NO_TILECONV=1"; do
  for c in resnet50 densenet121 resnet18_cifar unet; do
    echo "=== $c $v $(env $v timeout 300 python bench.py --config $c --no-cpu-baseline 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]), round(d["ms_per_step"],4))')"
  done
done; done > gpurun_out/r2b_ab2.log 2>&1
for c in resnet50 densenet121; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r2b_launches2_$c.csv python scripts/ncu_target.py $c > /dev/null 2>&1
done
