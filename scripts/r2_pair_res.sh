timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
for c in resnet50 resnet18_cifar unet; do
timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/r2_bench_$c.log 2>&1
python - $c <<'PY'
import json,sys
l=[x for x in open(f"gpurun_out/r2_bench_{sys.argv[1]}.log") if x.startswith("{")][-1]
d=json.loads(l); r=d["roofline"]
print(sys.argv[1], round(d["value"]), "img/s", round(d["ms_per_step"],3), "ms", round(r["frac"],3), r["bound"], {k: round(v,3) for k,v in d["kernel_classes_ms"].items()})
PY
timeout 120 python scripts/step_profile.py $c 8 2>&1 | head -9
done
