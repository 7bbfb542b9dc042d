# every bench config (N=1, no CPU baseline) + per-step profile of the top steps
timeout 900 python -m pytest tests -m gpu -q -x -k "unet or alexnet or gemm or vgg" 2>&1 | tail -2
for c in resnet50 densenet121 resnet18_cifar vgg16_cp alexnet unet; do
timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/r2_bench_$c.log 2>&1
python - $c <<'PY'
import json,sys
l=[x for x in open(f"gpurun_out/r2_bench_{sys.argv[1]}.log") if x.startswith("{")][-1]
d=json.loads(l); r=d["roofline"]
print(sys.argv[1], round(d["value"]), "img/s", round(d["ms_per_step"],3), "ms", "dom", d.get("roofline_kernel"), round(r["frac"],3), r["bound"])
PY
timeout 120 python scripts/step_profile.py $c 8 2>&1 | head -9
done
