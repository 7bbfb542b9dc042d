timeout 600 python -m pytest tests -m gpu -q -x -k "pair or resnet or unet or steps" 2>&1 | tail -2
timeout 300 python bench.py --config resnet50 --no-cpu-baseline > gpurun_out/r2_bench_resnet50.log 2>&1
python - resnet50 <<'PY'
import json,sys
l=[x for x in open(f"gpurun_out/r2_bench_{sys.argv[1]}.log") if x.startswith("{")][-1]
d=json.loads(l); r=d["roofline"]
print(sys.argv[1], round(d["value"]), "img/s", round(d["ms_per_step"],3), "ms", round(r["frac"],3), r["bound"], {k: round(v,3) for k,v in d["kernel_classes_ms"].items()})
PY
timeout 120 python scripts/step_profile.py resnet50 12 2>&1 | head -13
bash scripts/r2_tl.sh 2 | head -60
