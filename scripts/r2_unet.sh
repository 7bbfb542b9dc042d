timeout 900 python -m pytest tests -m gpu -q -x -k "unet or alexnet" 2>&1 | tail -4
for c in unet alexnet; do
timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/r2_bench_$c.log 2>&1; tail -1 gpurun_out/r2_bench_$c.log | cut -c1-300
timeout 120 python scripts/step_profile.py $c 10 2>&1 | head -12
done
