timeout 900 python -m pytest tests -m gpu -q -x -k "every_step or full_config or bf16_mode" > gpurun_out/r2b_tile_tests.log 2>&1; tail -3 gpurun_out/r2b_tile_tests.log
bash scripts/r2b_tiledbg.sh; grep gpu__time gpurun_out/r2b_tiledbg.log
for c in resnet50 densenet121 resnet18_cifar unet; do echo "=== $c $(timeout 300 python bench.py --config $c --no-cpu-baseline 2>/dev/null | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(round(d["value"]), round(d["ms_per_step"],4))')"; done
