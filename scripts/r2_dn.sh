timeout 1200 python -m pytest tests -m gpu -q -x -k "densenet or t4 or steps" 2>&1 | tail -2
timeout 300 python bench.py --config densenet121 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-120
timeout 120 python scripts/step_profile.py densenet121 300 > gpurun_out/r2_dn_steps.txt 2>&1; head -1 gpurun_out/r2_dn_steps.txt
