timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "bf16_mode or full_config or ragged or invariance" 2>&1 | tail -2
timeout 120 python scripts/step_profile.py resnet50 30 > gpurun_out/r2_pair_step_resnet50.log 2>&1
head -24 gpurun_out/r2_pair_step_resnet50.log
