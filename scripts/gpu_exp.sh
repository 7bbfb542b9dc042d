timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "=== resnet50"; python scripts/step_profile.py resnet50 400 | grep "tc_chain\|total" > gpurun_out/exp_ring.log 2>&1
