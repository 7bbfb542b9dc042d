timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "=== vgg"; python scripts/step_profile.py vgg16_cp 400 | grep "stem\|total" > gpurun_out/exp_pw.log 2>&1
