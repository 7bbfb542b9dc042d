set -x
timeout 400 python -m pytest tests -m gpu -x -q --timeout 120 -k "vgg or bf16" > gpurun_out/gpu_tests_all.log 2>&1 || exit 1
timeout 120 python scripts/step_profile.py vgg16_cp 30 > gpurun_out/step_vgg16.log 2>&1
