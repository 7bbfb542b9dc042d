# compute-sanitizer over every kernel family (logs -> gpurun_out/sanitize_<tool>.log)
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  : > gpurun_out/sanitize_$tool.log
  for g in c1 t2_3 t3 t4 resnet50_s vgg16_s alexnet_s; do
    echo "=== $tool $g" >> gpurun_out/sanitize_$tool.log
    timeout 900 $CS --tool $tool --print-limit 20 python scripts/sanitize_run.py $g >> gpurun_out/sanitize_$tool.log 2>&1
    echo "rc=$?" >> gpurun_out/sanitize_$tool.log
  done
done
grep -E "===|ERROR SUMMARY|rc=|ok:|Error|error" gpurun_out/sanitize_*.log | head -80
