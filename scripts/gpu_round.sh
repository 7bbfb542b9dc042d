# round artifacts: tests, smoke, bench lines for every config, ncu launch list + traffic of each config,
# ncu --set full of the top fused groups of each kernel family
set -x
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 400 python bench.py > gpurun_out/bench_default.log 2>&1
for c in densenet121 vgg16_cp resnet18_cifar; do timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
for c in resnet50 densenet121 vgg16_cp resnet18_cifar; do
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_$c.csv python scripts/ncu_target.py $c > /dev/null 2>&1
done
i=$(python scripts/ncu_group.py resnet50 226)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_chain -s $i -c 1 -o gpurun_out/full_r50_g226 python scripts/ncu_target.py resnet50 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mma_poolcat -c 1 -o gpurun_out/full_r50_poolcat python scripts/ncu_target.py resnet50 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_rank_mma -c 1 -o gpurun_out/full_r50_rank python scripts/ncu_target.py resnet50 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:mma_lean -c 1 -o gpurun_out/full_vgg_lean python scripts/ncu_target.py vgg16_cp > /dev/null 2>&1
