# round-2 artifacts: GPU tests, smoke, bench lines for every config, ncu launch lists (+DRAM bytes)
# of one step of each config, ncu --set full of the top CTA-pair groups
set -x
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/r2f_gpu_tests.log 2>&1; tail -3 gpurun_out/r2f_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2f_smoke.log 2>&1; tail -2 gpurun_out/r2f_smoke.log
timeout 600 python bench.py > gpurun_out/r2f_bench_resnet50.log 2>&1
for c in densenet121 vgg16_cp resnet18_cifar alexnet unet; do timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/r2f_bench_$c.log 2>&1; done
for c in resnet50 densenet121 vgg16_cp resnet18_cifar alexnet unet; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r2f_launches_$c.csv python scripts/ncu_target.py $c > /dev/null 2>&1
done
i=$(python scripts/ncu_group.py resnet50 226 tc_pair)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pair_chain -s $i -c 1 -o gpurun_out/r2f_pair226 python scripts/ncu_target.py resnet50 > /dev/null 2>&1
i=$(python scripts/ncu_group.py resnet50 58 tc_pair)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pair_chain -s $i -c 1 -o gpurun_out/r2f_pair58 python scripts/ncu_target.py resnet50 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_chain -s 20 -c 1 -o gpurun_out/r2f_dn_chain python scripts/ncu_target.py densenet121 > /dev/null 2>&1
ls gpurun_out/ | grep r2f
