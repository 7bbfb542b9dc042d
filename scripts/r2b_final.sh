# round-2 final artifacts: GPU suite, smoke, bench lines (every config, N=1), ablation + SiLU lines,
# ncu launch lists (+ DRAM bytes) of every config, ncu --set full of top tc_pair groups
set -x
O=gpurun_out/fin5
mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q --durations=5 > $O/gpu_tests.log 2>&1; tail -3 $O/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -2 $O/smoke.log
timeout 600 python bench.py > $O/bench_resnet50.log 2>&1; tail -1 $O/bench_resnet50.log | cut -c1-200
for c in densenet121 vgg16_cp resnet18_cifar alexnet unet resnet18_tt; do timeout 300 python bench.py --config $c --no-cpu-baseline > $O/bench_$c.log 2>&1; tail -1 $O/bench_$c.log | cut -c1-160; done
timeout 300 python bench.py --config resnet50 --variant cse_bound --no-cpu-baseline > $O/bench_resnet50_csebound.log 2>&1; tail -1 $O/bench_resnet50_csebound.log | cut -c1-160
for cfg in resnet50 densenet121 vgg16_cp resnet18_cifar alexnet unet; do
  for v in temco paper_schedule fusion_only skipopt_only decomposed; do
    timeout 300 python bench.py --config $cfg --variant $v --steps 10 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 >> $O/ablation.jsonl
  done
  timeout 300 python bench.py --config $cfg --act silu --no-cpu-baseline 2>/dev/null | tail -1 >> $O/silu.jsonl
done
for c in resnet50 densenet121 vgg16_cp resnet18_cifar alexnet unet resnet18_tt; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 3000 --csv --log-file $O/launches_$c.csv python scripts/ncu_target.py $c > /dev/null 2>&1
done
i=$(python scripts/ncu_group.py resnet50 72 tc_pair)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pair_chain -s $i -c 1 -o $O/ncu_pair72 python scripts/ncu_target.py resnet50 > /dev/null 2>&1
i=$(python scripts/ncu_group.py resnet50 211 tc_pair)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pair_chain -s $i -c 1 -o $O/ncu_pair211 python scripts/ncu_target.py resnet50 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tile_conv -s 0 -c 1 -o $O/ncu_tile0 python scripts/ncu_target.py resnet50 > /dev/null 2>&1
ls $O
