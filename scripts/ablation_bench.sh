#!/bin/bash
# the paper's ablation variants (Fig. 10/11) timed on the GPU,
# one bench.py line per (config, variant) -> gpurun_out/ablation_<config>.jsonl
mkdir -p gpurun_out
for cfg in ${CONFIGS:-resnet50 densenet121 vgg16_cp resnet18_cifar}; do
  : > gpurun_out/ablation_$cfg.jsonl
  for v in temco fusion_only skipopt_only decomposed; do
    timeout 300 python bench.py --config $cfg --variant $v --steps 10 --warmup 3 --no-cpu-baseline \
      2> gpurun_out/ablation_${cfg}_$v.err | tail -1 >> gpurun_out/ablation_$cfg.jsonl
  done
done
