# event timelines of CTA 0 for tc_pair launches (stage-1 group 72 = launch 4, stage-3 group 140 = 13, stage-4-ish 240 = 27)
for li in 4 13 27; do
WIN=12000 TEMCO_LIB=build/exp/libtemco_trace.so timeout 120 python scripts/pair_timeline.py resnet50 $li 12 > gpurun_out/r2b_tl_$li.log 2>&1
done
