for li in 21 3; do
TEMCO_PAIR_BIASMMA_ALL=1 WIN=8000 TEMCO_LIB=build/exp/libtemco_trace.so timeout 120 python scripts/pair_timeline.py resnet50 $li 12 > gpurun_out/r2b_tl3_$li.log 2>&1
done
