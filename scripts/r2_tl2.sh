for dbg in 0 2 6; do
PAIR_DBG=$dbg TEMCO_LIB=build/exp/libtemco_trace.so timeout 120 python scripts/pair_timeline.py resnet50 2 4 2>&1 | grep -E "launch|iss mma done|iss fconv  "
done
