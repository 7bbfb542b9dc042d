for dbg in 6 7; do
PAIR_DBG=$dbg TEMCO_LIB=build/exp/libtemco_trace.so timeout 120 python scripts/pair_timeline.py resnet50 ${1:-2} 8 2>&1 | grep -E "launch|iss fconv  |iss mma done|iss full|prod"
done
