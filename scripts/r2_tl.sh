for dbg in 0 3; do
EV_OFF=40 PAIR_DBG=$dbg TEMCO_LIB=build/exp/libtemco_trace.so timeout 120 python scripts/pair_timeline.py resnet50 14 24 2>&1 | grep -E "launch|iss|epi accF u0|prod"
done
