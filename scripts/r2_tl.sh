for dbg in ${2:-0}; do
WIN=16000 PAIR_DBG=$dbg TEMCO_LIB=build/exp/libtemco_trace.so timeout 120 python scripts/pair_timeline.py resnet50 ${1:-2} 0 2>&1 | grep -v "n="
done
