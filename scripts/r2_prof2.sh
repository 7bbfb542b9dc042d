PAIR_DBG=2 TEMCO_LIB=build/exp/libtemco_trace.so timeout 120 python scripts/pair_prof.py resnet50 > gpurun_out/r2_pprof_dbg2.log 2>&1
cat gpurun_out/r2_pprof_dbg2.log
