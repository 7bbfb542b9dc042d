for v in 3 7; do
TEMCO_TILE_DBG=$v timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,launch__grid_size -k regex:tile_conv -c 3 --csv python scripts/ncu_target.py resnet50 2>/dev/null | grep -E "gpu__time|grid" | awk -F'","' '{print "dbg'$v' rn", $(NF-2), $NF}'
TEMCO_TILE_DBG=$v timeout 300 ncu --metrics gpu__time_duration.sum,launch__grid_size -k regex:tile_conv -c 2 --csv python scripts/ncu_target.py densenet121 2>/dev/null | grep -E "gpu__time|grid" | awk -F'","' '{print "dbg'$v' dn", $(NF-2), $NF}'
done > gpurun_out/r2b_tiledbg.log 2>&1
