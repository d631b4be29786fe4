#!/bin/bash
# DRAM bytes of one sweep launch (ncu, one kernel, replayed): tools/ncu_traffic.sh c5 async [R]
WL=${1:-c5}; MODE=${2:-async}; RARG=${3:+--R $3}
mkdir -p gpurun_out
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
    --clock-control none -k regex:k_block -s 3 -c 1 --csv \
    python tools/profile_sweep.py --workload "$WL" --mode "$MODE" $RARG 2>/dev/null | grep -E '"(dram|gpu__|lts)' \
    | awk -F'","' '{print $(NF-2), $(NF-1), $NF}'
