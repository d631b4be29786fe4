#!/bin/bash
# Round evidence, part 2 (GPU box, repo root): ncu launch lists and full captures of the dominant
# kernels, compute-sanitizer over every default kernel, N2 / N4 tables.
#   bash tools/evidence_profile.sh r02  -> gpurun_out/r02/...
set -u
TAG=${1:-r02}; OUT=gpurun_out/$TAG; mkdir -p $OUT
for wl in c5 c4; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_${wl}_async.csv \
      python bench.py --workload $wl --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-dist > /dev/null 2>&1
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_block_duo -s 3 -c 1 \
      -o $OUT/full_${wl}_async -f python tools/profile_sweep.py --workload $wl > /dev/null 2>&1
done
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
    --clock-control none -k regex:k_block_duo -s 3 -c 1 --csv python tools/profile_sweep.py --workload c5 \
    --tune async_order=3,fronts=4 > $OUT/traffic_c5_fronts4.csv 2>/dev/null
for wl in c1 c3; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_${wl}_async.csv \
      python bench.py --workload $wl --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-dist > /dev/null 2>&1
done
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_cases.py > $OUT/sanitizer_$tool.log 2>&1
  echo "$tool rc=$?" >> $OUT/sanitizer_$tool.log
  tail -3 $OUT/sanitizer_$tool.log
done
timeout 900 python tools/local_iters.py --workload c5 > $OUT/n4_c5.txt 2>&1
timeout 900 python tools/local_iters.py --workload c4 > $OUT/n4_c4.txt 2>&1
timeout 900 python tools/local_iters.py --workload c2 > $OUT/n4_c2.txt 2>&1
timeout 900 python tools/nondeterminism.py --workload c1 --runs 200 > $OUT/n2_c1.txt 2>&1
timeout 900 python tools/nondeterminism.py --workload c1 --runs 200 --lead 3 > $OUT/n2_c1_lead3.txt 2>&1
timeout 900 python tools/nondeterminism.py --workload c2 --runs 100 > $OUT/n2_c2.txt 2>&1
ls -la $OUT | tail -30
