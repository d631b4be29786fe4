#!/bin/bash
# Round evidence, part 2 (GPU box, repo root): ncu launch lists and full captures of the dominant
# kernels, N2 / N4 tables, and the bounds-checking build over the GPU suite (compute-sanitizer was
# closed on the round-2 pool; where it is available, tools/sanitize_cases.py runs every default
# kernel family under it: compute-sanitizer --tool memcheck|racecheck|synccheck python tools/sanitize_cases.py).
#   python tools/build.py --check-bounds   # here, before the call (libbar_check.so travels with the repo)
#   bash tools/evidence_profile.sh r02     -> gpurun_out/r02/...
# then, here: python tools/ncu_summary.py full gpurun_out/r02/full_c5_async.ncu-rep profiles/r02_c5_async_full.txt \
#                 --traffic-json profiles/traffic_c5_async.json --R 1024   (and c4 with --R 512; launches for each list)
set -u
TAG=${1:-r02}; OUT=gpurun_out/$TAG; mkdir -p $OUT
for wl in c5 c4; do
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_block_duo -s 3 -c 1 \
      -o $OUT/full_${wl}_async -f python tools/profile_sweep.py --workload $wl > $OUT/ncu_full_$wl.log 2>&1
done
for wl in c5 c4 c1 c3; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_${wl}_async.csv \
      python bench.py --workload $wl --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-dist > /dev/null 2>&1
done
timeout 900 python tools/nondeterminism.py --workload c1 --runs 200 > $OUT/n2_c1.txt 2>&1
timeout 900 python tools/nondeterminism.py --workload c1 --runs 200 --lead 3 > $OUT/n2_c1_lead3.txt 2>&1
timeout 900 python tools/nondeterminism.py --workload c2 --runs 100 > $OUT/n2_c2.txt 2>&1
for wl in c5 c4 c2; do timeout 900 python tools/local_iters.py --workload $wl > $OUT/n4_$wl.txt 2>&1; done
if [ -f paper_conf_ipps_anzttdh12_b200/libbar_check.so ]; then
  BAR_LIB=paper_conf_ipps_anzttdh12_b200/libbar_check.so timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider \
      --timeout 400 > $OUT/check_tests.log 2>&1
  echo "BAR_CHECK failures: $(grep -c 'BAR_CHECK failed' $OUT/check_tests.log)"; tail -1 $OUT/check_tests.log
fi
ls -la $OUT | tail -30
