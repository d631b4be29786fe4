#!/bin/bash
# Bench line + ncu evidence for one workload/mode (run on the GPU box from the repo root).
#   tools/profile_round.sh c5 async   -> gpurun_out/{bench,launches,full}_<wl>_<mode>.*
set -u
WL=${1:-c5}; MODE=${2:-async}; EXTRA=${3:-}
mkdir -p gpurun_out
timeout 900 python bench.py --workload "$WL" --mode "$MODE" $EXTRA > gpurun_out/bench_${WL}_${MODE}.json 2> gpurun_out/bench_${WL}_${MODE}.err
tail -c 600 gpurun_out/bench_${WL}_${MODE}.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${WL}_${MODE}.csv \
    python bench.py --workload "$WL" --mode "$MODE" --steps 2 --warmup 1 --no-cpu-baseline --no-e2e $EXTRA > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_block -s 3 -c 1 \
    -o gpurun_out/full_${WL}_${MODE} -f python tools/profile_sweep.py --workload "$WL" --mode "$MODE" > /dev/null 2>&1
ls -la gpurun_out | tail -5
