#!/bin/bash
# Round evidence, part 1 (GPU box, repo root): the GPU test suite and the bench lines.
#   bash tools/evidence_bench.sh r02   -> gpurun_out/r02/{gputest.log, bench_*.json}
set -u
TAG=${1:-r02}; OUT=gpurun_out/$TAG; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw --format=csv > $OUT/smi.txt
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 400 > $OUT/gputest.log 2>&1
tail -3 $OUT/gputest.log
timeout 600 python bench.py > $OUT/bench_c5_async.json 2> $OUT/bench_c5_async.err
for m in sync-block jacobi; do
  timeout 600 python bench.py --mode $m --no-dist > $OUT/bench_c5_$m.json 2> $OUT/bench_c5_$m.err
done
for wl in c4 c3 c2 c1; do
  timeout 600 python bench.py --workload $wl $( [ $wl = c4 ] || echo "--steps 50 --warmup 5" ) > $OUT/bench_${wl}_async.json 2> $OUT/bench_${wl}_async.err
done
timeout 900 python bench.py --impl reference > $OUT/bench_reference_c5.json 2> $OUT/bench_reference_c5.err
for f in $OUT/bench_*.json; do echo "$f: $(tail -c 300 $f | head -c 300)"; done | cut -c1-200
