timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 900 python bench.py > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err; tail -c 2500 gpurun_out/bench_c5.json
for w in c1 c2 c3 c4; do timeout 600 python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench_$w.json 2>&1; tail -c 400 gpurun_out/bench_$w.json; echo; done
