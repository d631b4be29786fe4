timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 900 python bench.py > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err; tail -c 1200 gpurun_out/bench_c5.json
timeout 600 python bench.py --workload c4 --no-cpu-baseline > gpurun_out/bench_c4.json 2>&1
