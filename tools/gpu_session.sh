timeout 900 python bench.py > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err; tail -c 1500 gpurun_out/bench_c5.json
for w in c1 c2 c3 c4; do timeout 600 python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench_$w.json 2>&1; done
timeout 600 python bench.py --workload c5 --mode sync-block --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_sb.json 2>&1
timeout 600 python bench.py --workload c5 --mode jacobi --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_jac.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_ --csv --log-file gpurun_out/launches_c5.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_block_stage -s 3 -c 1 -o gpurun_out/prof_c5_async python tools/profile_sweep.py --workload c5 > gpurun_out/ncu_c5.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_block_stage -s 3 -c 1 -o gpurun_out/prof_c4_async python tools/profile_sweep.py --workload c4 > gpurun_out/ncu_c4.log 2>&1
