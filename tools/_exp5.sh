set -u
mkdir -p gpurun_out/exp5
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "duo or coded or large_subdomain or forced" > gpurun_out/exp5/tests.log 2>&1
tail -2 gpurun_out/exp5/tests.log
for wl in c5 c4; do
timeout 300 python tools/duo_phase_probe.py --workload $wl >> gpurun_out/exp5/probe.log 2>&1
done
cat gpurun_out/exp5/probe.log
timeout 900 python tools/kernel_ab.py --workload c5 --modes async,sync-block --reps 3 --rounds 2 --variants 'new:;gen:unroll_off=-1' > gpurun_out/exp5/ab_c5.log 2>&1
timeout 600 python tools/kernel_ab.py --workload c4 --modes async --reps 3 --rounds 2 --variants 'new:;gen:unroll_off=-1' > gpurun_out/exp5/ab_c4.log 2>&1
grep median gpurun_out/exp5/ab_c5.log gpurun_out/exp5/ab_c4.log
