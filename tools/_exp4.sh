set -u
mkdir -p gpurun_out/exp4
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "duo or coded or large_subdomain or forced" > gpurun_out/exp4/tests.log 2>&1
tail -2 gpurun_out/exp4/tests.log
for wl in c5 c4; do for t in "" "unroll_off=-1"; do
timeout 300 python tools/duo_phase_probe.py --workload $wl --tune "$t" >> gpurun_out/exp4/probe.log 2>&1
done; done
timeout 300 python tools/duo_phase_probe.py --workload c5 --mode sync-block >> gpurun_out/exp4/probe.log 2>&1
timeout 300 python tools/duo_phase_probe.py --workload c5 --k 1 >> gpurun_out/exp4/probe.log 2>&1
cat gpurun_out/exp4/probe.log
