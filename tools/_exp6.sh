set -u
mkdir -p gpurun_out/exp6
for t in "" "ghost_prefetch=-1" "slab_prefetch=1" "stage_bx=-1" "grid_cap=148"; do
timeout 300 python tools/duo_phase_probe.py --workload c5 --tune "$t" >> gpurun_out/exp6/probe.log 2>&1
done
timeout 300 python tools/duo_phase_probe.py --workload c5 --mode jacobi --k 1 >> gpurun_out/exp6/probe.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "duo or coded or large_subdomain or forced" > gpurun_out/exp6/tests.log 2>&1
tail -2 gpurun_out/exp6/tests.log
cat gpurun_out/exp6/probe.log
