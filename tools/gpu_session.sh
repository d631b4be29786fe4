timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -5
timeout 600 python tools/sweep_R.py --workload c4 --R 128,256,512 --modes async,sync-block 2>&1 | grep '^{'
timeout 900 python tools/sweep_R.py --workload c5 --R 256,512,1024 --modes async,sync-block 2>&1 | grep '^{'
timeout 300 python tools/sweep_R.py --workload c3 --R 128 --modes async,sync-block,jacobi 2>&1 | grep '^{'
timeout 300 python tools/sweep_R.py --workload c1 --R 128 --modes async,sync-block,jacobi 2>&1 | grep '^{'
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_block_pers -s 2 -c 1 -o gpurun_out/prof_c5_pers python tools/profile_sweep.py --workload c5 --R 1024 > gpurun_out/ncu_c5.log 2>&1
