timeout 900 python tools/nondeterminism.py --workload c1 --runs 200 > gpurun_out/r01_n2_c1.txt 2>&1
timeout 900 python tools/nondeterminism.py --workload c2 --runs 100 > gpurun_out/r01_n2_c2.txt 2>&1
timeout 900 python tools/nondeterminism.py --workload c1 --runs 100 --single-launch 0 > gpurun_out/r01_n2_c1_perlaunch.txt 2>&1
timeout 600 python tools/local_iters.py --workload c4 > gpurun_out/r01_n4_c4.txt 2>&1
timeout 600 python tools/local_iters.py --workload c5 > gpurun_out/r01_n4_c5.txt 2>&1
timeout 600 python tools/local_iters.py --workload c2 --R 128 > gpurun_out/r01_n4_c2.txt 2>&1
