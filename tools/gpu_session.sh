timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for m in async sync-block; do timeout 600 python tools/local_iters.py --workload c5 --mode $m 2>&1 | tail -9 | sed "s/^/$m /"; done
timeout 600 python tools/sweep_R.py --workload c5 --R 1024 --modes async,sync-block,jacobi 2>&1 | grep '^{'
timeout 600 python tools/sweep_R.py --workload c4 --R 128 --modes async,sync-block,jacobi 2>&1 | grep '^{'
