timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for w in c1 c2 c3; do timeout 300 python tools/sweep_R.py --workload $w --R 128 --modes async,sync-block 2>&1 | grep '^{'; done
timeout 300 python tools/sweep_R.py --workload c2 --R 448 --k 1,2,5,9 --modes async 2>&1 | grep '^{'
