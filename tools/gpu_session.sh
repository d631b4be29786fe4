set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
free -g | head -2; nproc
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -20
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -30
for w in c1 c2 c3 c4; do timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -3; done
