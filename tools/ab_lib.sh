#!/bin/bash
# A/B of two builds of libbar.so on the GPU box: tools/ab_lib.sh <workload> <mode> [R]
# (paper_conf_ipps_anzttdh12_b200/libbar_prev.so = the baseline build; BAR_LIB selects which
# file the Python binding loads — the library itself reads no environment; tuning aid only)
WL=${1:-c5}; MODE=${2:-async}; RARG=${3:+--R $3}
for rep in 1 2; do
  for lib in libbar_prev.so libbar.so; do
    BAR_LIB=paper_conf_ipps_anzttdh12_b200/$lib timeout 400 python tools/kernel_ab.py --workload "$WL" --modes "$MODE" \
        --reps 3 --variants "$lib:" $RARG 2>&1 | tail -1
  done
done
