#!/bin/bash
# Per-pass GB/s of a few shapes under lag settings (development tool).
for cfg in "IPT_COL_LAG=0" "IPT_COL_LAGD=1" "IPT_COL_LAGD=4" "IPT_COL_LAGD=0"; do
  for sh in 19769x2188 1902x4871 6314x5378 14414x6565; do
    for op in c2r r2c; do
      echo "== $cfg $sh $op"; env $cfg python tools/time_passes.py --shape $sh --eb 4 --reps 5 --op $op | python -c "import sys,json; d=json.loads(sys.stdin.readline()); print(d['eq37_GBps'], d['kernels'])"
    done
  done
done
