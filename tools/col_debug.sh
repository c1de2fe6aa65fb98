#!/bin/bash
# Column-pass decomposition (IPT_COL_DEBUG): 0 full pass, 1 loads only, 5 loads only without the
# dependency wait, 6 full pass with a relaxed arrival; per-kernel GB/s from tools/time_passes.py
# (algorithmic bytes = read + write of the matrix).  Extra args: env assignments.
mkdir -p gpurun_out
for sh in 14414x6565 14414x6568; do for eb in 4 8; do for d in 0 7; do
  echo "== $sh eb=$eb dbg=$d $*"
  env IPT_COL_DEBUG=$d "$@" python tools/time_passes.py --shape $sh --eb $eb --reps 5 | python -c "import sys,json; d=json.loads(sys.stdin.readline()); print(d['kernels']['col_shuffle'])"
done; done; done
