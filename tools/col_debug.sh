#!/bin/bash
# Column-pass decomposition (IPT_COL_DEBUG): 0 full pass, 1 loads only, 3 loads only without
# the dispatch ticket, 4 loads only without the row-index prepass; per-kernel GB/s from
# tools/time_passes.py (algorithmic bytes = read + write of the matrix).  Extra args: env.
mkdir -p gpurun_out
for sh in 14414x6565 14414x6568; do for eb in 4 8; do for d in 0 1 5 3; do
  echo "== $sh eb=$eb dbg=$d $*"
  env IPT_COL_DEBUG=$d "$@" python tools/time_passes.py --shape $sh --eb $eb --reps 5 | python -c "import sys,json; d=json.loads(sys.stdin.readline()); print(d['kernels']['col_shuffle'])"
done; done; done
