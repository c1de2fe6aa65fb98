#!/bin/bash
# Column-pass tuning sweep: bench.py (sweep config) under env variants.  usage: tools/col_sweep.sh TAG "ENV1" "ENV2" ...
TAG=$1; shift
mkdir -p gpurun_out
for v in "$@"; do
  echo "== $v" >> gpurun_out/col_sweep_$TAG.txt
  env $v timeout 300 python bench.py --no-cpu-baseline --steps 4 --warmup 3 2>>gpurun_out/col_sweep_$TAG.err | python -c "
import json,sys
d=json.loads(sys.stdin.readline()); print(d['value'], d['median_GBps_fp32'], d['median_GBps_fp64'], json.dumps(d['kernels']))" >> gpurun_out/col_sweep_$TAG.txt 2>&1
done
