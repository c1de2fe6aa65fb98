#!/bin/bash
# Skinny-engine tuning sweep: bench.py --config skinny under env variants.
# usage: tools/skinny_sweep.sh TAG "ENV1" "ENV2" ...
TAG=$1; shift
mkdir -p gpurun_out
for v in "$@"; do
  echo "== $v" >> gpurun_out/skinny_sweep_$TAG.txt
  env $v timeout 400 python bench.py --config skinny --no-cpu-baseline --steps 3 --warmup 3 2>>gpurun_out/skinny_sweep_$TAG.err | python -c "
import json,sys
d=json.loads(sys.stdin.readline()); print(d['value'], d['max_GBps'], json.dumps(d['kernels']))" >> gpurun_out/skinny_sweep_$TAG.txt 2>&1
done
