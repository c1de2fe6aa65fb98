#!/bin/bash
# One GPU session: parity tests, bench lines, ncu launch list and full captures.
# usage: tools/gpu_round.sh <tag> [tests|bench|ncu ...]
set -x
TAG=${1:-r01}; shift
STEPS=${@:-tests bench ncu}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
nvidia-smi > gpurun_out/nvidia_smi_$TAG.txt 2>&1
for s in $STEPS; do
case $s in
tests)
  timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log ;;
bench)
  timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
  timeout 600 python bench.py --config skinny --no-cpu-baseline > gpurun_out/bench_skinny_$TAG.json 2> gpurun_out/bench_skinny_$TAG.err ;;
ncu)
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
      python bench.py --profile-only --no-cpu-baseline > gpurun_out/ncu_launch_$TAG.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:col_ -s 20 -c 2 -f -o gpurun_out/col_$TAG \
      python bench.py --profile-only --no-cpu-baseline > gpurun_out/ncu_col_$TAG.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:row_ -s 20 -c 1 -f -o gpurun_out/row_$TAG \
      python bench.py --profile-only --no-cpu-baseline > gpurun_out/ncu_row_$TAG.log 2>&1 ;;
esac
done
ls -la gpurun_out
