#!/bin/bash
# Round deliverables: smoke, GPU tests, bench lines (sweep, skinny, batched), ncu launch list of
# the bench command, ncu --set full captures of the column and row kernels on one sweep shape.
# usage: tools/gpu_round2.sh <tag>
TAG=${1:-r01}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
timeout 600 python bench.py --config skinny --no-cpu-baseline > gpurun_out/bench_skinny_$TAG.json 2> gpurun_out/bench_skinny_$TAG.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref_$TAG.json 2> gpurun_out/bench_ref_$TAG.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --profile-only --no-cpu-baseline > gpurun_out/ncu_launch_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:col_ -c 1 -s 2 -f -o gpurun_out/col_$TAG \
    python tools/one_shape.py --m 14414 --n 6565 --eb 4 --reps 3 > gpurun_out/ncu_col_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:row_ -c 1 -s 2 -f -o gpurun_out/row_$TAG \
    python tools/one_shape.py --m 14414 --n 6565 --eb 4 --reps 3 > gpurun_out/ncu_row_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:row_rot -c 1 -s 2 -f -o gpurun_out/rowrot_$TAG \
    python tools/one_shape.py --m 17226 --n 6052 --eb 4 --reps 3 > gpurun_out/ncu_rowrot_$TAG.log 2>&1
ls -la gpurun_out | tail -5
timeout 600 ncu --set full --clock-control none --import-source on -k regex:record_block -c 1 -s 1 -f -o gpurun_out/rec_$TAG \
    python tools/one_shape.py --m 14414 --n 6565 --eb 12 --reps 2 > gpurun_out/ncu_rec_$TAG.log 2>&1
