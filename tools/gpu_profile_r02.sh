#!/bin/bash
# Round-2 evidence session: ncu launch list of the bench command, --set full captures of
# every kernel family, compute-sanitizer logs.  usage: tools/gpu_profile_r02.sh <tag> [ncu] [san]
TAG=${1:-r02}; shift
STEPS=${@:-ncu export san}
mkdir -p gpurun_out
NCU="ncu --set full --clock-control none --import-source on -f"
REP=/tmp/ncu_$TAG; mkdir -p $REP
for s in $STEPS; do
case $s in
ncu)
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
      python bench.py --profile-only --no-cpu-baseline --no-extras > gpurun_out/ncu_launch_$TAG.log 2>&1
  timeout 600 $NCU -k regex:col_tile -c 1 -s 2 -o $REP/col_$TAG \
      python tools/one_shape.py --m 14414 --n 6565 --eb 4 --reps 3 > gpurun_out/ncu_col_$TAG.log 2>&1
  # TMA-staged column pass: C2R shuffle of a 16-byte-pitch shape (14414 x 6564 fp32)
  timeout 600 $NCU -k regex:col_tile -c 1 -s 2 -o $REP/coltma_$TAG \
      python tools/one_shape.py --m 14414 --n 6564 --eb 4 --reps 3 > gpurun_out/ncu_coltma_$TAG.log 2>&1
  # R2C shuffle (scattered source rows, cp.async hulls)
  timeout 600 $NCU -k regex:col_tile -c 1 -s 2 -o $REP/colr2c_$TAG \
      python tools/one_shape.py --m 6565 --n 14414 --eb 4 --reps 3 > gpurun_out/ncu_colr2c_$TAG.log 2>&1
  timeout 600 $NCU -k regex:row_pipe -c 1 -s 2 -o $REP/rowpipe_$TAG \
      python tools/one_shape.py --m 14414 --n 6565 --eb 4 --reps 3 > gpurun_out/ncu_rowpipe_$TAG.log 2>&1
  timeout 600 $NCU -k regex:row_rot -c 1 -s 2 -o $REP/rowrot_$TAG \
      python tools/one_shape.py --m 13497 --n 16245 --eb 8 --reps 3 > gpurun_out/ncu_rowrot_$TAG.log 2>&1
  # chunked fused pass (gcd 2, rows of 24 KB)
  timeout 600 $NCU -k regex:row_chunk -c 1 -s 2 -o $REP/rowchunk_$TAG \
      python tools/one_shape.py --m 17226 --n 6052 --eb 4 --reps 3 > gpurun_out/ncu_rowchunk_$TAG.log 2>&1
  # separate rotation pass at HBM scale (gcd 6600): col_tile_kernel<4,0,128> is COL_ROT
  timeout 600 $NCU -k regex:col_pipe_kernel -c 1 -s 1 -o $REP/colrot_$TAG \
      python tools/one_shape.py --m 19800 --n 13200 --eb 4 --reps 2 > gpurun_out/ncu_colrot_$TAG.log 2>&1
  # cluster row pass (rows of 240 KB fp64)
  timeout 600 $NCU -k regex:row_cluster -c 1 -s 1 -o $REP/rowcluster_$TAG \
      python tools/one_shape.py --m 30011 --n 40009 --eb 8 --reps 2 > gpurun_out/ncu_rowcluster_$TAG.log 2>&1
  # skinny engine: column pass and register row shuffle (AoS -> SoA, 2^26 x 5 fields)
  timeout 600 $NCU -k regex:skinny_col -c 1 -s 1 -o $REP/skinnycol_$TAG \
      python tools/one_shape.py --m 67108864 --n 5 --eb 4 --reps 2 > gpurun_out/ncu_skinnycol_$TAG.log 2>&1
  timeout 600 $NCU -k regex:skinny_reg -c 1 -s 2 -o $REP/skinnyreg_$TAG \
      python tools/one_shape.py --m 67108864 --n 5 --eb 4 --reps 2 > gpurun_out/ncu_skinnyreg_$TAG.log 2>&1
  # AoS consumer kernel, coalesced variant, S = 4 and 7
  # (S = 1..4, copy then store, direct / vector / coalesced, 2 launches each: skip to S = 4
  # coalesced copy)
  timeout 600 $NCU -k regex:aos_kernel -s 40 -c 2 -o $REP/aos_$TAG \
      python tools/aos_bench.py --count 16777216 --max-words 4 --reps 1 > gpurun_out/ncu_aos_$TAG.log 2>&1 ;;
san)
  for tool in memcheck racecheck synccheck; do
    timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_driver.py \
        > gpurun_out/sanitizer_${tool}_$TAG.log 2>&1
    echo "rc=$?" >> gpurun_out/sanitizer_${tool}_$TAG.log
  done ;;
export)
  # keep what travels back small: raw metrics + SASS source counters as text
  for r in $REP/*.ncu-rep; do
    b=$(basename $r .ncu-rep)
    ncu -i $r --page raw --csv > gpurun_out/${b}_raw.csv 2>/dev/null
    ncu -i $r --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/${b}_sass.csv.gz
    python tools/ncu_summary.py $r > gpurun_out/${b}_summary.txt 2>&1
  done ;;
esac
done
du -sh gpurun_out
