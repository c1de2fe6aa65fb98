ncu --set full --clock-control none --import-source on -k regex:row_ -c 1 -s 2 -f -o gpurun_out/rowrot_c2 python tools/one_shape.py --m 6314 --n 5378 --eb 4 --reps 3 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:row_ -c 1 -s 2 -f -o gpurun_out/rowrot_c2_r2c python tools/one_shape.py --m 6314 --n 5378 --eb 4 --reps 3 --op r2c > /dev/null 2>&1
