NCU="ncu --set full --clock-control none --import-source on -f"
timeout 600 $NCU -k regex:row_rot -c 1 -s 2 -o /tmp/rr16 python tools/one_shape.py --m 15952 --n 11216 --eb 4 --reps 3 > gpurun_out/ncu_rr16.log 2>&1
python tools/ncu_summary.py /tmp/rr16.ncu-rep > gpurun_out/rr16_summary.txt 2>&1
python tools/ncu_source.py /tmp/rr16.ncu-rep 30 > gpurun_out/rr16_source.txt 2>&1
ncu -i /tmp/rr16.ncu-rep --page raw --csv > gpurun_out/rr16_raw.csv 2>&1
