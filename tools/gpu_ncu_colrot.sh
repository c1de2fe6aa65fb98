NCU="ncu --set full --clock-control none --import-source on -f"
timeout 600 $NCU -k regex:col_pipe_kernel -c 1 -s 1 -o /tmp/colrot python tools/one_shape.py --m 19800 --n 13200 --eb 4 --reps 2 > gpurun_out/ncu_colrot_fix.log 2>&1
python tools/ncu_summary.py /tmp/colrot.ncu-rep > gpurun_out/colrot_fix_summary.txt 2>&1
