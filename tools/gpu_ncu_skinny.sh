NCU="ncu --set full --clock-control none -f"
for op in aos_to_soa soa_to_aos; do
  timeout 600 $NCU -k regex:skinny_col -c 1 -s 1 -o /tmp/skc_$op python tools/skinny_one.py 8 $op > gpurun_out/ncu_skc_$op.log 2>&1
  python tools/ncu_summary.py /tmp/skc_$op.ncu-rep > gpurun_out/skc_${op}_summary.txt 2>&1
  ncu -i /tmp/skc_$op.ncu-rep --page raw --csv > gpurun_out/skc_${op}_raw.csv 2>&1
done
