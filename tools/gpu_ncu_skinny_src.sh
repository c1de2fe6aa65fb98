NCU="ncu --set full --clock-control none --import-source on -f"
for N in 24 25; do
  timeout 600 $NCU -k regex:skinny_col -c 1 -s 1 -o /tmp/sks_$N python tools/skinny_one.py $N aos_to_soa > /dev/null 2>&1
  python tools/ncu_source.py /tmp/sks_$N.ncu-rep 30 > gpurun_out/sks_${N}_source.txt 2>&1
done
