# ncu captures of the skinny kernels on cfg3 (args: kernel regex, n)
K=${1:-skinny_col}; N=${2:-8}
NCU="ncu --set full --clock-control none -f"
for op in aos_to_soa soa_to_aos; do
  timeout 600 $NCU -k regex:$K -c 1 -s 1 -o /tmp/sk_$op python tools/skinny_one.py $N $op > gpurun_out/ncu_sk_${K}_${N}_$op.log 2>&1
  python tools/ncu_summary.py /tmp/sk_$op.ncu-rep > gpurun_out/sk_${K}_${N}_${op}_summary.txt 2>&1
  ncu -i /tmp/sk_$op.ncu-rep --page raw --csv > gpurun_out/sk_${K}_${N}_${op}_raw.csv 2>&1
done
