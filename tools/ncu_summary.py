"""Summarise an ncu report (raw page) into the metrics we track; optional JSON output.

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep [--json out.json --key name --alg-bytes B]
"""
import csv
import io
import json
import subprocess
import sys

KEYS = ['Kernel Name', 'gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 'launch__registers_per_thread',
        'launch__grid_size', 'launch__block_size', 'launch__cluster_dim_x', 'launch__shared_mem_per_block_dynamic',
        'launch__occupancy_limit_shared_mem', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'smsp__inst_executed.sum', 'sm__instruction_throughput.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed',
        'lts__t_sectors_srcunit_tex_op_read.sum', 'lts__t_sectors_srcunit_tex_op_write.sum',
        'lts__throughput.avg.pct_of_peak_sustained_elapsed', 'l1tex__throughput.avg.pct_of_peak_sustained_active']


def raw(path):
    out = subprocess.run(['ncu', '-i', path, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    return [{h: (v, u) for h, u, v in zip(hdr, units, r)} for r in rows[2:]]


def main():
    path = sys.argv[1]
    for rec in raw(path):
        for k in KEYS:
            if k in rec:
                print(f'{k:80s} {rec[k][0]:>24s} {rec[k][1]}')
        if '--json' in sys.argv:
            out = sys.argv[sys.argv.index('--json') + 1]
            key = sys.argv[sys.argv.index('--key') + 1]
            alg = float(sys.argv[sys.argv.index('--alg-bytes') + 1])
            scale = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}
            rd = float(rec['dram__bytes_read.sum'][0]) * scale[rec['dram__bytes_read.sum'][1]]
            wr = float(rec['dram__bytes_write.sum'][0]) * scale[rec['dram__bytes_write.sum'][1]]
            try:
                d = json.load(open(out))
            except Exception:
                d = {}
            d[key] = {'dram_bytes_per_launch': rd + wr, 'dram_read': rd, 'dram_write': wr,
                      'algorithmic_bytes_per_launch': alg, 'kernel': rec['Kernel Name'][0],
                      'duration_us': float(rec['gpu__time_duration.sum'][0]), 'source': path}
            json.dump(d, open(out, 'w'), indent=1)


if __name__ == '__main__':
    main()
