"""Top stall sites of one kernel in an ncu report: SASS lines with the most warp-stall samples.

    python tools/ncu_stalls.py gpurun_out/prof.ncu-rep [min_pct]
"""
import csv
import io
import subprocess
import sys

path = sys.argv[1]
minpct = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
out = subprocess.run(['ncu', '-i', path, '--page', 'source', '--csv', '--print-source', 'sass'],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = next(i for i, r in enumerate(rows) if 'Source' in r and 'Instructions Executed' in r)
h = rows[hi]
isrc, ia, ist, iad = h.index('Source'), h.index('Instructions Executed'), \
    h.index('Warp Stall Sampling (All Samples)'), h.index('Address')
body = [r for r in rows[hi + 1:] if len(r) > ist and r[ist].isdigit()]
tot = sum(int(r[ist]) for r in body) or 1
print('total samples', tot, 'instructions', len(body))
for idx, r in enumerate(body):
    if int(r[ist]) >= minpct / 100 * tot:
        print('--')
        for rr in body[max(0, idx - 4):idx + 1]:
            print(f"{rr[iad][-5:]} {100*int(rr[ist])/tot:5.1f}% {rr[ia]:>9} {rr[isrc][:90]}")
