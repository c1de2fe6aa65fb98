"""Per-source-line instruction / stall breakdown of an ncu report (needs -lineinfo).

    python tools/ncu_source.py gpurun_out/prof.ncu-rep [top]
"""
import csv
import io
import subprocess
import sys

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(['ncu', '-i', path, '--page', 'source', '--csv', '--print-source', 'cuda,sass'],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
# find header row
hi = next(i for i, r in enumerate(rows) if 'Source' in r and 'Instructions Executed' in r)
h = rows[hi]
isrc, ia, ist = h.index('Source'), h.index('Instructions Executed'), h.index('Warp Stall Sampling (All Samples)')
iline = h.index('#') if '#' in h else None
res = []
for r in rows[hi + 1:]:
    if len(r) <= ia:
        continue
    try:
        n = int(r[ia] or 0)
        s = int(r[ist] or 0)
    except ValueError:
        continue
    res.append((n, s, (r[iline] if iline is not None else ''), r[isrc][:110]))
tot = sum(x[0] for x in res) or 1
tots = sum(x[1] for x in res) or 1
print('total instr', tot, 'total stall samples', tots)
for n, s, ln, src in sorted(res, key=lambda x: -x[0])[:top]:
    print(f'{100*n/tot:5.1f}% instr {100*s/tots:5.1f}% stall  L{ln:>5} {src}')
