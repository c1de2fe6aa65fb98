"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per kernel
launches, total time and share of the profiled device time (cold-cache, serialised).

    python tools/launch_summary.py gpurun_out/launches.csv [--json out.json]
"""
import csv
import json
import re
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
h = rows[hi]
ik, iv, im, iu = h.index('Kernel Name'), h.index('Metric Value'), h.index('Metric Name'), h.index('Metric Unit')
agg = defaultdict(lambda: [0, 0.0])
for r in rows[hi + 1:]:
    if len(r) <= iv or r[im] != 'gpu__time_duration.sum':
        continue
    name = r[ik]
    m = re.search(r'(\w+_kernel)<([^>]*)>', name) or re.search(r'(\w+)\(', name)
    key = (m.group(1) + ('<' + m.group(2) + '>' if m.lastindex and m.lastindex > 1 else '')) if m else name[:60]
    if 'ipt::' not in name and '<unnamed>::' not in name.split('(')[0][:0] and not any(
            k in name for k in ('row_', 'col_', 'skinny_')):
        key = 'other: ' + name[:50]
    scale = {'ns': 1e-6, 'us': 1e-3, 'ms': 1.0, 'usecond': 1e-3, 'nsecond': 1e-6, 'msecond': 1.0}.get(r[iu], 1e-6)
    agg[key][0] += 1
    agg[key][1] += float(r[iv].replace(',', '')) * scale
ours = {k: v for k, v in agg.items() if not k.startswith('other')}
tot = sum(v[1] for v in ours.values()) or 1.0
out = []
for k, (n, ms) in sorted(ours.items(), key=lambda kv: -kv[1][1]):
    out.append({'kernel': k, 'launches': n, 'ms': round(ms, 3), 'share_of_ipt_time': round(ms / tot, 4)})
    print(f'{k:45s} {n:6d} {ms:10.3f} ms  {100 * ms / tot:5.1f}%')
other = sum(v[1] for k, v in agg.items() if k.startswith('other'))
print(f'other (torch fill/flush) {sum(v[0] for k, v in agg.items() if k.startswith("other"))} launches {other:.3f} ms')
if '--json' in sys.argv:
    json.dump(out, open(sys.argv[sys.argv.index('--json') + 1], 'w'), indent=1)
