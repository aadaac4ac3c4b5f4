"""Summarise an ncu --page source --print-source sass CSV: top instructions by
executed count and by stall samples."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ie = hdr.index('Instructions Executed'); ss = hdr.index('Warp Stall Sampling (All Samples)'); src = hdr.index('Source')
data = []
for r in rows[2:]:
    try:
        data.append((int(r[ie] or 0), int(r[ss] or 0), r[src].strip(), r[0]))
    except Exception:
        pass
tot_i = sum(d[0] for d in data); tot_s = sum(d[1] for d in data)
print('instructions', tot_i, 'samples', tot_s, 'n', len(data))
k = int(sys.argv[2]) if len(sys.argv) > 2 else 25
print('--- by samples')
for d in sorted(data, key=lambda x: -x[1])[:k]:
    print(f'{100*d[1]/max(tot_s,1):5.1f}% s {100*d[0]/max(tot_i,1):5.1f}% i  {d[2][:70]}  {d[3][-5:]}')
# instruction mix by opcode
from collections import Counter
c = Counter()
for d in data:
    op = d[2].split()[0] if d[2] else '?'
    if op.startswith('@'): op = d[2].split()[1]
    c[op.split('.')[0]] += d[0]
print('--- opcode mix (executed)')
for op, v in c.most_common(18):
    print(f'{op:10s} {100*v/tot_i:5.1f}%')
