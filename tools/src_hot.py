"""Aggregate an ncu 'cuda,sass' source CSV by CUDA source line: stall samples
and executed instructions per line (top N)."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
k = int(sys.argv[2]) if len(sys.argv) > 2 else 30
per = {}
fname = None
cur_line = None
for r in rows:
    if not r:
        continue
    if r[0] == 'File Path':
        fname = r[1].split('/')[-1]; continue
    if r[0] in ('Function Name', 'Line No'):
        if r[0] == 'Line No':
            hdr = r
        continue
    # cuda rows: first col = line number, second = source text; sass rows have '' line no
    if r[0].strip():
        cur_line = (fname, int(r[0]), r[1].strip()[:80])
        continue
    try:
        s = int(r[4] or 0); ie = int(r[7] or 0)
    except (ValueError, IndexError):
        continue
    d = per.setdefault(cur_line, [0, 0])
    d[0] += s; d[1] += ie
ts = sum(v[0] for v in per.values()) or 1
ti = sum(v[1] for v in per.values()) or 1
print('samples', ts, 'instructions', ti)
for key, v in sorted(per.items(), key=lambda x: -x[1][0])[:k]:
    print(f'{100*v[0]/ts:5.1f}% s {100*v[1]/ti:5.1f}% i  {key[0]}:{key[1]}  {key[2]}')
