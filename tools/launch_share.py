"""Per-kernel share of device time from an ncu --metrics gpu__time_duration.sum CSV
(cold-cache, serialised launches: compare shares, not absolute times).
  python tools/launch_share.py launches.csv [prefix1,prefix2]   # keep only these kernels"""
import csv, io, sys, collections
rows = [r for r in csv.reader(io.StringIO(open(sys.argv[1]).read())) if r]
hdr = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
h = rows[hdr]
ki, mi, vi = h.index('Kernel Name'), h.index('Metric Name'), h.index('Metric Value')
tot = collections.defaultdict(float); cnt = collections.Counter()
for r in rows[hdr + 1:]:
    if len(r) <= vi or r[mi] != 'gpu__time_duration.sum':
        continue
    name = r[ki].split('(')[0].replace('void ', '')
    if len(sys.argv) > 2 and not any(name.startswith(pfx) for pfx in sys.argv[2].split(',')):
        continue
    v = float(r[vi].replace(',', ''))
    tot[name] += v; cnt[name] += 1
S = sum(tot.values())
print(f'{"kernel":60s} {"launches":>8s} {"total":>12s} {"share":>7s}')
for k, v in sorted(tot.items(), key=lambda x: -x[1]):
    print(f'{k[:60]:60s} {cnt[k]:8d} {v:12.0f} {100*v/S:6.1f}%')
print('unit of total: as in the CSV (ns for gpu__time_duration.sum)')
