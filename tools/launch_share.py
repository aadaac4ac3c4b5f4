"""Per-kernel totals of an `ncu --metrics gpu__time_duration.sum --csv`
launch list: total time, launches and share of all listed launches."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if r and r[0] == 'ID'][0]
hdr = rows[hi]
ki, vi, mi, ui = hdr.index('Kernel Name'), hdr.index('Metric Value'), hdr.index('Metric Name'), hdr.index('Metric Unit')
tot, cnt = collections.Counter(), collections.Counter()
scale = {'ns': 1e-3, 'nsecond': 1e-3, 'us': 1.0, 'usecond': 1.0, 'ms': 1e3, 'msecond': 1e3}
for r in rows[hi + 1:]:
    if len(r) <= vi or r[mi] != 'gpu__time_duration.sum':
        continue
    name = r[ki]
    if 'mfl_block<' in name:
        k = 'mfl_block_m' if name.split('<')[1].split(',')[1].strip() == '128' else 'mfl_block_l'
    else:
        k = name.split('(')[0].split('<')[0].replace('void ', '').replace('glp::', '')
    tot[k] += float(r[vi].replace(',', '')) * scale.get(r[ui], 1.0)
    cnt[k] += 1
T = sum(tot.values())
print(f'{"kernel":24s} {"us total":>12s} {"launches":>9s} {"share":>7s}')
for k, v in tot.most_common():
    print(f'{k:24s} {v:12.1f} {cnt[k]:9d} {v / T:7.3f}')
print(f'{"all":24s} {T:12.1f} {sum(cnt.values()):9d}')
