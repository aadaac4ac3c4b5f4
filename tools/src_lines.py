"""Per-source-line totals from `ncu --page source --csv --print-source cuda,sass`:
stall samples and executed warp instructions (top N by instructions)."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
k = int(sys.argv[2]) if len(sys.argv) > 2 else 40
per, fname, cur, hdr = {}, None, None, None
for r in rows:
    if not r: continue
    if r[0] == 'File Path': fname = r[1].split('/')[-1]; continue
    if r[0] == 'Function Name': continue
    if r[0] == 'Line No': hdr = r; si = hdr.index('Warp Stall Sampling (All Samples)'); ii = hdr.index('Instructions Executed'); continue
    if r[0].strip():
        cur = (fname, int(r[0]), r[1].strip()[:90]); continue
    try: s = int(r[si] or 0); ie = int(r[ii] or 0)
    except (ValueError, IndexError): continue
    d = per.setdefault(cur, [0, 0]); d[0] += s; d[1] += ie
ts = sum(v[0] for v in per.values()) or 1; ti = sum(v[1] for v in per.values()) or 1
print('samples', ts, 'instructions', ti)
for key, (s, ie) in sorted(per.items(), key=lambda x: -x[1][1])[:k]:
    print(f'{100*ie/ti:5.1f}% i {100*s/ts:5.1f}% s  {key[0]}:{key[1]}  {key[2]}')
