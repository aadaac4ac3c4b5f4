"""Executed warp instructions by SASS opcode from an ncu 'cuda,sass' source CSV."""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
ops = collections.Counter(); tot = 0
for r in rows:
    if len(r) > 8 and r[0] == '' and r[2].startswith('0x'):
        try: ie = int(r[7] or 0)
        except ValueError: continue
        sass = r[3].strip()
        if sass.startswith('@'): sass = sass.split(None, 1)[1]
        op = sass.split()[0] if sass else '?'
        ops[op] += ie; tot += ie
print('total warp instructions', tot)
for op, v in ops.most_common(int(sys.argv[2]) if len(sys.argv) > 2 else 30):
    print(f'{100*v/tot:5.1f}%  {op}')
