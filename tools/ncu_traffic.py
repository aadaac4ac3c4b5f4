"""DRAM traffic per launch of each MFL kernel class from one `ncu --set full`
capture of a whole run (all launches), for bench.py's roofline.traffic:
  python tools/ncu_traffic.py REPORT.ncu-rep WORKLOAD [iterations]
Merges {WORKLOAD: {kernel: bytes_per_launch, "_source": ...}} into
profiles/traffic.json.  Kernel classes use bench.py's names; a launch is what
bench.py's kernel statistics count as one (mfl_giant = count + finish of one
iteration, so its bytes are divided by the iteration count)."""
import csv, io, json, os, subprocess, sys, collections

rep, workload = sys.argv[1], sys.argv[2]
iters = int(sys.argv[3]) if len(sys.argv) > 3 else None
out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(out)))
hdr = r[0]
ki, rd, wr = hdr.index('Kernel Name'), hdr.index('dram__bytes_read.sum'), hdr.index('dram__bytes_write.sum')
units = r[1]
scale = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}


def cls(name):
    if 'mfl_block<' in name:  # template args: <VAR, BLOCK, ...>
        return 'mfl_block_m' if name.split('<')[1].split(',')[1].strip() == '128' else 'mfl_block_l'
    for k in ('mfl_low', 'mfl_warp', 'mfl_giant', 'mfl_mono', 'mfl_wt_warp', 'mfl_wt_block'):
        if k in name:
            return k
    return None


tot = collections.defaultdict(float)
cnt = collections.Counter()
for row in r[2:]:
    c = cls(row[ki])
    if not c:
        continue
    b = float(row[rd].replace(',', '')) * scale[units[rd]] + float(row[wr].replace(',', '')) * scale[units[wr]]
    tot[c] += b
    cnt[c] += 1
res = {}
for c in tot:
    n = iters if (c == 'mfl_giant' and iters) else cnt[c]
    res[c] = round(tot[c] / n)
res['_source'] = f'{os.path.basename(rep)}: ncu --set full, {sum(cnt.values())} launches, dram__bytes_read.sum + dram__bytes_write.sum'
path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), 'profiles', 'traffic.json')
allv = json.load(open(path)) if os.path.exists(path) else {}
allv[workload] = res
json.dump(allv, open(path, 'w'), indent=1)
print(json.dumps(res, indent=1))
