"""Static SASS instruction count per kernel of a .so (cuobjdump -sass)."""
import re, subprocess, sys
out = subprocess.run(['cuobjdump', '-sass', sys.argv[1]], capture_output=True, text=True).stdout
cur = None; cnt = {}
for line in out.splitlines():
    m = re.match(r'\s+Function : (\S+)', line)
    if m: cur = m.group(1); cnt[cur] = 0; continue
    if cur and re.match(r'\s+/\*[0-9a-f]{4}\*/', line): cnt[cur] += 1
pat = sys.argv[2] if len(sys.argv) > 2 else ''
for k, v in sorted(cnt.items()):
    if pat in k: print(v, k)
