"""Build kernel A/B variants of libglp.so under build/ (name=DEF1,DEF2 ...).
  python tools/build_variants.py base= ef=GLP_STREAM_POLICY=1 ...
Each variant is loaded on the GPU with GLP_LIB=build/<name>.so."""
import os, sys
from concurrent.futures import ThreadPoolExecutor
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigmod_yelhls21_b200 import _build
os.makedirs(os.path.join(_build.ROOT, 'build'), exist_ok=True)
jobs = []
for spec in sys.argv[1:]:
    name, _, defs = spec.partition('=')
    jobs.append((os.path.join(_build.ROOT, 'build', name + '.so'), [d for d in defs.split(',') if d]))
with ThreadPoolExecutor(len(jobs)) as ex:
    for out in ex.map(lambda j: _build.build(out=j[0], defines=j[1]), jobs):
        print(out)
