"""Build diagnostic library variants in parallel (-D defines) into build_variants/.

    python tools/build_variants.py name:DEF1=1,DEF2=2 name2:DEF3 ...
"""
import os, sys
from concurrent.futures import ThreadPoolExecutor
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_huangd0lc23_b200 import build as B

os.makedirs(os.path.join(ROOT, "build_variants"), exist_ok=True)
jobs = []
for spec in sys.argv[1:]:
    name, _, defs = spec.partition(":")
    jobs.append((name, [d for d in defs.split(",") if d]))
with ThreadPoolExecutor(8) as ex:
    for name, out in zip([j[0] for j in jobs], ex.map(lambda j: B.build(defines=j[1], out=os.path.join(ROOT, "build_variants", f"{j[0]}.so")), jobs)):
        print(name, out)
