"""Build libcrocco tuning variants into build/variants/ (timed by tools/kbench.py on the GPU).
usage: python tools/build_variants.py name:DEF1,DEF2 name2:DEF3 ..."""
import os, sys
from concurrent.futures import ThreadPoolExecutor
sys.path.insert(0, os.getcwd())
from paper_conf_ipps_davissngmb23_b200 import build as B
os.makedirs("build/variants", exist_ok=True)
for f in os.listdir("build/variants"):
    os.remove(os.path.join("build/variants", f))
specs = []
for a in sys.argv[1:]:
    name, _, defs = a.partition(":")
    specs.append((name, [d for d in defs.split(",") if d]))
with ThreadPoolExecutor(4) as ex:
    list(ex.map(lambda s: B.build(force=True, defines=s[1], out=f"build/variants/libcrocco_{s[0]}.so"), specs))
print("built", [s[0] for s in specs])
