"""Build k_bnd_sym tuning variants (EFIT_SYM_UNR x EFIT_SYM_BUF) into tune/*.so (git-ignored)."""
import os, sys
from concurrent.futures import ThreadPoolExecutor
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_anteparawkbml23_b200 import build as b
variants = [tuple(map(int, v.split("x"))) for v in sys.argv[1:]] or [(2, 3), (2, 4), (3, 3), (1, 6), (4, 2)]
os.makedirs(os.path.join(ROOT, "tune"), exist_ok=True)
def one(v):
    u, n = v
    return b.build(force=True, defines=[f"EFIT_SYM_UNR={u}", f"EFIT_SYM_BUF={n}"],
                   out=os.path.join(ROOT, "tune", f"libefit_u{u}b{n}.so"))
with ThreadPoolExecutor(len(variants)) as ex:
    for p in ex.map(one, variants):
        print(p)
