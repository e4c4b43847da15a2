"""Build k_bnd_sym tuning variants into tune/*.so (git-ignored).  Variant "u2b3w1m2" = EFIT_SYM_UNR=2,
EFIT_SYM_BUF=3, EFIT_SYM_WG=1, EFIT_SYM_MINB=2 (m optional)."""
import os, re, shutil, sys
from concurrent.futures import ThreadPoolExecutor
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_anteparawkbml23_b200 import build as b
variants = sys.argv[1:] or ["u2b3w1", "u2b2w2", "u1b3w2", "u2b3w2", "u1b4w2"]
tdir = os.path.join(ROOT, "tune")
shutil.rmtree(tdir, ignore_errors=True)
os.makedirs(tdir)
def one(v):
    u, n, w, m = re.fullmatch(r"u(\d+)b(\d+)w(\d+)(?:m(\d+))?", v).groups()
    return b.build(force=True, defines=[f"EFIT_SYM_UNR={u}", f"EFIT_SYM_BUF={n}", f"EFIT_SYM_WG={w}",
                                        f"EFIT_SYM_MINB={m or 0}"],
                   out=os.path.join(tdir, f"libefit_{v}.so"))
with ThreadPoolExecutor(len(variants)) as ex:
    for p in ex.map(one, variants):
        print(p)
