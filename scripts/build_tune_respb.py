"""Build k_response_mma tuning variants into tune/*.so (git-ignored): "np4m3" = EFIT_RESPB_NP=4,
EFIT_RESPB_MINB=3 (ring depth, min CTAs per SM)."""
import os, re, shutil, sys
from concurrent.futures import ThreadPoolExecutor
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_anteparawkbml23_b200 import build as b
variants = sys.argv[1:] or ["np4m3", "np4m2", "np16m2"]
tdir = os.path.join(ROOT, "tune")
shutil.rmtree(tdir, ignore_errors=True)
os.makedirs(tdir)
def one(v):
    npv, m = re.fullmatch(r"np(\d+)m(\d+)", v).groups()
    return b.build(force=True, defines=[f"EFIT_RESPB_NP={npv}", f"EFIT_RESPB_MINB={m}"],
                   out=os.path.join(tdir, f"libefit_{v}.so"))
with ThreadPoolExecutor(len(variants)) as ex:
    for p in ex.map(one, variants):
        print(p)
for f in os.listdir(os.path.join(ROOT, "paper_conf_sc_anteparawkbml23_b200", "csrc")):
    if ".libefit_" in f:
        os.remove(os.path.join(ROOT, "paper_conf_sc_anteparawkbml23_b200", "csrc", f))
