"""Static per-kernel SASS instruction-class summary of the built library (cuobjdump -sass):
python scripts/sass_summary.py [lib.so] > profiles/r02_sass_summary.txt.  Classes that prove the
B200 paths: DMMA (FP64 tensor cores, m8n8k4), LDG.*.256 (256-bit streaming loads), UBLKCP (TMA 1-D
bulk copies), SYNCS (mbarriers), ACQBULK (griddepcontrol.wait, PDL), plus the FP64 ALU mix."""
import collections
import re
import subprocess
import sys

lib = sys.argv[1] if len(sys.argv) > 1 else "paper_conf_sc_anteparawkbml23_b200/libefit_b200.so"
txt = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
classes = [("DMMA", r"\bDMMA\."), ("LDG.256", r"\bLDG\.E[^ ]*\.256\b"), ("LDG(other)", r"\bLDG\b"),
           ("UBLKCP", r"\bUBLKCP\b"), ("SYNCS", r"\bSYNCS\."), ("ACQBULK", r"\bACQBULK\b"),
           ("DFMA", r"\bDFMA\b"), ("DADD", r"\bDADD\b"), ("DMUL", r"\bDMUL\b"), ("MUFU", r"\bMUFU\."),
           ("SHFL", r"\bSHFL\."), ("LDS", r"\bLDS\b"), ("STS", r"\bSTS\b"), ("STG", r"\bSTG\b"),
           ("BAR", r"\bBAR\."), ("ATOM", r"\b(RED|ATOMG|ATOM)\b")]
cur, counts, total = None, collections.OrderedDict(), collections.Counter()
for line in txt.splitlines():
    m = re.match(r"\s*Function : (\S+)", line)
    if m:
        cur = m.group(1)
        counts[cur] = collections.Counter()
        continue
    if cur is None or not re.search(r"/\*[0-9a-f]{4}\*/", line):
        continue
    counts[cur]["instructions"] += 1
    for name, pat in classes:
        if re.search(pat, line):
            counts[cur][name] += 1
            if name == "LDG.256":
                break
print(f"# cuobjdump -sass {lib}: static instruction counts per kernel (sm_100a)")
hdr = ["instructions"] + [c[0] for c in classes]
print("kernel," + ",".join(hdr))
for k, c in counts.items():
    dem = subprocess.run(["c++filt", k], capture_output=True, text=True).stdout.strip()
    print(f"\"{dem[:110]}\"," + ",".join(str(c[h]) for h in hdr))
    for h in hdr:
        total[h] += c[h]
print("TOTAL," + ",".join(str(total[h]) for h in hdr))
