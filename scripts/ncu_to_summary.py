"""Update profiles/ncu_summary.json from an `ncu --set full` report (round 2): DRAM bytes read +
written per launch, duration, registers, grid/block for the named kernels (first launch of each).
python scripts/ncu_to_summary.py report.ncu-rep tag k_bnd_sym k_response ..."""
import csv
import json
import os
import subprocess
import sys

rep, tag, names = sys.argv[1], sys.argv[2], sys.argv[3:]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr, units, data = rows[0], rows[1], rows[2:]
col = {h: i for i, h in enumerate(hdr)}


def val(r, key):
    v = r[col[key]].replace(",", "")
    try:
        return float(v)
    except ValueError:
        return None


path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_summary.json")
summ = json.load(open(path)) if os.path.exists(path) else {}
summ.update({"config": "C4", "world": 1, "round": 2,
             "source": f"ncu --set full --clock-control none, bench.py C4 513^2 ({tag}); profiles/r02_summary.md"})
for name in names:
    for r in data:
        if name in r[col["Kernel Name"]]:
            scale = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
            rd = val(r, "dram__bytes_read.sum") * scale.get(units[col["dram__bytes_read.sum"]], 1.0)
            wr = val(r, "dram__bytes_write.sum") * scale.get(units[col["dram__bytes_write.sum"]], 1.0)
            dur = val(r, "gpu__time_duration.sum")
            du = units[col["gpu__time_duration.sum"]]
            dur_us = dur / 1e3 if du == "nsecond" else (dur * 1e3 if du == "msecond" else dur)
            summ[name] = {"dram_bytes_read": rd, "dram_bytes_write": wr, "dram_bytes_per_launch": rd + wr,
                          "duration_us": round(dur_us, 3),
                          "registers_per_thread": val(r, "launch__registers_per_thread"),
                          "grid": val(r, "launch__grid_size"), "block": val(r, "launch__block_size"),
                          "source": f"{tag} (round 2 capture)"}
            break
json.dump(summ, open(path, "w"), indent=1)
print(json.dumps({k: summ[k] for k in names if k in summ}, indent=1))
