"""Per-kernel totals of an ncu launch list (--metrics gpu__time_duration.sum --csv).
    python tools/launch_summary.py gpurun_out/build_launches.csv [--skip N]"""
import csv
import json
import re
import sys
from collections import defaultdict

path = sys.argv[1]
skip = int(sys.argv[sys.argv.index("--skip") + 1]) if "--skip" in sys.argv else 0
rows = [r for r in csv.reader(open(path)) if len(r) > 10]
hdr = rows[0]
ik, iu, iv = hdr.index("Kernel Name"), hdr.index("Metric Unit"), hdr.index("Metric Value")
tot, cnt = defaultdict(float), defaultdict(int)
for r in rows[1 + skip:]:
    if r[hdr.index("Metric Name")] != "gpu__time_duration.sum":
        continue
    name = re.sub(r"\(.*", "", r[ik]).replace("void ", "").replace("ganns::", "")
    v = float(r[iv].replace(",", ""))
    v *= {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "nsecond": 1e-6, "ms": 1.0, "msecond": 1.0}.get(r[iu], 1.0)
    tot[name] += v
    cnt[name] += 1
out = {k: {"launches": cnt[k], "total_ms": round(tot[k], 3), "mean_us": round(tot[k] / cnt[k] * 1e3, 2)}
       for k in sorted(tot, key=lambda k: -tot[k])}
print(json.dumps(out, indent=1))
