"""Per-source-line instruction and stall-sample shares from an ncu report."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
fname, res = None, []
for r in rows:
    if len(r) >= 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if len(r) > 8 and r[0].isdigit() and r[2] == "-":
        res.append((int(r[7]), int(r[4]), fname, int(r[0]), r[1].strip()[:85]))
tot = sum(x[0] for x in res) or 1
ts = sum(x[1] for x in res) or 1
print(f"total warp instructions {tot}, stall samples {ts}")
for x in sorted(res, key=lambda x: -x[1])[:top]:
    print(f"{x[0] / tot * 100:5.1f}% inst {x[1] / ts * 100:5.1f}% samples  {x[2]}:{x[3]}  {x[4]}")
