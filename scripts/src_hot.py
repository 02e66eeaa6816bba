"""Per-CUDA-source-line totals from `ncu --page source --csv --print-source cuda,sass`."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
cur = None
out = []
ix = None
for r in rows:
    if len(r) >= 2 and r[0] == "File Path":
        cur = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        ix = {h: i for i, h in enumerate(r)}
        continue
    if cur and ix and r and r[0].isdigit():
        try:
            ins = float(r[ix["Instructions Executed"]] or 0)
            smp = float(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
        except (ValueError, IndexError):
            continue
        if ins or smp:
            out.append((ins, smp, cur, int(r[0]), r[1].strip()[:90]))
tot = sum(o[0] for o in out) or 1
ts = sum(o[1] for o in out) or 1
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
for o in sorted(out, key=lambda o: -o[0])[:n]:
    print(f"{o[0] / tot:6.1%} inst {o[1] / ts:6.1%} stall  {o[2]}:{o[3]}  {o[4]}")
