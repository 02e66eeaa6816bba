"""Per-CUDA-source-line warp-stall samples of one stall reason (column of
`ncu --page source --csv --print-source cuda,sass`), e.g. stall_long_sb."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
col = sys.argv[2]
cur = None
ix = None
out = []
for r in rows:
    if len(r) >= 2 and r[0] == "File Path":
        cur = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        ix = {h: i for i, h in enumerate(r)}
        continue
    if cur and ix and r and r[0].isdigit():
        try:
            v = float(r[ix[col]] or 0)
        except (ValueError, IndexError, KeyError):
            continue
        if v:
            out.append((v, cur, int(r[0]), r[1].strip()[:90]))
tot = sum(o[0] for o in out) or 1
for o in sorted(out, key=lambda o: -o[0])[: int(sys.argv[3]) if len(sys.argv) > 3 else 15]:
    print(f"{o[0] / tot:6.1%}  {o[1]}:{o[2]}  {o[3]}")
