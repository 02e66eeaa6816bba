"""Top CUDA source lines by one stall reason, from
`ncu --page source --csv --print-source cuda,sass` (usage: file reason [n])."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
reason = sys.argv[2]
n = int(sys.argv[3]) if len(sys.argv) > 3 else 15
cur, ix, acc = None, None, {}
for r in rows:
    if len(r) >= 2 and r[0] == "File Path":
        cur = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        ix = {}
        for i, h in enumerate(r):
            ix.setdefault(h, i)
        continue
    if cur and ix and r and r[0].isdigit() and reason in ix:
        try:
            v = float(r[ix[reason]] or 0)
        except ValueError:
            continue
        if v:
            k = (cur, int(r[0]))
            acc[k] = (acc.get(k, (0, ""))[0] + v, r[1].strip()[:90])
tot = sum(v[0] for v in acc.values()) or 1
for (f, ln), (v, src) in sorted(acc.items(), key=lambda kv: -kv[1][0])[:n]:
    print(f"{v / tot:6.1%} {f}:{ln}  {src}")
