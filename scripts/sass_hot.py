"""Summarise an `ncu --page source --print-source sass --csv` dump: top SASS
instructions by executed count and by stall samples, grouped in address ranges."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
data = [r for r in rows[2:] if r and r[0].startswith("0x")]
end = next((i for i, r in enumerate(rows[2:]) if r and r[0] == "Kernel Name"), None)
data = [r for r in (rows[2:2 + end] if end else rows[2:]) if r and r[0].startswith("0x")]
tot_inst = sum(float(r[ix["Instructions Executed"]] or 0) for r in data)
tot_samp = sum(float(r[ix["Warp Stall Sampling (All Samples)"]] or 0) for r in data)
print(f"total warp-instructions {tot_inst:.4g}, stall samples {tot_samp:.4g}")
stall_cols = [h for h in hdr if h.startswith("stall_")]
agg = {h: sum(float(r[ix[h]] or 0) for r in data) for h in stall_cols}
print("stalls:", ", ".join(f"{k[6:]}={v / max(tot_samp, 1):.2f}" for k, v in sorted(agg.items(), key=lambda kv: -kv[1])[:8]))
window = int(sys.argv[2]) if len(sys.argv) > 2 else 40
# contiguous windows of instructions
for start in range(0, len(data), window):
    seg = data[start:start + window]
    ins = sum(float(r[ix["Instructions Executed"]] or 0) for r in seg)
    smp = sum(float(r[ix["Warp Stall Sampling (All Samples)"]] or 0) for r in seg)
    if ins / tot_inst > 0.02 or smp / max(tot_samp, 1) > 0.03:
        ops = [r[ix["Source"]].split()[0] if r[ix["Source"]].strip() else "" for r in seg]
        top = {}
        for o in ops:
            top[o] = top.get(o, 0) + 1
        print(f"[{seg[0][ix['Address']]}..] inst {ins / tot_inst:5.1%} samples {smp / max(tot_samp, 1):5.1%} "
              f"ops {sorted(top.items(), key=lambda kv: -kv[1])[:6]}")
