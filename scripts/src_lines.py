"""Per-CUDA-source-line totals (stall samples, instructions) of one kernel in an
ncu report: python scripts/src_lines.py REPORT KERNEL_REGEX [x [N]] (x: sort by instructions)."""
import csv,sys,collections
rep,kern=sys.argv[1],sys.argv[2]
import subprocess
out=subprocess.run(['ncu','-i',rep,'--page','source','--csv','-k','regex:'+kern,'--print-source','cuda,sass'],capture_output=True,text=True).stdout
rows=list(csv.reader(out.splitlines()))
fname=None; hdr=None; agg=[]
for r in rows:
    if not r: continue
    if r[0]=='File Path': fname=r[1].split('/')[-1]; continue
    if r[0]=='Line No': hdr=r; continue
    if hdr is None or r[0]=='' : continue
    if r[0] in ('Function Name',): continue
    try:
        d=dict(zip(hdr[2:],r[2:]))
        agg.append((fname,int(r[0]),r[1][:90],int(d['Warp Stall Sampling (All Samples)']),int(d['Instructions Executed'])))
    except Exception as e: pass
ts=sum(a[3] for a in agg); ti=sum(a[4] for a in agg)
print('total samples',ts,'instr',ti)
key=3 if len(sys.argv)<4 else 4
for a in sorted(agg,key=lambda a:-a[key])[:int(sys.argv[4]) if len(sys.argv)>4 else 45]:
    print(f"{a[0][:14]:14s}{a[1]:5d} s={a[3]*100/ts:5.1f}% i={a[4]*100/ti:5.1f}%  {a[2]}")
