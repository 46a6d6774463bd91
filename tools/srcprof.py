import csv, sys
rows=list(csv.reader(open(sys.argv[1])))
curfile=None; h=None; lines=[]
def num(x):
    try: return float(x)
    except: return 0.0
for r in rows:
    if not r: continue
    if r[0]=='File Path': curfile=r[1].split('/')[-1]; continue
    if r[0]=='Line No': h=r; ie=h.index('Instructions Executed'); ss=h.index('Warp Stall Sampling (All Samples)'); continue
    if r[0] in ('Function Name',): continue
    if h is None or r[0]=='' : continue
    try: li=int(r[0])
    except: continue
    lines.append((curfile, li, r[1][:95], num(r[ie]), num(r[ss])))
ti=sum(x[3] for x in lines); ts=sum(x[4] for x in lines)
print('total inst', ti, 'samples', ts)
for f,li,src,inst,smp in sorted(lines, key=lambda x:-x[4])[:int(sys.argv[2]) if len(sys.argv)>2 else 50]:
    print(f"{f[:14]:14s}{li:4d} {inst/ti*100:5.1f}% {smp/ts*100:5.1f}%  {src}")
