import csv, sys, re
# usage: region_prof.py cs.csv encode.cu  -> instruction/sample share per function region of encode.cu
rows=list(csv.reader(open(sys.argv[1])))
src=open(sys.argv[2]).read().splitlines()
# function regions: line of each top-level function definition
regions=[]
for i,l in enumerate(src,1):
    m=re.match(r'^(?:__global__|__device__|static|cudaError_t|inline).*?\b(\w+)\(', l)
    if m and not l.strip().endswith(';'): regions.append((i,m.group(1)))
def region(li):
    name='?'
    for st,nm in regions:
        if li>=st: name=nm
    return name
def num(x):
    try: return float(x)
    except: return 0.0
cur=None; h=None; agg={}
for r in rows:
    if not r: continue
    if r[0]=='File Path': cur=r[1].split('/')[-1]; continue
    if r[0]=='Line No': h=r; ie=h.index('Instructions Executed'); ss=h.index('Warp Stall Sampling (All Samples)'); continue
    if h is None or r[0]=='': continue
    try: li=int(r[0])
    except: continue
    key=region(li) if cur==sys.argv[2].split('/')[-1] else cur
    a=agg.setdefault(key,[0,0]); a[0]+=num(r[ie]); a[1]+=num(r[ss])
ti=sum(v[0] for v in agg.values()); ts=sum(v[1] for v in agg.values())
N=float(sys.argv[3]) if len(sys.argv)>3 else 1
for k,v in sorted(agg.items(), key=lambda x:-x[1][1]):
    print(f"{k:24s} inst {v[0]/ti*100:5.1f}%  ({v[0]/N:9.0f}/chunk)  samples {v[1]/ts*100:5.1f}%")
