#!/bin/bash
# summarize gpurun_out/enc_<cls>.ncu-rep: duration, inst/chunk, IPC, stall mix, top source lines
for c in "$@"; do
  echo "=== $c"
  ncu -i gpurun_out/enc_$c.ncu-rep --page raw --csv 2>/dev/null > /tmp/raw_$c.csv
  python - $c <<'PY'
import csv,sys
r=list(csv.reader(open(f'/tmp/raw_{sys.argv[1]}.csv')))
d=dict(zip(r[0],r[2]))
N=16384
print('dur ms', d.get('gpu__time_duration.sum'), 'inst/chunk %.0f'%(float(d['smsp__inst_executed.sum'])/N), 'ipc', d.get('sm__inst_executed.avg.per_cycle_active'), 'warps/SM', d.get('sm__warps_active.avg.per_cycle_active'))
st={k.replace('smsp__pcsamp_warps_issue_stalled_',''):float(v) for k,v in d.items() if k.startswith('smsp__pcsamp_warps_issue_stalled_') and not k.endswith('not_issued')}
tot=sum(st.values())
print(' '.join(f"{k}:{v/tot*100:.0f}%" for k,v in sorted(st.items(), key=lambda x:-x[1])[:7]))
PY
  ncu -i gpurun_out/enc_$c.ncu-rep --page source --csv --print-source cuda,sass 2>/dev/null > /tmp/cs_$c.csv
  python tools/srcprof.py /tmp/cs_$c.csv ${TOPN:-25}
done
