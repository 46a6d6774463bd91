"""Per-CUDA-line instruction / stall-sample totals from an ncu report
(`--page source --print-source cuda,sass`): python tools/srcline_prof.py rep.ncu-rep [top]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
cur_file, cur_line, h = "?", None, None
agg = {}
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        cur_file = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        h = r
        ie = h.index("Instructions Executed")
        ss = h.index("Warp Stall Sampling (All Samples)")
        continue
    if h is None:
        continue
    if r[0]:
        if r[0].isdigit():
            cur_line = (cur_file, int(r[0]), r[1][:90])
        continue
    try:
        inst, smp = float(r[ie] or 0), float(r[ss] or 0)
    except ValueError:
        continue
    a = agg.setdefault(cur_line, [0.0, 0.0])
    a[0] += inst
    a[1] += smp
ti = sum(v[0] for v in agg.values()) or 1
ts = sum(v[1] for v in agg.values()) or 1
print(f"total warp-inst {ti:.4g}  samples {ts:.0f}")
for k, v in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    f, li, src = k if k else ("?", 0, "")
    print(f"{f[:12]:12s}{li:5d} {v[0]/ti*100:5.1f}% {v[1]/ts*100:5.1f}%  {src}")
