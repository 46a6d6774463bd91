"""Headline metrics of an ncu report (one kernel): python tools/ncu_brief.py rep.ncu-rep"""
import csv, io, subprocess, sys
want = ["gpu__time_duration.sum", "smsp__inst_executed.sum", "sm__inst_executed.avg.per_cycle_active",
        "sm__warps_active.avg.per_cycle_active", "launch__registers_per_thread",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "dram__bytes_read.sum", "dram__bytes_write.sum"]
for rep in sys.argv[1:]:
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    h, u, v = rows[0], rows[1], rows[2]
    print(rep)
    for w in want:
        if w in h:
            i = h.index(w)
            print(f"  {w:75s} {v[i]:>14s} {u[i]}")
    st = [(h[i], float(v[i].replace(',', '') or 0)) for i in range(len(h))
          if h[i].startswith("smsp__pcsamp_warps_issue_stalled_") and not h[i].endswith("_not_issued")]
    tot = sum(x for _, x in st) or 1
    print("  stalls:", ", ".join(f"{k.replace('smsp__pcsamp_warps_issue_stalled_', '')} {x / tot:.2f}"
                                  for k, x in sorted(st, key=lambda t: -t[1])[:8]))
