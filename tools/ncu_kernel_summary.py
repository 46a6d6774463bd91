"""Key metrics of one ncu --set full capture (any kernel) as JSON:
python tools/ncu_kernel_summary.py rep.ncu-rep [label] > profiles/ncu_<label>.json"""
import csv, io, json, subprocess, sys

rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(io.StringIO(raw)))
d, u = dict(zip(rr[0], rr[2])), dict(zip(rr[0], rr[1]))
KEYS = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__inst_executed.avg.per_cycle_active", "smsp__inst_executed.sum", "sm__warps_active.avg.per_cycle_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic", "launch__grid_size",
        "launch__block_size", "launch__occupancy_limit_shared_mem", "launch__occupancy_limit_registers"]
out = {"label": sys.argv[2] if len(sys.argv) > 2 else rep}
for k in KEYS:
    if k in d:
        v = d[k]
        try:
            v = float(v.replace(",", ""))
        except ValueError:
            pass
        out[k] = v if u.get(k, "") in ("", None) else {"value": v, "unit": u.get(k)}
st = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(v) for k, v in d.items()
      if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")
      and v.replace(".", "").isdigit()}
t = sum(st.values()) or 1
out["stall_share"] = {k: round(v / t, 3) for k, v in sorted(st.items(), key=lambda x: -x[1])[:8]}
print(json.dumps(out, indent=1))
