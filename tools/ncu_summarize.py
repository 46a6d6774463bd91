"""Summarize the ncu captures of tools/ncu_bench.sh into profiles/ (run here, no GPU).
usage: python tools/ncu_summarize.py r01"""
import csv, io, json, os, subprocess, sys
R = sys.argv[1] if len(sys.argv) > 1 else "r01"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_pact_map17_b200._build import source_hash  # noqa: E402
out = {}
# launch list -> per-kernel share
rows = list(csv.reader(open(os.path.join(ROOT, "gpurun_out", f"launches_{R}.csv"))))
hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hi]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
per = {}
for r in rows[hi + 1:]:
    if len(r) <= vi:
        continue
    name = r[ki].split("(")[0].replace("lzr::<unnamed>::", "").replace("void ", "")
    v = float(r[vi].replace(",", ""))
    unit = r[ui]
    ns = v * {"ns": 1, "usecond": 1e3, "us": 1e3, "msecond": 1e6, "ms": 1e6, "nsecond": 1}.get(unit, 1)
    per.setdefault(name, []).append(ns)
tot = sum(sum(v) for k, v in per.items() if k.startswith("lzr_"))
out["launches"] = {k: {"count": len(v), "mean_us": sum(v) / len(v) / 1e3,
                       "share_of_lzr_time": (sum(v) / tot if k.startswith("lzr_") else None)}
                   for k, v in per.items()}
# full capture of the encode kernel
rep = os.path.join(ROOT, "gpurun_out", f"encode_full_{R}.ncu-rep")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(io.StringIO(raw)))
d = dict(zip(rr[0], rr[2]))
u = dict(zip(rr[0], rr[1]))
def val(k):
    x = float(d[k].replace(",", ""))
    unit = u.get(k, "")
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
            "msecond": 1e-3, "ms": 1e-3, "us": 1e-6, "ns": 1e-9, "second": 1}.get(unit, 1)
    return x * mult
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__inst_executed.avg.per_cycle_active", "smsp__inst_executed.sum",
        "sm__warps_active.avg.per_cycle_active", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "launch__shared_mem_per_block_dynamic", "launch__grid_size", "launch__block_size"]
full = {k: val(k) for k in keys if k in d}
stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(v) for k, v in d.items()
          if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")}
st = sum(stalls.values())
full["stall_share"] = {k: round(v / st, 3) for k, v in sorted(stalls.items(), key=lambda x: -x[1])[:8]}
full["dram_bytes_per_launch"] = full.get("dram__bytes_read.sum", 0) + full.get("dram__bytes_write.sum", 0)
out["encode_full"] = full
workload = "cfg2: 256 MiB mix per GPU, C=W=4096, m=4, M=259"
summ_path = os.path.join(ROOT, "profiles", "encode_ncu_summary.json")
summ = json.load(open(summ_path)) if os.path.exists(summ_path) else {}
bpath = os.path.join(ROOT, "gpurun_out", f"build_{R}.txt")
build = open(bpath).read().strip() if os.path.exists(bpath) else source_hash()
summ[workload] = {"round": R, "build": build, "dram_bytes_per_launch": full["dram_bytes_per_launch"],
                  "duration_s": full.get("gpu__time_duration.sum"),
                  "warp_inst_per_launch": full.get("smsp__inst_executed.sum"),
                  "ipc": full.get("sm__inst_executed.avg.per_cycle_active"),
                  "smem_pipe_pct": full.get("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed"),
                  "stall_share": full.get("stall_share"),
                  "source": f"profiles/ncu_{R}.json (ncu --set full, one encode launch of bench.py)"}
json.dump(summ, open(summ_path, "w"), indent=1)
json.dump(out, open(os.path.join(ROOT, "profiles", f"ncu_{R}.json"), "w"), indent=1)
print(json.dumps(out, indent=1))
