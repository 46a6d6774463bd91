"""Per-SASS-instruction execution counts of an ncu report, normalised per unit:
python tools/sass_counts.py rep.ncu-rep UNITS [min_per_unit]"""
import csv, subprocess, sys
rep, units = sys.argv[1], float(sys.argv[2])
lo = float(sys.argv[3]) if len(sys.argv) > 3 else 1.0
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout.splitlines()
r = list(csv.reader(txt))
h = r[1]
ie, ss = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
tot = sum(float(x[ie] or 0) for x in r[2:])
print(f"total {tot:.4g}  per unit {tot / units:.1f}")
for i, x in enumerate(r[2:]):
    c = float(x[ie] or 0) / units
    if c >= lo:
        print(f"{i:5d} {c:8.1f} {x[ss]:>6s}  {x[1][:80]}")
