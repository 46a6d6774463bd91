"""SASS instruction count of one encode kernel instantiation by source phase
(code-size / i-cache budget).  usage: python tools/sass_by_phase.py enc.sass Li4ELi1"""
import collections, re, sys
sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.abspath(__file__)))
from phase_ranges import ranges, phase_of
RS = ranges()
txt = open(sys.argv[1]).read().split("\n")
tag = sys.argv[2]
inside = False; cur = None; cnt = collections.Counter()
for line in txt:
    if line.startswith("//--------------------- .text."):
        inside = tag in line
        continue
    if not inside:
        continue
    m = re.search(r'line (\d+)', line) if "//##" in line else None
    if m:
        f = re.search(r'File "([^"]+)"', line)
        cur = ((f.group(1).split("/")[-1]) if f else "?", int(m.group(1)))
        continue
    if re.search(r"/\*[0-9a-f]{4}\*/", line):
        cnt[cur] += 1
agg = collections.Counter()
for key, c in cnt.items():
    f, l = key if key else ("?", 0)
    nm = phase_of(l, RS) if f == "encode.cu" else f
    agg[nm] += c
print("total", sum(agg.values()))
for k, v in agg.most_common():
    print(f"{v:6d} {k}")
