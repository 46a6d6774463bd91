"""Opcode histogram of every kernel in liblzr.so (cuobjdump -sass): the
instructions that show the sm_100a features in use (UBLKCP = cp.async.bulk TMA,
SYNCS = mbarrier, CREDUX/REDUX = warp reductions, MATCH = match.any, VOTE,
SHFL, ATOMS/RED) plus totals.  usage: python tools/sass_hist.py > profiles/sass_hist_<round>.txt"""
import collections, os, re, subprocess, sys

LIB = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_pact_map17_b200", "liblzr.so")
txt = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True).stdout
KEYS = ["UBLKCP", "SYNCS", "CREDUX", "REDUX", "MATCH", "VOTE", "SHFL", "ATOMS", "ATOMG", "RED", "BAR",
        "LDS", "STS", "LDG", "STG", "FLO", "POPC", "BREV", "STL", "LDL"]
cur, hist = None, {}
for line in txt.splitlines():
    m = re.match(r"\s+Function : (\S+)", line)
    if m:
        cur = m.group(1)
        hist[cur] = collections.Counter()
        continue
    m = re.search(r"/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)(?:\.[A-Z0-9_.]+)?", line)
    if cur and m:
        hist[cur][m.group(1)] += 1
print(f"# cuobjdump -sass {os.path.basename(LIB)} (sm_100a); static instruction counts per kernel")
for fn, c in sorted(hist.items()):
    name = re.sub(r"_ZN3lzr\d+_GLOBAL__N__\w+?_\d+_(\w+?)_cu_\w+?\d+(lzr_\w+?)E", r"\2", fn)
    tot = sum(c.values())
    keys = " ".join(f"{k}={c[k]}" for k in KEYS if c[k])
    print(f"{fn[:120]}\n    total={tot} {keys}")
