"""Phase line ranges of csrc/encode.cu, derived from its own markers (function
definitions and the '// ---- ' phase comments), for the profiling summaries."""
import os, re
SRC = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                   "paper_conf_pact_map17_b200", "csrc", "encode.cu")


def ranges(path=SRC):
    lines = open(path).read().split("\n")
    marks = []
    for i, l in enumerate(lines, 1):
        m = re.match(r"__device__ __forceinline__ \w+ (\w+)\(", l) or re.match(r"__global__ .* (\w+)\(", l)
        if m:
            marks.append((i, m.group(1)))
            continue
        m = re.match(r"\s*// ---- (.*)", l)
        if m:
            marks.append((i, m.group(1)[:28]))
    out = []
    for j, (i, nm) in enumerate(marks):
        end = marks[j + 1][0] - 1 if j + 1 < len(marks) else len(lines)
        out.append((nm, i, end))
    return out


def phase_of(line, rs):
    for nm, a, b in rs:
        if a <= line <= b:
            return nm
    return "encode.cu other"
