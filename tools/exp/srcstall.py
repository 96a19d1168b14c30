"""Aggregate an ncu source-page CSV (`ncu -i X --page source --csv --print-source cuda,sass`): warp
stall samples per CUDA source line with the top reasons, and per SASS opcode.
Usage: srcstall.py page.csv [top] [--sass]"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2].isdigit() else 30
fname, hdr = None, None
per_line = collections.defaultdict(lambda: [0, collections.Counter(), ""])
per_op = collections.defaultdict(lambda: [0, collections.Counter()])
tot = 0
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        i_s = hdr.index("Warp Stall Sampling (All Samples)")
        reasons = [(j, h) for j, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
        continue
    if hdr is None or len(r) <= i_s:
        continue
    try:
        s = int(r[i_s])
    except ValueError:
        continue
    if s == 0:
        continue
    if r[0]:  # CUDA source line (aggregate of the SASS rows that follow it)
        tot += s
        e = per_line[(fname, r[0])]
        e[0] += s
        e[2] = e[2] or r[1][:80]
        for j, h in reasons:
            if r[j].isdigit() and int(r[j]):
                e[1][h[6:]] += int(r[j])
        continue
    if not r[2].startswith("0x"):
        continue
    t = r[3].split()
    op = t[1] if t and t[0].startswith("@") and len(t) > 1 else (t[0] if t else "?")
    o = per_op[op.split(".")[0]]
    o[0] += s
    for j, h in reasons:
        if r[j].isdigit() and int(r[j]):
            o[1][h[6:]] += int(r[j])
print("total samples", tot)
for (f, ln), (s, rs, src) in sorted(per_line.items(), key=lambda x: -x[1][0])[:top]:
    print(f"{100*s/tot:5.1f}% {f}:{ln:5s} {src:80s} {' '.join(f'{k}={v}' for k, v in rs.most_common(3))}")
print("--- per SASS opcode")
for op, (s, rs) in sorted(per_op.items(), key=lambda x: -x[1][0])[:25]:
    print(f"{100*s/tot:5.1f}% {op:10s} {' '.join(f'{k}={v}' for k, v in rs.most_common(4))}")
