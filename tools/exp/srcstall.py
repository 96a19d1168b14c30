"""Aggregate ncu source-page (cuda,sass) CSV: stall samples per CUDA source line, top reasons."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
fname, hdr, out, tot = None, None, [], 0
for r in rows:
    if not r: continue
    if r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = r; continue
    if hdr is None or r[0] == "" or r[0] == "Function Name": continue
    try: s = int(r[4])
    except ValueError: continue
    reasons = {h: int(v) for h, v in zip(hdr[31:48], r[31:48]) if v.isdigit() and int(v) > 0}
    tot += s
    out.append((s, fname, r[0], r[1][:70], sorted(reasons.items(), key=lambda x: -x[1])[:3], r[7]))
out.sort(key=lambda x: -x[0])
print("total samples", tot)
for s, f, ln, src, rs, ie in out[:top]:
    print(f"{100*s/tot:5.1f}% {f}:{ln:5s} ie={ie:>10s} {src:70s} {' '.join(f'{k[6:]}={v}' for k,v in rs)}")
