"""Top CUDA source lines for one stall reason from an ncu source-page (cuda,sass) CSV."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1]))); reason = sys.argv[2]; top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
fname, hdr, out, tot = None, None, [], 0
for r in rows:
    if not r: continue
    if r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = r; idx = hdr.index(reason); continue
    if hdr is None or not r[0].isdigit(): continue
    v = int(r[idx]) if r[idx].isdigit() else 0
    tot += v; out.append((v, fname, r[0], r[1][:90]))
out.sort(key=lambda x: -x[0]); print(reason, "total", tot)
for v, f, ln, src in out[:top]: print(f"{100*v/tot:5.1f}% {f}:{ln} {src}")
