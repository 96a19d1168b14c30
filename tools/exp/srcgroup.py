"""Group ncu source-page rows by line ranges of l1_gram.cu (phase attribution)."""
import csv, sys, re
rows = list(csv.reader(open(sys.argv[1])))
ranges = [tuple(x.split(":")) for x in sys.argv[2:]]  # name:lo-hi
fname, hdr = None, None
agg = {}
tot_s = tot_i = 0
for r in rows:
    if not r: continue
    if r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = r; continue
    if hdr is None or r[0] == "" or not r[0].isdigit(): continue
    s, ie = int(r[4]), int(r[7]) if r[7].isdigit() else 0
    tot_s += s; tot_i += ie
    key = fname
    if fname == "l1_gram.cu":
        ln = int(r[0]); key = "l1:other"
        for name, span in ranges:
            lo, hi = map(int, span.split("-"))
            if lo <= ln <= hi: key = name
    a = agg.setdefault(key, [0, 0]); a[0] += s; a[1] += ie
print(f"total samples {tot_s} instr {tot_i/1e9:.2f}G")
for k, (s, i) in sorted(agg.items(), key=lambda x: -x[1][0]):
    print(f"{k:20s} samples {100*s/tot_s:5.1f}%  instr {100*i/tot_i:5.1f}%")
