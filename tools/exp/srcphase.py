"""Group an ncu source CSV (--print-source cuda,sass) by l1_gram.cu line ranges; per group: samples,
SASS opcode mix of stall samples and instructions executed. Usage: srcphase.py page.csv name:lo-hi ..."""
import collections, csv, sys
rows = list(csv.reader(open(sys.argv[1])))
ranges = [(x.split(":")[0], tuple(map(int, x.split(":")[1].split("-")))) for x in sys.argv[2:]]
fname, hdr, cur = None, None, None
agg = collections.defaultdict(lambda: [0, 0, collections.Counter(), collections.Counter()])
tot = 0
for r in rows:
    if not r: continue
    if r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r[0] == "Line No":
        hdr = r; i_s = hdr.index("Warp Stall Sampling (All Samples)"); i_ie = hdr.index("Instructions Executed")
        reasons = [(j, h) for j, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
        continue
    if hdr is None or len(r) <= i_s: continue
    if r[0]:
        key = fname
        if fname == "l1_gram.cu":
            ln = int(r[0]); key = "l1:other"
            for name, (lo, hi) in ranges:
                if lo <= ln <= hi: key = name
        elif fname == "rotation.cuh": key = "evd_step"
        cur = key
        continue
    if not r[2].startswith("0x") or cur is None: continue
    try: s = int(r[4]); ie = int(r[7]) if r[7].isdigit() else 0
    except ValueError: continue
    t = r[3].split(); op = t[1] if t and t[0].startswith("@") and len(t) > 1 else (t[0] if t else "?")
    a = agg[cur]; a[0] += s; a[1] += ie; a[2][op.split(".")[0]] += s; a[3][op.split(".")[0]] += ie
    tot += s
ti = sum(a[1] for a in agg.values())
for k, (s, ie, ops, iops) in sorted(agg.items(), key=lambda x: -x[1][0]):
    print(f"{k:14s} samples {100*s/tot:5.1f}%  instr {100*ie/ti:5.1f}%  top-stall-ops {dict(ops.most_common(4))}")
    print(f"{'':14s} instr mix {dict((o, round(100*v/max(ie,1),1)) for o, v in iops.most_common(8))}")
