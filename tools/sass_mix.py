"""Instruction mix and hot SASS lines of one kernel in an ncu report:
python tools/sass_mix.py rep.ncu-rep [frac]"""
import collections, csv, subprocess, sys
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[1]
d = [r for r in rows[2:] if len(r) == len(h)]
ie, src, ss = h.index("Instructions Executed"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
tot = sum(int(r[ie] or 0) for r in d)
print("total warp instructions", tot)
ops = collections.Counter()
for r in d:
    t = r[src].split()
    if not t:
        continue
    op = t[1] if t[0].startswith("@") else t[0]
    ops[op.split(".")[0]] += int(r[ie] or 0)
for k, v in ops.most_common(25):
    print(f"{k:12s} {v:10d} {v / tot:.3f}")
fr = float(sys.argv[2]) if len(sys.argv) > 2 else 1 / 300
for i, r in enumerate(d):
    if int(r[ie] or 0) > tot * fr:
        print(i, r[ie], r[ss], r[src][:100])
