"""Per-instruction stall breakdown over an SASS index range of an ncu report (source page)."""
import csv, subprocess, sys
rep, lo, hi = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[1]
d = [r for r in rows[2:] if len(r) == len(h)]
cols = [i for i, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
tot = {h[i]: 0 for i in cols}
isrc, iss = h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
for r in d[lo:hi]:
    for i in cols:
        tot[h[i]] += int(r[i] or 0)
print("range total", sum(int(r[iss] or 0) for r in d[lo:hi]), {k: v for k, v in sorted(tot.items(), key=lambda t: -t[1]) if v})
if len(sys.argv) > 4:
    for j, r in enumerate(d[lo:hi]):
        s = int(r[iss] or 0)
        if s >= int(sys.argv[4]):
            top = sorted(((int(r[i] or 0), h[i]) for i in cols), reverse=True)[:2]
            print(lo + j, s, r[isrc].strip()[:70], top)
