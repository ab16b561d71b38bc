"""Top SASS lines by stall samples from an ncu report (ncu -i X --page source --csv --print-source sass)."""
import csv, subprocess, sys
rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]
ia, isrc, iss = hdr.index("Address"), hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)")
data = [r for r in rows[2:] if len(r) == len(hdr)]
tot = sum(int(r[iss] or 0) for r in data)
print("total samples", tot)
for idx, r in sorted(enumerate(data), key=lambda t: -int(t[1][iss] or 0))[:n]:
    print(f"{idx:5d} {int(r[iss]):6d} {r[isrc].strip()[:90]}")
