"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) per kernel: count, total, share."""
import csv, collections, json, sys
lines = [l for l in open(sys.argv[1]) if l.startswith('"')]
rows = list(csv.reader(lines))
h = rows[0]
ik, iv, iu = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
tot, cnt = collections.defaultdict(float), collections.Counter()
for r in rows[1:]:
    if len(r) != len(h):
        continue
    name = r[ik].replace("void ", "").split("(")[0]
    v = float(r[iv].replace(",", ""))
    v = v / 1e3 if r[iu] == "ns" else (v * 1e3 if r[iu] == "ms" else v)  # -> us
    tot[name] += v
    cnt[name] += 1
T = sum(tot.values())
out = []
for k in sorted(tot, key=lambda k: -tot[k]):
    out.append({"kernel": k, "launches": cnt[k], "total_ms": round(tot[k] / 1e3, 3), "share": round(tot[k] / T, 4),
                "avg_us": round(tot[k] / cnt[k], 2)})
    print(f"{k[:70]:70s} n={cnt[k]:5d} total={tot[k]/1e3:9.2f} ms share={tot[k]/T:.3f} avg={tot[k]/cnt[k]:8.1f} us")
if len(sys.argv) > 2:
    json.dump({"source": sys.argv[1], "launches": sum(cnt.values()), "total_ms": round(T / 1e3, 3), "kernels": out},
              open(sys.argv[2], "w"), indent=1)
