"""Key metrics of ncu --set full reports -> JSON (profiles/)."""
import csv, json, subprocess, sys
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__t_bytes.sum", "sm__cycles_elapsed.avg",
        "l1tex__throughput.avg.pct_of_peak_sustained_active", "sm__memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__cycles_active.avg"]
out = {}
for rep in sys.argv[2:]:
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(txt.splitlines()))
    h, units, v = rows[0], rows[1], rows[2]
    d = {"kernel": v[h.index("Kernel Name")][:120]}
    for k in KEYS:
        if k in h:
            i = h.index(k)
            d[k] = f"{v[i]} {units[i]}".strip()
    stalls = {}
    for i, x in enumerate(h):
        if x.startswith("smsp__pcsamp_warps_issue_stalled_") and not x.endswith("not_issued"):
            try:
                stalls[x.replace("smsp__pcsamp_warps_issue_stalled_", "")] = int(float(v[i]))
            except ValueError:
                pass
    d["stall_samples_top"] = dict(sorted(stalls.items(), key=lambda t: -t[1])[:8])
    out[rep.split("/")[-1]] = d
json.dump(out, open(sys.argv[1], "w"), indent=1)
print(json.dumps(out, indent=1)[:3000])
