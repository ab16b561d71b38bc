"""SM clock / power / throttle trace (nvidia-smi every 50 ms) across generations of the configs[3]
bench workload (prefill then 128 decode steps), to see which phase runs power-capped.
  python tools/clock_trace.py [runs]"""
import os
import subprocess
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402


def main():
    import bench
    import synth
    from paper_conf_cluster_zhaowplw25_b200 import runtime as R
    from paper_conf_cluster_zhaowplw25_b200 import plan as PL
    wl = bench.WORKLOADS["opt66b"]
    L, h1, h2, B = wl["L"], wl["h1"], wl["h2"], wl["b_per_gpu"]
    bits = bench.workload_bits(wl)
    g = R.build_layers(L, h1, h2, bits)
    plan = R.Plan(bits, [0] * L, h1, h2, B, wl["eta"], wl["xi"], wl["s"], wl["n_dec"])
    ws = R.PipelineWorkspace(plan, g, 0)
    arr = R.layer_array(g)
    x0 = torch.empty((B, wl["s"], h1), dtype=torch.float32, device="cuda")
    synth.device_fill_f32(x0.data_ptr(), 1, 0, x0.numel(), 1.0, False)
    out = torch.zeros((B, 1 + wl["n_dec"], h1), dtype=torch.float32, device="cuda")
    R.sq_pipeline_run(plan, 0, g, None, x0, out, ws, arr=arr)
    torch.cuda.synchronize()
    lines = []
    p = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,power.draw,clocks_event_reasons.sw_power_cap",
                          "--format=csv,noheader,nounits", "-lms", "50", "-i", "0"], stdout=subprocess.PIPE, text=True)
    th = threading.Thread(target=lambda: [lines.append((time.time(), l.strip())) for l in p.stdout], daemon=True)
    th.start()
    time.sleep(1.0)
    marks = []
    for _ in range(int(sys.argv[1]) if len(sys.argv) > 1 else 2):
        t0 = time.time()
        st = R.sq_pipeline_run(plan, 0, g, None, x0, out, ws, arr=arr)
        marks.append((t0, t0 + st["t_prefill_ms"] / 1e3, t0 + st["t_total_ms"] / 1e3))
    time.sleep(0.5)
    p.terminate()
    for (a, b, c) in marks:
        for name, lo, hi in (("prefill", a, b), ("decode", b, c)):
            s = [l for t, l in lines if lo + 0.1 < t < hi - 0.05]
            cl = [float(x.split(",")[0]) for x in s]
            pw = [float(x.split(",")[1]) for x in s]
            cap = sum(1 for x in s if "Active" in x.split(",")[2])
            if cl:
                print(f"{name}: {len(cl)} samples, SM MHz median {sorted(cl)[len(cl) // 2]:.0f} (min {min(cl):.0f}, "
                      f"max {max(cl):.0f}), power median {sorted(pw)[len(pw) // 2]:.0f} W, power-cap active {cap}/{len(s)}")


if __name__ == "__main__":
    main()
