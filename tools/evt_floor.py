"""Event-timing floor: a trivial torch kernel timed the way gemv_sweep times a GEMV
(sleep, event, launch, event), to separate timer/launch floor from kernel time."""
import statistics
import torch

x = torch.zeros(1, device="cuda")
for _ in range(5):
    x.add_(1)
ts = []
for _ in range(20):
    torch.cuda._sleep(200_000)
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(); x.add_(1); e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1) * 1e3)
print("trivial kernel us: median", statistics.median(ts), "min", min(ts), "all", sorted(ts)[:5])
ts = []
for _ in range(20):
    torch.cuda._sleep(200_000)
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(100):
        x.add_(1)
    e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1) * 1e3 / 100)
print("100 back-to-back trivial kernels, us each: median", statistics.median(ts))
