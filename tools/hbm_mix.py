"""HBM ceilings for read/write mixes on this B200 (context for the roofline of write-dominated
launches): write-only (fill_), copy (read+write 1:1, as MEASURED_PEAKS.json), read-only (sum)."""
import torch
n = 1 << 30  # 4 GiB fp32
a = torch.empty(n, device="cuda")
b = torch.empty(n, device="cuda")
a.fill_(1.0)
def t(fn, reps=10):
    best = 1e9
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best
for _ in range(3): b.copy_(a)
w = t(lambda: b.fill_(2.0))
c = t(lambda: b.copy_(a))
r = t(lambda: a.sum())
print("write-only fill_: %.0f GB/s" % (4 * n / w / 1e6))
print("copy (r+w):       %.0f GB/s" % (8 * n / c / 1e6))
print("read-only sum:    %.0f GB/s" % (4 * n / r / 1e6))
