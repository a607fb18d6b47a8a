import torch, time
n = 2 * 1024**3  # 8 GiB of fp32
a = torch.empty(n, device='cuda'); b = torch.empty(n, device='cuda')
for name, fn, nbytes in [("fill (write only)", lambda: a.fill_(1.0), 4 * n), ("copy (read+write)", lambda: a.copy_(b), 8 * n)]:
    fn(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10): fn()
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 10
    print(name, round(ms, 3), "ms", round(nbytes / ms / 1e6, 1), "GB/s")
