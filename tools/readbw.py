"""Read-only HBM bandwidth on the bench's batch size (ceiling check for streaming kernels)."""
import torch, json
n = 2 * 1_708_000_000 // 4
x = torch.randint(0, 1 << 30, (n,), dtype=torch.int32, device="cuda")
res = {}
for name, fn in [("sum_i32", lambda: x.sum()), ("max_i32", lambda: x.max()),
                 ("copy_half", lambda: x[: n // 2].copy_(x[n // 2:]))]:
    for _ in range(3): fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
    s.record()
    for _ in range(10): fn()
    e.record(); torch.cuda.synchronize()
    ms = s.elapsed_time(e) / 10
    nbytes = x.numel() * 4 if name != "copy_half" else x.numel() * 4
    res[name] = round(nbytes / ms / 1e6, 1)
print(json.dumps({"GB/s": res}))
