import torch, json
x = torch.randn(512**3, device="cuda")
y = torch.empty_like(x)
def t(f, reps=50):
    for _ in range(5): f()
    torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps): f()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / reps
nb = x.numel() * 4
r = {}
r["read_sum_us"] = t(lambda: x.sum()) * 1e3
r["read_amax_us"] = t(lambda: x.amax()) * 1e3
r["write_fill_us"] = t(lambda: y.fill_(1.0)) * 1e3
r["copy_us"] = t(lambda: y.copy_(x)) * 1e3
r["read_GBs"] = nb / (r["read_sum_us"] * 1e-6) / 1e9
r["read_amax_GBs"] = nb / (r["read_amax_us"] * 1e-6) / 1e9
r["write_GBs"] = nb / (r["write_fill_us"] * 1e-6) / 1e9
r["copy_GBs(rd+wr)"] = 2 * nb / (r["copy_us"] * 1e-6) / 1e9
print(json.dumps(r))
