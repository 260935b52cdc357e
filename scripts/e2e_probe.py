"""Break the end-to-end host API time into its parts (pinned buffers)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_hpdc_yudztt0c22_b200 as szx
import synth
x = synth.nyx_like(0, 512, device="cuda").reshape(-1).contiguous()
n = x.numel()
xh = x.cpu().pin_memory()
sh = torch.empty(szx.compress_bound(n, szx.F32, 128), dtype=torch.uint8, pin_memory=True)
yh = torch.empty(n, dtype=torch.float32, pin_memory=True)
d = torch.empty_like(x)
def t(f, k=5):
    f(); torch.cuda.synchronize()
    ts = []
    for _ in range(k):
        t0 = time.perf_counter(); f(); torch.cuda.synchronize(); ts.append(time.perf_counter() - t0)
    return min(ts) * 1e3
print("h2d 537MB ms", t(lambda: d.copy_(xh, non_blocking=True)))
print("d2h 537MB ms", t(lambda: yh.copy_(d, non_blocking=True)))
print("compress_host ms", t(lambda: szx.compress_host(xh, 1e-3, "rel", 128, out=sh)))
s_h = szx.compress_host(xh, 1e-3, "rel", 128, out=sh)
print("decompress_host ms", t(lambda: szx.decompress_host(s_h, out=yh)))
