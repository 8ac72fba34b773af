"""e2e sweep for the pipelined host path: GB/s of culzss_compress_host on
pinned buffers (c2 csource 128 MiB), plus raw pinned H2D / D2H bandwidth.
Run once per CULZSS_GROUP_KB value (the knob is read once per process)."""
import os, statistics, sys, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_ozsoys11_b200 import culzss, datagen
n = 128 << 20
x = datagen.generate(sys.argv[1] if len(sys.argv) > 1 else "csource", n, 2)
hin = torch.from_numpy(x).pin_memory()
hout = torch.empty(culzss.max_compressed_size(n), dtype=torch.uint8).pin_memory()
def t(fn, k=8):
    ts = []
    for i in range(k + 3):
        torch.cuda.synchronize(); e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); e1.synchronize()
        if i >= 3: ts.append(e0.elapsed_time(e1))
    return statistics.median(ts)
ms = t(lambda: culzss.compress_host_ptr(hin.data_ptr(), n, hout.data_ptr(), hout.numel()))
d = torch.empty(n, dtype=torch.uint8, device="cuda")
h2d = t(lambda: d.copy_(hin, non_blocking=True))
d2h = t(lambda: hin.copy_(d, non_blocking=True))
print(f"group_kb={os.environ.get('CULZSS_GROUP_KB','8192')} e2e {n/ms/1e6:.1f} GB/s ({ms:.3f} ms)  h2d {n/h2d/1e6:.1f} GB/s  d2h {n/d2h/1e6:.1f} GB/s")
