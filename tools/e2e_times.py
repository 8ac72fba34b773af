"""Per-call times of culzss_compress_host on pinned buffers (c2 csource 128 MiB): the spread behind
bench.py's e2e mean."""
import os, sys, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_ozsoys11_b200 import culzss, datagen
n = 128 << 20
x = datagen.generate("csource", n, 2)
hin = torch.from_numpy(x).pin_memory()
hout = torch.empty(culzss.max_compressed_size(n), dtype=torch.uint8).pin_memory()
ts = []
for i in range(25):
    torch.cuda.synchronize(); e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(); culzss.compress_host_ptr(hin.data_ptr(), n, hout.data_ptr(), hout.numel()); e1.record(); e1.synchronize()
    ts.append(e0.elapsed_time(e1))
print(" ".join(f"{t:.2f}" for t in ts))
