"""Per-call times of culzss_decompress_host on pinned buffers (c2 csource 128 MiB stream)."""
import os, statistics, sys, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_ozsoys11_b200 import culzss, datagen
n = 128 << 20
x = datagen.generate("csource", n, 2)
s = culzss.compress_host(x)
sin = torch.from_numpy(s.copy()).pin_memory()
out = torch.empty(n, dtype=torch.uint8).pin_memory()
ts = []
for i in range(12):
    torch.cuda.synchronize(); e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(); culzss.decompress_host_ptr(sin.data_ptr(), s.size, out.data_ptr(), n); e1.record(); e1.synchronize()
    ts.append(e0.elapsed_time(e1))
print(os.environ.get("CULZSS_DGROUP_KB", "8192"), round(statistics.median(ts[3:]), 3), "ms", round(n / statistics.median(ts[3:]) / 1e6, 1), "GB/s")
