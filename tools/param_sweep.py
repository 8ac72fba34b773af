"""NEXT-4: parameter variants on B200 -- compression GB/s and ratio of the c2 input
(csource 128 MiB) for window W (up to 256), max match F and chunk S (64 B .. 64 KiB; above 4 KiB
in tiles) around the paper's W = 128, F = 128, S = 4096 (PAPER.md:1@22727-23374 window sweep, @36001 tuning API).  Each setting's stream is checked
byte-exact against the oracle on its first 64 chunks.  Device time from the library's events, L2
flushed between calls, median of 5."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
from paper_conf_cluster_ozsoys11_b200 import culzss, datagen

kind = sys.argv[1] if len(sys.argv) > 1 else "csource"
n = 128 << 20
x_np = datagen.generate(kind, n, 2)
x = torch.from_numpy(x_np).cuda()
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
culzss.set_profiling(True)
rows = []
settings = [(4096, W, 128) for W in (8, 16, 32, 64, 128, 192, 255, 256)] + \
           [(4096, 128, F) for F in (18, 32, 64, 258)] + [(4096, 256, 256)] + \
           [(S, 128, 128) for S in (256, 512, 1024, 2048, 8192, 16384, 65536)] + [(65536, 256, 256)]
for S, W, F in settings:
    p = culzss.Params.make(S=S, W=W, F=F)
    out = torch.empty(culzss.max_compressed_size(n, p), dtype=torch.uint8, device="cuda")
    ts = []
    for it in range(7):
        flush.fill_(1)
        torch.cuda.synchronize()
        on = culzss.compress_into(x, out, p)
        if it >= 2:
            ts.append(culzss.last_kernel_ms("call"))
    ms = statistics.median(ts)
    s = out[:on].cpu().numpy().tobytes()
    C = (n + S - 1) // S
    sizes = np.frombuffer(s, "<u4", count=C, offset=32).astype(np.int64)
    ref, _ = oracle.compress_range(x_np, 0, 64, S=S, W=W, F=F)
    exact = s[32 + 4 * C:32 + 4 * C + len(ref)] == ref
    # decompression of the same stream (culzss_decompress, CUDA events), exact round trip
    dec = torch.empty(n, dtype=torch.uint8, device="cuda")
    dts = []
    for it in range(5):
        flush.fill_(1)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        culzss.decompress(out[:on], dec)
        e1.record()
        e1.synchronize()
        if it >= 2:
            dts.append(e0.elapsed_time(e1))
    rt = bool(torch.equal(dec, x))
    del dec
    rows.append({"S": S, "W": W, "F": F, "GBps": n / ms / 1e6, "ratio": on / n, "exact_first_64_chunks": exact,
                 "decompress_GBps": n / statistics.median(dts) / 1e6, "roundtrip_exact": rt})
    print(json.dumps(rows[-1]), flush=True)
