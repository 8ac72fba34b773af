import sys, os, statistics, torch
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
from paper_conf_cluster_ozsoys11_b200 import culzss, datagen
n = 128 << 20
for kind in ("csource", "runs20"):
    x = torch.from_numpy(datagen.generate(kind, n, 2)).cuda()
    for S in (8192, 65536):
        p = culzss.Params.make(S=S)
        out = torch.empty(culzss.max_compressed_size(n, p), dtype=torch.uint8, device="cuda")
        on = culzss.compress_into(x, out, p)
        dec = torch.empty(n, dtype=torch.uint8, device="cuda")
        ts = []
        for it in range(5):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(); culzss.decompress(out[:on], dec); e1.record(); e1.synchronize()
            if it >= 2: ts.append(e0.elapsed_time(e1))
        print(kind, S, round(n / (statistics.median(ts) / 1000) / 1e9, 1), "GB/s", bool(torch.equal(dec, x)))
