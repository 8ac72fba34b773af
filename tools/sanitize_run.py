"""Workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
small compress + decompress calls through the C ABI on C1 and adversarial inputs,
both search versions, both walk machines, packed small chunks, the host API.

    compute-sanitizer --tool racecheck python tools/sanitize_run.py
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_cluster_ozsoys11_b200 import culzss, datagen  # noqa: E402


def main():
    rng = np.random.default_rng(1)
    inputs = {
        "c1_english_64k": datagen.generate("english", 64 << 10, 1),
        "runs20": datagen.generate("runs20", 3 * 4096 + 77, 3),
        "tarmix": datagen.generate("tarmix", 5 * 4096 + 5, 5),
        "random": datagen.generate("random", 2 * 4096 + 1, 4),
        "period7": np.tile(rng.integers(0, 256, 7, dtype=np.uint8), 2000),
        "zeros": np.zeros(9000, np.uint8),
    }
    n_calls = 0
    for env_tx in (None, "0"):
        if env_tx is None:
            os.environ.pop("CULZSS_WALK_TOKEN_SWITCH", None)
        else:
            os.environ["CULZSS_WALK_TOKEN_SWITCH"] = env_tx
        for name, x in inputs.items():
            xd = torch.from_numpy(x.copy()).cuda()
            for p in (None, culzss.Params.make(version=2), culzss.Params.make(S=256), culzss.Params.make(S=1000, W=255, F=258)):
                if p is not None and p.version == 2 and env_tx is not None:
                    continue
                s = culzss.compress(xd, p)
                y = culzss.decompress(s)
                assert torch.equal(y, xd), name
                n_calls += 2
            L, D = culzss.match_search(xd)
            tok = culzss.parse_tokens(xd)
            n_calls += 2
    x = inputs["c1_english_64k"]
    hin = torch.from_numpy(x.copy()).pin_memory()
    hout = torch.empty(culzss.max_compressed_size(x.size), dtype=torch.uint8).pin_memory()
    on = culzss.compress_host_ptr(hin.data_ptr(), x.size, hout.data_ptr(), hout.numel())
    hdec = torch.empty(x.size, dtype=torch.uint8).pin_memory()
    culzss.decompress_host_ptr(hout.data_ptr(), on, hdec.data_ptr(), x.size)
    assert torch.equal(hdec, hin)
    torch.cuda.synchronize()
    print(f"sanitize workload ok: {n_calls + 2} library calls")


if __name__ == "__main__":
    main()
