import torch, numpy as np, sys
sys.path.insert(0, '.')
import oracle as O
from paper_conf_cluster_ozsoys11_b200 import culzss, datagen
for kind in ("csource", "random", "runs20"):
    x = datagen.generate(kind, 300001, seed=3)
    s = culzss.compress(torch.from_numpy(x).cuda())
    y = culzss.decompress(s)
    print(kind, bool((y.cpu().numpy() == x).all()))
