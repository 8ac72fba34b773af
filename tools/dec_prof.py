import sys, torch
sys.path.insert(0, '.')
from paper_conf_cluster_ozsoys11_b200 import culzss, datagen
kind = sys.argv[1] if len(sys.argv) > 1 else 'csource'
x = torch.from_numpy(datagen.generate(kind, 64 << 20, 2)).cuda()
s = culzss.compress(x)
y = torch.empty_like(x)
for _ in range(3):
    culzss.decompress(s, y)
torch.cuda.synchronize()
print('ok', torch.equal(x, y))
