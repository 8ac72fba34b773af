# Host simulation: false 3-gram candidates (bucket hit within W, different 3-gram) of the
# per-lane 512-bucket tables, golden-ratio multiplicative hash vs a strong 64-bit mixer.
# Usage: python tools/hash_sim.py csource random tarmix english
import numpy as np, sys
sys.path.insert(0,'/root/repo')
from paper_conf_cluster_ozsoys11_b200 import datagen
import inspect
def gen(name, n):
    return np.asarray(datagen.generate(name, n, 2), np.uint8)
def _unused(name, n):
    f = getattr(datagen, name)
    return np.frombuffer(bytes(f(n, seed=2)) if 'seed' in inspect.signature(f).parameters else bytes(f(n)), np.uint8)
def sim(data, hfun, nb, W=128):
    false = tot = 0
    for c0 in range(0, len(data)-4096+1, 4096):
        ch = data[c0:c0+4096].astype(np.uint32)
        g = ch[:-2] | (ch[1:-1]<<8) | (ch[2:]<<16)
        h = hfun(g, nb)
        for l in range(32):
            b0 = 128*l
            tab = {}
            for q in range(max(0,b0-W), b0): tab[h[q]] = q
            for p in range(b0, min(b0+128, len(g))):
                q = tab.get(h[p])
                if q is not None and p-q <= W:
                    tot += 1
                    if g[q] != g[p]: false += 1
                tab[h[p]] = p
    return false, tot
def hmul(g, nb):
    x = (g * np.uint32(0x9E3779B1 << 8 & 0xFFFFFFFF)).astype(np.uint32)
    return (x.astype(np.uint64) * nb >> 32).astype(np.int64)
def hideal(g, nb):
    x = g.astype(np.uint64)
    x = (x * 0xff51afd7ed558ccd) & 0xFFFFFFFFFFFFFFFF
    x ^= x >> 33
    x = (x * 0xc4ceb9fe1a85ec53) & 0xFFFFFFFFFFFFFFFF
    x ^= x >> 33
    return (x % nb).astype(np.int64)
for name in sys.argv[1:]:
    d = gen(name, 4096*16)
    print(name, 'mul', sim(d, hmul, 512), 'ideal', sim(d, hideal, 512))
