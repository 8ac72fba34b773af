"""Host model of the chunk kernel's walk balance: per-position walk iterations from
the exact greedy parse (exact 3-gram candidate chains; one iteration per candidate plus LCP
extension steps and the token step), then the warp-maximum cost of three segment layouts and of
probing two rejected candidates per iteration.

    python tools/walk_sim.py [csource|tarmix|...] [chunks]
"""
import heapq
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cluster_ozsoys11_b200 import datagen  # noqa: E402

W = F = 128


def position_costs(c, pair=False):
    m = len(c)
    last, cands = {}, [[] for _ in range(m)]
    for p in range(m - 2):
        lst = last.setdefault(bytes(c[p:p + 3]), [])
        cands[p] = [p - q for q in reversed(lst) if p - q <= W]
        lst.append(p)
    cost, ln = [0] * m, [1] * m
    for p in range(m):
        if not cands[p]:
            continue
        cap, bestL, bestD, it, rej = min(F, m - p), 2, 0, 0, 0
        for d in cands[p]:
            L = 0
            while L < cap and c[p - d + L] == c[p + L]:
                L += 1
            L = min(L, cap)
            if L > bestL:
                it += 1 + max(0, (L - 1) // 8)
                bestL, bestD = L, d
            else:
                rej += 1
            if bestL == cap:
                break
        it += (rej + 1) // 2 if pair else rej
        cost[p], ln[p] = it + 1, (bestL if bestD else 1)
    return cost, ln, cands


def seg(cost, ln, cands, s0, s1):
    p, w = s0, 0
    while p < s1:
        w += cost[p]
        p += ln[p] if cands[p] else 1
    return w + 1


def main():
    kind = sys.argv[1] if len(sys.argv) > 1 else "csource"
    nch = int(sys.argv[2]) if len(sys.argv) > 2 else 16
    x = datagen.generate(kind, nch * 4096, seed=2)
    tot = dict(static64=0, two32=0, dyn32=0, pair_probe=0, average=0)
    for ci in range(nch):
        c = x[ci * 4096:(ci + 1) * 4096]
        cost, ln, cands = position_costs(c)
        a = [seg(cost, ln, cands, 64 * t, 64 * t + 64) for t in range(64)]
        tot["static64"] += max(a[:32]) + max(a[32:])
        tot["average"] += sum(a) / 32
        b = [seg(cost, ln, cands, 32 * t, 32 * t + 32) + seg(cost, ln, cands, 2048 + 32 * t, 2080 + 32 * t)
             for t in range(64)]
        tot["two32"] += max(b[:32]) + max(b[32:])
        works = [seg(cost, ln, cands, 32 * i, 32 * i + 32) for i in range(128)]
        h = [(0, l) for l in range(64)]
        fin = [0] * 64
        for w in works:  # greedy list scheduling in segment order
            t, l = heapq.heappop(h)
            fin[l] = t + w + 2
            heapq.heappush(h, (fin[l], l))
        tot["dyn32"] += max(fin[:32]) + max(fin[32:])
        cost2, ln2, cands2 = position_costs(c, pair=True)
        a2 = [seg(cost2, ln2, cands2, 64 * t, 64 * t + 64) for t in range(64)]
        tot["pair_probe"] += max(a2[:32]) + max(a2[32:])
    print(kind, {k: round(v) for k, v in tot.items()})


if __name__ == "__main__":
    main()
