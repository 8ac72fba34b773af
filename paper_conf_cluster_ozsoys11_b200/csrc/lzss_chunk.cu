// lzss_chunk.cu -- the fused per-chunk kernel: SURVEY §8(a) rows a1-a4.
//
//   a1  stage     chunk c = in[cS, min((c+1)S, n)) into shared memory with
//                 coalesced 16-byte loads (PAPER.md:1@20938 §III.D coalescing;
//                 chunk independence PAPER.md:1@30360 §V, reading R5)
//   a2  search    L(p) = max_{1<=d<=min(W,p)} min(run_d(p), F, m-p), D(p) the
//                 smallest d attaining it (PAPER.md:1@5312 §II.A.1 "looks for
//                 the longest substring in the search buffer that matches the
//                 lookahead buffer"; R6 overlap, R7 smallest d)
//   a3  parse     greedy: literal if L(p) < 3 else (D, L), p jumps over the
//                 match (PAPER.md:1@15206 "the uncoded head pointer will jump
//                 over them"; PAPER.md:1@17800 V2 redundant-match removal)
//   a4  bit-pack  flag 0 + byte | flag 1 + (D-1) + (L-3), MSB first, zero pad
//                 (PAPER.md:1@4785, @23049-23282; readings R9-R11)
//
// B200 design, one warp per chunk, everything in shared memory:
//   * Phase 1 builds exact 3-gram hash chains over the chunk, 32 positions per
//     step: __match_any_sync groups equal hashes inside the step, a 1024-entry
//     head table carries the latest position across steps.  link[p] = distance
//     to the previous position with the same hash (0 = none within W).
//     Every d with run_d(p) >= 3 shares p's 3-gram, hence its hash, so walking
//     the chain while the distance stays <= W visits every candidate, nearest
//     first -- the window-offset search of the paper without the brute force.
//   * Phase 2 parses: lane l owns the 128-position segment [128l, 128l+128)
//     and runs the greedy parse from its segment start speculatively,
//     evaluating L/D only where its parse lands (the V1 "jump over" saving,
//     PAPER.md:1@32329 §V).  Rounds of shuffles then hand each lane the true
//     entry point (the previous lane's exit); a lane whose entry moved
//     re-parses only until it meets its own earlier path, after which the
//     greedy path is identical.  The result is the exact serial greedy parse.
//   * Phase 3 bit-packs: per-lane bit counts, warp exclusive scan, each lane
//     ORs its tokens into the payload words.
//
// The match search compares 4 bytes per step (XOR of two 32-bit words, first
// differing byte by __ffs), i.e. packed byte compares with early out.

#include "culzss_internal.h"

namespace culzss {
namespace {

constexpr uint32_t kFull = 0xffffffffu;
constexpr uint16_t kLiteral = 0xFFFF;
constexpr uint16_t kNoPos = 0xFFFF;

__device__ __forceinline__ uint32_t load4(const uint32_t *cw, int x) {
    // bytes x..x+3 of the chunk (little endian), from two aligned words
    uint32_t lo = cw[x >> 2], hi = cw[(x >> 2) + 1];
    return __funnelshift_r(lo, hi, (x & 3) * 8);
}

__device__ __forceinline__ uint32_t byte_at(const uint32_t *cw, int x) {
    return reinterpret_cast<const uint8_t *>(cw)[x];
}

__device__ __forceinline__ uint32_t hash3(uint32_t key24) {
    return (key24 * 0x9E3779B1u) >> (32 - kHashBits);
}

// Longest common prefix of chunk[q..] and chunk[p..], capped at cap (>= 1).
// Reads at most 3 bytes past p + cap (zero pad covers m + 16).
__device__ __forceinline__ int lcp(const uint32_t *cw, int q, int p, int cap) {
    int k = 0;
    while (true) {
        uint32_t x = load4(cw, q + k) ^ load4(cw, p + k);
        if (x) {
            k += (__ffs(x) - 1) >> 3;
            break;
        }
        k += 4;
        if (k >= cap) break;
    }
    return k < cap ? k : cap;
}

// Token at position p: ((D-1) << 8) | (L-3) for a match, kLiteral otherwise.
__device__ __forceinline__ uint16_t eval_pos(const uint32_t *cw, const uint8_t *link, int p, int m,
                                             int W, int F) {
    int cap = min(F, m - p);
    if (cap < 3) return kLiteral;
    int d = link[p];
    int bestL = 2, bestD = 0;
    while (d) {
        int q = p - d;
        // a candidate can only win if it also matches at offset bestL
        if (bestL < 3 || byte_at(cw, q + bestL) == byte_at(cw, p + bestL)) {
            int L = lcp(cw, q, p, cap);
            if (L > bestL) {
                bestL = L;
                bestD = d;
                if (L == cap) break;
            }
        }
        int l2 = link[q];
        if (!l2) break;
        d += l2;
        if (d > W) break;
    }
    return bestD ? (uint16_t)(((bestD - 1) << 8) | (bestL - 3)) : kLiteral;
}

__device__ __forceinline__ int tok_len(uint16_t t) { return t == kLiteral ? 1 : (t & 0xFF) + 3; }

__device__ __forceinline__ bool mask_test(uint64_t lo, uint64_t hi, int off) {
    return off < 64 ? (lo >> off) & 1ull : (hi >> (off - 64)) & 1ull;
}
__device__ __forceinline__ void mask_set(uint64_t &lo, uint64_t &hi, int off) {
    if (off < 64) lo |= 1ull << off; else hi |= 1ull << (off - 64);
}

// Walk the greedy parse from `entry` inside segment [s0, s1) until the walk
// leaves the segment or lands on a position of the current path (lo, hi).
// On return (lo, hi) is the path from `entry` and exitp its exit.
__device__ __forceinline__ void walk(const uint32_t *cw, const uint8_t *link, uint16_t *ld, int m,
                                     int W, int F, int s0, int s1, int entry, uint64_t &lo,
                                     uint64_t &hi, int &exitp) {
    uint64_t nlo = 0, nhi = 0;
    int p = entry;
    while (p < s1) {
        int off = p - s0;
        if (mask_test(lo, hi, off)) break;
        uint16_t t = eval_pos(cw, link, p, m, W, F);
        ld[p] = t;
        mask_set(nlo, nhi, off);
        p += tok_len(t);
    }
    if (p < s1) {  // merged with the old path at p: keep its positions >= p
        int off = p - s0;
        if (off < 64) {
            lo &= ~0ull << off;
        } else {
            lo = 0;
            hi &= ~0ull << (off - 64);
        }
        lo |= nlo;
        hi |= nhi;
    } else {
        lo = nlo;
        hi = nhi;
        exitp = p;
    }
}

template <int MODE>
__global__ void __launch_bounds__(kWarpsPerCta * 32, kCtasPerSm)
chunk_kernel(const uint8_t *__restrict__ in, uint64_t n, Geometry g, uint8_t *__restrict__ bucket,
             uint32_t *__restrict__ sizes, void *__restrict__ dbg) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int lane = threadIdx.x & 31;
    const int wid = threadIdx.x >> 5;
    WarpSmem &sm = reinterpret_cast<WarpSmem *>(smem_raw)[wid];
    const uint64_t C = (n + g.S - 1) / g.S;
    const uint64_t c = (uint64_t)blockIdx.x * kWarpsPerCta + wid;
    if (c >= C) return;  // whole warp leaves together
    const uint64_t start = c * g.S;
    const int m = (int)min((uint64_t)g.S, n - start);
    const int W = g.W, F = g.F;
    const uint8_t *src = in + start;
    uint8_t *cb = reinterpret_cast<uint8_t *>(sm.cw);

    // ---------------- a1: stage the chunk (16-byte coalesced loads) --------
    if ((reinterpret_cast<uintptr_t>(src) & 15) == 0) {
        const int nvec = m >> 4;
        const uint4 *s4 = reinterpret_cast<const uint4 *>(src);
        uint4 *d4 = reinterpret_cast<uint4 *>(sm.cw);
        for (int i = lane; i < nvec; i += 32) d4[i] = __ldcs(s4 + i);
        for (int i = (nvec << 4) + lane; i < m; i += 32) cb[i] = src[i];
    } else {
        for (int i = lane; i < m; i += 32) cb[i] = src[i];
    }
    if (lane < 16) cb[m + lane] = 0;  // zero pad: lcp may read 3 bytes past m
    for (int i = lane; i < (1 << kHashBits) / 2; i += 32)
        reinterpret_cast<uint32_t *>(sm.u.s.head)[i] = 0xFFFFFFFFu;
    __syncwarp();

    // ---------------- a2 (part 1): 3-gram hash chains -----------------------
    const uint32_t lt = (1u << lane) - 1u;
    const uint32_t gt = ~lt & ~(1u << lane);
    uint8_t *link = sm.u.s.link;
    uint16_t *head = sm.u.s.head;
    for (int base = 0; base < m; base += 32) {
        const int p = base + lane;
        const bool valid = p + 2 < m;
        uint32_t h = 0x10000u + lane;  // unique dummy for lanes without a 3-gram
        if (valid) h = hash3(load4(sm.cw, p) & 0xFFFFFFu);
        const uint32_t grp = __match_any_sync(kFull, h);
        if (p < m) {
            uint32_t lk = 0;
            if (valid) {
                const uint32_t lower = grp & lt;
                const int q = lower ? base + 31 - __clz(lower) : (int)head[h];
                if (q != kNoPos && p - q <= W) lk = (uint32_t)(p - q);
            }
            link[p] = (uint8_t)lk;
        }
        __syncwarp();
        if (valid && !(grp & gt)) head[h] = (uint16_t)p;
        __syncwarp();
    }

    if (MODE == kModeDumpMatch) {
        // every position, for per-position parity (a2)
        uint8_t *LD = reinterpret_cast<uint8_t *>(dbg) + 2 * start;
        for (int p = lane; p < m; p += 32) {
            uint16_t t = eval_pos(sm.cw, link, p, m, W, F);
            uint32_t L = t == kLiteral ? 0 : (t & 0xFF) + 3;
            uint32_t D = t == kLiteral ? 0 : (t >> 8) + 1;
            LD[2 * p] = (uint8_t)L;
            LD[2 * p + 1] = (uint8_t)D;
        }
        return;
    }

    // ---------------- a3: speculative segment-parallel greedy parse --------
    const int s0 = lane * kSeg;
    const int s1 = max(s0, min(s0 + kSeg, m));
    uint64_t lo = 0, hi = 0;
    int exitp = s0;
    walk(sm.cw, link, sm.ld, m, W, F, s0, s1, s0, lo, hi, exitp);
    int cur = s0;
    while (true) {
        int entry = __shfl_up_sync(kFull, exitp, 1);
        if (lane == 0) entry = 0;
        const bool chg = entry != cur;
        if (chg) {
            walk(sm.cw, link, sm.ld, m, W, F, s0, s1, entry, lo, hi, exitp);
            cur = entry;
        }
        if (!__any_sync(kFull, chg)) break;
    }

    if (MODE == kModeDumpTokens) {
        uint32_t *tok = reinterpret_cast<uint32_t *>(dbg) + start;
        for (int p = s0; p < s1; p++) {
            uint32_t v = 0;
            if (mask_test(lo, hi, p - s0)) {
                uint16_t t = sm.ld[p];
                v = t == kLiteral ? 1u : ((uint32_t)((t & 0xFF) + 3) << 16) | ((t >> 8) + 1);
            }
            tok[p] = v;
        }
        return;
    }

    // ---------------- a4: bit-pack ----------------------------------------
    int nbits = 9 * __popcll(lo) + 9 * __popcll(hi);
    {
        uint64_t w = lo;
        while (w) {
            int b = __ffsll(w) - 1;
            w &= w - 1;
            if (sm.ld[s0 + b] != kLiteral) nbits += 8;
        }
        w = hi;
        while (w) {
            int b = __ffsll(w) - 1;
            w &= w - 1;
            if (sm.ld[s0 + 64 + b] != kLiteral) nbits += 8;
        }
    }
    int incl = nbits;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(kFull, incl, o);
        if (lane >= o) incl += y;
    }
    const int excl = incl - nbits;
    const int total = __shfl_sync(kFull, incl, 31);
    const int nwords = (total + 31) >> 5;
    uint32_t *ow = sm.u.ow;
    __syncwarp();  // link/head are dead from here on
    for (int i = lane; i < nwords + 1; i += 32) ow[i] = 0;
    __syncwarp();
    {
        uint64_t acc = 0;
        int nacc = excl & 31;
        int wi = excl >> 5;
#pragma unroll 1
        for (int half = 0; half < 2; half++) {
            uint64_t w = half ? hi : lo;
            while (w) {
                const int b = __ffsll(w) - 1;
                w &= w - 1;
                const int p = s0 + half * 64 + b;
                const uint16_t t = sm.ld[p];
                uint32_t val;
                int nb;
                if (t == kLiteral) {
                    val = cb[p];
                    nb = 9;
                } else {
                    val = 0x10000u | t;
                    nb = 17;
                }
                acc = (acc << nb) | val;
                nacc += nb;
                if (nacc >= 32) {
                    nacc -= 32;
                    atomicOr(&ow[wi++], (uint32_t)(acc >> nacc));
                }
            }
        }
        if (nacc > 0) atomicOr(&ow[wi], (uint32_t)(acc << (32 - nacc)));
    }
    __syncwarp();

    // payload -> bucket c (bytes in stream order: big-endian words)
    const int nbytes = (total + 7) >> 3;
    const uint64_t stride = bucket_stride(g.S);
    uint4 *dst = reinterpret_cast<uint4 *>(bucket + c * stride);
    const uint4 *o4 = reinterpret_cast<const uint4 *>(ow);
    for (int i = lane; i < (nbytes + 15) >> 4; i += 32) {
        uint4 v = o4[i];
        v.x = __byte_perm(v.x, 0, 0x0123);
        v.y = __byte_perm(v.y, 0, 0x0123);
        v.z = __byte_perm(v.z, 0, 0x0123);
        v.w = __byte_perm(v.w, 0, 0x0123);
        dst[i] = v;
    }
    if (lane == 0) sizes[c] = (uint32_t)nbytes;
}

template <int MODE>
cudaError_t launch_mode(const uint8_t *in, uint64_t n, Geometry g, uint8_t *bucket,
                        uint32_t *sizes, void *dbg, cudaStream_t st) {
    const uint64_t C = (n + g.S - 1) / g.S;
    if (C == 0) return cudaSuccess;
    const size_t smem = sizeof(WarpSmem) * kWarpsPerCta;
    static bool attr_set = false;  // benign race: idempotent
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(chunk_kernel<MODE>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    const uint64_t blocks = (C + kWarpsPerCta - 1) / kWarpsPerCta;
    chunk_kernel<MODE><<<(unsigned)blocks, kWarpsPerCta * 32, smem, st>>>(in, n, g, bucket, sizes,
                                                                         dbg);
    count_launch();
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_chunk_kernel(int mode, const uint8_t *in, uint64_t n, Geometry g,
                                uint8_t *bucket, uint32_t *sizes, void *dbg, cudaStream_t st) {
    switch (mode) {
        case kModeCompress: return launch_mode<kModeCompress>(in, n, g, bucket, sizes, dbg, st);
        case kModeDumpMatch: return launch_mode<kModeDumpMatch>(in, n, g, bucket, sizes, dbg, st);
        default: return launch_mode<kModeDumpTokens>(in, n, g, bucket, sizes, dbg, st);
    }
}

}  // namespace culzss
