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
// B200 design: a PAIR of warps per 4 KiB chunk, one chunk per
// 64-thread CTA, nine CTAs per SM (24.8 KB of shared memory each: a chunk's
// memory is released as soon as it finishes), everything in shared memory:
//   * Chain build (a2, part 1; warp 0).  Lane l owns the 128-position build
//     segment [128l, 128l + 128) and a private 512-bucket u8 hash table
//     ([lane][bucket]); it inserts the W positions before its segment, then
//     its own positions in order, recording link[p] = distance to the previous
//     position with the same 3-gram hash (0 = none within W; four links per
//     4-position group formed bytewise with vadd4/vsub4/vcmpleu4).  Every d
//     with run_d(p) >= 3 shares p's 3-gram, hence its hash, so walking the
//     chain while the distance stays <= W visits every candidate, nearest
//     first -- the paper's window-offset search without the brute force.
//   * Lazy greedy walk (a2 part 2 + a3; both warps).  Walk lane t (0..63) runs
//     the greedy parse over the 64-position segment [64t, 64t + 64) from its
//     start, evaluating L/D only where the parse lands -- the V1 "jump over"
//     saving (PAPER.md:1@32329 §V).  Machine 1 is a flat state machine per
//     lane: every iteration is one 8-byte compare (big-endian words of an
//     unskewed chunk copy, equal leading bytes by a 64-bit clz) of one
//     candidate -- an 8-byte reject test at [bestL-7, bestL] once bestL >= 8,
//     else an LCP step -- and positions without a candidate are skipped with a
//     64-bit mask.  A warp one of whose lanes spends 16 iterations on one token
//     switches to machine 2, the same walk with two exact prunes (run skip,
//     chain switch; see walk_spec).  Fix-up rounds then hand each lane its true
//     entry (the previous lane's exit); a lane whose entry moved re-walks only
//     until it meets its earlier path.  The result is exactly the serial
//     greedy parse.
//   * Bit-pack (a4): each lane emits its path's tokens (positions combined in
//     32-bit pairs), a 64-lane scan of bit counts places them, edge words are
//     OR-ed, and the payload goes to the chunk's bucket with 16-byte stores.
//   * params.version = 2 replaces the build and walk by the paper's V2 search
//     (every position, every offset, warp argmax); chunks of S = 64..2048 are
//     packed 4096 / S to a pair (PACK); chunks of S > 4096 are compressed in
//     4096-position tiles (TILED); W = 256 adds d = 256 as one extra candidate
//     (the u8 links hold <= 255).

#include "culzss_internal.h"

namespace culzss {
namespace {

constexpr uint32_t kFull = 0xffffffffu;
constexpr uint32_t kTabBias = 0x1000;   // table entry = position + bias; 0 = empty
constexpr uint32_t kHashMul = 0x9E3779B1u << 8;
constexpr int kSparseLinks = 24;  // candidate-mask filter: at most this many linked positions per lane of the warp
// Memoised token encoding in ld[] (u16).  W <= 128: 0 = not evaluated,
// 2 = literal, (D << 8) | (L - 3) = match (>= 0x100; L - 3 fits 8 bits for
// F <= 258).  W > 128 (BW; W = 256 needs D = 256): 0 = not evaluated,
// 1 = literal, ((D - 1) << 8 | (L - 3)) + 2 = match, which fits 16 bits for
// F <= 258 at W <= 255 and for F <= 256 at W = 256.
template <bool BW>
struct Memo {
    static constexpr uint16_t kLit = BW ? 1 : 2;
    __device__ static __forceinline__ uint32_t match(int D, int L) {
        return BW ? ((((uint32_t)D - 1) << 8) | (uint32_t)(L - 3)) + 2u : ((uint32_t)D << 8) | (uint32_t)(L - 3);
    }
    __device__ static __forceinline__ bool is_match(uint32_t t) { return BW ? t >= 2 : t >= 0x100; }
    // the token's 17 bits: flag 1 | D - 1 | L - 3 (reading R11)
    __device__ static __forceinline__ uint32_t code(uint32_t t) {
        return BW ? ((t - 2) | 0x10000u) : t + (0x10000u - 0x100u);
    }
    __device__ static __forceinline__ int len(uint32_t t) { return is_match(t) ? (int)(code(t) & 0xFF) + 3 : 1; }
    __device__ static __forceinline__ int dist(uint32_t t) { return (int)((code(t) >> 8) & 0xFF) + 1; }
};

// skewed byte index of chunk position x (4 pad bytes per 128 positions)
__device__ __forceinline__ int sk(int x) { return (int)((unsigned)x + (((unsigned)x >> 7) << 2)); }
// skewed u16 index of position x
__device__ __forceinline__ int sk2(int x) { return x + ((x >> 7) << 1); }

__device__ __forceinline__ uint32_t load4(const uint32_t *cw, int x) {
    // bytes x..x+3 of the chunk (little endian), from two aligned words; the
    // pad word after each segment repeats the next segment's first word.
    // Word index of sk(x) = x/4 + x/128; the funnel shift masks its amount to
    // 5 bits, so 8x selects the byte offset within the word.
    const unsigned ux = (unsigned)x;
    const unsigned wi = (ux >> 2) + (ux >> 7);
    return __funnelshift_r(cw[wi], cw[wi + 1], ux << 3);
}

// The walks compare on an unskewed, byte-swapped (big-endian words) copy of
// the chunk: bytes x..x+7 are two funnel shifts of three aligned words with
// byte x in the most significant position, so the number of equal leading
// bytes of two such values is a count of leading zeros of their XOR.
struct Be8 {
    uint32_t hi, lo;  // bytes x..x+3, x+4..x+7
};
__device__ __forceinline__ Be8 load8(const uint32_t *__restrict__ u, int x) {
    const uint32_t *w = u + ((unsigned)x >> 2);
    const uint32_t a = w[0], b = w[1], c = w[2];
    const unsigned sh = (unsigned)x << 3;  // the funnel shift masks it to 5 bits
    return Be8{__funnelshift_l(b, a, sh), __funnelshift_l(c, b, sh)};
}

// first candidate position >= p of the lane's segment [s0, s1), or s1 (p if
// p >= s1 already).  cm: candidate bits of positions s0..s0+63, position
// s0+i at bit 63-i (reversed: next = count of leading zeros)
__device__ __forceinline__ int next_cand(uint64_t cm, int p, int s0, int s1) {
    // branch-free: for p >= s1 the min gives s1 and the max restores p
    const int nc = min(p + __clzll(cm << min(p - s0, 63)), s1);  // clz(0) = 64: past the segment
    return max(nc, p);
}

__device__ __forceinline__ bool is_cand(uint64_t cm, int o) { return (cm << o) >> 63; }

// byte offset (into the per-lane-interleaved table) of the 3-gram hash of a
// little-endian word whose low 3 bytes are the 3-gram: hash h = top 8 bits of
// (w << 8) * K (== w * (K << 8)); entry [h][lane] lives at byte 64 h + 2 lane
__device__ __forceinline__ uint32_t hash_off(uint32_t w) { return ((w * kHashMul) >> 18) & 0x3FC0u; }
// W <= 128 variant: 9-bit hash h of the same product, u8 entries [lane][h]
// at byte 512 lane + h (one add per address; lanes' buckets are random, so
// the bank spread is the same as the interleaved layout's)
__device__ __forceinline__ uint32_t hash9(uint32_t w) { return (w * kHashMul) >> 23; }


// Run-boundary mask (the run-skip prune): bit x of bnd (u32
// words, position-indexed) = chunk[x] != chunk[x+1]; every bit from the
// chunk's last position on is set.  run_len / run_start read it with ffs /
// clz (a run of equal bytes of length up to 128 spans at most 5 words).
//
// length of the run of equal bytes starting at p, capped at cap (>= 1)
__device__ __forceinline__ int run_len(const uint32_t *__restrict__ bnd, int p, int cap) {
    int x = p;
    uint32_t w = bnd[x >> 5] >> (x & 31);
    int r = 0;
    while (!w) {  // no boundary in the rest of this word
        r += 32 - (x & 31);
        if (r >= cap) return cap;
        x = (x | 31) + 1;
        w = bnd[x >> 5];
    }
    return min(r + __ffs(w), cap);
}
// first position of the run of equal bytes that contains q, or lo if that
// run starts at or before lo (lo < q)
__device__ __forceinline__ int run_start(const uint32_t *__restrict__ bnd, int q, int lo) {
    int x = q - 1;  // the run starts after the last boundary bit below q
    while (x >= lo) {
        const uint32_t w = bnd[x >> 5] << (31 - (x & 31));  // bit 31 = position x
        if (w) return max(x - (int)__clz(w) + 1, lo);
        x = (x & ~31) - 1;
    }
    return lo;
}

// The same two run queries read on the fly from the big-endian chunk copy u
// (for eval_pos: a fix-up re-walk may run in a warp without the mask).
__device__ __forceinline__ int run_len_u(const uint32_t *__restrict__ u, int p, int cap) {
    const Be8 f = load8(u, p);
    const uint64_t B = (uint64_t)(f.hi >> 24) * 0x0101010101010101ull;
    uint64_t v = (((uint64_t)f.hi << 32) | f.lo) ^ B;
    int k = 0;
    while (!v) {
        k += 8;
        if (k >= cap) return cap;
        const Be8 w = load8(u, p + k);
        v = (((uint64_t)w.hi << 32) | w.lo) ^ B;
    }
    return min(k + (__clzll(v) >> 3), cap);
}
__device__ __forceinline__ int run_start_u(const uint32_t *__restrict__ u, int q, int lo) {
    const Be8 f = load8(u, q);
    const uint64_t B = (uint64_t)(f.hi >> 24) * 0x0101010101010101ull;
    int x = q;  // the run covers [x, q]
    while (x > lo) {
        const int a = max(x - 8, lo);  // bytes [a, x): the first x - a of the 8 loaded
        const Be8 w = load8(u, a);
        const uint64_t v = ((((uint64_t)w.hi << 32) | w.lo) ^ B) >> (8 * (8 - (x - a)));
        if (v) return x - (__ffsll(v) - 1) / 8;  // equal bytes just below x
        x = a;
    }
    return lo;
}

// Longest common prefix of the chunk at q and at p (q < p), capped at cap,
// 8 bytes per step on the big-endian copy u.
__device__ __forceinline__ int lcp8(const uint32_t *__restrict__ u, int q, int p, int cap) {
    int k = 0;
    while (k < cap) {
        const Be8 a = load8(u, q + k), b = load8(u, p + k);
        const int fb = __clzll(((uint64_t)(a.hi ^ b.hi) << 32) | (a.lo ^ b.lo)) >> 3;
        k += fb;
        if (fb < 8) break;
    }
    return min(k, cap);
}

// first entry > dmin of the chain through position z (link hops, chain
// offset already applied), starting from distance d0 = that of z; 0 if the
// chain ends or passes wlim first
__device__ __forceinline__ int chain_after(const uint8_t *__restrict__ link, int p, int o, int d0, int dmin,
                                           int wlim) {
    int d = d0;
    while (d <= dmin) {
        const int l2 = link[sk(p - d + o)];
        if (!l2) return 0;
        d += l2;
    }
    return d <= wlim ? d : 0;
}

// (L, D) at one position p by the chain walk with the same two exact prunes
// as the walk state machine below (a plain loop: fix-up re-walks only).
// m: end of p's chunk, cstart: its start.  Returns the memo encoding.  At
// W = 256 the links hold distances <= 255 and d = 256 is one extra candidate.
template <bool BW>
__device__ uint32_t eval_pos(const uint32_t *__restrict__ u, const uint8_t *__restrict__ link, int p, int m,
                             int cstart, int W, int F) {
    const int cap = min(F, m - p);
    int d = link[sk(p)];
    if (cap < 3) return Memo<BW>::kLit;
    const int wlim = min(W, p - cstart);
    int t = -1;  // run length at p (computed when first needed)
    int bestL = 2, bestD = 0, o = 0, nrej = 0;
    while (d) {
        const int q = p - d;
        const int L = lcp8(u, q, p, cap);
        const bool upd = L > bestL;
        if (upd) {
            bestL = L;
            bestD = d;
            if (L == cap) break;
        }
        nrej = upd ? 0 : nrej + 1;
        if (L >= 3 && t < 0) t = run_len_u(u, p, cap);
        if (L >= 3 && L < t) {
            // run skip: q's match ended with the run of equal bytes it sits in
            const int lo = p - wlim;
            const int r0 = run_start_u(u, q, lo);
            const int qs = max(q + L - t, r0);
            if (qs < q) {
                const int L2 = lcp8(u, qs, p, cap);
                if (L2 > bestL) {
                    bestL = L2;
                    bestD = p - qs;
                    if (L2 == cap) break;
                }
                if (r0 <= lo) break;
                o = 0;  // resume on p's own chain after the run start
                nrej = 0;
                d = chain_after(link, p, 0, p - r0, p - r0, wlim);
                continue;
            }
        }
        if (nrej >= 2 && bestL >= 3 && bestL - 2 > o) {
            // chain switch: every better candidate matches bytes [bestL-2, bestL]
            o = bestL - 2;
            nrej = 0;
            const int e = link[sk(p + o)];
            d = e ? chain_after(link, p, o, e, d, wlim) : 0;
            continue;
        }
        const int l2 = link[sk(q + o)];
        d = (l2 && d + l2 <= wlim) ? d + l2 : 0;
    }
    if (BW && W == 256 && wlim == 256 && bestL < cap) {  // the one distance the u8 links cannot hold
        const int L = lcp8(u, p - 256, p, cap);
        if (L > bestL) {
            bestL = L;
            bestD = 256;
        }
    }
    return bestD ? Memo<BW>::match(bestD, bestL) : Memo<BW>::kLit;
}

// Run-boundary mask of a warp's half of the chunk plus the words before and
// after it that run_start / run_len reach from it (W <= 255 back, F <= 258
// ahead: kBndWarpLo / kBndWarpWords), built on demand by the whole warp when it switches to the pruned
// walk, into the warp's own copy (kBndWarpWords words; bnd points at its
// word 0, so bnd[w] is mask word w).  The skewed words of one 32-position
// group lie in one 128-position segment; the group's next word is the pad
// word (a copy of the next segment's first word) at a segment end.
__device__ __forceinline__ void build_bnd_warp(const uint32_t *__restrict__ cw, uint32_t *__restrict__ bnd,
                                               int half, int lane, int m) {
    const int w0 = max(64 * half - kBndWarpLo, 0), w1 = min(64 * half + kBndWarpWords - kBndWarpLo, kChunkMax / 32);
#pragma unroll 1
    for (int w = w0 + lane; w < w1; w += 32) {
        const uint32_t *c = cw + (sk(32 * w) >> 2);
        uint32_t a = c[0], bits = 0;
#pragma unroll
        for (int gi = 0; gi < 8; gi++) {
            const uint32_t an = c[gi + 1];
            const uint32_t v = a ^ __funnelshift_r(a, an, 8);  // byte j: chunk[x+j] ^ chunk[x+j+1]
            const uint32_t nz = (((v & 0x7F7F7F7Fu) + 0x7F7F7F7Fu) | v) & 0x80808080u;
            bits |= ((nz >> 7) * 0x10204080u >> 28) << (4 * gi);  // bit j = byte j nonzero
            a = an;
        }
        const int lim = m - 1 - 32 * w;  // bits from the last position m-1 on are set
        if (lim < 32) bits |= lim <= 0 ? 0xFFFFFFFFu : ~((1u << lim) - 1);
        bnd[w] = bits;
    }
    __syncwarp();
}

// Speculative greedy walk over segment [s0, s1) from s0 as a branch-free
// state machine: every iteration of every active lane does exactly one
// 8-byte compare of its current candidate d at offset `off` (on the unskewed
// chunk copy u) and then updates its state with selects:
//   * once bestL >= 8 a candidate first gets an 8-byte reject test of bytes
//     [bestL-7, bestL] (it can only win if bytes [0, bestL] match); then (or
//     directly, below 8, where the first LCP step decides as cheaply) its
//     LCP 8 bytes per iteration;
//   * a finished candidate moves to the next one on the hash chain
//     (d += link[p-d]) or finishes the token;
//   * a finished token is memoised in ld[] and p jumps over candidate-free
//     positions (literals) with the lane's candidate mask; the new token's
//     first candidate is loaded in the same iteration.
// A warp still walking after `sw` iterations, or one of whose lanes has spent
// `tx` iterations on one token (runs and structured binary: long chains of
// true 3-gram candidates), continues in a second machine with
// two exact prunes, after building its run-boundary mask;
// there a finished candidate moves to the next one on the chain it was found
// on (d += link[p-d+o]) or, in a rarely taken branch:
//   - run skip: a candidate whose match L (3 <= L < t, t = the run of equal
//     bytes at p) ended because the run it sits in ended: the start
//     qs = max(end - t, run start) of that run dominates every other start in
//     it (nearer ones match less, farther ones at most as much), so qs is
//     evaluated next and the walk then resumes after the run start on p's
//     chain;
//   - chain switch: after two candidates in a row that did not improve,
//     continue on the chain of p's 3-gram at offset o = bestL-2 (any better
//     candidate matches those bytes too), from its first entry beyond d.
// Both keep the candidates in increasing d, so the strict '>' still leaves
// the smallest d on ties (reading R7).
// ALLPOS (per-position parity dump, row a2): every candidate position of the
// segment is evaluated and (L, D) written to dump instead.
// Returns the exit (first position >= s1 the greedy path reaches).
template <bool ALLPOS, bool BW>
__device__ __forceinline__ int walk_spec(const uint32_t *__restrict__ u, const uint8_t *__restrict__ link,
                                         const uint32_t *__restrict__ cw, uint32_t *__restrict__ bnd, uint64_t cm,
                                         uint16_t *__restrict__ ld, uint8_t *__restrict__ dump, int m, int mbuf,
                                         int cstart, int W, int F, int s0, int s1, int half, int lane, int sw,
                                         int tx, bool &anym) {
    // token starts stay inside the lane's segment, which never crosses a
    // 128-position skew boundary: p-indexed arrays use a constant offset
    const int so = (s0 >> 7) << 2;
    const uint8_t *lks = link + so;
    uint16_t *lds = ld + (so >> 1);
    int p = next_cand(cm, s0, s0, s1);
    bool active = p < s1;
    uint32_t nm = 0;  // matches found on the path
    int d = 0, cap = 0;
    // W = 256: the links hold distances <= 255; d = 256 is evaluated as one
    // extra candidate when the chain ends (t256: done), first if p has no link
    bool t256 = false;
    auto begin_token = [&]() {
        d = lks[p];
        cap = min(F, m - p);
        t256 = BW && W == 256 && d == 0;
        d = t256 ? 256 : d;
    };
    if (active) begin_token();
    int k = 0, bestL = 2, bestD = 0;
    int qr = 0;  // reject-test mode (int: no byte-register repacking)
    auto finish_token = [&]() {
        if (ALLPOS) {
            dump[2 * p] = (uint8_t)(bestD ? bestL : 0);
            dump[2 * p + 1] = (uint8_t)bestD;
        } else {
            lds[p] = (uint16_t)(bestD ? Memo<BW>::match(bestD, bestL) : Memo<BW>::kLit);
        }
        nm |= bestD;
        p = next_cand(cm, p + (ALLPOS ? 1 : (bestD ? bestL : 1)), s0, s1);
        active = p < s1;
        if (active) begin_token();
        bestL = 2;
        bestD = 0;
        k = 0;
        qr = 0;
    };
    // W = 256: when p's chain is exhausted, try d = 256 once
    auto last256 = [&](bool fin) { return BW && fin && W == 256 && !t256 && bestL < cap && p - cstart >= 256; };
    // ---- machine 1: plain chain walk, until the warp has walked sw
    // iterations or one of its lanes has spent tx on its current token ------
    int it = 0, ti = 0;  // warp iterations, iterations of the lane's current token
#pragma unroll 1
    for (; it < sw && __any_sync(kFull, active) && !__any_sync(kFull, active && ti >= tx); it++) {
        ti++;
        if (active) {
            const int q = p - d;
            const int off = qr ? bestL - 7 : k;
            // next chain member, loaded with the compare words every iteration
            // (volatile: kept off the candidate-change path's latency)
            int lq;
            asm volatile("ld.volatile.shared.u8 %0, [%1];"
                         : "=r"(lq)
                         : "r"((uint32_t)__cvta_generic_to_shared(link + sk(q))));
            const Be8 vq = load8(u, q + off), vp = load8(u, p + off);
            const uint32_t xh = vq.hi ^ vp.hi, xl = vq.lo ^ vp.lo;
            const int fb = __clzll(((uint64_t)xh << 32) | xl) >> 3;  // equal leading bytes (<= 8), branch-free
            const bool cand_done = fb < 8 || (!qr && k + 8 >= cap);
            const int L = min(k + fb, cap);
            const bool upd = !qr && cand_done && L > bestL;
            bestL = upd ? L : bestL;
            bestD = upd ? d : bestD;
            k = qr ? 0 : k + 8;
            qr = qr && fb < 8 ? 1 : 0;
            bool tok_done = false;
            if (cand_done) {
                const int l2 = bestL == cap ? 0 : lq;
                int nd = d + l2;
                tok_done = l2 == 0 || nd > W;
                if (last256(tok_done)) {
                    tok_done = false;
                    nd = 256;
                    t256 = true;
                }
                d = nd;
                k = 0;
                qr = bestL >= 8 ? 1 : 0;
            }
            if (tok_done) {
                finish_token();
                ti = 0;
            }
        }
    }
    if (__any_sync(kFull, active)) {
        // ---- machine 2: the same walk with the two exact prunes ------------
        build_bnd_warp(cw, bnd, half, lane, mbuf);
        const int wl0 = min(W, p - cstart);
        int wlim = wl0;          // window limit of p: min(W, p - chunk start)
        int o = 0;               // chain offset (chain switch)
        int rs = 0;              // run skip: distance of the run start to resume after (0: none; > W: stop)
        int nrej = 0;            // candidates since the last improvement
        bool runp = false;       // bytes p..p+3 are equal (latched when off == 0)
#pragma unroll 1
        while (__any_sync(kFull, active)) {
            if (active) {
                const int q = p - d;
                const int off = qr ? bestL - 7 : k;
                int lq;
                asm volatile("ld.volatile.shared.u8 %0, [%1];"
                             : "=r"(lq)
                             : "r"((uint32_t)__cvta_generic_to_shared(link + sk(q + o))));
                const Be8 vq = load8(u, q + off), vp = load8(u, p + off);
                const uint32_t xh = vq.hi ^ vp.hi, xl = vq.lo ^ vp.lo;
                const int fb = __clzll(((uint64_t)xh << 32) | xl) >> 3;
                runp = off == 0 ? vp.hi == __byte_perm(vp.hi, 0, 0x3333) : runp;
                const bool cand_done = fb < 8 || (!qr && k + 8 >= cap);
                const int L = min(k + fb, cap);
                const bool lval = !qr && cand_done;  // L is the finished candidate's match length
                const bool upd = lval && L > bestL;
                bestL = upd ? L : bestL;
                bestD = upd ? d : bestD;
                k = qr ? 0 : k + 8;
                qr = qr && fb < 8 ? 1 : 0;
                bool tok_done = false;
                if (cand_done) {
                    nrej = upd ? 0 : nrej + 1;
                    int nd = d + lq;
                    bool fin = lq == 0 || nd > wlim || bestL == cap;  // default: follow the chain
                    if (!fin || rs) {
                        if (rs) {  // qs done: resume after the run start on p's own chain
                            nd = rs <= wlim ? chain_after(link, p, 0, rs, rs, wlim) : 0;
                            fin = nd == 0 || bestL == cap;
                            o = 0;
                            rs = 0;
                            nrej = 0;
                        } else if (lval && runp && L >= 3) {
                            const int t = run_len(bnd, p, cap);
                            if (L < t) {
                                const int lo = p - wlim;
                                const int r0 = run_start(bnd, q, lo);
                                const int qs = max(q + L - t, r0);
                                if (qs < q) {  // run skip (else q starts its run: follow the chain)
                                    nd = p - qs;
                                    rs = r0 > lo ? p - r0 : 0x7FFF;
                                }
                            }
                        } else if (nrej >= 2 && bestL >= 3 && bestL - 2 > o) {  // chain switch
                            o = bestL - 2;
                            nrej = 0;
                            const int e = link[sk(p + o)];
                            nd = e ? chain_after(link, p, o, e, d, wlim) : 0;
                            fin = nd == 0;
                        }
                    }
                    if (last256(fin)) {
                        fin = false;
                        nd = 256;
                        o = 0;
                        rs = 0;
                        t256 = true;
                    }
                    d = nd;
                    tok_done = fin;
                    k = 0;
                    qr = bestL >= 8 ? 1 : 0;
                }
                if (tok_done) {
                    finish_token();
                    wlim = min(W, p - cstart);
                    o = 0;
                    rs = 0;
                    nrej = 0;
                }
            }
        }
    }
    anym = nm != 0;
    return p;
}

// Re-walk from a corrected entry (fix-up rounds; short).  On a lane's first
// re-walk every memoised token start (ld != 0) belongs to its speculative
// path, so reaching one adopts the speculative exit: the greedy path from
// there is the same.  A later re-walk of the same lane (rare: its entry moved
// twice) cannot tell which earlier walk a memoised start belongs to and walks
// to the segment end, reusing memoised tokens.
template <bool BW>
__device__ int walk_fix(const uint32_t *__restrict__ u, const uint8_t *__restrict__ link, uint64_t cm,
                        uint16_t *__restrict__ ld, int m, int cstart, int W, int F, int s0, int s1, int entry,
                        int spec_exit, bool first) {
    int p = entry;
    while (true) {
        p = next_cand(cm, p, s0, s1);
        if (p >= s1) return p;
        uint32_t t = ld[sk2(p)];
        if (t && first) return spec_exit;
        if (!t) {
            t = eval_pos<BW>(u, link, p, m, cstart, W, F);
            ld[sk2(p)] = (uint16_t)t;
        }
        p += Memo<BW>::len(t);
    }
}

// ---------------------------------------------------------------------------
// Version 2: the paper's V2 search (PAPER.md:1@13703-14454 §III.B: "each
// thread ... is responsible for one character of the uncoded lookahead
// buffer" and searches the whole window buffer for it; "all the matches are
// searched ... redundant ones are eliminated" @17800) as the north star's
// warp-cooperative kernel: (L, D) of EVERY position over EVERY window offset.
// Lane l owns the offsets d = l + 1 + 32k (k < K; K = 4 for W <= 128, 8
// above); warp h sweeps half the chunk's positions from the top down, one
// 32-bit word (4 positions) per step, with the diagonal run recurrence
//     R_d(p) = (chunk[p] == chunk[p-d]) ? min(R_d(p+1) + 1, F) : 0,
// whose equalities come from one packed 32-bit compare (XOR + exact
// zero-byte test) of bytes p..p+3 against p-d..p-d+3 per offset -- the
// compare count of the roofline's compare term, with no
// data-dependent early-out loop.  R_d(p) <= m - p because the sweep starts
// at the chunk end with R = 0 (and restarts at every packed chunk boundary);
// pairs with d > p - chunk start or d > W never match.  The argmax over d is
// one __reduce_max_sync per position over (L << 8) | (256 - d): the largest L,
// ties to the smallest d (reading R7); L < 3 is a literal (R4).  The result is
// the same (L, D) table the lazy walk evaluates on demand, so the greedy parse
// and the bit-pack downstream are shared.
//
// bytes x..x+3 (little endian) of the unskewed chunk copy U (x >= 0)
__device__ __forceinline__ uint32_t v2_bytes4(const uint32_t *__restrict__ U, int x) {
    const uint32_t a = (uint32_t)x >> 2;
    return __funnelshift_r(U[a], U[a + 1], (uint32_t)x << 3);  // the shift is taken mod 32
}

// prmt with the selector's sign-replicate bit honoured (__byte_perm masks it)
__device__ __forceinline__ uint32_t prmt_sx(uint32_t a, uint32_t b, uint32_t sel) {
    uint32_t r;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
    return r;
}

// P16 (F <= 254): two offsets' keys per register as 16-bit halves,
// updated by the 16x2 forms (VIADDMNMX.U16x2, VIMNMX.U16x2); a position's
// two "differs" half-masks come from one sign-replicating byte permute of the
// two offsets' per-byte difference bits.
template <int K, bool P16>
__device__ void v2_search_all(const uint32_t *__restrict__ U, uint16_t *__restrict__ ld, int m, int W, int F,
                              int half, int lane, int smask) {
    // warp 0: positions [0, M0), warp 1: [M0, m); M0 is a word boundary
    const int M0 = ((m >> 1) + 3) & ~3;
    const int r0 = half ? M0 : 0, r1 = half ? m : M0;
    if (r0 >= r1) return;
    uint32_t R[K];     // (R_d << 8) | (256 - d) at the last position swept
    uint32_t dead[K];  // all ones: offset beyond W (never matches)
#pragma unroll
    for (int k = 0; k < K; k++) {
        const int d = lane + 1 + 32 * k;
        dead[k] = d <= W ? 0u : 0xFFFFFFFFu;
        // the run at r1 (the carry into the sweep): 0 at the chunk end or at a
        // packed chunk boundary, else measured directly
        int r = 0;
        if (r1 < m && (r1 & smask) != 0 && d <= W && d <= (r1 & smask)) {
            const int cap = min(F, min((r1 | smask) + 1, m) - r1);
            while (r < cap) {
                const uint32_t x = v2_bytes4(U, r1 + r) ^ v2_bytes4(U, r1 - d + r);
                if (x) {
                    r += (__ffs(x) - 1) >> 3;
                    break;
                }
                r += 4;
            }
            r = min(r, cap);
        }
        R[k] = ((uint32_t)r << 8) | (uint32_t)(256 - d);
    }
    // P16: offsets 2q (low half) and 2q + 1 (high half) share register q
    uint32_t R2[K / 2], c2[K / 2], fk2[K / 2];
#pragma unroll
    for (int q = 0; q < K / 2; q++) {
        c2[q] = (uint32_t)(256 - (lane + 1 + 64 * q)) | ((uint32_t)(256 - (lane + 33 + 64 * q)) << 16);
        fk2[q] = c2[q] | ((uint32_t)F << 8) | ((uint32_t)F << 24);
        R2[q] = (R[2 * q] & 0xFFFFu) | (R[2 * q + 1] << 16);
    }
    // One step: the 4 positions of word p0.  EDGE steps (the first W
    // positions of a chunk, where d > p - chunk start, and the buffer's last,
    // partial word) mask the invalid pairs; the others are straight-line: for
    // offset d_k = lane + 1 + 32k the bytes p0 - d_k .. + 3 lie in the aligned
    // words at byte offsets p0 - c4 - 32k and + 4 (c4 = d_0 rounded up to a
    // multiple of 4), shifted by the same amount for every k.
    const int c4 = (lane + 4) & ~3;
    const uint32_t shq = 8u * (uint32_t)((-(lane + 1)) & 3);
    const unsigned char *Ub = reinterpret_cast<const unsigned char *>(U);
    uint32_t mine = 0;  // the argmax key of position (block base) + lane
    auto flush = [&](int blk) {  // positions blk .. blk + 31 (those of this warp)
        const int p = blk + lane;
        const uint32_t key = P16 ? (mine & 0xFFFFu) : mine;
        if (p >= r0 && p < r1)
            ld[sk2(p)] = key >= (3u << 8) ? (uint16_t)Memo<true>::match((int)(256 - (key & 0xFF)), (int)(key >> 8))
                                          : Memo<true>::kLit;
    };
    auto step = [&](int p0, bool edge) {
        const uint32_t P = U[p0 >> 2];
        const int lowp = p0 & smask;               // position of p0 in its chunk
        const unsigned char *qa = Ub + (p0 - c4);
        uint32_t rk[K][4];  // key (R << 8) | c of positions p0 + j, per offset
        uint32_t nzv[K];    // P16: per-byte difference bits, per offset
#pragma unroll
        for (int k = 0; k < K; k++) {
            const int d = lane + 1 + 32 * k;
            uint32_t Q;
            if (!edge) {
                const uint32_t *w = reinterpret_cast<const uint32_t *>(qa - 32 * k);
                Q = __funnelshift_r(w[0], w[1], shq);
            } else {
                // before the buffer start (-3 <= q < 0 holds valid bytes) the
                // first word shifted into place
                const int q = p0 - d;
                Q = q >= 0 ? v2_bytes4(U, q) : v2_bytes4(U, 0) << (8 * min(-q, 3));
            }
            // byte j of x is 0 iff positions p0 + j and p0 + j - d hold equal bytes
            // (a dead offset, d > W, never matches)
            uint32_t x = (P ^ Q) | dead[k];
            if (edge) {
#pragma unroll
                for (int j = 0; j < 4; j++)
                    if (d > lowp + j || p0 + j >= m) x |= 0xFFu << (8 * j);
            }
            if constexpr (P16) {
                nzv[k] = ((x & 0x7F7F7F7Fu) + 0x7F7F7F7Fu) | x;  // bit 7 of byte j: differs
            } else {
                // the recurrence carried on the key (R << 8) | c itself: +256 per
                // equal byte, capped at (F << 8) | c, back to c (R = 0) on a difference
                const uint32_t c = (uint32_t)(256 - d), fk = ((uint32_t)F << 8) | c;
                uint32_t r = R[k];
                r = (x & 0xFF000000u) ? c : min(r + 256u, fk);
                rk[k][3] = r;
                r = (x & 0x00FF0000u) ? c : min(r + 256u, fk);
                rk[k][2] = r;
                r = (x & 0x0000FF00u) ? c : min(r + 256u, fk);
                rk[k][1] = r;
                r = (x & 0x000000FFu) ? c : min(r + 256u, fk);
                rk[k][0] = r;
                R[k] = r;
            }
        }
        uint32_t bj[4];
        if constexpr (P16) {
            uint32_t rk2[K / 2][4];
#pragma unroll
            for (int q = 0; q < K / 2; q++) {
                uint32_t r = R2[q];
#pragma unroll
                for (int j = 3; j >= 0; j--) {
                    // halves 0xFFFF where position p0 + j differs for offset 2q / 2q + 1
                    const uint32_t msk = prmt_sx(nzv[2 * q], nzv[2 * q + 1],
                                                 (uint32_t)((8 + j) | ((8 + j) << 4) | ((12 + j) << 8) | ((12 + j) << 12)));
                    r = __viaddmin_u16x2(r, 0x01000100u, fk2[q]);
                    r = (r & ~msk) | (c2[q] & msk);
                    rk2[q][j] = r;
                }
                R2[q] = r;
            }
#pragma unroll
            for (int j = 0; j < 4; j++) {
                uint32_t mm = rk2[0][j];
#pragma unroll
                for (int q = 1; q < K / 2; q++) mm = __vmaxu2(mm, rk2[q][j]);
                bj[j] = __vmaxu2(mm, __byte_perm(mm, 0, 0x1032));  // the larger key in both halves
            }
        } else {
            // the lane's best key per position: three-input maxima over its offsets
    #pragma unroll
            for (int j = 0; j < 4; j++) {
                uint32_t b = rk[0][j];
    #pragma unroll
                for (int k = 1; k < K; k += 2)
                    b = k + 1 < K ? __vimax3_u32(b, rk[k][j], rk[k + 1][j]) : max(b, rk[k][j]);
                bj[j] = b;
            }

        }
        uint32_t best0 = bj[0], best1 = bj[1], best2 = bj[2], best3 = bj[3];
        best0 = __reduce_max_sync(kFull, best0);
        best1 = __reduce_max_sync(kFull, best1);
        best2 = __reduce_max_sync(kFull, best2);
        best3 = __reduce_max_sync(kFull, best3);
        // lane t keeps the key of position (p0 & ~31) + t; the warp stores a
        // block of 32 positions once its lowest word is done
        const unsigned t = (unsigned)(lane - (p0 & 31));
        const uint32_t s01 = (t & 1) ? best1 : best0, s23 = (t & 1) ? best3 : best2;
        const uint32_t sv = (t & 2) ? s23 : s01;
        mine = t < 4 ? sv : mine;
        if ((p0 & 31) == 0) flush(p0);
    };
    int p0 = (r1 - 1) & ~3;
    if (p0 + 4 > m) {  // the buffer's last, partial word
        step(p0, true);
        p0 -= 4;
    }
#pragma unroll 1
    while (p0 >= r0) {
        if (((p0 + 4) & smask) == 0) {  // a chunk ends above this word: no carry into it
#pragma unroll
            for (int k = 0; k < K; k++) R[k] = (uint32_t)(256 - (lane + 1 + 32 * k));
#pragma unroll
            for (int q = 0; q < K / 2; q++) R2[q] = c2[q];
        }
        // straight-line steps down to the first W positions of p0's chunk
        // (they always read bytes >= 0: p0 - d >= chunk start)
        const int fe = max(r0, (p0 & ~smask) + ((W + 3) & ~3));
#pragma unroll 1
        for (; p0 >= fe; p0 -= 4) step(p0, false);
#pragma unroll 1
        for (; p0 >= r0 && (p0 & smask) < W; p0 -= 4) step(p0, true);
    }
    if (r0 & 31) flush(r0 & ~31);  // the last, partial block
}

// greedy parse over a fully evaluated token table: jump from p to the end of
// segment [.., s1); returns the exit (first position >= s1 on the path)
__device__ __forceinline__ int v2_jump(const uint16_t *ld, int p, int s1) {
#pragma unroll 1
    while (p < s1) p += Memo<true>::len(ld[sk2(p)]);  // version 2 runs in the W > 128 instantiation
    return p;
}

__device__ __forceinline__ void pair_sync(int id) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(kWalkLanes) : "memory");
}

template <int MODE, bool SMALLW, bool V2, bool PACK, bool TILED>
__global__ void __launch_bounds__(kChunksPerCta * kWalkLanes, kCtasPerSm)
chunk_kernel(const uint8_t *__restrict__ in, uint64_t n, Geometry g, uint8_t *__restrict__ bucket,
             uint32_t *__restrict__ sizes, void *__restrict__ dbg) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int lane = threadIdx.x & 31;
    const int pair = threadIdx.x / kWalkLanes;     // chunk slot in the CTA
    const int half = (threadIdx.x >> 5) % kWarpsPerChunk;  // warp within the chunk
    const int t64 = threadIdx.x % kWalkLanes;      // walk lane 0..63
    const int bar = 1 + pair;                      // named barrier of the warp pair
    WarpSmem &sm = reinterpret_cast<WarpSmem *>(smem_raw)[pair];
    const uint64_t C = (n + g.S - 1) / g.S;
    // the pair's chunks [c, c + K): K = 1 (S > 2048 or not a power of two) or
    // 4096 / S small chunks packed back to back into one 4096-position buffer
    const uint64_t c = ((uint64_t)blockIdx.x * kChunksPerCta + pair) * g.K;
    // programmatic dependent launch: the scan grid may be scheduled as soon as
    // every CTA of this grid has started (it waits for our results itself)
    asm volatile("griddepcontrol.launch_dependents;");
    if (c >= C) return;  // both warps of the pair leave together
    const uint64_t start = c * g.S;
    // !TILED: the buffer's length (one chunk, or K packed small chunks);
    // TILED: the chunk's length (S > 4096)
    const int m0 = (int)min((uint64_t)g.K * g.S, n - start);
    const int smask = PACK ? (int)g.smask : 4095;  // !PACK: one chunk, no inner bounds
    const int W = g.W, F = g.F;
    uint8_t *cb = reinterpret_cast<uint8_t *>(sm.cw);
    uint8_t *link = sm.a.link;
    // TILED (S > 4096; DESIGN.md §5 "large chunks"): the chunk is compressed
    // in tiles of one 4096-position buffer each -- chunk bytes [B0, B0 + m),
    // B0 = the tile's first parse position minus Hh >= W bytes of window
    // history; parse region [T0, T1) in buffer coordinates (the last Fh >= F - 1
    // positions of a non-last tile are lookahead only); the greedy path enters
    // the tile at Eb and leaves it at the first position >= T1 it reaches.  The
    // tiles' bits are appended to the chunk's bucket 16-byte unit by unit; the
    // last partial unit is carried to the next tile.
    const int Hh = TILED ? (W + 63) & ~63 : 0, Fh = TILED ? (F - 1 + 63) & ~63 : 0;
    int tileT1c = 0, Ec = 0;  // previous tile's parse end, the path's entry (chunk coordinates)
    int boff = 0;             // payload bits of the earlier tiles
    uint32_t cy0 = 0, cy1 = 0, cy2 = 0, cy3 = 0;  // their last, partial 16-byte unit (payload words)
#pragma unroll 1
    for (int tile = 0;; tile++) {
        if (TILED && tile > 0) pair_sync(bar);  // the previous tile's shared-memory reads are done
        const int B0 = TILED && tile > 0 ? tileT1c - Hh : 0;
        const int m = TILED ? min(kChunkMax, m0 - B0) : m0;
        const bool last = !TILED || m0 - B0 <= kChunkMax;
        const int T0 = TILED && tile > 0 ? Hh : 0;
        const int T1 = last ? m : kChunkMax - Fh;
        const int Eb = Ec - B0;
        const uint8_t *src = in + start + B0;

        // ---------------- a1: stage the chunk (16-byte coalesced loads) --------
        // a full chunk overwrites every data byte, so nothing needs clearing and
        // no barrier has to order the clearing before the data stores (bytes past
        // the chunk end are only ever read beyond a match's cap)
        const bool full = m == kChunkMax;
        {
            uint4 *z4 = reinterpret_cast<uint4 *>(sm.cw);
            const uint4 z = make_uint4(0, 0, 0, 0);
            if (!full) {
                for (int i = t64; i < (int)(sizeof(sm.cw) / 16); i += kWalkLanes) z4[i] = z;
            }
            uint4 *t4 = reinterpret_cast<uint4 *>(sm.a.u.tab);
            // u8 tables: empty = (s0 - 129) mod 256 = 0x7F (even lanes) / 0xFF (odd)
    #pragma unroll 4
            for (int i = t64; i < (int)(sizeof(sm.a.u.tab) / 16); i += kWalkLanes) {
                // u8 tables: lane (i >> 5)'s 512 bytes hold its empty value
                const uint32_t e = SMALLW ? ((i >> 5) & 1 ? 0xFFFFFFFFu : 0x7F7F7F7Fu) : 0u;
                t4[i] = make_uint4(e, e, e, e);
            }
        }
        if (!full) pair_sync(bar);  // (uniform per pair)
        if ((reinterpret_cast<uintptr_t>(src) & 15) == 0) {
            // a 16-byte group never straddles a 128-position segment
            const int nvec = m >> 4;
            const uint4 *s4 = reinterpret_cast<const uint4 *>(src);
    #pragma unroll 4
            for (int i = t64; i < nvec; i += kWalkLanes) {
                const uint4 v = __ldcs(s4 + i);
                uint32_t *d = sm.cw + (sk(i << 4) >> 2);
                d[0] = v.x;
                d[1] = v.y;
                d[2] = v.z;
                d[3] = v.w;
            }
            for (int i = (nvec << 4) + t64; i < m; i += kWalkLanes) cb[sk(i)] = src[i];
        } else {
            for (int i = t64; i < m; i += kWalkLanes) cb[sk(i)] = src[i];
        }
        pair_sync(bar);
        // pad word of 128-segment `lane` = first word of the next segment (0 past the end)
        if (half == 0) sm.cw[33 * lane + 32] = lane < 31 ? sm.cw[33 * (lane + 1)] : 0u;
        pair_sync(bar);

        // ---------------- a2 part 1: per-lane 3-gram hash chains (warp 0) ------
        // Lane l of warp 0 owns the 128-position build segment [128 l, 128 l + 128)
        // and its own hash table; straight-line: every position is hashed and
        // inserted; the last two positions (no 3-gram) get link 0 after.
        if (!V2 && half == 0) {
            const int b0 = lane * kSeg;
            const int b1 = min(b0 + kSeg, m);
            unsigned char *tabl = reinterpret_cast<unsigned char *>(sm.a.u.tab) + (SMALLW ? 512 * lane : 2 * lane);
            if (b0 < m) {
                // the W positions before the segment (pre-insert, no links)
    #pragma unroll 4
                for (int q = max(0, b0 - W) & ~3; q < b0; q += 4) {
                    const uint32_t w0 = sm.cw[sk(q) >> 2], w1 = sm.cw[(sk(q) >> 2) + 1];
    #pragma unroll
                    for (int j = 0; j < 4; j++) {
                        const uint32_t key = __funnelshift_r(w0, w1, 8 * j);
                        if (SMALLW)
                            tabl[hash9(key)] = (uint8_t)(q + j);
                        else
                            *reinterpret_cast<uint16_t *>(tabl + hash_off(key)) = (uint16_t)(q + j + kTabBias);
                    }
                }
                // own segment: links
                const uint32_t w4 = (uint32_t)min(W, 255) * 0x01010101u;
    #pragma unroll 1
                for (int wi = 0; wi < 4; wi++) {
                    const int pb = b0 + 32 * wi;
                    if (pb < b1) {
    #pragma unroll
                        for (int i = 0; i < 8; i++) {
                            const int p = pb + 4 * i;
                            const uint32_t w0 = sm.cw[sk(p) >> 2], w1 = sm.cw[(sk(p) >> 2) + 1];
                            uint32_t lw = 0;
                            if (SMALLW) {
                                // entries hold position mod 256: every live entry is
                                // within 256 of p, the empty value maps to 0 or > 128.
                                // Entries are read and replaced in position order
                                // (a repeated hash in the group sees its predecessor),
                                // then the four distances are formed bytewise.
                                uint32_t E = 0;
    #pragma unroll
                                for (int j = 0; j < 4; j++) {
                                    uint8_t *e = tabl + hash9(__funnelshift_r(w0, w1, 8 * j));
                                    E |= (uint32_t)*e << (8 * j);
                                    *e = (uint8_t)(p + j);
                                }
                                const uint32_t D = __vsub4(__vadd4(((uint32_t)p & 0xFFu) * 0x01010101u, 0x03020100u), E);
                                // at most W, and never before the chunk start (packed
                                // small chunks; a 4-group lies in one chunk)
                                uint32_t lim = w4;
                                if (PACK) {
                                    const uint32_t rel = (uint32_t)min(p & smask, 252);
                                    lim = __vminu4(w4, __vadd4(rel * 0x01010101u, 0x03020100u));
                                }
                                lw = D & __vcmpleu4(D, lim);  // distance, or 0 past the window
                            } else {
    #pragma unroll
                                for (int j = 0; j < 4; j++) {
                                    const uint32_t key = __funnelshift_r(w0, w1, 8 * j);
                                    uint16_t *e = reinterpret_cast<uint16_t *>(tabl + hash_off(key));
                                    const uint32_t dist = (uint32_t)(p + j + kTabBias) - *e;
                                    *e = (uint16_t)(p + j + kTabBias);
                                    // links are u8: distances <= 255 (W = 256 adds d = 256 in the walk)
                                    const bool ok = dist <= (uint32_t)min(W, 255) && (!PACK || dist <= (uint32_t)((p + j) & smask));
                                    lw |= (ok ? dist : 0u) << (8 * j);
                                }
                            }
                            *reinterpret_cast<uint32_t *>(link + sk(p)) = lw;
                        }
                    }
                }
            }
            // positions m-2 and m-1 have no 3-gram: never candidates
    #pragma unroll
            for (int t = 1; t <= 2; t++) {
                const int x = m - t;
                if (x >= b0 && x < b1) link[sk(x)] = 0;
            }
        }
        pair_sync(bar);  // tab is dead from here on
        if (V2) {
            // version 2: (L, D) of every position by the warp-cooperative search,
            // on an unskewed little-endian copy of the chunk (+ zero tail)
            uint32_t *U = sm.a.u.w.ucw;
            for (int j = t64; j < kUcwWords; j += kWalkLanes) U[j] = j < kChunkMax / 4 ? sm.cw[j + (j >> 5)] : 0u;
            pair_sync(bar);
            // 16-bit keys whenever (R << 8) | (256 - d) + 256 fits them: F <= 254
            if (W <= 128 && F <= 254)
                v2_search_all<4, true>(U, sm.a.u.w.ld, m, W, F, half, lane, smask);
            else if (W <= 128)
                v2_search_all<4, false>(U, sm.a.u.w.ld, m, W, F, half, lane, smask);
            else if (F <= 254)
                v2_search_all<8, true>(U, sm.a.u.w.ld, m, W, F, half, lane, smask);
            else
                v2_search_all<8, false>(U, sm.a.u.w.ld, m, W, F, half, lane, smask);
            pair_sync(bar);
        }

        if (V2 && MODE == kModeDumpMatch) {
            // every position's evaluated token, for per-position parity (a2)
            uint8_t *LD = reinterpret_cast<uint8_t *>(dbg) + 2 * start;
            for (int p = t64; p < m; p += kWalkLanes) {
                const uint32_t t = sm.a.u.w.ld[sk2(p)];
                LD[2 * p] = (uint8_t)(Memo<true>::is_match(t) ? Memo<true>::len(t) : 0);
                LD[2 * p + 1] = (uint8_t)(Memo<true>::is_match(t) ? Memo<true>::dist(t) : 0);
            }
            return;
        }

        // ---------------- a3: lazy greedy walk, speculative per 64-segment -----
        const int s0 = t64 * kWSeg;
        // <= s0 for lanes past the chunk end (TILED: outside the parse region)
        const int s1 = TILED ? (s0 >= T0 && s0 < T1 ? min(s0 + kWSeg, T1) : s0) : min(s0 + kWSeg, m);
        const int ce = PACK ? min((s0 | smask) + 1, m) : m;  // end of the segment's chunk (matches stop there)
        const int cst = PACK ? (s0 & ~smask) : 0;  // start of the segment's chunk
        uint16_t *ld = sm.a.u.w.ld;
        uint32_t *ucw = sm.a.u.w.ucw;
        // the warp's run-boundary mask (free until the bit-pack staging), indexed by mask word
        uint32_t *bnd = reinterpret_cast<uint32_t *>(sm.a.u.w.pad) + kBndWarpWords * half + kBndWarpLo - 64 * half;
        if (!V2) {
            // zero the memoised tokens (their bytes held the hash tables) and
            // unskew the chunk for the walks' compares
            uint4 *l4 = reinterpret_cast<uint4 *>(ld);
            const uint4 z = make_uint4(0, 0, 0, 0);
    #pragma unroll 4
            for (int i = t64; i < (int)(sizeof(sm.a.u.w.ld) / 16); i += kWalkLanes) l4[i] = z;
    #pragma unroll 4
            for (int j = t64; j < kUcwWords; j += kWalkLanes)
                ucw[j] = j < kChunkMax / 4 ? __byte_perm(sm.cw[j + (j >> 5)], 0, 0x0123) : 0u;  // + zero tail
        }
        // candidate mask: bit i = position s0 + i (< s1) has a chain link
        uint32_t rc0 = 0, rc1 = 0;
        uint32_t h[2] = {0, 0};
        if (V2) {
            // every position holds its evaluated token
            const int r = max(s1 - s0, 0);
            rc0 = r >= 32 ? 0xFFFFFFFFu : ~(0xFFFFFFFFu >> r);
            rc1 = r <= 32 ? 0u : (r >= 64 ? 0xFFFFFFFFu : ~(0xFFFFFFFFu >> (r - 32)));
        } else if (s0 < s1) {
            const int so = (s0 >> 7) << 2;  // constant skew inside the segment
    #pragma unroll
            for (int w = 0; w < kWSeg / 4; w++) {
                const uint32_t lw = *reinterpret_cast<const uint32_t *>(link + so + s0 + 4 * w);
                const uint32_t nz = (((lw & 0x7F7F7F7Fu) + 0x7F7F7F7Fu) | lw) & 0x80808080u;
                h[w >> 3] |= ((nz >> 7) * 0x10204080u >> 28) << (4 * (w & 7));  // bit j = byte j nonzero
            }
            if (!SMALLW && W == 256) {
                // W = 256: a position whose 3-gram recurs exactly 256 back is a
                // candidate too (the u8 links stop at 255; the walk adds d = 256)
                for (int i = max(s0, cst + 256); i < min(s1, ce - 2); i++) {
                    if (((load4(sm.cw, i) ^ load4(sm.cw, i - 256)) & 0xFFFFFFu) == 0)
                        h[(i - s0) >> 5] |= 1u << ((i - s0) & 31);
                }
            }
            if (s1 - s0 < 64) {  // positions >= s1 (garbage links)
                const int r = s1 - s0;
                h[0] &= r >= 32 ? 0xFFFFFFFFu : (1u << r) - 1;
                h[1] &= r <= 32 ? 0u : (1u << (r - 32)) - 1;
            }
        }
        // a position whose chain is one hash collision and nothing more has
        // no candidate at all: a literal, never evaluated.  Checked where
        // every lane of the warp has sparse links (incompressible data,
        // whose candidates are nearly all collisions; on text the chains
        // continue and the check would only cost)
        if (!V2 && SMALLW && __all_sync(kFull, __popc(h[0]) + __popc(h[1]) <= kSparseLinks)) {
#pragma unroll
            for (int hw = 0; hw < 2; hw++) {
                uint32_t keep = h[hw];
#pragma unroll 1
                for (uint32_t b = h[hw]; b; b &= b - 1) {
                    const int p = s0 + 32 * hw + __ffs(b) - 1;
                    const int d = link[sk(p)];
                    const int l2 = link[sk(p - d)];
                    const bool eq3 = ((load4(sm.cw, p) ^ load4(sm.cw, p - d)) & 0xFFFFFFu) == 0;
                    if (!eq3 && (l2 == 0 || d + l2 > W)) keep &= ~(1u << (p - s0 - 32 * hw));
                }
                h[hw] = keep;
            }
        }
        if (!V2) {
            rc0 = __brev(h[0]);
            rc1 = __brev(h[1]);
        }
        pair_sync(bar);
        bool anym = true;  // the speculative path holds a match (V2: not tracked)
        const uint64_t cm = ((uint64_t)rc0 << 32) | rc1;
        if (MODE == kModeDumpMatch) {
            // every candidate position through the production walk machine (a2)
            uint8_t *LD = reinterpret_cast<uint8_t *>(dbg) + 2 * (start + B0);
            walk_spec<true, !SMALLW>(ucw, link, sm.cw, bnd, cm, ld, LD, ce, m, cst, W, F, s0, s1, half, lane, (int)g.sw,
                            (int)g.tx, anym);
            if (last) return;
            tileT1c = B0 + T1;
            continue;
        }
        const int spec_exit =
            V2 ? v2_jump(ld, s0, s1) : walk_spec<false, !SMALLW>(ucw, link, sm.cw, bnd, cm, ld, nullptr, ce, m, cst, W, F, s0, s1, half, lane,
                                         (int)g.sw, (int)g.tx, anym);
        int exitp = TILED && s0 < T0 ? Eb : spec_exit;  // window-history lanes hand on the tile's entry
        int cur = s0;
        bool first = true;
        volatile uint32_t *xf = sm.a.u.w.xfer;
        // two barriers per round: exits and "changed" flags use slots alternating
        // with the round's parity, so a slot is rewritten only two rounds later,
        // after every read of it
        int par = 0;
    #pragma unroll 1
        while (true) {
            // entry of walk lane t64 = exit of lane t64 - 1 (warp 1 lane 0 reads
            // warp 0 lane 31 through shared memory)
            int entry = __shfl_up_sync(kFull, exitp, 1);
            if (lane == 31) xf[2 * par + half] = (uint32_t)exitp;
            pair_sync(bar);
            if (lane == 0) entry = half ? (int)xf[2 * par + half - 1] : 0;
            const bool chg = (!TILED || (s0 >= T0 && s0 < T1)) && entry != cur;
            const bool any = __any_sync(kFull, chg);
            if (lane == 0) xf[4 + 2 * par + half] = any;
            pair_sync(bar);
            bool go = false;
    #pragma unroll
            for (int k = 0; k < kWarpsPerChunk; k++) go |= xf[4 + 2 * par + k] != 0;
            if (!go) break;
            par ^= 1;
            if (chg) {
                exitp = V2 ? v2_jump(ld, entry, s1)
                           : walk_fix<!SMALLW>(ucw, link, cm, ld, ce, cst, W, F, s0, s1, entry, spec_exit, first);
                first = false;
                cur = entry;
            }
        }

        // TILED: the tile's exit (ucw is dead after the walks; read after the next barrier)
        if (TILED && !last && t64 == (T1 - 1) / kWSeg) ucw[0] = (uint32_t)exitp;
        if (MODE == kModeDumpTokens) {
            uint32_t *tok = reinterpret_cast<uint32_t *>(dbg) + start + B0;
            for (int p = s0; p < s1; p++) tok[p] = 0;
            int p = cur;
            while (p < s1) {
                if (!is_cand(cm, p - s0)) {
                    tok[p] = 1;
                    p++;
                } else {
                    const uint32_t t = ld[sk2(p)];
                    tok[p] = Memo<!SMALLW>::is_match(t) ? ((uint32_t)Memo<!SMALLW>::len(t) << 16) | (uint32_t)Memo<!SMALLW>::dist(t)
                                                        : 1u;
                    p += Memo<!SMALLW>::len(t);
                }
            }
            if (last) return;
            pair_sync(bar);
            Ec = B0 + (int)ucw[0];
            tileT1c = B0 + T1;
            continue;
        }
        pair_sync(bar);  // link is dead: staging may overwrite it
        if (TILED && !last) Ec = B0 + (int)ucw[0];

        // ---------------- a4: bit-pack ----------------------------------------
        // Each walk lane emits its path's tokens MSB-first into its own staging
        // words starting at bit 0 (a token is up to 3 literals of a candidate-free
        // run, an evaluated literal, or a match); after the scan of bit counts the
        // staged words are shifted into place.
        uint32_t *stage = reinterpret_cast<uint32_t *>(sm.a.link) + t64 * kStageWords;
        int nbits = 0;
        {
            // Uniform position scan (no token jumps): every position >= the lane's
            // true entry is either inside a path match (covered) or a path token
            // start; a token start's memoised ld[] is its token whichever walk
            // wrote it, and is 0 for candidate-free positions (literals).  Each
            // position emits 0, 9 or 17 bits.
            uint64_t acc = 0;
            int nacc = 0;
            uint32_t *sp = stage;  // next staging word
            int cov = cur;  // positions < cov are covered (by the previous lane or a match)
            const int so = (s0 >> 7) << 2;
            const uint32_t *ldw = reinterpret_cast<const uint32_t *>(ld + (so >> 1) + s0);  // 2 tokens / word
            const uint32_t *cbw = reinterpret_cast<const uint32_t *>(cb + so + s0);         // 4 bytes / word
            const int ng = (s1 - s0 + 3) >> 2;
            // append pn (<= 26) bits; acc keeps < 32 pending bits between calls
            auto put = [&](uint32_t pv, int pn) {
                acc = (acc << pn) | pv;
                nacc += pn;
                if (nacc >= 32) {
                    nacc -= 32;
                    *sp++ = (uint32_t)(acc >> nacc);
                }
            };
            if (__all_sync(kFull, !anym && cur == s0 && s1 - s0 == kWSeg)) {
                // every lane of the warp walks its whole segment from its start
                // and found no match: 64 literals each (incompressible data),
                // emitted branch-free in 18-bit pairs (bit positions static)
    #pragma unroll
                for (int i = 0; i < kWSeg / 4; i++) {
                    const uint32_t bytes = cbw[i];
                    put(((bytes & 0xFFu) << 9) | ((bytes >> 8) & 0xFFu), 18);
                    put((((bytes >> 16) & 0xFFu) << 9) | (bytes >> 24), 18);
                }
            } else {
                // groups wholly inside a match are skipped.  Positions are
                // combined in pairs in 32 bits first: a pair is at most a literal
                // and a match (26 bits), since a match covers the next position.
                // Only a chunk's last lane can have a partial last group: full
                // groups skip the segment-end test.
                auto group = [&](int i, bool chk) {
                    const uint32_t bytes = cbw[i];
                    const uint32_t t01 = ldw[2 * i], t23 = ldw[2 * i + 1];
                    uint32_t pv = 0;
                    int pn = 0;
    #pragma unroll
                    for (int j = 0; j < 4; j++) {
                        const int p = s0 + 4 * i + j;
                        const uint32_t t = (j < 2 ? t01 : t23) >> (16 * (j & 1)) & 0xFFFFu;
                        const bool on = p >= cov && (!chk || p < s1);
                        const bool mt = on && Memo<!SMALLW>::is_match(t);
                        const int nb = mt ? 17 : (on ? 9 : 0);
                        const uint32_t val = mt ? Memo<!SMALLW>::code(t) : (on ? (bytes >> (8 * j)) & 0xFFu : 0u);  // 1|D-1|L-3
                        cov = mt ? p + Memo<!SMALLW>::len(t) : cov;
                        pv = (pv << nb) | val;
                        pn += nb;
                        if (j & 1) {
                            put(pv, pn);
                            pv = 0;
                            pn = 0;
                        }
                    }
                };
                const int ngf = (s1 - s0) >> 2;  // full groups
                int i = max(0, (cov - s0) >> 2);
    #pragma unroll 1
                for (; i < ngf; i = max(i + 1, (cov - s0) >> 2)) group(i, false);
                if (i == ngf && ngf < ng) group(i, true);
            }
            const int nw = (int)(sp - stage);
            nbits = 32 * nw + nacc;
            if (nacc > 0) *sp = (uint32_t)(acc << (32 - nacc));
        }
        // exclusive scan of bit counts over the 64 walk lanes
        int incl = nbits;
    #pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(kFull, incl, o);
            if (lane >= o) incl += y;
        }
        if (lane == 31) xf[half] = (uint32_t)incl;
        pair_sync(bar);
        int before = 0, total = 0;
    #pragma unroll
        for (int k = 0; k < kWarpsPerChunk; k++) {
            const int v = (int)xf[k];
            before += k < half ? v : 0;
            total += v;
        }
        incl += before;
        int excl = incl - nbits;
        const int cb0 = TILED ? (boff & 127) : 0;  // TILED: bits of the carried partial unit come first
        excl += cb0;
        total += cb0;
        const uint64_t stride = bucket_stride(g.S);
        const int kk = (m + (int)g.S - 1) / (int)g.S;  // chunks in this pair
        int cbits = total, cword = 0;                  // this lane's chunk: total bits, first payload word
        if (PACK) {
            // packed chunks: a chunk's lanes are lpc consecutive lanes of one warp;
            // bit offsets restart at each chunk, whose payload words start at its
            // bucket offset in ow (the same layout as the buckets in HBM)
            const int lpc = (int)g.S / kWSeg;
            const int first = lane & ~(lpc - 1);
            const int cbase = __shfl_sync(kFull, excl, first);
            cbits = __shfl_sync(kFull, excl + nbits, first + lpc - 1) - cbase;
            excl -= cbase;
            cword = (t64 / lpc) * (int)(stride / 4);
        }
        // (TILED: every word of the last, partial 16-byte unit, which is carried)
        const int nwords = PACK ? kk * (int)(stride / 4) : (TILED ? 4 * ((total + 127) >> 7) + 4 : ((total + 31) >> 5) + 1);
        uint32_t *ow = reinterpret_cast<uint32_t *>(ld);  // ld is dead: payload words
    #pragma unroll 4
        for (int i = t64; i < nwords; i += kWalkLanes)
            ow[i] = TILED && i < 4 ? (i == 0 ? cy0 : i == 1 ? cy1 : i == 2 ? cy2 : cy3) : 0u;
        pair_sync(bar);
        {
            // shift the lane's staged words to bit offset excl; output words shared
            // with the neighbouring lanes (first, last, spill) are OR-ed atomically
            const int sh = excl & 31;
            const int base = cword + (excl >> 5);
            const int nsw = (nbits + 31) >> 5;
            if (nsw) {
                // word i of the output = bits of staged words i-1, i shifted by sh
                // (funnel shift: sh = 0 gives the word itself); the first and last
                // (and the spill word) are shared with neighbours
                uint32_t prev = stage[0];
                atomicOr(&ow[base], prev >> sh);
    #pragma unroll 1
                for (int i = 1; i < nsw - 1; i++) {
                    const uint32_t v = stage[i];
                    ow[base + i] = __funnelshift_r(v, prev, sh);
                    prev = v;
                }
                if (nsw > 1) {
                    const uint32_t v = stage[nsw - 1];
                    atomicOr(&ow[base + nsw - 1], __funnelshift_r(v, prev, sh));
                    prev = v;
                }
                const uint32_t o = sh ? prev << (32 - sh) : 0u;
                if (o) atomicOr(&ow[base + nsw], o);
            }
        }
        pair_sync(bar);

        // payload(s) -> bucket c.. (bytes in stream order: big-endian words); with
        // packed chunks the kk buckets are contiguous in HBM as in ow
        const int nbytes = (cbits + 7) >> 3;
        uint4 *dst = reinterpret_cast<uint4 *>(bucket + c * stride) + (TILED ? boff >> 7 : 0);
        const uint4 *o4 = reinterpret_cast<const uint4 *>(ow);
        // TILED: a non-last tile writes its whole 16-byte units and carries the rest
        const int n16 = PACK ? kk * (int)(stride / 16) : (TILED && !last ? total >> 7 : (nbytes + 15) >> 4);
        if (TILED && !last) {
            const uint32_t *cyw = ow + 4 * (total >> 7);
            cy0 = cyw[0], cy1 = cyw[1], cy2 = cyw[2], cy3 = cyw[3];
        }
        for (int i = t64; i < n16; i += kWalkLanes) {
            uint4 v = o4[i];
            v.x = __byte_perm(v.x, 0, 0x0123);
            v.y = __byte_perm(v.y, 0, 0x0123);
            v.z = __byte_perm(v.z, 0, 0x0123);
            v.w = __byte_perm(v.w, 0, 0x0123);
            dst[i] = v;
        }
        if (PACK) {
            const int lpc = (int)g.S / kWSeg;
            if ((t64 & (lpc - 1)) == 0 && t64 / lpc < kk) sizes[c + t64 / lpc] = (uint32_t)nbytes;
        } else if (t64 == 0 && last) {
            sizes[c] = TILED ? (uint32_t)(((boff & ~127) + total + 7) >> 3) : (uint32_t)nbytes;
        }
        if (last) break;
        boff = (boff & ~127) + total;
        tileT1c = B0 + T1;
    }  // tiles
}

template <int MODE, bool SMALLW, bool V2, bool PACK, bool TILED = false>
cudaError_t launch_mode(const uint8_t *in, uint64_t n, Geometry g, uint8_t *bucket,
                        uint32_t *sizes, void *dbg, cudaStream_t st) {
    const uint64_t C = (n + g.S - 1) / g.S;
    if (C == 0) return cudaSuccess;
    const size_t smem = sizeof(WarpSmem) * kChunksPerCta;
    static std::atomic<uint64_t> attr_devs{0};  // per device (the opt-in is per device context)
    cudaError_t e = set_smem_attr_once(chunk_kernel<MODE, SMALLW, V2, PACK, TILED>, (int)smem, attr_devs);
    if (e != cudaSuccess) return e;
    const uint64_t pairs = (C + g.K - 1) / g.K;
    const uint64_t blocks = (pairs + kChunksPerCta - 1) / kChunksPerCta;
    chunk_kernel<MODE, SMALLW, V2, PACK, TILED><<<(unsigned)blocks, kChunksPerCta * kWalkLanes, smem, st>>>(in, n, g, bucket,
                                                                                            sizes, dbg);
    count_launch();
    return cudaGetLastError();
}

template <int MODE>
cudaError_t launch_w(const uint8_t *in, uint64_t n, Geometry g, uint8_t *bucket, uint32_t *sizes,
                     void *dbg, cudaStream_t st) {
    const bool pack = g.K > 1;
    if (g.S > (uint32_t)kChunkMax)  // large chunks (version 0 only): compressed in tiles
        return g.W <= 128 ? launch_mode<MODE, true, false, false, true>(in, n, g, bucket, sizes, dbg, st)
                          : launch_mode<MODE, false, false, false, true>(in, n, g, bucket, sizes, dbg, st);
    if (g.V == 2)
        return pack ? launch_mode<MODE, false, true, true>(in, n, g, bucket, sizes, dbg, st)
                    : launch_mode<MODE, false, true, false>(in, n, g, bucket, sizes, dbg, st);
    if (g.W <= 128)
        return pack ? launch_mode<MODE, true, false, true>(in, n, g, bucket, sizes, dbg, st)
                    : launch_mode<MODE, true, false, false>(in, n, g, bucket, sizes, dbg, st);
    return pack ? launch_mode<MODE, false, false, true>(in, n, g, bucket, sizes, dbg, st)
                : launch_mode<MODE, false, false, false>(in, n, g, bucket, sizes, dbg, st);
}

}  // namespace

cudaError_t launch_chunk_kernel(int mode, const uint8_t *in, uint64_t n, Geometry g,
                                uint8_t *bucket, uint32_t *sizes, void *dbg, cudaStream_t st) {
    switch (mode) {
        case kModeCompress: return launch_w<kModeCompress>(in, n, g, bucket, sizes, dbg, st);
        case kModeDumpMatch: return launch_w<kModeDumpMatch>(in, n, g, bucket, sizes, dbg, st);
        default: return launch_w<kModeDumpTokens>(in, n, g, bucket, sizes, dbg, st);
    }
}

}  // namespace culzss
