/*
 * culzss_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct single-threaded CPU implementation of the
 * chunked LZSS method of Ozsoy & Swany, "CULZSS: LZSS Lossless Data
 * Compression on CUDA" (IEEE CLUSTER 2011), written from the paper text
 * (/root/reference/PAPER.md, one physical line; citations are
 * PAPER.md:1@<byte offset> §<section>) and the readings R1..R18 fixed in
 * SURVEY.md §8(c) / DESIGN.md §3.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares NO code, header,
 * table or constant with the CUDA path (paper_conf_cluster_ozsoys11_b200/csrc);
 * neither side includes or links the other.
 *
 * Every function is the definition written out: no hashing, no blocking, no
 * vectorisation.  The match search is the literal double loop of the
 * paper's LZSS description (PAPER.md:1@5188 §II.A.1: "For every character
 * in the uncoded buffer, the searching process looks for the longest
 * substring in the search buffer that matches the lookahead buffer").
 *
 * Parity status per function:
 *   oracle_match_at          pinned: brute force (tests/test_oracle_bruteforce.py),
 *                            Figure 1 (tests/golden/figure1.txt), window/cap edges
 *   oracle_compress_chunk    pinned: Figure 1 token sequence, hand-worked bit
 *                            vectors, closed-form payload sizes, all-literal bound
 *   oracle_compress          pinned: header layout, closed-form stream length
 *   oracle_decompress        pinned: round trip + hand-built corrupt streams
 */
#include <stdint.h>
#include <stddef.h>
#include <string.h>

/* status codes: same numeric values the public C-ABI documents
 * (include/culzss.h); restated here, not included, to keep the two
 * sides independent. */
#define OR_OK 0
#define OR_ERR_INVALID_ARG 1
#define OR_ERR_BUFFER_TOO_SMALL 3
#define OR_ERR_CORRUPT 4

#define OR_HEADER_BYTES 32u

/* ------------------------------------------------------------------ */
/* Parameters.  R1 W=128 (PAPER.md:1@22955 §III.D "window buffer size of
 * 128 bytes"), R2 F=128 (lookahead not stated; reading), R3 S=4096
 * (PAPER.md:1@20422 "4KB block size"), R4 MIN=3 (PAPER.md:1@5848 "in our
 * case it is three").  The 16-bit match code (PAPER.md:1@23195: "8 bits for
 * the match offset and 8 bits for the match length") bounds W<=256 (d-1 in
 * 8 bits, R9) and F<=MIN+255 (L-MIN in 8 bits, R10). */
int oracle_params_valid(uint32_t S, uint32_t W, uint32_t F, uint32_t MIN)
{
    if (MIN != 3) return 0;
    if (S < 1) return 0;
    if (W < 1 || W > 256) return 0;
    if (F < MIN || F > MIN + 255) return 0;
    return 1;
}

/* ------------------------------------------------------------------ */
/* Longest match at position p of a chunk of length m (SURVEY §8(a) a2,
 * §8(c)).  R5: the window never reaches before the chunk start (d <= p) and
 * the lookahead never passes the chunk end (cap = min(F, m-p)).  R6: the
 * source may run into the lookahead (overlap allowed).  R7: ascending d with
 * strict '>' keeps the smallest d on ties.  Results with L < MIN are
 * reported as (0,0): no match. */
void oracle_match_at(const uint8_t *chunk, size_t m, size_t p,
                     uint32_t W, uint32_t F, uint32_t MIN,
                     uint32_t *outL, uint32_t *outD)
{
    size_t cap = m - p;
    if (cap > F) cap = F;
    size_t bestL = 0, bestD = 0;
    size_t dmax = p < W ? p : W;
    for (size_t d = 1; d <= dmax; d++) {
        size_t L = 0;
        while (L < cap && chunk[p - d + L] == chunk[p + L]) L++;
        if (L > bestL) { bestL = L; bestD = d; }
        if (bestL == cap) break;
    }
    if (bestL < MIN) { bestL = 0; bestD = 0; }
    *outL = (uint32_t)bestL;
    *outD = (uint32_t)bestD;
}

/* All positions of one chunk (used only for the per-position K1 parity). */
void oracle_match_all(const uint8_t *chunk, size_t m, uint32_t W, uint32_t F,
                      uint32_t MIN, uint16_t *L, uint16_t *D)
{
    for (size_t p = 0; p < m; p++) {
        uint32_t l, d;
        oracle_match_at(chunk, m, p, W, F, MIN, &l, &d);
        L[p] = (uint16_t)l;
        D[p] = (uint16_t)d;
    }
}

/* ------------------------------------------------------------------ */
/* Greedy parse (R8; PAPER.md:1@15206 "the uncoded head pointer will jump
 * over them").  Token i is written as tok[i] = (flag<<31)|(a<<16)|b with
 * flag 0: literal, b = the byte; flag 1: match, a = D, b = L.
 * Returns the number of tokens. */
size_t oracle_tokens_chunk(const uint8_t *chunk, size_t m, uint32_t W,
                           uint32_t F, uint32_t MIN, uint32_t *tok)
{
    size_t p = 0, nt = 0;
    while (p < m) {
        uint32_t L, D;
        oracle_match_at(chunk, m, p, W, F, MIN, &L, &D);
        if (L >= MIN) {
            tok[nt++] = 0x80000000u | (D << 16) | L;
            p += L;
        } else {
            tok[nt++] = chunk[p];
            p += 1;
        }
    }
    return nt;
}

/* ------------------------------------------------------------------ */
/* Bit writer, MSB first (R11). */
typedef struct { uint8_t *buf; size_t bitpos; } bitw;

static void bw_put(bitw *w, uint32_t value, unsigned nbits)
{
    for (unsigned i = 0; i < nbits; i++) {
        unsigned bit = (value >> (nbits - 1 - i)) & 1u;
        size_t byte = w->bitpos >> 3;
        unsigned off = (unsigned)(w->bitpos & 7);
        if (off == 0) w->buf[byte] = 0;
        if (bit) w->buf[byte] |= (uint8_t)(0x80u >> off);
        w->bitpos++;
    }
}

/* One chunk -> its payload (SURVEY §8(c) pseudo-code, PAPER.md:1@4785 flags,
 * PAPER.md:1@23049 16-bit match code).  Literal: flag 0 + 8-bit byte.
 * Match: flag 1 + 8-bit (D-1) + 8-bit (L-MIN).  Zero padded to a byte.
 * out must hold ceil(9*m/8) bytes.  Returns the payload size in bytes. */
size_t oracle_compress_chunk(const uint8_t *chunk, size_t m, uint32_t W,
                             uint32_t F, uint32_t MIN, uint8_t *out)
{
    bitw w = { out, 0 };
    size_t p = 0;
    while (p < m) {
        uint32_t L, D;
        oracle_match_at(chunk, m, p, W, F, MIN, &L, &D);
        if (L >= MIN) {
            bw_put(&w, 1, 1);
            bw_put(&w, D - 1, 8);
            bw_put(&w, L - MIN, 8);
            p += L;
        } else {
            bw_put(&w, 0, 1);
            bw_put(&w, chunk[p], 8);
            p += 1;
        }
    }
    return (w.bitpos + 7) >> 3;
}

/* ------------------------------------------------------------------ */
/* Stream container (R12): 32-byte little-endian header, u32 size table
 * (the paper's "list of block compression sizes", PAPER.md:1@18853 §III.C),
 * then the payloads in chunk order. */
static void put_le(uint8_t *dst, uint64_t v, int nbytes)
{
    for (int i = 0; i < nbytes; i++) dst[i] = (uint8_t)(v >> (8 * i));
}

static uint64_t get_le(const uint8_t *src, int nbytes)
{
    uint64_t v = 0;
    for (int i = 0; i < nbytes; i++) v |= (uint64_t)src[i] << (8 * i);
    return v;
}

static uint64_t n_chunks(uint64_t n, uint32_t S) { return (n + S - 1) / S; }

/* Upper bound of the stream length: header + table + sum ceil(9 m_c / 8). */
uint64_t oracle_max_compressed_size(uint64_t n, uint32_t S)
{
    uint64_t C = n_chunks(n, S);
    uint64_t full = n / S, tail = n % S;
    uint64_t bound = OR_HEADER_BYTES + 4 * C + full * ((9ull * S + 7) / 8);
    if (tail) bound += (9 * tail + 7) / 8;
    return bound;
}

void oracle_write_header(uint8_t *out, uint64_t n, uint32_t S, uint32_t W,
                         uint32_t F, uint32_t MIN)
{
    memset(out, 0, OR_HEADER_BYTES);
    out[0] = 'C'; out[1] = 'L'; out[2] = 'Z'; out[3] = 'S';
    put_le(out + 4, 1, 2);                    /* format version */
    put_le(out + 6, OR_HEADER_BYTES, 2);
    put_le(out + 8, S, 4);
    put_le(out + 12, n_chunks(n, S), 4);
    put_le(out + 16, n, 8);
    put_le(out + 24, W, 2);
    put_le(out + 26, F, 2);
    out[28] = (uint8_t)MIN;
}

/* Whole stream.  *out_n: in = capacity of out, out = bytes written (or the
 * required bound on OR_ERR_BUFFER_TOO_SMALL). */
int oracle_compress(const uint8_t *in, uint64_t n, uint8_t *out,
                    uint64_t *out_n, uint32_t S, uint32_t W, uint32_t F,
                    uint32_t MIN)
{
    if (!oracle_params_valid(S, W, F, MIN)) return OR_ERR_INVALID_ARG;
    uint64_t C = n_chunks(n, S);
    if (C > 0xFFFFFFFFull) return OR_ERR_INVALID_ARG;
    uint64_t bound = oracle_max_compressed_size(n, S);
    if (*out_n < bound) { *out_n = bound; return OR_ERR_BUFFER_TOO_SMALL; }
    oracle_write_header(out, n, S, W, F, MIN);
    uint64_t pos = OR_HEADER_BYTES + 4 * C;
    for (uint64_t c = 0; c < C; c++) {
        uint64_t start = c * S;
        uint64_t m = n - start < S ? n - start : S;
        size_t sz = oracle_compress_chunk(in + start, (size_t)m, W, F, MIN, out + pos);
        put_le(out + OR_HEADER_BYTES + 4 * c, sz, 4);
        pos += sz;
    }
    *out_n = pos;
    return OR_OK;
}

/* Compress chunks [c0, c1) of an input of total length n into payload only
 * (no header, no table): sizes[c - c0] receives each payload size.  This is
 * the per-rank unit of the sharded stream and the unit of the
 * all-core timing fan-out (PAPER.md:1@11659, the Pthread decomposition). */
int oracle_compress_range(const uint8_t *in, uint64_t n, uint64_t c0,
                          uint64_t c1, uint8_t *payload, uint64_t *payload_n,
                          uint32_t *sizes, uint32_t S, uint32_t W, uint32_t F,
                          uint32_t MIN)
{
    if (!oracle_params_valid(S, W, F, MIN)) return OR_ERR_INVALID_ARG;
    uint64_t pos = 0;
    for (uint64_t c = c0; c < c1; c++) {
        uint64_t start = c * S;
        if (start >= n) return OR_ERR_INVALID_ARG;
        uint64_t m = n - start < S ? n - start : S;
        size_t sz = oracle_compress_chunk(in + start, (size_t)m, W, F, MIN, payload + pos);
        sizes[c - c0] = (uint32_t)sz;
        pos += sz;
    }
    *payload_n = pos;
    return OR_OK;
}

/* ------------------------------------------------------------------ */
/* Decoder (PAPER.md:1@6743 §II.A.2: "The encoding flags are read ... If a
 * flag indicates encoded, the number of the characters and the starting
 * position is gathered ... If it is not encoded, the character is output
 * directly"; per-chunk independence via the size list, PAPER.md:1@18853). */
typedef struct { const uint8_t *buf; uint64_t nbits; uint64_t pos; } bitr;

static int br_get(bitr *r, unsigned nbits, uint32_t *v)
{
    uint32_t x = 0;
    for (unsigned i = 0; i < nbits; i++) {
        if (r->pos >= r->nbits) return 0;
        unsigned bit = (r->buf[r->pos >> 3] >> (7 - (r->pos & 7))) & 1u;
        x = (x << 1) | bit;
        r->pos++;
    }
    *v = x;
    return 1;
}

int oracle_decompressed_size(const uint8_t *in, uint64_t in_n, uint64_t *n)
{
    if (in_n < OR_HEADER_BYTES) return OR_ERR_CORRUPT;
    if (in[0] != 'C' || in[1] != 'L' || in[2] != 'Z' || in[3] != 'S') return OR_ERR_CORRUPT;
    *n = get_le(in + 16, 8);
    return OR_OK;
}

int oracle_decompress(const uint8_t *in, uint64_t in_n, uint8_t *out,
                      uint64_t *out_n)
{
    if (in_n < OR_HEADER_BYTES) return OR_ERR_CORRUPT;
    if (in[0] != 'C' || in[1] != 'L' || in[2] != 'Z' || in[3] != 'S') return OR_ERR_CORRUPT;
    if (get_le(in + 4, 2) != 1 || get_le(in + 6, 2) != OR_HEADER_BYTES) return OR_ERR_CORRUPT;
    uint32_t S = (uint32_t)get_le(in + 8, 4);
    uint64_t C = get_le(in + 12, 4);
    uint64_t n = get_le(in + 16, 8);
    uint32_t W = (uint32_t)get_le(in + 24, 2);
    uint32_t F = (uint32_t)get_le(in + 26, 2);
    uint32_t MIN = in[28];
    if (in[29] || in[30] || in[31]) return OR_ERR_CORRUPT;
    if (!oracle_params_valid(S, W, F, MIN)) return OR_ERR_CORRUPT;
    if (C != n_chunks(n, S)) return OR_ERR_CORRUPT;
    if (in_n < OR_HEADER_BYTES + 4 * C) return OR_ERR_CORRUPT;
    uint64_t total = 0;
    for (uint64_t c = 0; c < C; c++) total += get_le(in + OR_HEADER_BYTES + 4 * c, 4);
    if (OR_HEADER_BYTES + 4 * C + total != in_n) return OR_ERR_CORRUPT;
    if (*out_n < n) { *out_n = n; return OR_ERR_BUFFER_TOO_SMALL; }

    uint64_t pos = OR_HEADER_BYTES + 4 * C;
    for (uint64_t c = 0; c < C; c++) {
        uint64_t size_c = get_le(in + OR_HEADER_BYTES + 4 * c, 4);
        uint64_t start = c * S;
        uint64_t m = n - start < S ? n - start : S;
        bitr r = { in + pos, size_c * 8, 0 };
        uint8_t *dst = out + start;
        uint64_t produced = 0;
        while (produced < m) {
            uint32_t flag, a, b;
            if (!br_get(&r, 1, &flag)) return OR_ERR_CORRUPT;
            if (flag == 0) {
                if (!br_get(&r, 8, &a)) return OR_ERR_CORRUPT;
                dst[produced++] = (uint8_t)a;
            } else {
                if (!br_get(&r, 8, &a) || !br_get(&r, 8, &b)) return OR_ERR_CORRUPT;
                uint64_t d = (uint64_t)a + 1, L = (uint64_t)b + MIN;
                if (d > W || d > produced || L > F || L > m - produced) return OR_ERR_CORRUPT;
                for (uint64_t k = 0; k < L; k++) {       /* forward, overlap-safe */
                    dst[produced] = dst[produced - d];
                    produced++;
                }
            }
        }
        /* consumed bits must round up to exactly size_c with zero padding */
        if ((r.pos + 7) / 8 != size_c) return OR_ERR_CORRUPT;
        while (r.pos < r.nbits) {
            uint32_t bit;
            br_get(&r, 1, &bit);
            if (bit) return OR_ERR_CORRUPT;
        }
        pos += size_c;
    }
    *out_n = n;
    return OR_OK;
}
