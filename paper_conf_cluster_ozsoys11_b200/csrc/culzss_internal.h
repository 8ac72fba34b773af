// Internal declarations shared by the CUDA translation units of libculzss.
// Not part of the ABI (the ABI is include/culzss.h).  Shares nothing with
// oracle/ (independence rule).
#pragma once
#include <atomic>
#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>

namespace culzss {

// Geometry of the fused chunk kernel.
constexpr int kChunkMax = 4096;     // the kernel's buffer: chunks of S <= 4096 in one piece
constexpr int kChunkTiledMax = 1 << 16;  // S in (4096, 65536]: compressed in 4096-position tiles
constexpr int kSeg = 128;           // positions per lane segment (32 x 128 = 4096)
constexpr int kHashBits = 8;        // per-lane 3-gram hash table, W > 128: 256 u16 heads
constexpr int kHashBitsSmallW = 9;  // W <= 128: 512 u8 heads (relative positions)
constexpr int kChunksPerCta = 1;    // chunks per CTA (each chunk's smem is released when it finishes)
constexpr int kWarpsPerChunk = 2;   // warp 0 builds the hash chains; all warps walk
constexpr int kWalkLanes = 32 * kWarpsPerChunk;   // 64 walk segments per chunk
constexpr int kWSeg = kChunkMax / kWalkLanes;     // 64 positions per walk segment
constexpr int kCtasPerSm = 9;

struct Geometry {
    uint32_t S, W, F;               // chunk, window, max match (MIN is 3)
    uint32_t V = 0;                 // kernel version: 0 = lazy hash-chain search,
                                    // 2 = the paper's V2 all-position search
    uint32_t K = 1;                 // chunks per warp pair: 4096 / S for S in {64, 128, ..., 2048},
                                    // else 1 (small chunks packed into one 4096-position buffer)
    uint32_t smask = 4095;          // S - 1 when K > 1: position p's chunk is [p & ~smask, +S)
    uint32_t tx = 16;               // iterations one lane may spend on one token before its warp
                                    // switches to the pruned walk machine (B200 sweep:
                                    // profiles/r2_walk_switch.md), ...
    uint32_t sw = 1u << 30;         // ... or walk iterations of the warp in total (off by default).
                                    // CULZSS_WALK_TOKEN_SWITCH / CULZSS_WALK_SWITCH override both, for
                                    // tuning and for the tests that cover each machine on its own
};
// Chunk packing for the fused kernel: chunks of S = 64 .. 2048
// (powers of two) share one warp pair, K = 4096 / S of them, so every 64-position
// walk segment lies inside one chunk.
inline void set_packing(Geometry *g) {
    const uint32_t S = g->S;
    const bool pack = S >= 64 && S <= 2048 && (S & (S - 1)) == 0;
    g->K = pack ? 4096 / S : 1;
    g->smask = pack ? S - 1 : 4095;
}

// Per-chunk (warp pair) shared memory.  Per-position arrays use a SKEWED layout: 4 pad
// bytes after every 128-position segment, so that the 32 lanes (one segment
// each) scanning the same relative offset hit 32 different banks.  The pad
// word of a segment duplicates the first word of the next one, so an
// unaligned 4-byte load is two aligned word loads anywhere in the chunk.
// During the chain build `tab` holds the per-lane hash heads; afterwards the
// same bytes hold the memoised tokens (`ld`) and an unskewed copy of the
// chunk for the walks.  After the walks link (+ pad) becomes per-lane bit
// staging and `ld` the packed payload words.
constexpr int kSkewBytes = kChunkMax + 4 * (kChunkMax / kSeg);   // 4224
// per-walk-lane bit staging: a segment emits at most 9 bits per position (a
// 17-bit match covers >= 3 positions) + one 17-bit token crossing its end
constexpr int kStageWords = ((kWSeg * 9 + 17 + 31) / 32) | 1;   // odd stride: conflict-free
constexpr int kStagePad = (kWalkLanes * kStageWords * 4 > kSkewBytes ? kWalkLanes * kStageWords * 4 - kSkewBytes : 0) + 16;
constexpr int kUcwWords = kChunkMax / 4 + 4;  // + zero tail: 8-byte loads read 3 words
struct __align__(16) WarpSmem {
    uint32_t cw[kSkewBytes / 4];                     // chunk bytes (skewed).  No tail: reads past the
                                                     // chunk end only feed bytes beyond every match's cap
    struct {
        uint8_t link[kSkewBytes];                    // distance to previous same-hash position
        union {
            uint16_t tab[(1 << kHashBits) * 32];     // [hash][lane]: u16 position + 0x1000 (W > 128)
                                                     // or [lane][bucket] u8 position mod 256, 512 buckets (W <= 128)
            struct {
                uint8_t pad[kStagePad];              // staging = link + pad (after the walks)
                uint32_t xfer[8];                    // cross-warp exchange (exits, flags, bit counts)
                uint16_t ld[kChunkMax + 2 * (kChunkMax / kSeg)];  // memoised token (0 = not evaluated)
                uint32_t ucw[kUcwWords];             // unskewed chunk copy for the walks' 8-byte compares
                                                     // (random access: the skew buys nothing there)
            } w;
        } u;
    } a;
};
static_assert(sizeof(WarpSmem) <= 24848, "smem layout");
// a warp's run-boundary mask words (walk machine 2): its 64 + the 8 before
// (run_start reaches back W <= 255) + the 9 after (run_len reaches F <= 258)
constexpr int kBndWarpLo = 8, kBndWarpWords = 64 + kBndWarpLo + 9;
static_assert(kWarpsPerChunk * kBndWarpWords * 4 <= kStagePad, "both warps' run-boundary masks fit in the staging pad");
static_assert(offsetof(WarpSmem, a.u.w.xfer) - offsetof(WarpSmem, a.link) >= kWalkLanes * kStageWords * 4,
              "staging (over link + pad) must not reach xfer / ld");
static_assert((kChunkMax * 9 / 8 + 16) <= sizeof(WarpSmem::a.u.w.ld), "payload words fit in ld");

__host__ __device__ inline uint64_t bucket_stride(uint32_t S) { return (((uint64_t)S * 9 + 7) / 8 + 15) / 16 * 16; }

enum ChunkMode { kModeCompress = 0, kModeDumpMatch = 1, kModeDumpTokens = 2 };

// Launchers (return cudaError_t of the launch).
cudaError_t launch_chunk_kernel(int mode, const uint8_t *in, uint64_t n, Geometry g,
                                uint8_t *bucket, uint32_t *sizes, void *dbg,
                                cudaStream_t st);
cudaError_t launch_scan(const uint32_t *sizes, uint64_t C, uint64_t *offsets,
                        uint64_t *total, uint64_t *status_ws, cudaStream_t st, bool zero_ws = true);
uint64_t scan_workspace_words(uint64_t C);
cudaError_t launch_compact(const uint8_t *bucket, uint64_t stride, const uint32_t *sizes,
                           const uint64_t *offsets, uint64_t C, uint8_t *out_payload,
                           uint32_t *out_table, cudaStream_t st);
cudaError_t launch_header(uint8_t *out, uint64_t n, Geometry g, cudaStream_t st);
cudaError_t launch_decode(const uint8_t *payload, uint64_t pay_len, const uint32_t *sizes,
                          const uint64_t *offsets, uint64_t C, uint64_t n, Geometry g,
                          uint8_t *out, uint32_t *err, uint32_t *tb_scratch, cudaStream_t st);
uint64_t decode_scratch_bytes(uint64_t C);

void count_launch(int k = 1);

// cudaFuncSetAttribute opt-ins (dynamic shared memory above 48 KB) apply to
// the CURRENT device only: done once per (kernel, device), tracked in a
// per-kernel bit mask of device ordinals.
template <typename K>
cudaError_t set_smem_attr_once(K kernel, int bytes, std::atomic<uint64_t> &done) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const uint64_t bit = dev < 64 ? 1ull << dev : 0;
    if (bit && (done.load(std::memory_order_relaxed) & bit)) return cudaSuccess;
    e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess && bit) done.fetch_or(bit, std::memory_order_relaxed);
    return e;
}

}  // namespace culzss

namespace culzss {
// packed small chunks: K buckets of bucket_stride(S) bytes must fit in the ld area (S = 64 is the largest)
static_assert((kChunkMax / 64) * (((64 * 9 + 7) / 8 + 15) / 16 * 16) <= sizeof(WarpSmem::a.u.w.ld), "packed buckets fit in ld");
static_assert((kChunkMax / 128) * (((128 * 9 + 7) / 8 + 15) / 16 * 16) <= sizeof(WarpSmem::a.u.w.ld), "packed buckets fit in ld");
}  // namespace culzss
