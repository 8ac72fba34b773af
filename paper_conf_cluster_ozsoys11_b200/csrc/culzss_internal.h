// Internal declarations shared by the CUDA translation units of libculzss.
// Not part of the ABI (the ABI is include/culzss.h).  Shares nothing with
// oracle/ (independence rule).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace culzss {

// Geometry of the fused chunk kernel.
constexpr int kChunkMax = 4096;     // largest chunk the kernel stages (S <= 4096)
constexpr int kSeg = 128;           // positions per lane in the parse (32 x 128 = 4096)
constexpr int kHashBits = 10;       // 3-gram hash table: 1024 heads per chunk
constexpr int kWarpsPerCta = 4;     // one warp per chunk
constexpr int kCtasPerSm = 3;

struct Geometry {
    uint32_t S, W, F;               // chunk, window, max match (MIN is 3)
};

// Per-warp shared memory.  The output words alias link/head, which are dead
// once the parse finishes.
struct __align__(16) WarpSmem {
    uint32_t cw[(kChunkMax + 16) / 4];                 // chunk bytes + zero pad
    uint16_t ld[kChunkMax];                            // token at parse positions
    union {
        struct {
            uint8_t link[kChunkMax];                   // distance to previous same-hash position
            uint16_t head[1 << kHashBits];             // latest position per hash
        } s;
        uint32_t ow[(kChunkMax + 2 * (1 << kHashBits)) / 4];   // packed payload words
    } u;
};
static_assert(sizeof(WarpSmem) == 18448, "smem layout");
static_assert((kChunkMax * 9 + 7) / 8 + 8 <= sizeof(WarpSmem::u), "payload fits alias");

__host__ __device__ inline uint64_t bucket_stride(uint32_t S) { return (((uint64_t)S * 9 + 7) / 8 + 15) / 16 * 16; }

enum ChunkMode { kModeCompress = 0, kModeDumpMatch = 1, kModeDumpTokens = 2 };

// Launchers (return cudaError_t of the launch).
cudaError_t launch_chunk_kernel(int mode, const uint8_t *in, uint64_t n, Geometry g,
                                uint8_t *bucket, uint32_t *sizes, void *dbg,
                                cudaStream_t st);
cudaError_t launch_scan(const uint32_t *sizes, uint64_t C, uint64_t *offsets,
                        uint64_t *total, uint64_t *status_ws, cudaStream_t st);
uint64_t scan_workspace_words(uint64_t C);
cudaError_t launch_compact(const uint8_t *bucket, uint64_t stride, const uint32_t *sizes,
                           const uint64_t *offsets, uint64_t C, uint8_t *out_payload,
                           uint32_t *out_table, cudaStream_t st);
cudaError_t launch_header(uint8_t *out, uint64_t n, Geometry g, cudaStream_t st);
cudaError_t launch_decode(const uint8_t *payload, const uint32_t *sizes,
                          const uint64_t *offsets, uint64_t C, uint64_t n, Geometry g,
                          uint8_t *out, uint32_t *err, cudaStream_t st);

void count_launch(int k = 1);

}  // namespace culzss
