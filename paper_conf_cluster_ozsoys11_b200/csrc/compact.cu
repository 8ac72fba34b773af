// compact.cu -- SURVEY §8(a) row a5: device exclusive scan of the per-chunk
// compressed sizes and compaction of the payloads into one stream.
//
// The paper leaves this serial on the CPU: "there is a final separate process
// to concatenate only the compressed data into a continuous stream of data by
// getting rid of the empty parts of the bucket" (PAPER.md:1@17241 §III.B.3),
// and names porting it to the GPU as future work (PAPER.md:1@37261-37485
// §VII).  Here it is two kernels:
//   scan_kernel     single-pass decoupled look-back exclusive scan over the
//                   u32 sizes (tiles of 2048 sizes per 256-thread CTA; CTA
//                   order from an atomic ticket so the look-back never waits
//                   on an unscheduled CTA); writes u64 offsets and the total.
//   compact_kernel  one warp per chunk copies its payload from the bucket to
//                   32 + 4C + offset[c] and its size into the table.
// The header is written by header_kernel (one thread).

#include "culzss_internal.h"

namespace culzss {
namespace {

constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr int kTile = kScanThreads * kScanItems;
constexpr uint64_t kFlagAgg = 1ull << 62;
constexpr uint64_t kFlagPre = 2ull << 62;
constexpr uint64_t kValMask = (1ull << 62) - 1;

__device__ __forceinline__ uint64_t ld_acquire(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(uint64_t *p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// status_ws layout: [0] ticket counter, [1 .. ntiles] tile status (zeroed).
__global__ void __launch_bounds__(kScanThreads)
scan_kernel(const uint32_t *__restrict__ sizes, uint64_t C, uint64_t *__restrict__ offsets,
            uint64_t *__restrict__ total, uint64_t *__restrict__ ws) {
    __shared__ uint64_t warp_sums[kScanThreads / 32];
    __shared__ uint64_t tile_prefix;
    __shared__ uint32_t tile_id;
    // programmatic dependent launch: the grid may start while its predecessor
    // (the chunk kernel) drains; wait for its results, and let the compaction
    // grid get scheduled behind this one
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;");
    if (threadIdx.x == 0) tile_id = (uint32_t)atomicAdd(reinterpret_cast<unsigned long long *>(ws), 1ull);
    __syncthreads();
    const uint64_t tile = tile_id;
    uint64_t *status = ws + 1;
    const uint64_t base = tile * kTile + (uint64_t)threadIdx.x * kScanItems;

    uint64_t v[kScanItems];
    uint64_t local = 0;
#pragma unroll
    for (int i = 0; i < kScanItems; i++) {
        v[i] = base + i < C ? sizes[base + i] : 0;
        local += v[i];
    }
    // block exclusive scan of per-thread sums
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint64_t incl = local;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint64_t y = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) warp_sums[wid] = incl;
    __syncthreads();
    uint64_t wpre = 0, agg = 0;
#pragma unroll
    for (int w = 0; w < kScanThreads / 32; w++) {
        if (w < wid) wpre += warp_sums[w];
        agg += warp_sums[w];
    }
    // decoupled look-back (one thread)
    if (threadIdx.x == 0) {
        if (tile == 0) {
            st_release(&status[0], kFlagPre | agg);
            tile_prefix = 0;
        } else {
            st_release(&status[tile], kFlagAgg | agg);
            uint64_t pre = 0;
            int64_t t = (int64_t)tile - 1;
            while (t >= 0) {
                uint64_t s = ld_acquire(&status[t]);
                if (s & kFlagPre) {
                    pre += s & kValMask;
                    break;
                }
                if (s & kFlagAgg) {
                    pre += s & kValMask;
                    t--;
                }
            }
            st_release(&status[tile], kFlagPre | (pre + agg));
            tile_prefix = pre;
        }
    }
    __syncthreads();
    uint64_t run = tile_prefix + wpre + incl - local;
#pragma unroll
    for (int i = 0; i < kScanItems; i++) {
        if (base + i < C) offsets[base + i] = run;
        run += v[i];
    }
    const uint64_t ntiles = (C + kTile - 1) / kTile;
    if (tile == ntiles - 1 && threadIdx.x == 0) *total = tile_prefix + agg;
}

// One warp per chunk: payload bytes bucket -> out_payload + offsets[c];
// sizes[c] -> out_table[c].  Destination is byte aligned: interior words are
// written as aligned u32 (assembled with funnel shifts), the two edge words
// byte by byte (they are shared with the neighbouring chunks).
__global__ void __launch_bounds__(256)
compact_kernel(const uint8_t *__restrict__ bucket, uint64_t stride,
               const uint32_t *__restrict__ sizes, const uint64_t *__restrict__ offsets,
               uint64_t C, uint8_t *__restrict__ out_payload, uint32_t *__restrict__ out_table) {
    asm volatile("griddepcontrol.wait;" ::: "memory");  // programmatic dependent launch (after the scan)
    const int lane = threadIdx.x & 31;
    const uint64_t c = (uint64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
    if (c >= C) return;
    const uint32_t len = sizes[c];
    if (lane == 0 && out_table) {
        // the table itself is 4-byte aligned in the stream only if out is; use bytes
        uint8_t *t = reinterpret_cast<uint8_t *>(out_table) + 4 * c;
        t[0] = (uint8_t)len; t[1] = (uint8_t)(len >> 8); t[2] = (uint8_t)(len >> 16); t[3] = (uint8_t)(len >> 24);
    }
    const uint8_t *src = bucket + c * stride;        // 16-byte aligned; +16 B slack at the end
    uint8_t *dst = out_payload + offsets[c];
    const uintptr_t d0 = reinterpret_cast<uintptr_t>(dst);
    const uintptr_t d1 = d0 + len;
    const uintptr_t a0 = (d0 + 3) & ~(uintptr_t)3;   // first aligned word start
    const uintptr_t a1 = d1 & ~(uintptr_t)3;         // end of aligned words
    if (a0 >= a1) {
        for (uint32_t i = lane; i < len; i += 32) dst[i] = src[i];
        return;
    }
    const uint32_t head = (uint32_t)(a0 - d0), tail_start = (uint32_t)(a1 - d0);
    if (lane < head) dst[lane] = src[lane];
    for (uint32_t i = tail_start + lane; i < len; i += 32) dst[i] = src[i];
    const uint32_t *s4 = reinterpret_cast<const uint32_t *>(src);
    uint32_t *o4 = reinterpret_cast<uint32_t *>(a0);
    const uint32_t nw = (uint32_t)((a1 - a0) >> 2);
    for (uint32_t j = lane; j < nw; j += 32) {
        const uint32_t s = head + 4 * j;            // source byte offset of this word
        const uint32_t lo = s4[s >> 2], hi = (s & 3) ? s4[(s >> 2) + 1] : 0u;  // hi only when it is used
        o4[j] = __funnelshift_r(lo, hi, (s & 3) * 8);
    }
}

__global__ void header_kernel(uint8_t *out, uint64_t n, Geometry g) {
    const uint64_t C = (n + g.S - 1) / g.S;
    uint8_t h[32] = {'C', 'L', 'Z', 'S', 1, 0, 32, 0};
    for (int i = 0; i < 4; i++) h[8 + i] = (uint8_t)(g.S >> (8 * i));
    for (int i = 0; i < 4; i++) h[12 + i] = (uint8_t)(C >> (8 * i));
    for (int i = 0; i < 8; i++) h[16 + i] = (uint8_t)(n >> (8 * i));
    h[24] = (uint8_t)g.W; h[25] = (uint8_t)(g.W >> 8);
    h[26] = (uint8_t)g.F; h[27] = (uint8_t)(g.F >> 8);
    h[28] = 3;
    for (int i = 0; i < 32; i++) out[i] = h[i];
}

}  // namespace

uint64_t scan_workspace_words(uint64_t C) { return 1 + (C + kTile - 1) / kTile; }

// Kernel launch with programmatic stream serialization (PDL): the grid may be
// scheduled before its stream predecessor kernel finishes; the kernel's
// griddepcontrol.wait orders its reads after that kernel's writes.
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*k)(KArgs...), unsigned grid, unsigned block, cudaStream_t st, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(block);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}

cudaError_t launch_scan(const uint32_t *sizes, uint64_t C, uint64_t *offsets, uint64_t *total,
                        uint64_t *ws, cudaStream_t st, bool zero_ws) {
    if (zero_ws) {
        cudaError_t e = cudaMemsetAsync(ws, 0, scan_workspace_words(C) * sizeof(uint64_t), st);
        if (e != cudaSuccess) return e;
    }
    if (C == 0) return cudaMemsetAsync(total, 0, sizeof(uint64_t), st);
    const uint64_t ntiles = (C + kTile - 1) / kTile;
    cudaError_t e = launch_pdl(scan_kernel, (unsigned)ntiles, kScanThreads, st, sizes, C, offsets, total, ws);
    count_launch();
    return e;
}

cudaError_t launch_compact(const uint8_t *bucket, uint64_t stride, const uint32_t *sizes,
                           const uint64_t *offsets, uint64_t C, uint8_t *out_payload,
                           uint32_t *out_table, cudaStream_t st) {
    if (C == 0) return cudaSuccess;
    cudaError_t e = launch_pdl(compact_kernel, (unsigned)((C + 7) / 8), 256, st, bucket, stride, sizes, offsets, C,
                               out_payload, out_table);
    count_launch();
    return e;
}

cudaError_t launch_header(uint8_t *out, uint64_t n, Geometry g, cudaStream_t st) {
    header_kernel<<<1, 1, 0, st>>>(out, n, g);
    count_launch();
    return cudaGetLastError();
}

}  // namespace culzss
