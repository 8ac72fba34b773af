// api.cu -- the C ABI of libculzss.so (include/culzss.h) and its host
// orchestration: parameter validation, stream-ordered workspace, the launch
// sequence, the device error word, and the one sync that returns *out_n.
//
// The paper's API (PAPER.md:1@10268-10919 §III): a dynamically loaded
// in-memory library that "gets initialized when loaded, detects GPUs, and
// determines capabilities"; Gpu_compress() "compresses it into the given
// memory region, and returns ... the compressed data and its length".

#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>
#include <algorithm>

#include <nvtx3/nvToolsExt.h>

#include "../../include/culzss.h"
#include "culzss_internal.h"

namespace culzss {

static std::atomic<uint64_t> g_launches{0};
void count_launch(int k) { g_launches.fetch_add((uint64_t)k, std::memory_order_relaxed); }

namespace {

thread_local int t_last_cuda_error = 0;
thread_local int t_profiling = 0;  // 0 off, 1 call + per-kernel events, 2 call events only
struct KernelTimes {
    float chunk = -1, scan = -1, compact = -1, decode = -1, call = -1;
};
thread_local KernelTimes t_times;

int g_device_count = -1;
std::once_flag g_init_once;

void lib_init() {
    std::call_once(g_init_once, [] {
        int n = 0;
        if (cudaGetDeviceCount(&n) != cudaSuccess) {
            n = 0;
            cudaGetLastError();
        }
        g_device_count = n;
        // keep freed workspace in the stream-ordered pool between calls
        for (int d = 0; d < n; d++) {
            cudaMemPool_t pool;
            if (cudaDeviceGetDefaultMemPool(&pool, d) == cudaSuccess) {
                uint64_t thr = UINT64_MAX;
                cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
            }
        }
        cudaGetLastError();
    });
}

// NVTX range around each ABI call (visible in nsys / ncu --nvtx timelines;
// a no-op unless a tool is attached)
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

struct LibLoad {
    LibLoad() { /* device detection is lazy: CUDA may not be usable at dlopen time */ }
} g_libload;

culzss_status cuda_fail(cudaError_t e) {
    t_last_cuda_error = (int)e;
    return CULZSS_ERR_CUDA;
}

#define CK(expr)                                      \
    do {                                              \
        cudaError_t _e = (expr);                      \
        if (_e != cudaSuccess) return cuda_fail(_e);  \
    } while (0)

culzss_status check_params(const culzss_params *p, Geometry *g) {
    culzss_params d;
    culzss_default_params(&d);
    if (!p) p = &d;
    if (p->min_match != 3 || p->chunk_size < 1 || p->window < 1 || p->window > 256 ||
        p->max_match < 3 || p->max_match > 258 || p->reserved != 0)
        return CULZSS_ERR_INVALID_ARG;
    // W = 256 (the paper's "offsets are upto 256", PAPER.md:1@23151 §III.D):
    // version 0 only, and F <= 256 (the walk's 16-bit token memo holds
    // 256 x 254 match codes + literal + not-evaluated)
    // S up to 64 KiB ("the decision on the length of the blocks is a
    // configuration parameter", PAPER.md:1@30360 §V): version 0 compresses
    // chunks above 4 KiB in tiles; version 2 is built for S <= 4096
    if ((p->version != 0 && p->version != 2) || p->chunk_size > (uint32_t)kChunkTiledMax ||
        (p->version == 2 && p->chunk_size > (uint32_t)kChunkMax) ||
        (p->window == 256 && (p->version != 0 || p->max_match > 256)))
        return CULZSS_ERR_UNSUPPORTED;
    g->V = p->version;
    if (const char *e = getenv("CULZSS_WALK_SWITCH")) g->sw = (uint32_t)atol(e);
    if (const char *e = getenv("CULZSS_WALK_TOKEN_SWITCH")) g->tx = (uint32_t)atol(e);
    g->S = p->chunk_size;
    g->W = p->window;
    g->F = p->max_match;
    set_packing(g);
    return CULZSS_OK;
}

uint64_t n_chunks(uint64_t n, uint32_t S) { return (n + S - 1) / S; }

uint64_t payload_bound(uint64_t n, uint32_t S) {
    uint64_t full = n / S, tail = n % S;
    uint64_t b = full * ((9ull * S + 7) / 8);
    if (tail) b += (9 * tail + 7) / 8;
    return b;
}

bool is_device_ptr(const void *ptr) {
    if (!ptr) return false;
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, ptr) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

bool overlap(const void *a, size_t na, const void *b, size_t nb) {
    uintptr_t x = (uintptr_t)a, y = (uintptr_t)b;
    return na && nb && x < y + nb && y < x + na;
}

// Stream-ordered workspace that frees itself on scope exit.
struct Workspace {
    cudaStream_t st;
    void *p = nullptr;
    explicit Workspace(cudaStream_t s) : st(s) {}
    cudaError_t alloc(size_t bytes) { return cudaMallocAsync(&p, bytes ? bytes : 16, st); }
    ~Workspace() {
        if (p) cudaFreeAsync(p, st);
    }
};

// Pinned host word for the 8-byte D2H of a device total (one per thread).
uint64_t *host_word() {
    thread_local uint64_t *w = nullptr;
    if (!w) {
        if (cudaMallocHost(&w, 64) != cudaSuccess) {
            cudaGetLastError();
            w = nullptr;
        }
    }
    return w;
}

// Profiling: events recorded on the call's stream at stage boundaries with
// no intermediate host sync; elapsed times are read after the call's own
// final synchronisation.  Stages: 0 call start, 1 after the fused chunk
// kernel's predecessor (header), 2 after chunk, 3 after scan, 4 after
// compact, 5 call end (after the D2H of the total).
struct Prof {
    static constexpr int kN = 6;
    cudaEvent_t e[kN] = {};
    bool used[kN] = {};
    bool ready = false;
    void rec(int i, cudaStream_t st) {
        if (!t_profiling) return;
        if (t_profiling == 2 && i != 0 && i != kN - 1) return;  // nothing between the call's kernels
        if (!ready) {
            for (auto &x : e) cudaEventCreate(&x);
            ready = true;
        }
        cudaEventRecord(e[i], st);
        used[i] = true;
    }
    float between(int a, int b) {
        float v = -1;
        if (ready && used[a] && used[b] && cudaEventElapsedTime(&v, e[a], e[b]) != cudaSuccess) {
            cudaGetLastError();
            v = -1;
        }
        return v;
    }
    void reset() {
        for (auto &u : used) u = false;
    }
};
// CUDA events and streams belong to the device that was current when they
// were created: the per-thread state is kept per device ordinal.
constexpr int kMaxDevices = 64;
int cur_device() {
    int d = 0;
    if (cudaGetDevice(&d) != cudaSuccess) {
        cudaGetLastError();
        d = 0;
    }
    return d >= 0 && d < kMaxDevices ? d : 0;
}
thread_local Prof t_prof_dev[kMaxDevices];
#define t_prof (t_prof_dev[cur_device()])

void prof_finish_compress() {
    if (!t_profiling) return;
    t_times.chunk = t_prof.between(1, 2);
    t_times.scan = t_prof.between(2, 3);
    t_times.compact = t_prof.between(3, 4);
    t_times.call = t_prof.between(0, 5);
}

// Workspace of compress_core for C chunks: bucket | sizes | offsets | scan ws
struct CoreLayout {
    uint64_t sizes_off, offs_off, ws_off, total;
    CoreLayout(uint64_t C, uint32_t S) {
        const uint64_t bucket_bytes = C * bucket_stride(S) + 16;
        sizes_off = (bucket_bytes + 255) / 256 * 256;
        offs_off = sizes_off + (C * 4 + 255) / 256 * 256;
        ws_off = offs_off + (C * 8 + 255) / 256 * 256;
        total = ws_off + scan_workspace_words(C) * 8;
    }
};

// Core compression of n bytes at device `in` into: payload region `pay`
// (capacity checked by callers), table `table` (may be null), total payload
// bytes -> device word `dev_total`.  Sizes go to `sizes` (device, C words).
// `wsp`: a CoreLayout-sized device workspace, or null to allocate one on st.
culzss_status compress_core(const uint8_t *in, uint64_t n, const Geometry &g, uint8_t *pay,
                            uint32_t *table, uint32_t *sizes_out, uint64_t *dev_total,
                            cudaStream_t st, void *wsp = nullptr, bool prof = true) {
    const uint64_t C = n_chunks(n, g.S);
    const uint64_t stride = bucket_stride(g.S);
    const CoreLayout lay(C, g.S);
    const uint64_t sizes_off = lay.sizes_off, offs_off = lay.offs_off, ws_off = lay.ws_off;
    Workspace ws(st);
    if (!wsp) {
        CK(ws.alloc(lay.total));
        wsp = ws.p;
    }
    uint8_t *base = static_cast<uint8_t *>(wsp);
    uint8_t *bucket = base;
    uint32_t *sizes = sizes_out ? sizes_out : reinterpret_cast<uint32_t *>(base + sizes_off);
    uint64_t *offsets = reinterpret_cast<uint64_t *>(base + offs_off);
    uint64_t *scanws = reinterpret_cast<uint64_t *>(base + ws_off);

    // the scan's look-back status words are cleared before the chunk kernel,
    // so nothing but kernels sits between the chunk kernel and the scan
    CK(cudaMemsetAsync(scanws, 0, scan_workspace_words(C) * sizeof(uint64_t), st));
    if (prof) t_prof.rec(1, st);
    CK(launch_chunk_kernel(kModeCompress, in, n, g, bucket, sizes, nullptr, st));
    if (prof) t_prof.rec(2, st);
    CK(launch_scan(sizes, C, offsets, dev_total, scanws, st, false));
    if (prof) t_prof.rec(3, st);
    CK(launch_compact(bucket, stride, sizes, offsets, C, pay, table, st));
    if (prof) t_prof.rec(4, st);
    return CULZSS_OK;
}

}  // namespace
}  // namespace culzss

using namespace culzss;

extern "C" {

void culzss_default_params(culzss_params *p) {
    if (!p) return;
    p->chunk_size = 4096;
    p->window = 128;
    p->max_match = 128;
    p->min_match = 3;
    p->version = 0;
    p->reserved = 0;
}

size_t culzss_max_compressed_size(size_t n, const culzss_params *p) {
    culzss_params d;
    culzss_default_params(&d);
    if (!p) p = &d;
    if (p->chunk_size < 1) return 0;
    uint64_t C = n_chunks(n, p->chunk_size);
    return (size_t)(32 + 4 * C + payload_bound(n, p->chunk_size));
}

int culzss_device_count(void) {
    lib_init();
    return g_device_count;
}

uint64_t culzss_launch_count(void) { return g_launches.load(); }

void culzss_set_profiling(int mode) { t_profiling = mode == 1 || mode == 2 ? mode : 0; }

float culzss_last_kernel_ms(const char *name) {
    if (!name) return -1;
    if (!strcmp(name, "chunk")) return t_times.chunk;
    if (!strcmp(name, "scan")) return t_times.scan;
    if (!strcmp(name, "compact")) return t_times.compact;
    if (!strcmp(name, "decode")) return t_times.decode;
    if (!strcmp(name, "call")) return t_times.call;
    return -1;
}

const char *culzss_status_string(culzss_status s) {
    switch (s) {
        case CULZSS_OK: return "ok";
        case CULZSS_ERR_INVALID_ARG: return "invalid argument";
        case CULZSS_ERR_UNSUPPORTED: return "unsupported parameters";
        case CULZSS_ERR_BUFFER_TOO_SMALL: return "buffer too small";
        case CULZSS_ERR_CORRUPT: return "corrupt stream";
        case CULZSS_ERR_CUDA: return "CUDA error";
        case CULZSS_ERR_NO_DEVICE: return "no CUDA device";
    }
    return "unknown status";
}

int culzss_last_cuda_error(void) { return t_last_cuda_error; }

culzss_status culzss_write_header(void *out, size_t n_total, const culzss_params *p,
                                  culzss_stream_t stream) {
    lib_init();
    if (g_device_count <= 0) return CULZSS_ERR_NO_DEVICE;
    Geometry g;
    culzss_status s = check_params(p, &g);
    if (s != CULZSS_OK) return s;
    if (!is_device_ptr(out)) return CULZSS_ERR_INVALID_ARG;
    if (n_chunks(n_total, g.S) > 0xFFFFFFFFull) return CULZSS_ERR_INVALID_ARG;
    cudaError_t e = launch_header(static_cast<uint8_t *>(out), n_total, g, (cudaStream_t)stream);
    return e == cudaSuccess ? CULZSS_OK : cuda_fail(e);
}

culzss_status culzss_compress(const void *in, size_t n, void *out, size_t *out_n,
                              const culzss_params *p, culzss_stream_t stream) {
    NvtxRange nvtx_("culzss_compress");
    lib_init();
    if (g_device_count <= 0) return CULZSS_ERR_NO_DEVICE;
    if (!out_n) return CULZSS_ERR_INVALID_ARG;
    Geometry g;
    culzss_status s = check_params(p, &g);
    if (s != CULZSS_OK) return s;
    const uint64_t C = n_chunks(n, g.S);
    if (C > 0xFFFFFFFFull) return CULZSS_ERR_INVALID_ARG;
    const uint64_t bound = 32 + 4 * C + payload_bound(n, g.S);
    if (*out_n < bound) {
        *out_n = (size_t)bound;
        return CULZSS_ERR_BUFFER_TOO_SMALL;
    }
    if (!is_device_ptr(out) || (n && !is_device_ptr(in))) return CULZSS_ERR_INVALID_ARG;
    if (overlap(in, n, out, bound)) return CULZSS_ERR_INVALID_ARG;
    cudaStream_t st = (cudaStream_t)stream;
    uint8_t *o = static_cast<uint8_t *>(out);
    uint64_t *hw = host_word();
    if (!hw) return cuda_fail(cudaErrorMemoryAllocation);
    if (n == 0) {
        t_prof.reset();
        CK(launch_header(o, n, g, st));
        CK(cudaStreamSynchronize(st));
        *out_n = 32;
        return CULZSS_OK;
    }
    // workspace (core layout + the device total) is taken from the stream-
    // ordered pool before the call's first event: the device-timed region
    // holds the kernels and the 8-byte read-back, not host-side allocation
    const CoreLayout lay(C, g.S);
    const uint64_t tot_off = (lay.total + 255) / 256 * 256;
    Workspace ws(st);
    CK(ws.alloc(tot_off + 256));
    uint64_t *dev_total = reinterpret_cast<uint64_t *>(static_cast<uint8_t *>(ws.p) + tot_off);
    t_prof.reset();
    t_prof.rec(0, st);
    CK(launch_header(o, n, g, st));
    s = compress_core(static_cast<const uint8_t *>(in), n, g, o + 32 + 4 * C,
                      reinterpret_cast<uint32_t *>(o + 32), nullptr, dev_total, st, ws.p);
    if (s != CULZSS_OK) return s;
    CK(cudaMemcpyAsync(hw, dev_total, 8, cudaMemcpyDeviceToHost, st));
    t_prof.rec(5, st);
    CK(cudaStreamSynchronize(st));
    prof_finish_compress();
    *out_n = (size_t)(32 + 4 * C + *hw);
    return CULZSS_OK;
}

culzss_status culzss_compress_chunks(const void *in_slice, size_t slice_n, void *payload,
                                     size_t *payload_n, uint32_t *chunk_sizes,
                                     const culzss_params *p, culzss_stream_t stream) {
    NvtxRange nvtx_("culzss_compress_chunks");
    lib_init();
    if (g_device_count <= 0) return CULZSS_ERR_NO_DEVICE;
    if (!payload_n) return CULZSS_ERR_INVALID_ARG;
    Geometry g;
    culzss_status s = check_params(p, &g);
    if (s != CULZSS_OK) return s;
    const uint64_t bound = payload_bound(slice_n, g.S);
    if (*payload_n < bound) {
        *payload_n = (size_t)bound;
        return CULZSS_ERR_BUFFER_TOO_SMALL;
    }
    cudaStream_t st = (cudaStream_t)stream;
    if (slice_n == 0) {
        *payload_n = 0;
        return CULZSS_OK;
    }
    if (n_chunks(slice_n, g.S) > 0xFFFFFFFFull) return CULZSS_ERR_INVALID_ARG;
    if (!is_device_ptr(in_slice) || !is_device_ptr(payload) || !is_device_ptr(chunk_sizes))
        return CULZSS_ERR_INVALID_ARG;
    if (overlap(in_slice, slice_n, payload, bound) || overlap(in_slice, slice_n, chunk_sizes, 4 * n_chunks(slice_n, g.S)) ||
        overlap(payload, bound, chunk_sizes, 4 * n_chunks(slice_n, g.S)))
        return CULZSS_ERR_INVALID_ARG;
    uint64_t *hw = host_word();
    if (!hw) return cuda_fail(cudaErrorMemoryAllocation);
    // workspace before the first event (see culzss_compress)
    const CoreLayout lay(n_chunks(slice_n, g.S), g.S);
    const uint64_t tot_off = (lay.total + 255) / 256 * 256;
    Workspace ws(st);
    CK(ws.alloc(tot_off + 256));
    uint64_t *dev_total = reinterpret_cast<uint64_t *>(static_cast<uint8_t *>(ws.p) + tot_off);
    t_prof.reset();
    t_prof.rec(0, st);
    s = compress_core(static_cast<const uint8_t *>(in_slice), slice_n, g,
                      static_cast<uint8_t *>(payload), nullptr, chunk_sizes, dev_total, st, ws.p);
    if (s != CULZSS_OK) return s;
    CK(cudaMemcpyAsync(hw, dev_total, 8, cudaMemcpyDeviceToHost, st));
    t_prof.rec(5, st);
    CK(cudaStreamSynchronize(st));
    prof_finish_compress();
    *payload_n = (size_t)*hw;
    return CULZSS_OK;
}

culzss_status culzss_compress_chunks_async(const void *in_slice, size_t slice_n, void *payload,
                                           size_t payload_cap, uint32_t *chunk_sizes, uint64_t *dev_total,
                                           const culzss_params *p, culzss_stream_t stream) {
    NvtxRange nvtx_("culzss_compress_chunks_async");
    lib_init();
    if (g_device_count <= 0) return CULZSS_ERR_NO_DEVICE;
    Geometry g;
    culzss_status s = check_params(p, &g);
    if (s != CULZSS_OK) return s;
    const uint64_t bound = payload_bound(slice_n, g.S);
    if (payload_cap < bound) return CULZSS_ERR_BUFFER_TOO_SMALL;
    const uint64_t C = n_chunks(slice_n, g.S);
    if (C > 0xFFFFFFFFull) return CULZSS_ERR_INVALID_ARG;
    if (!is_device_ptr(dev_total) || (reinterpret_cast<uintptr_t>(dev_total) & 7)) return CULZSS_ERR_INVALID_ARG;
    cudaStream_t st = (cudaStream_t)stream;
    if (slice_n == 0) {
        CK(cudaMemsetAsync(dev_total, 0, 8, st));
        return CULZSS_OK;
    }
    if (!is_device_ptr(in_slice) || !is_device_ptr(payload) || !is_device_ptr(chunk_sizes))
        return CULZSS_ERR_INVALID_ARG;
    if (overlap(in_slice, slice_n, payload, bound) || overlap(in_slice, slice_n, chunk_sizes, 4 * C) ||
        overlap(payload, bound, chunk_sizes, 4 * C) || overlap(dev_total, 8, payload, bound) ||
        overlap(dev_total, 8, chunk_sizes, 4 * C) || overlap(dev_total, 8, in_slice, slice_n))
        return CULZSS_ERR_INVALID_ARG;
    const CoreLayout lay(C, g.S);
    Workspace ws(st);  // freed stream-ordered on st after the kernels
    CK(ws.alloc(lay.total));
    return compress_core(static_cast<const uint8_t *>(in_slice), slice_n, g, static_cast<uint8_t *>(payload),
                         nullptr, chunk_sizes, dev_total, st, ws.p, false);
}

// Pipelined host-memory compression: the chunks go in groups of ~8 MiB.
// Group k's H2D, fused kernel, scan and compaction (into its own staging
// region) run on compute stream k % 3, so the H2D of one group overlaps the
// kernels of the previous ones; its size table goes straight to its final
// host position.  Its payload's host position needs the totals of all
// earlier groups: the scan writes each group total into mapped host memory
// (no copy-engine round trip), the host waits for group k-2 (the GPU has
// groups k-1 and k queued) and issues that payload's D2H on its own stream.
namespace {
constexpr int kPipeStreams = 3;
struct HostPipe {
    cudaStream_t cs[kPipeStreams] = {}, ds = {}, hs = {};  // compute streams, D2H stream, H2D stream
    cudaEvent_t ev_in = {};
    std::vector<cudaEvent_t> ev, evh;  // per group: kernels + table copy done; its H2D done
    uint64_t *htot = nullptr;  // mapped pinned: the scan kernel writes group totals here
    uint64_t *dtot = nullptr;  // its device alias
    size_t htot_n = 0;
    bool ok = false;
    bool init(size_t groups) {
        if (!ok) {
            for (auto &c : cs)
                if (cudaStreamCreateWithFlags(&c, cudaStreamNonBlocking) != cudaSuccess) return false;
            if (cudaStreamCreateWithFlags(&ds, cudaStreamNonBlocking) != cudaSuccess ||
                cudaStreamCreateWithFlags(&hs, cudaStreamNonBlocking) != cudaSuccess ||
                cudaEventCreateWithFlags(&ev_in, cudaEventDisableTiming) != cudaSuccess)
                return false;
            ok = true;
        }
        while (ev.size() < groups) {
            cudaEvent_t e, f;
            if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return false;
            if (cudaEventCreateWithFlags(&f, cudaEventDisableTiming) != cudaSuccess) return false;
            ev.push_back(e);
            evh.push_back(f);
        }
        if (htot_n < groups) {
            if (htot) cudaFreeHost(htot);
            htot = nullptr;
            if (cudaHostAlloc(&htot, groups * 8, cudaHostAllocMapped) != cudaSuccess) return false;
            if (cudaHostGetDevicePointer(&dtot, htot, 0) != cudaSuccess) return false;
            htot_n = groups;
        }
        return true;
    }
};
thread_local HostPipe t_pipe_dev[kMaxDevices];  // streams/events of the current device
}  // namespace

culzss_status culzss_compress_host(const void *in_host, size_t n, void *out_host, size_t *out_n,
                                   const culzss_params *p, culzss_stream_t stream) {
    NvtxRange nvtx_("culzss_compress_host");
    lib_init();
    if (g_device_count <= 0) return CULZSS_ERR_NO_DEVICE;
    if (!out_n || (n && !in_host) || !out_host) return CULZSS_ERR_INVALID_ARG;
    Geometry g;
    culzss_status s = check_params(p, &g);
    if (s != CULZSS_OK) return s;
    const uint64_t C = n_chunks(n, g.S);
    if (C > 0xFFFFFFFFull) return CULZSS_ERR_INVALID_ARG;
    const uint64_t bound = 32 + 4 * C + payload_bound(n, g.S);
    if (*out_n < bound) {
        *out_n = (size_t)bound;
        return CULZSS_ERR_BUFFER_TOO_SMALL;
    }
    cudaStream_t st = (cudaStream_t)stream;
    // group size: 8 MiB, 16 MiB from 512 MiB of input on (fewer per-group host
    // waits; B200: c2 128 MiB 44.8 GB/s at 8 MiB vs 38.4 at 16; c3 1 GiB 51.2 vs
    // 52.5).  CULZSS_GROUP_KB overrides (pipeline tuning knob)
    static const uint64_t group_env = [] {
        const char *e = getenv("CULZSS_GROUP_KB");
        const long v = e ? atol(e) : 0;
        return v > 0 ? (uint64_t)v << 10 : 0ull;
    }();
    const uint64_t group_bytes = group_env ? group_env : (n >= (512ull << 20) ? 16ull << 20 : 8ull << 20);
    const uint64_t gc = std::max<uint64_t>(1, group_bytes / g.S);  // chunks per group
    const uint64_t G = (C + gc - 1) / gc;
    if (G <= 1) {  // one group: no overlap to gain
        Workspace ws(st);
        const uint64_t in_bytes = (n + 255) / 256 * 256;
        CK(ws.alloc(in_bytes + bound));
        uint8_t *din = static_cast<uint8_t *>(ws.p);
        uint8_t *dout = din + in_bytes;
        if (n) CK(cudaMemcpyAsync(din, in_host, n, cudaMemcpyHostToDevice, st));
        size_t on = (size_t)bound;
        s = culzss_compress(din, n, dout, &on, p, stream);
        if (s != CULZSS_OK) return s;
        CK(cudaMemcpyAsync(out_host, dout, on, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        *out_n = on;
        return CULZSS_OK;
    }
    HostPipe &hp = t_pipe_dev[cur_device()];
    if (!hp.init(G)) return cuda_fail(cudaErrorMemoryAllocation);
    // device: input | header + table (contiguous, as in the stream) | per-group
    // staging at its worst-case offset | group totals | two core workspaces
    const CoreLayout lay(gc, g.S);
    const uint64_t in_bytes = (n + 255) / 256 * 256;
    const uint64_t ht_bytes = (32 + 4 * C + 255) / 256 * 256;
    const uint64_t stg_bytes = (payload_bound(n, g.S) + 255) / 256 * 256;
    const uint64_t core_bytes = (lay.total + 255) / 256 * 256;
    Workspace ws(st);
    CK(ws.alloc(in_bytes + ht_bytes + stg_bytes + kPipeStreams * core_bytes));
    uint8_t *din = static_cast<uint8_t *>(ws.p);
    uint8_t *dht = din + in_bytes;
    uint8_t *dstg = dht + ht_bytes;
    uint8_t *dcore = dstg + stg_bytes;
    uint8_t *hout = static_cast<uint8_t *>(out_host);
    const uint8_t *hin = static_cast<const uint8_t *>(in_host);
    struct Drain {  // on an error return, no internal stream may still use ws
        HostPipe &hp;
        bool done = false;
        ~Drain() {
            if (done) return;
            for (auto cs : hp.cs) cudaStreamSynchronize(cs);
            cudaStreamSynchronize(hp.ds);
            cudaStreamSynchronize(hp.hs);
            cudaGetLastError();
        }
    } drain{hp};
    t_prof.reset();
    t_prof.rec(0, st);
    CK(launch_header(dht, n, g, st));
    CK(cudaEventRecord(hp.ev_in, st));  // the workspace and header exist
    for (auto cs : hp.cs) CK(cudaStreamWaitEvent(cs, hp.ev_in, 0));
    CK(cudaStreamWaitEvent(hp.ds, hp.ev_in, 0));
    CK(cudaStreamWaitEvent(hp.hs, hp.ev_in, 0));
    // every group's H2D up front, back to back on the H2D stream: the
    // host->device copy engine never waits for the issue loop below
    for (uint64_t k = 0; k < G; k++) {
        const uint64_t c0 = k * gc, c1 = std::min(C, c0 + gc);
        const uint64_t b0 = c0 * g.S, nb = std::min<uint64_t>(n, c1 * g.S) - b0;
        CK(cudaMemcpyAsync(din + b0, hin + b0, nb, cudaMemcpyHostToDevice, hp.hs));
        CK(cudaEventRecord(hp.evh[k], hp.hs));
    }
    CK(cudaMemcpyAsync(hout, dht, 32, cudaMemcpyDeviceToHost, hp.ds));
    uint64_t base = 0;  // payload bytes of the groups whose D2H is issued
    auto issue_payload = [&](uint64_t k) -> culzss_status {
        CK(cudaEventSynchronize(hp.ev[k]));
        const uint64_t t = hp.htot[k];
        if (t) {
            CK(cudaStreamWaitEvent(hp.ds, hp.ev[k], 0));
            CK(cudaMemcpyAsync(hout + 32 + 4 * C + base, dstg + payload_bound(k * gc * g.S, g.S), t,
                               cudaMemcpyDeviceToHost, hp.ds));
        }
        base += t;
        return CULZSS_OK;
    };
    for (uint64_t k = 0; k < G; k++) {
        cudaStream_t cs = hp.cs[k % kPipeStreams];
        const uint64_t c0 = k * gc, c1 = std::min(C, c0 + gc);
        const uint64_t b0 = c0 * g.S, nb = std::min<uint64_t>(n, c1 * g.S) - b0;
        CK(cudaStreamWaitEvent(cs, hp.evh[k], 0));
        s = compress_core(din + b0, nb, g, dstg + payload_bound(b0, g.S),
                          reinterpret_cast<uint32_t *>(dht + 32) + c0, nullptr, hp.dtot + k, cs,
                          dcore + (k % kPipeStreams) * core_bytes, false);  // no per-group profiling events in the issue loop
        if (s != CULZSS_OK) return s;
        CK(cudaMemcpyAsync(hout + 32 + 4 * c0, dht + 32 + 4 * c0, 4 * (c1 - c0), cudaMemcpyDeviceToHost,
                           cs));
        CK(cudaEventRecord(hp.ev[k], cs));
        if (k >= 2) {
            s = issue_payload(k - 2);
            if (s != CULZSS_OK) return s;
        }
    }
    for (uint64_t k = G >= 2 ? G - 2 : 0; k < G; k++) {
        s = issue_payload(k);
        if (s != CULZSS_OK) return s;
    }
    // the caller's stream resumes after everything (the workspace is freed on it)
    CK(cudaEventRecord(hp.ev_in, hp.ds));
    CK(cudaStreamWaitEvent(st, hp.ev_in, 0));
    for (auto cs : hp.cs) {
        CK(cudaEventRecord(hp.ev[0], cs));
        CK(cudaStreamWaitEvent(st, hp.ev[0], 0));
    }
    t_prof.rec(5, st);
    CK(cudaStreamSynchronize(st));
    drain.done = true;
    if (t_profiling) t_times.call = t_prof.between(0, 5);
    *out_n = (size_t)(32 + 4 * C + base);
    return CULZSS_OK;
}

// Parse and validate the 32-byte header from host bytes (readings R12, R13).
static culzss_status parse_header(const uint8_t *h, Geometry *g, uint64_t *n, uint64_t *C) {
    auto le = [&](int off, int nb) {
        uint64_t v = 0;
        for (int i = 0; i < nb; i++) v |= (uint64_t)h[off + i] << (8 * i);
        return v;
    };
    if (h[0] != 'C' || h[1] != 'L' || h[2] != 'Z' || h[3] != 'S') return CULZSS_ERR_CORRUPT;
    if (le(4, 2) != 1 || le(6, 2) != 32 || h[29] || h[30] || h[31]) return CULZSS_ERR_CORRUPT;
    culzss_params p;
    p.chunk_size = (uint32_t)le(8, 4);
    p.window = (uint16_t)le(24, 2);
    p.max_match = (uint16_t)le(26, 2);
    p.min_match = h[28];
    p.version = 0;
    p.reserved = 0;
    if (p.min_match != 3 || p.chunk_size < 1 || p.window < 1 || p.window > 256 ||
        p.max_match < 3 || p.max_match > 258)
        return CULZSS_ERR_CORRUPT;
    *n = le(16, 8);
    *C = le(12, 4);
    if (*C != n_chunks(*n, p.chunk_size)) return CULZSS_ERR_CORRUPT;
    culzss_status s = check_params(&p, g);
    return s == CULZSS_OK ? CULZSS_OK : CULZSS_ERR_UNSUPPORTED;
}

static culzss_status read_header(const void *in, size_t in_n, Geometry *g, uint64_t *n,
                                 uint64_t *C, cudaStream_t st) {
    if (in_n < 32) return CULZSS_ERR_CORRUPT;
    uint64_t *hw = host_word();
    if (!hw) return cuda_fail(cudaErrorMemoryAllocation);
    uint8_t *h = reinterpret_cast<uint8_t *>(hw);
    CK(cudaMemcpyAsync(h, in, 32, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    return parse_header(h, g, n, C);
}

culzss_status culzss_decompressed_size(const void *in, size_t in_n, size_t *n,
                                       culzss_stream_t stream) {
    lib_init();
    if (g_device_count <= 0) return CULZSS_ERR_NO_DEVICE;
    if (!n || !is_device_ptr(in)) return CULZSS_ERR_INVALID_ARG;
    Geometry g;
    uint64_t nn, C;
    culzss_status s = read_header(in, in_n, &g, &nn, &C, (cudaStream_t)stream);
    if (s == CULZSS_OK || s == CULZSS_ERR_UNSUPPORTED) *n = (size_t)nn;
    return s == CULZSS_ERR_UNSUPPORTED ? CULZSS_OK : s;
}

// Enqueue the decode of C chunks (n output bytes) from `payload` (pay_len
// bytes) with the u32 size table at `table_src` (device, any alignment:
// copied to an aligned workspace) on st, without a host sync: scan of the
// sizes, walk + decode kernels; malformed chunks OR bits into *err (device).
static culzss_status decompress_enqueue(const uint8_t *payload, uint64_t pay_len, const void *table_src, uint64_t C,
                                        uint64_t n, const Geometry &g, uint8_t *out, cudaStream_t st, uint32_t *err,
                                        bool prof) {
    // workspace: aligned copy of the table | offsets | scan ws | total | records
    const uint64_t tab_off = 0;
    const uint64_t offs_off = (C * 4 + 255) / 256 * 256;
    const uint64_t ws_off = offs_off + (C * 8 + 255) / 256 * 256;
    const uint64_t tot_off = ws_off + (scan_workspace_words(C) * 8 + 255) / 256 * 256;
    const uint64_t tb_off = tot_off + 256;
    Workspace ws(st);  // freed stream-ordered on st
    CK(ws.alloc(tb_off + decode_scratch_bytes(C)));
    uint8_t *base = static_cast<uint8_t *>(ws.p);
    uint32_t *sizes = reinterpret_cast<uint32_t *>(base + tab_off);
    uint64_t *offsets = reinterpret_cast<uint64_t *>(base + offs_off);
    uint64_t *scanws = reinterpret_cast<uint64_t *>(base + ws_off);
    uint64_t *total = reinterpret_cast<uint64_t *>(base + tot_off);
    CK(cudaMemcpyAsync(sizes, table_src, C * 4, cudaMemcpyDeviceToDevice, st));
    CK(launch_scan(sizes, C, offsets, total, scanws, st));
    // the walk kernel checks the table against the payload length (no sync here)
    if (prof) t_prof.rec(1, st);
    CK(launch_decode(payload, pay_len, sizes, offsets, C, n, g, out, err, reinterpret_cast<uint32_t *>(base + tb_off),
                     st));
    if (prof) t_prof.rec(2, st);
    return CULZSS_OK;
}

// Synchronous decode: enqueue, then one sync for the device error word.
static culzss_status decompress_core(const uint8_t *payload, uint64_t pay_len, const void *table_src, uint64_t C,
                                     uint64_t n, const Geometry &g, uint8_t *out, cudaStream_t st) {
    Workspace ew(st);
    CK(ew.alloc(256));
    uint32_t *err = static_cast<uint32_t *>(ew.p);
    CK(cudaMemsetAsync(err, 0, 4, st));
    uint64_t *hw = host_word();
    if (!hw) return cuda_fail(cudaErrorMemoryAllocation);
    t_prof.reset();
    culzss_status s = decompress_enqueue(payload, pay_len, table_src, C, n, g, out, st, err, true);
    if (s != CULZSS_OK) return s;
    CK(cudaMemcpyAsync(hw, err, 4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (t_profiling) t_times.decode = t_prof.between(1, 2);
    if (reinterpret_cast<uint32_t *>(hw)[0]) return CULZSS_ERR_CORRUPT;
    return CULZSS_OK;
}

culzss_status culzss_decompress(const void *in, size_t in_n, void *out, size_t *out_n,
                                const culzss_params *, culzss_stream_t stream) {
    NvtxRange nvtx_("culzss_decompress");
    lib_init();
    if (g_device_count <= 0) return CULZSS_ERR_NO_DEVICE;
    if (!out_n || !is_device_ptr(in)) return CULZSS_ERR_INVALID_ARG;
    cudaStream_t st = (cudaStream_t)stream;
    Geometry g;
    uint64_t n, C;
    culzss_status s = read_header(in, in_n, &g, &n, &C, st);
    if (s != CULZSS_OK) return s;
    if (in_n < 32 + 4 * C) return CULZSS_ERR_CORRUPT;
    if (*out_n < n) {
        *out_n = (size_t)n;
        return CULZSS_ERR_BUFFER_TOO_SMALL;
    }
    if (n == 0) {
        if (in_n != 32) return CULZSS_ERR_CORRUPT;
        *out_n = 0;
        return CULZSS_OK;
    }
    if (!is_device_ptr(out) || overlap(in, in_n, out, n)) return CULZSS_ERR_INVALID_ARG;
    const uint8_t *src = static_cast<const uint8_t *>(in);
    s = decompress_core(src + 32 + 4 * C, in_n - 32 - 4 * C, src + 32, C, n, g, static_cast<uint8_t *>(out), st);
    if (s == CULZSS_OK) *out_n = (size_t)n;
    return s;
}

culzss_status culzss_decompress_chunks(const void *payload, size_t payload_n, const uint32_t *chunk_sizes,
                                       size_t slice_n, void *out, const culzss_params *p,
                                       culzss_stream_t stream) {
    NvtxRange nvtx_("culzss_decompress_chunks");
    lib_init();
    if (g_device_count <= 0) return CULZSS_ERR_NO_DEVICE;
    Geometry g;
    culzss_status s = check_params(p, &g);
    if (s != CULZSS_OK) return s;
    if (slice_n == 0) return payload_n == 0 ? CULZSS_OK : CULZSS_ERR_CORRUPT;
    const uint64_t C = n_chunks(slice_n, g.S);
    if (!is_device_ptr(payload) || !is_device_ptr(chunk_sizes) || !is_device_ptr(out) ||
        overlap(payload, payload_n, out, slice_n) || overlap(chunk_sizes, 4 * C, out, slice_n))
        return CULZSS_ERR_INVALID_ARG;
    return decompress_core(static_cast<const uint8_t *>(payload), payload_n, chunk_sizes, C, slice_n, g,
                           static_cast<uint8_t *>(out), (cudaStream_t)stream);
}

// Host-memory decompression, the inverse of culzss_compress_host: the
// header and size table are read from host memory, the output is decoded in
// groups of ~8 MiB on the three compute streams (H2D of the group's table
// slice and payload, scan + walk + decode), and each group's output is copied
// back on the copy stream as soon as its kernels finish, so both copy
// directions overlap the kernels.  Device errors OR into one word checked at
// the single final sync.
culzss_status culzss_decompress_host(const void *in_host, size_t in_n, void *out_host, size_t *out_n,
                                     const culzss_params *, culzss_stream_t stream) {
    NvtxRange nvtx_("culzss_decompress_host");
    lib_init();
    if (g_device_count <= 0) return CULZSS_ERR_NO_DEVICE;
    if (!out_n || !in_host || !out_host) return CULZSS_ERR_INVALID_ARG;
    if (in_n < 32) return CULZSS_ERR_CORRUPT;
    const uint8_t *hin = static_cast<const uint8_t *>(in_host);
    Geometry g;
    uint64_t n, C;
    culzss_status s = parse_header(hin, &g, &n, &C);
    if (s != CULZSS_OK) return s;
    if (in_n < 32 + 4 * C) return CULZSS_ERR_CORRUPT;
    if (*out_n < n) {
        *out_n = (size_t)n;
        return CULZSS_ERR_BUFFER_TOO_SMALL;
    }
    if (n == 0) {
        if (in_n != 32) return CULZSS_ERR_CORRUPT;
        *out_n = 0;
        return CULZSS_OK;
    }
    // payload offsets from the host copy of the table (u64 prefix sums)
    std::vector<uint64_t> off(C + 1, 0);
    for (uint64_t c = 0; c < C; c++) {
        uint32_t v;
        memcpy(&v, hin + 32 + 4 * c, 4);
        off[c + 1] = off[c] + v;
    }
    const uint64_t pay_len = in_n - 32 - 4 * C;
    if (off[C] != pay_len) return CULZSS_ERR_CORRUPT;
    cudaStream_t st = (cudaStream_t)stream;
    static const uint64_t dgroup_env = [] {  // CULZSS_DGROUP_KB: decode group size (output bytes)
        const char *e = getenv("CULZSS_DGROUP_KB");
        const long v = e ? atol(e) : 0;
        return v > 0 ? (uint64_t)v << 10 : 0ull;
    }();
    const uint64_t dgroup_bytes = dgroup_env ? dgroup_env : (n >= (512ull << 20) ? 16ull << 20 : 8ull << 20);
    const uint64_t gc = std::max<uint64_t>(1, dgroup_bytes / g.S);  // chunks per group
    const uint64_t G = (C + gc - 1) / gc;
    HostPipe &hp = t_pipe_dev[cur_device()];
    if (!hp.init(G)) return cuda_fail(cudaErrorMemoryAllocation);
    // device: table | payload | output | error word
    const uint64_t tab_bytes = (4 * C + 255) / 256 * 256;
    const uint64_t pay_bytes = (pay_len + 255) / 256 * 256;
    const uint64_t out_bytes = (n + 255) / 256 * 256;
    Workspace ws(st);
    CK(ws.alloc(tab_bytes + pay_bytes + out_bytes + 256));
    uint8_t *dtab = static_cast<uint8_t *>(ws.p);
    uint8_t *dpay = dtab + tab_bytes;
    uint8_t *dout = dpay + pay_bytes;
    uint32_t *err = reinterpret_cast<uint32_t *>(dout + out_bytes);
    uint8_t *hout = static_cast<uint8_t *>(out_host);
    struct Drain {  // on an error return, no internal stream may still use ws
        HostPipe &hp;
        bool done = false;
        ~Drain() {
            if (done) return;
            for (auto cs : hp.cs) cudaStreamSynchronize(cs);
            cudaStreamSynchronize(hp.ds);
            cudaStreamSynchronize(hp.hs);
            cudaGetLastError();
        }
    } drain{hp};
    t_prof.reset();
    t_prof.rec(0, st);
    CK(cudaMemsetAsync(err, 0, 4, st));
    CK(cudaEventRecord(hp.ev_in, st));  // the workspace exists and the error word is clear
    for (auto cs : hp.cs) CK(cudaStreamWaitEvent(cs, hp.ev_in, 0));
    CK(cudaStreamWaitEvent(hp.ds, hp.ev_in, 0));
    CK(cudaStreamWaitEvent(hp.hs, hp.ev_in, 0));
    // every group's H2D (table slice + payload) up front on the H2D stream
    for (uint64_t k = 0; k < G; k++) {
        const uint64_t c0 = k * gc, c1 = std::min(C, c0 + gc);
        CK(cudaMemcpyAsync(dtab + 4 * c0, hin + 32 + 4 * c0, 4 * (c1 - c0), cudaMemcpyHostToDevice, hp.hs));
        if (off[c1] > off[c0])
            CK(cudaMemcpyAsync(dpay + off[c0], hin + 32 + 4 * C + off[c0], off[c1] - off[c0],
                               cudaMemcpyHostToDevice, hp.hs));
        CK(cudaEventRecord(hp.evh[k], hp.hs));
    }
    for (uint64_t k = 0; k < G; k++) {
        cudaStream_t cs = hp.cs[k % kPipeStreams];
        const uint64_t c0 = k * gc, c1 = std::min(C, c0 + gc);
        const uint64_t b0 = c0 * g.S, nb = std::min<uint64_t>(n, c1 * g.S) - b0;
        CK(cudaStreamWaitEvent(cs, hp.evh[k], 0));
        s = decompress_enqueue(dpay + off[c0], off[c1] - off[c0], dtab + 4 * c0, c1 - c0, nb, g, dout + b0, cs, err,
                               false);
        if (s != CULZSS_OK) return s;
        CK(cudaEventRecord(hp.ev[k], cs));
        CK(cudaStreamWaitEvent(hp.ds, hp.ev[k], 0));
        CK(cudaMemcpyAsync(hout + b0, dout + b0, nb, cudaMemcpyDeviceToHost, hp.ds));
    }
    // the caller's stream resumes after everything (the workspace is freed on it)
    CK(cudaEventRecord(hp.ev_in, hp.ds));
    CK(cudaStreamWaitEvent(st, hp.ev_in, 0));
    for (auto cs : hp.cs) {
        CK(cudaEventRecord(hp.ev[0], cs));
        CK(cudaStreamWaitEvent(st, hp.ev[0], 0));
    }
    uint64_t *hw = host_word();
    if (!hw) return cuda_fail(cudaErrorMemoryAllocation);
    CK(cudaMemcpyAsync(hw, err, 4, cudaMemcpyDeviceToHost, st));
    t_prof.rec(5, st);
    CK(cudaStreamSynchronize(st));
    drain.done = true;
    if (t_profiling) t_times.call = t_prof.between(0, 5);
    if (reinterpret_cast<uint32_t *>(hw)[0]) return CULZSS_ERR_CORRUPT;
    *out_n = (size_t)n;
    return CULZSS_OK;
}

static culzss_status debug_entry(int mode, const void *in, size_t n, void *dst,
                                 const culzss_params *p, culzss_stream_t stream) {
    lib_init();
    if (g_device_count <= 0) return CULZSS_ERR_NO_DEVICE;
    Geometry g;
    culzss_status s = check_params(p, &g);
    if (s != CULZSS_OK) return s;
    if (mode == kModeDumpMatch && g.F > 255) return CULZSS_ERR_UNSUPPORTED;
    if (n == 0) return CULZSS_OK;
    if (!is_device_ptr(in) || !is_device_ptr(dst)) return CULZSS_ERR_INVALID_ARG;
    cudaStream_t st = (cudaStream_t)stream;
    CK(launch_chunk_kernel(mode, static_cast<const uint8_t *>(in), n, g, nullptr, nullptr, dst, st));
    CK(cudaStreamSynchronize(st));
    return CULZSS_OK;
}

culzss_status culzss_match_search(const void *in, size_t n, uint8_t *LD, const culzss_params *p,
                                  culzss_stream_t stream) {
    return debug_entry(kModeDumpMatch, in, n, LD, p, stream);
}

culzss_status culzss_parse_tokens(const void *in, size_t n, uint32_t *tok, const culzss_params *p,
                                  culzss_stream_t stream) {
    return debug_entry(kModeDumpTokens, in, n, tok, p, stream);
}

}  // extern "C"
