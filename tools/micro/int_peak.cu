// Integer-pipe peak microbenchmark:
// dependent-free streams of LOP3, IADD3 and IMAD on every SM, timed with
// CUDA events.  The chunk kernel's compare term is charged
// against the ALU-pipe figure: XOR / zero-byte tests / funnel-free compares
// are LOP3 / IADD3, which issue only on the ALU pipe.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o int_peak tools/micro/int_peak.cu
//   ./int_peak [device] > profiles/int_peak.json       (one JSON object)
//
// Each thread runs 8 independent accumulator chains through an unrolled
// loop of inline-PTX instructions (lop3.b32 / add of three operands that
// ptxas fuses into IADD3 / mad.lo.u32 -> IMAD), so issue, not latency, binds
// (8 chains x 16 warps per SMSP).  Check the SASS with
//   cuobjdump -sass int_peak | grep -c LOP3    (etc.)
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int kChains = 8;
constexpr int kUnroll = 16;

template <int OP>
__global__ void __launch_bounds__(512) k_int(uint32_t *out, int iters, uint32_t s) {
    uint32_t a[kChains];
#pragma unroll
    for (int i = 0; i < kChains; i++) a[i] = threadIdx.x * 2654435761u + i * 0x9E3779B9u + s;
    const uint32_t b = s ^ 0x5bd1e995u, c = s + 0x27d4eb2du;
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
#pragma unroll
            for (int i = 0; i < kChains; i++) {
                if (OP == 0) {  // LOP3 (ALU pipe): a = (a ^ b) & c | ...  one lop3
                    asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(a[i]) : "r"(b), "r"(c));
                } else if (OP == 1) {  // IADD3 (ALU pipe)
                    asm volatile("{ .reg .u32 t; add.u32 t, %0, %1; add.u32 %0, t, %2; }"
                                 : "+r"(a[i]) : "r"(b), "r"(c));
                } else if (OP == 2) {  // IMAD (FMA pipe)
                    asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(a[i]) : "r"(b), "r"(c));
                } else {  // LOP3 and IMAD interleaved (both pipes)
                    if (i & 1)
                        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(a[i]) : "r"(b), "r"(c));
                    else
                        asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(a[i]) : "r"(b), "r"(c));
                }
            }
        }
    }
    uint32_t r = 0;
#pragma unroll
    for (int i = 0; i < kChains; i++) r ^= a[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = r;
}

template <int OP>
double run(int sms, uint32_t *d, cudaEvent_t e0, cudaEvent_t e1, int blocks_per_sm, int threads) {
    const int iters = 2000;
    const int blocks = sms * blocks_per_sm;
    k_int<OP><<<blocks, threads>>>(d, 10, 1);  // warm-up
    cudaDeviceSynchronize();
    float best = 1e30f;
    for (int rep = 0; rep < 5; rep++) {
        cudaEventRecord(e0);
        k_int<OP><<<blocks, threads>>>(d, iters, rep + 2);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    // ops = 32-bit integer instructions per thread (one IADD3 = one op)
    const double ops = (double)blocks * threads * iters * kUnroll * kChains;
    return ops / (best * 1e-3) / 1e12;  // Tops/s
}

int main(int argc, char **argv) {
    int dev = argc > 1 ? atoi(argv[1]) : 0, sms = 0, clk_khz = 0;  // device ordinal (bench.py passes its rank's)
    cudaSetDevice(dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev);
    cudaDeviceProp prop;
    cudaGetDeviceProperties(&prop, dev);
    const int threads = 512, bps = 4;  // 64 warps per SM
    uint32_t *d;
    cudaMalloc(&d, (size_t)sms * bps * threads * 4);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const double lop3 = run<0>(sms, d, e0, e1, bps, threads);
    const double iadd3 = run<1>(sms, d, e0, e1, bps, threads);
    const double imad = run<2>(sms, d, e0, e1, bps, threads);
    const double mixed = run<3>(sms, d, e0, e1, bps, threads);
    cudaError_t err = cudaGetLastError();
    printf("{\"gpu\": \"%s\", \"sms\": %d, \"clock_mhz_attr\": %.0f, "
           "\"lop3_tops\": %.3f, \"iadd3_tops\": %.3f, \"imad_tops\": %.3f, \"lop3_imad_mixed_tops\": %.3f, "
           "\"alu_lanes_per_sm_clk_at_attr_clock\": %.1f, \"what\": \"dependent-free int32 instruction streams, "
           "8 chains x 64 warps per SM, best of 5, CUDA events (tools/micro/int_peak.cu)\", \"cuda_error\": \"%s\"}\n",
           prop.name, sms, clk_khz / 1e3, lop3, iadd3, imad, mixed,
           lop3 * 1e12 / (sms * clk_khz * 1e3), cudaGetErrorString(err));
    return err == cudaSuccess ? 0 : 1;
}
