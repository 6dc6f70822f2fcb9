// intpeak.cu — integer-pipe peak microbenchmark on one B200 ("Measure with the
// microbenchmark ... Do not assume 64 vs 128").  The denominators of bench.py's K3 roofline come from here.
//
// Four kernels, each a loop of independent dependency chains (8 per thread, 32 warps per SM so the 4-cycle
// fixed latency is hidden), with every operand another chain's value (no constant folding, no hoisting):
//   alu   LOP3 (majority / mux LUTs: not reassociable), IADD3, PRMT, SHF   -> the ALU pipe only
//   fma   IMAD (mad.lo.u32)                                                 -> the FMA pipe only
//   mix   half ALU, half IMAD, interleaved, 3 register sources per op       -> both pipes
//   mix2  the same with 2 register sources + an immediate per op            -> both pipes (issue-bound)
// Reported: lane-ops per second (CUDA events) and lane-ops per SM per clock (clock64 in every CTA), plus the
// SM clock during the run derived from the two.  cuobjdump -sass of this file shows the loop bodies
// (tools/intpeak_sass.txt); every counted op is one SASS instruction.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/intpeak tools/intpeak.cu
// Run:   tools/intpeak [iters]   (prints one JSON object)
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x)                                                                          \
    do {                                                                               \
        cudaError_t e = (x);                                                           \
        if (e != cudaSuccess) {                                                        \
            fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); \
            exit(1);                                                                   \
        }                                                                              \
    } while (0)

__device__ __forceinline__ uint32_t maj(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t r;
    asm volatile("lop3.b32 %0, %1, %2, %3, 0xE8;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
    return r;
}
__device__ __forceinline__ uint32_t mux(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t r;
    asm volatile("lop3.b32 %0, %1, %2, %3, 0xCA;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
    return r;
}
__device__ __forceinline__ uint32_t add3(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t r;
    asm volatile("{ .reg .u32 t; add.u32 t, %1, %2; add.u32 %0, t, %3; }" : "=r"(r) : "r"(a), "r"(b), "r"(c));
    return r;
}
__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b) {
    uint32_t r;
    asm volatile("prmt.b32 %0, %1, %2, 0x7531;" : "=r"(r) : "r"(a), "r"(b));
    return r;
}
__device__ __forceinline__ uint32_t shf(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t r;
    asm volatile("shf.l.wrap.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
    return r;
}
__device__ __forceinline__ uint32_t lop_i(uint32_t a, uint32_t b) {  // two register operands + immediate
    uint32_t r;
    asm volatile("lop3.b32 %0, %1, %2, 0x5a5a5a5a, 0xE8;" : "=r"(r) : "r"(a), "r"(b));
    return r;
}
__device__ __forceinline__ uint32_t imad_i(uint32_t a, uint32_t c) {  // a * imm + c
    uint32_t r;
    asm volatile("mad.lo.u32 %0, %1, 0x9e3779b1, %2;" : "=r"(r) : "r"(a), "r"(c));
    return r;
}
__device__ __forceinline__ uint32_t imad(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t r;
    asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
    return r;
}

constexpr int kChains = 8;

// MODE 0 = alu, 1 = fma, 2 = mix, 3 = mix2.  Per iteration every chain does 4 ops -> 32 ops per thread per iteration.
template <int MODE>
__global__ void __launch_bounds__(1024, 1) intpeak_kernel(int iters, uint32_t seed, uint32_t *out,
                                                          unsigned long long *cycles) {
    uint32_t a[kChains];
#pragma unroll
    for (int k = 0; k < kChains; k++) a[k] = seed * (threadIdx.x + 1) + k * 0x9e3779b9u + blockIdx.x;
    __syncthreads();
    const long long c0 = clock64();
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int k = 0; k < kChains; k++) {
            const uint32_t b = a[(k + 1) % kChains], c = a[(k + 3) % kChains];
            uint32_t x = a[k];
            if (MODE == 0) {
                x = maj(x, b, c);
                x = add3(x, b, c);
                x = prmt(x, b);
                x = shf(x, c, b);
            } else if (MODE == 1) {
                x = imad(x, b, c);
                x = imad(x, c, b);
                x = imad(x, b, c);
                x = imad(x, c, b);
            } else if (MODE == 2) {
                x = mux(x, b, c);
                x = imad(x, b, c);
                x = maj(x, c, b);
                x = imad(x, c, b);
            } else {
                x = lop_i(x, b);
                x = imad_i(x, c);
                x = lop_i(x, c);
                x = imad_i(x, b);
            }
            a[k] = x;
        }
    }
    __syncthreads();
    const long long c1 = clock64();
    uint32_t r = 0;
#pragma unroll
    for (int k = 0; k < kChains; k++) r ^= a[k];
    if (r == 0x12345678u) out[blockIdx.x * blockDim.x + threadIdx.x] = r;  // keep the chains live
    if (threadIdx.x == 0) atomicAdd(cycles, (unsigned long long)(c1 - c0));
}

template <int MODE>
double run(int iters, int sms, double *lanes_per_sm_clk, double *mhz) {
    const int threads = 1024, blocks = sms;  // one 32-warp CTA per SM
    uint32_t *out;
    unsigned long long *cyc;
    CK(cudaMalloc(&out, sizeof(uint32_t) * threads * blocks));
    CK(cudaMalloc(&cyc, sizeof(unsigned long long)));
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    double best = 0;
    for (int rep = 0; rep < 5; rep++) {
        CK(cudaMemset(cyc, 0, sizeof(unsigned long long)));
        CK(cudaEventRecord(e0));
        intpeak_kernel<MODE><<<blocks, threads>>>(iters, 12345u + rep, out, cyc);
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        CK(cudaGetLastError());
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, e0, e1));
        unsigned long long c = 0;
        CK(cudaMemcpy(&c, cyc, sizeof(c), cudaMemcpyDeviceToHost));
        const double ops = (double)threads * blocks * iters * kChains * 4;
        const double rate = ops / (ms * 1e-3);
        const double cyc_per_cta = (double)c / blocks;
        if (rep > 0 && rate > best) {  // rep 0 warms the clocks
            best = rate;
            *lanes_per_sm_clk = ops / blocks / cyc_per_cta;
            *mhz = cyc_per_cta / (ms * 1e-3) / 1e6;
        }
    }
    CK(cudaFree(out));
    CK(cudaFree(cyc));
    return best;
}

int main(int argc, char **argv) {
    const int iters = argc > 1 ? atoi(argv[1]) : 200000;
    int dev = 0, sms = 0;
    CK(cudaGetDevice(&dev));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    cudaDeviceProp prop;
    CK(cudaGetDeviceProperties(&prop, dev));
    double l[4], f[4], r[4];
    r[0] = run<0>(iters, sms, &l[0], &f[0]);
    r[1] = run<1>(iters, sms, &l[1], &f[1]);
    r[2] = run<2>(iters, sms, &l[2], &f[2]);
    r[3] = run<3>(iters, sms, &l[3], &f[3]);
    printf("{\"gpu\": \"%s\", \"sms\": %d, \"iters\": %d, \"threads_per_sm\": 1024, \"chains_per_thread\": %d,\n",
           prop.name, sms, iters, kChains);
    const char *names[4] = {"alu", "fma", "mix", "mix2"};
    const char *what[4] = {"LOP3/IADD3/PRMT/SHF (ALU pipe)", "IMAD (FMA pipe)",
                           "LOP3 + IMAD interleaved, three register sources each (ALU+FMA)",
                           "LOP3 + IMAD interleaved, two register sources + an immediate each (ALU+FMA)"};
    for (int k = 0; k < 4; k++)
        printf(" \"%s\": {\"what\": \"%s\", \"lane_ops_per_s\": %.6e, \"lane_ops_per_sm_per_clk\": %.2f, \"sm_mhz\": %.0f}%s\n",
               names[k], what[k], r[k], l[k], f[k], k < 3 ? "," : "");
    printf("}\n");
    return 0;
}
