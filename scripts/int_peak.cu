// int_peak.cu -- measured integer issue / pipe throughput of one B200 SM (the ALU
// roofline denominator of the SA kernel must be measured, not assumed).
//
// Each thread runs 8 independent dependency chains of one opcode (32 per loop iteration), so the
// pipe, not the 4-cycle latency, bounds the rate.  Every CTA records %clock64 and %globaltimer at
// start and end: the SM clock of the run is measured, not assumed.  Output (stdout, one JSON line
// per opcode): warp instructions of that opcode per SM clock per SM = instructions / (event time x
// measured clock), over the whole launch (waves included).
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o int_peak int_peak.cu
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdint>
#include <vector>

constexpr int kIters = 4096;
constexpr int kChains = 8;

enum Op { IADD3, LOP3, IMAD, PRMT, IDP4A, IDP2A, SHF, MIX_IMAD_LOP3, MIX_SA_PASS, MIX_IMAD_IADD3_IND,
          NOPS };
static const char* kNames[NOPS] = {"IADD3", "LOP3", "IMAD", "PRMT", "IDP.4A", "IDP.2A", "SHF",
                                   "IMAD+LOP3", "SA pass (PRMT,IMAD,IDP.2A,IDP.4A)",
                                   "IMAD | IADD3 (independent chains)"};
// opcode instructions per chain per inner step (the mixes issue several)
static const int kPerStep[NOPS] = {1, 1, 1, 1, 1, 1, 1, 2, 4, 1};

template <int OP>
__device__ __forceinline__ void step(uint32_t (&a)[kChains], uint32_t b, uint32_t c) {
#pragma unroll
    for (int i = 0; i < kChains; ++i) {
        // (IADD3 / LOP3 take a second chain as an operand so the compiler cannot fold the steps)
        if constexpr (OP == IADD3) a[i] = a[i] + a[(i + 4) & 7] + c;
        if constexpr (OP == LOP3) a[i] = (a[i] & a[(i + 4) & 7]) ^ c;
        if constexpr (OP == IMAD) a[i] = a[i] * b + c;
        if constexpr (OP == PRMT) a[i] = __byte_perm(a[i], b, 0x5140u + i);
        if constexpr (OP == IDP4A) a[i] = __dp4a(a[i], b, c);
        if constexpr (OP == IDP2A) a[i] = __dp2a_lo(a[i], b, c);
        if constexpr (OP == SHF) a[i] = __funnelshift_l(a[i], b, c);
        if constexpr (OP == MIX_IMAD_LOP3) a[i] = ((a[i] * b + c) & a[(i + 4) & 7]) ^ c;
        if constexpr (OP == MIX_IMAD_IADD3_IND) {  // even chains on the FMA pipe, odd on the ALU pipe
            if (i & 1) a[i] = a[i] + a[(i + 2) & 7] + c;
            else a[i] = a[i] * b + c;
        }
        if constexpr (OP == MIX_SA_PASS) {  // the SA pass of sa_group.cuh per position pair
            const uint32_t f2 = a[i] * 0x10001u + __byte_perm(a[i], 0u, 0x4044u);
            a[i] = __dp2a_lo(f2, b, a[i]);
            a[i] = __dp4a(a[i], 0x00010001u, c);
        }
    }
}

template <int OP>
__global__ void __launch_bounds__(512) kern(uint32_t* out, unsigned long long* clk, uint32_t seed) {
    uint32_t a[kChains];
#pragma unroll
    for (int i = 0; i < kChains; ++i) a[i] = seed * (threadIdx.x + 1) + i;
    const uint32_t b = seed ^ 0x9e3779b9u, c = seed + 7u;
    __syncthreads();
    unsigned long long t0 = 0, g0 = 0;
    if (threadIdx.x == 0) {
        asm volatile("mov.u64 %0, %%clock64;" : "=l"(t0));
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g0));
    }
#pragma unroll 1
    for (int it = 0; it < kIters; ++it) {
        step<OP>(a, b, c);
        step<OP>(a, b, c);
        step<OP>(a, b, c);
        step<OP>(a, b, c);
    }
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < kChains; ++i) s ^= a[i];
    if (s == 0x12345678u) out[blockIdx.x] = s;  // keeps the chains alive
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long t1, g1;
        asm volatile("mov.u64 %0, %%clock64;" : "=l"(t1));
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g1));
        clk[2 * blockIdx.x] = t1 - t0;
        clk[2 * blockIdx.x + 1] = g1 - g0;
    }
}

template <int OP>
void run(int sms, uint32_t* out, unsigned long long* clk) {
    const int ctas_per_sm = 4, threads = 512;  // 64 warps per SM: every SMSP has 16 to pick from
    const int blocks = sms * ctas_per_sm;
    kern<OP><<<blocks, threads>>>(out, clk, 1u);  // warm-up
    cudaDeviceSynchronize();
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    kern<OP><<<blocks, threads>>>(out, clk, 3u);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    std::vector<unsigned long long> h(2 * blocks);
    cudaMemcpy(h.data(), clk, sizeof(unsigned long long) * 2 * blocks, cudaMemcpyDeviceToHost);
    double cyc = 0, ns = 0;
    for (int i = 0; i < blocks; ++i) {
        cyc += (double)h[2 * i];
        ns += (double)h[2 * i + 1];
    }
    const double mhz = cyc / ns * 1e3;  // SM clock of the run (clock64 over globaltimer per CTA)
    // opcode warp instructions per SM over the whole launch (event time x measured clock)
    const double winstr = (double)ctas_per_sm * (threads / 32) * kIters * 4.0 * kChains * kPerStep[OP];
    const double sm_cycles = (double)ms * 1e-3 * mhz * 1e6;
    const double per_clk = winstr / sm_cycles;
    printf("{\"op\": \"%s\", \"warp_instr_per_clk_per_sm\": %.4f, \"lane_ops_per_clk_per_sm\": %.2f, "
           "\"sm_mhz\": %.0f, \"kernel_ms\": %.4f, \"tops_at_measured_clock\": %.3f}\n",
           kNames[OP], per_clk, per_clk * 32, mhz, ms, per_clk * 32 * sms * mhz * 1e6 / 1e12);
    fflush(stdout);
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    uint32_t* out;
    unsigned long long* clk;
    cudaMalloc(&out, sizeof(uint32_t) * sms * 8);
    cudaMalloc(&clk, sizeof(unsigned long long) * 2 * sms * 8);
    run<IADD3>(sms, out, clk);
    run<LOP3>(sms, out, clk);
    run<IMAD>(sms, out, clk);
    run<PRMT>(sms, out, clk);
    run<IDP4A>(sms, out, clk);
    run<IDP2A>(sms, out, clk);
    run<SHF>(sms, out, clk);
    run<MIX_IMAD_LOP3>(sms, out, clk);
    run<MIX_SA_PASS>(sms, out, clk);
    run<MIX_IMAD_IADD3_IND>(sms, out, clk);
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        fprintf(stderr, "CUDA error: %s\n", cudaGetErrorString(e));
        return 1;
    }
    return 0;
}
