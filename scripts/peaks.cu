// peaks.cu — the two peak microbenchmarks SURVEY.md §8(d) asks for before quoting a roofline:
//   (1) LOP3 issue rate: 148 x 8 blocks x 256 threads, 8 independent u32 chains per thread of
//       x = lop3(x, y, z) (opaque inline PTX so the compiler cannot fold it), unrolled, looped.
//       LOP3/clk/SM is taken from the SM's own clock64 (per-SM first start .. last end), so it does
//       not depend on the clock the GPU happened to run at; the rate per second uses CUDA events.
//   (2) Streaming HBM: c[i] = a[i] & b[i] over uint4 (2 reads + 1 write, the traffic shape of the
//       paper's simulation table, 12 B per node-word), 3 x 2.67 GiB.
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o peaks scripts/peaks.cu
// Prints one JSON line. Measurement tooling only (not part of libcec).
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

#define CK(x)                                                                         \
    do {                                                                              \
        cudaError_t e_ = (x);                                                         \
        if (e_ != cudaSuccess) {                                                      \
            fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
            return 1;                                                                 \
        }                                                                             \
    } while (0)

__device__ __forceinline__ uint32_t lop3(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t r;
    asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
    return r;
}

__device__ __forceinline__ unsigned smid() {
    unsigned r;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
    return r;
}

constexpr int CHAINS = 8, UNROLL = 64;

__global__ void __launch_bounds__(256) lop3_peak(uint32_t *out, int iters, unsigned long long *sm_t0,
                                                  unsigned long long *sm_t1) {
    uint32_t x[CHAINS];
    const uint32_t y = threadIdx.x * 0x9E3779B9u, z = blockIdx.x * 0x85EBCA6Bu;
    for (int c = 0; c < CHAINS; ++c) x[c] = threadIdx.x + c;
    __syncthreads();
    const unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int u = 0; u < UNROLL; ++u)
#pragma unroll
            for (int c = 0; c < CHAINS; ++c) x[c] = lop3(x[c], y, z);
    }
    __syncthreads();
    const unsigned long long t1 = clock64();
    uint32_t acc = 0;
    for (int c = 0; c < CHAINS; ++c) acc ^= x[c];
    if (acc == 0x12345678u) out[0] = acc;  // keeps the chains live
    if (threadIdx.x == 0) {
        const unsigned s = smid();
        atomicMin(&sm_t0[s], t0);
        atomicMax(&sm_t1[s], t1);
    }
}

__global__ void stream_and(const uint4 *__restrict__ a, const uint4 *__restrict__ b, uint4 *__restrict__ c, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        const uint4 p = a[i], q = b[i];
        c[i] = make_uint4(p.x & q.x, p.y & q.y, p.z & q.z, p.w & q.w);
    }
}

int main() {
    cudaDeviceProp prop;
    CK(cudaGetDeviceProperties(&prop, 0));
    const int sms = prop.multiProcessorCount;
    int clk_khz = 0;
    CK(cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0));
    // ---- (1) LOP3 ----
    const int blocks = sms * 8, threads = 256, iters = 2000;
    uint32_t *out;
    unsigned long long *t0, *t1;
    CK(cudaMalloc(&out, 4));
    CK(cudaMalloc(&t0, 8 * 1024));
    CK(cudaMalloc(&t1, 8 * 1024));
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    lop3_peak<<<blocks, threads>>>(out, 50, t0, t1);  // warm-up
    CK(cudaDeviceSynchronize());
    double best_rate = 0, best_per_clk = 0, best_mhz = 0, best_ms = 0;
    for (int rep = 0; rep < 5; ++rep) {
        CK(cudaMemset(t0, 0xFF, 8 * 1024));
        CK(cudaMemset(t1, 0, 8 * 1024));
        CK(cudaEventRecord(e0));
        lop3_peak<<<blocks, threads>>>(out, iters, t0, t1);
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, e0, e1));
        std::vector<unsigned long long> h0(1024), h1(1024);
        CK(cudaMemcpy(h0.data(), t0, 8 * 1024, cudaMemcpyDeviceToHost));
        CK(cudaMemcpy(h1.data(), t1, 8 * 1024, cudaMemcpyDeviceToHost));
        const double ops = (double)blocks * threads * iters * UNROLL * CHAINS;
        double cyc = 0;
        int n = 0;
        for (int s = 0; s < 1024; ++s)
            if (h1[s] > 0 && h0[s] != ~0ull) {
                cyc += (double)(h1[s] - h0[s]);
                ++n;
            }
        cyc /= n;  // mean per-SM busy cycles
        const double per_clk = ops / n / cyc;
        const double rate = ops / (ms * 1e-3);
        if (rate > best_rate) {
            best_rate = rate;
            best_per_clk = per_clk;
            best_mhz = cyc / (ms * 1e-3) / 1e6;
            best_ms = ms;
        }
    }
    // ---- (2) streaming 2R+1W ----
    const size_t n4 = (size_t)(8ull << 30) / 3 / sizeof(uint4);
    uint4 *a, *b, *c;
    CK(cudaMalloc(&a, n4 * sizeof(uint4)));
    CK(cudaMalloc(&b, n4 * sizeof(uint4)));
    CK(cudaMalloc(&c, n4 * sizeof(uint4)));
    CK(cudaMemset(a, 0x5A, n4 * sizeof(uint4)));
    CK(cudaMemset(b, 0x3C, n4 * sizeof(uint4)));
    const int sgrid = sms * 8, sthreads = 512;
    stream_and<<<sgrid, sthreads>>>(a, b, c, n4);
    CK(cudaDeviceSynchronize());
    double best_gbs = 0;
    for (int rep = 0; rep < 5; ++rep) {
        CK(cudaEventRecord(e0));
        stream_and<<<sgrid, sthreads>>>(a, b, c, n4);
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, e0, e1));
        const double gbs = 3.0 * n4 * sizeof(uint4) / (ms * 1e-3) / 1e9;
        if (gbs > best_gbs) best_gbs = gbs;
    }
    printf("{\"device\": \"%s\", \"sms\": %d, \"max_sm_mhz\": %.0f, "
           "\"lop3\": {\"per_clk_per_sm\": %.2f, \"tlop3_per_s\": %.3f, \"sm_mhz_during\": %.0f, \"ms\": %.3f, "
           "\"blocks\": %d, \"threads\": %d, \"chains\": %d}, "
           "\"stream_2r1w\": {\"gbs\": %.1f, \"bytes\": %zu}}\n",
           prop.name, sms, clk_khz / 1e3, best_per_clk, best_rate / 1e12, best_mhz, best_ms, blocks, threads, CHAINS,
           best_gbs, 3 * n4 * sizeof(uint4));
    return 0;
}
