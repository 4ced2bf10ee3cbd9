// Micro-benchmark of the integer pipes the comparer binds on (sm_100a).
// Measures warp-instruction throughput of POPC, LOP3 and the comparer's inner-loop mix.
// Output: one line per variant with ops/clk/SM, using the measured SM clock
// (CTA 0's clock64 delta over its own globaltimer delta: the SM clock while it ran).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ uint32_t lop3_xor_or(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t d; asm volatile("lop3.b32 %0, %1, %2, %3, 0xBE;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; // (a^b)|c
}
__device__ __forceinline__ uint32_t lop3_or_xor(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t d; asm volatile("lop3.b32 %0, %1, %2, %3, 0xF6;" : "=r"(d) : "r"(a), "r"(b), "r"(c)); return d; // a|(b^c)
}

// Variant 0: POPC only; 8 independent chains, each iteration x = popc(x) + x (IADD)... use popc into acc via IADD3-free: acc ^= popc
template <int V>
__global__ void kern(const uint32_t* __restrict__ in, uint32_t* out, int iters, unsigned long long* clk) {
    uint32_t r[8];
    for (int i = 0; i < 8; i++) r[i] = in[(threadIdx.x + i) & 255] + blockIdx.x;
    uint32_t g0 = in[300], g1 = in[301], nt = in[302];
    uint32_t acc = 0;
    unsigned long long t0 = clock64(), gt0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt0));
    if (V == 0) {          // POPC throughput: popc on 8 independent values per iter, values perturbed by one LOP3 every 4 iters
        uint32_t s[8] = {0,0,0,0,0,0,0,0};
        for (int it = 0; it < iters; it++) {
#pragma unroll
            for (int i = 0; i < 8; i++) s[i] += __popc(r[i] ^ it);
        }
        for (int i = 0; i < 8; i++) acc += s[i];
    } else if (V == 1) {   // LOP3 throughput: 8 independent chains of lop3
        for (int it = 0; it < iters; it++) {
#pragma unroll
            for (int i = 0; i < 8; i++) r[i] = lop3_xor_or(r[i], g0, g1);
#pragma unroll
            for (int i = 0; i < 8; i++) r[i] = lop3_or_xor(r[i], g1, g0);
        }
        for (int i = 0; i < 8; i++) acc ^= r[i];
    } else if (V == 2) {   // comparer mix: 2 LOP3 + POPC + IADD per comparison, OR-reduce sign, 8 items
        uint32_t wl[8], wh[8], wn[8];
        for (int i = 0; i < 8; i++) { wl[i] = r[i]; wh[i] = r[i] * 3u; wn[i] = r[i] & 0x100u; }
        for (int it = 0; it < iters; it++) {
            uint32_t gl = g0 ^ it, gh = g1 + it;
            int32_t d[8];
#pragma unroll
            for (int i = 0; i < 8; i++) {
                uint32_t y = lop3_or_xor(lop3_xor_or(wl[i], gl, wn[i]), wh[i], gh);
                d[i] = (int32_t)__popc(y) + (int32_t)nt;
            }
            int32_t o = (d[0] | d[1] | d[2] | d[3]) | (d[4] | d[5] | d[6] | d[7]);
            if (o < 0) acc += 1;
        }
    } else if (V == 3) {   // same mix with popc replaced by a LOP (alu bound only)
        uint32_t wl[8], wh[8], wn[8];
        for (int i = 0; i < 8; i++) { wl[i] = r[i]; wh[i] = r[i] * 3u; wn[i] = r[i] & 0x100u; }
        for (int it = 0; it < iters; it++) {
            uint32_t gl = g0 ^ it, gh = g1 + it;
            int32_t d[8];
#pragma unroll
            for (int i = 0; i < 8; i++) {
                uint32_t y = lop3_or_xor(lop3_xor_or(wl[i], gl, wn[i]), wh[i], gh);
                d[i] = (int32_t)(y >> 27) + (int32_t)nt;
            }
            int32_t o = (d[0] | d[1] | d[2] | d[3]) | (d[4] | d[5] | d[6] | d[7]);
            if (o < 0) acc += 1;
        }
    }
    unsigned long long t1 = clock64(), gt1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt1));
    if (threadIdx.x == 0 && blockIdx.x == 0) { clk[0] = t1 - t0; clk[1] = gt1 - gt0; }
    if (acc == 0x12345678u) out[0] = acc;
}

int main() {
    int dev = 0; cudaDeviceProp prop; CK(cudaGetDeviceProperties(&prop, dev));
    int sms = prop.multiProcessorCount;
    uint32_t* in; uint32_t* out; unsigned long long* clk;
    CK(cudaMalloc(&in, 4096)); CK(cudaMalloc(&out, 64)); CK(cudaMalloc(&clk, 16));
    uint32_t h[1024]; for (int i = 0; i < 1024; i++) h[i] = 0x9E3779B9u * (i + 1);
    h[302] = (uint32_t)-7;  // nt = -(t+1), t = 6
    CK(cudaMemcpy(in, h, 4096, cudaMemcpyHostToDevice));
    const char* names[4] = {"popc x8 (+IADD)", "lop3 x16", "comparer mix 2LOP3+POPC+ADD", "mix without POPC"};
    for (int v = 0; v < 4; v++) {
        for (int rep = 0; rep < 2; rep++) {
            int iters = 20000, threads = 256, blocks = sms * 8;
            CK(cudaMemset(clk, 0, 16));
            cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
            cudaEventRecord(a);
            if (v == 0) kern<0><<<blocks, threads>>>(in, out, iters, clk);
            if (v == 1) kern<1><<<blocks, threads>>>(in, out, iters, clk);
            if (v == 2) kern<2><<<blocks, threads>>>(in, out, iters, clk);
            if (v == 3) kern<3><<<blocks, threads>>>(in, out, iters, clk);
            cudaEventRecord(b); CK(cudaEventSynchronize(b));
            float ms; cudaEventElapsedTime(&ms, a, b);
            unsigned long long c[2]; CK(cudaMemcpy(c, clk, 16, cudaMemcpyDeviceToHost));
            double mhz = (double)c[0] / (double)c[1] * 1e3;   // cycles per ns of CTA 0 -> MHz
            double units = (double)blocks * threads * iters;  // loop iterations (per thread)
            double per_iter_ops = (v == 0) ? 8 : (v == 1) ? 16 : 8;  // popcs / lop3s / comparisons
            double rate = units * per_iter_ops / (ms * 1e-3);
            double per_clk_sm = rate / (mhz * 1e6) / sms;
            if (rep == 1)
                printf("%-32s %8.3f ms  %.3e ops/s  sm_clk~%.0f MHz  %.2f ops/clk/SM\n", names[v], ms, rate, mhz, per_clk_sm);
        }
    }
    return 0;
}
