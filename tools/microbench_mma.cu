// Micro-benchmark of tcgen05.mma throughput on sm_100a (B200): one CTA per SM, one thread
// issues back-to-back 128 x N x K MMAs from shared-memory operands into two TMEM
// accumulators.  Variants: kind::i8 (s32 accumulate), kind::f16 (bf16, f32 accumulate),
// kind::f8f6f4 (e4m3, f32 accumulate); operand layout K-major SWIZZLE_NONE (interleaved
// 8x16-byte core matrices) or SWIZZLE_128B.  Prints MAC/clk/SM and the aggregate rate.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/microbench_mma tools/microbench_mma.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t desc(uint32_t a, uint32_t lbo, uint32_t sbo, uint32_t layout) {
    return (uint64_t)((a >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46) | ((uint64_t)layout << 61);
}

template <int KIND>
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc) {
    if (KIND == 0)
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, 1, 0;\ntcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n}\n"
                     ::"r"(d), "l"(a), "l"(b), "r"(idesc) : "memory");
    else if (KIND == 1)
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, 1, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                     ::"r"(d), "l"(a), "l"(b), "r"(idesc) : "memory");
    else
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, 1, 0;\ntcgen05.mma.cta_group::1.kind::f8f6f4 [%0], %1, %2, %3, p;\n}\n"
                     ::"r"(d), "l"(a), "l"(b), "r"(idesc) : "memory");
}

// KIND 0 = i8, 1 = bf16, 2 = e4m3; SW 0 = none, 1 = 128B swizzle
template <int KIND, int SW>
__global__ void __launch_bounds__(128, 1) kern(int iters, int N, unsigned long long* clk) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t bar;
    __shared__ uint32_t slot;
    uint8_t* A = sm;                 // 128 rows x 128 bytes
    uint8_t* B = sm + 128 * 128;     // 256 rows x 128 bytes
    for (int i = threadIdx.x; i < (128 + 256) * 128 / 16; i += blockDim.x)
        reinterpret_cast<uint4*>(sm)[i] = make_uint4(0x01010101u * (i & 3), 0, 0x01000100u, 0);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&slot)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tm = slot;
    if (threadIdx.x == 0) {
        uint32_t idesc;
        if (KIND == 0) idesc = (2u << 4) | (1u << 7) | (1u << 10);
        else if (KIND == 1) idesc = (1u << 4) | (1u << 7) | (1u << 10);
        else idesc = (1u << 4);
        idesc |= ((uint32_t)(N >> 3) << 17) | ((128u >> 4) << 24);
        const uint32_t a0 = su32(A), b0 = su32(B);
        unsigned long long t0 = clock64();
        for (int it = 0; it < iters; it++) {
#pragma unroll
            for (int ks = 0; ks < 4; ks++) {   // 4 K-steps of 32 bytes = one 128-byte row
                uint64_t ad, bd;
                if (SW == 0) {   // interleaved: k-step = 2 core matrices (LBO 128), SBO = 8 rows x 128 B
                    ad = desc(a0 + ks * 256, 128, 1024, 0);
                    bd = desc(b0 + ks * 256, 128, 1024, 0);
                } else {         // 128B swizzle: rows of 128 B, 8-row atoms of 1024 B, k-step = +32 B
                    ad = desc(a0 + ks * 32, 16, 1024, 2);
                    bd = desc(b0 + ks * 32, 16, 1024, 2);
                }
                mma<KIND>(tm + (it & 1) * 256, ad, bd, idesc);
            }
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)) : "memory");
        asm volatile("{\n.reg .pred P1;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n@!P1 bra W;\n}\n" ::"r"(su32(&bar)) : "memory");
        unsigned long long t1 = clock64();
        clk[blockIdx.x] = t1 - t0;
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tm) : "memory");
    }
}

template <int KIND, int SW>
int run(const char* name, int N, int sms) {
    const int iters = 20000;
    unsigned long long* d;
    CK(cudaMalloc(&d, sms * 8));
    auto fn = kern<KIND, SW>;
    const int smem = (128 + 256) * 128;
    CK(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    fn<<<sms, 128, smem>>>(100, N, d);
    CK(cudaDeviceSynchronize());
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    fn<<<sms, 128, smem>>>(iters, N, d);
    cudaEventRecord(e1);
    CK(cudaDeviceSynchronize());
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    unsigned long long h[1024]; CK(cudaMemcpy(h, d, sms * 8, cudaMemcpyDeviceToHost));
    double avg = 0; for (int i = 0; i < sms; i++) avg += h[i]; avg /= sms;
    const double kbytes = 128;   // K bytes per row per iteration
    const double k_elems = KIND == 1 ? kbytes / 2 : kbytes;
    const double macs = (double)iters * 128 * N * k_elems;
    printf("%-22s N=%3d  %8.3f ms  %7.1f MAC/clk/SM  %7.1f TOPS(2*MAC) agg  clk~%4.0f MHz\n", name, N, ms,
           macs / avg, 2 * macs * sms / (ms * 1e-3) / 1e12, avg / (ms * 1e-3) / 1e6);
    cudaFree(d);
    return 0;
}


// TMEM read throughput: W warps (W/4 per lane quarter) repeatedly load 32-column chunks
// (tcgen05.ld 32x32b.xC) and wait; bytes moved = 32 lanes x C cols x 4 B per warp-load.
template <int C, int INFLIGHT>
__global__ void __launch_bounds__(512, 1) tmem_rd(int iters, unsigned long long* clk, int* sink) {
    __shared__ uint32_t slot;
    const int warp = threadIdx.x >> 5;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&slot)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tm = slot + (((uint32_t)(warp & 3) * 32u) << 16);
    uint32_t acc = 0;
    unsigned long long t0 = clock64();
    for (int it = 0; it < iters; it++) {
        uint32_t v[INFLIGHT][C];
#pragma unroll
        for (int f = 0; f < INFLIGHT; f++) {
            const uint32_t col = (uint32_t)(((it * INFLIGHT + f) * C + (warp >> 2) * 64) & 511);
            if (C == 32)
                asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
                    : "=r"(v[f][0]), "=r"(v[f][1]), "=r"(v[f][2]), "=r"(v[f][3]), "=r"(v[f][4]), "=r"(v[f][5]), "=r"(v[f][6]), "=r"(v[f][7]),
                      "=r"(v[f][8]), "=r"(v[f][9]), "=r"(v[f][10]), "=r"(v[f][11]), "=r"(v[f][12]), "=r"(v[f][13]), "=r"(v[f][14]), "=r"(v[f][15]),
                      "=r"(v[f][16]), "=r"(v[f][17]), "=r"(v[f][18]), "=r"(v[f][19]), "=r"(v[f][20]), "=r"(v[f][21]), "=r"(v[f][22]), "=r"(v[f][23]),
                      "=r"(v[f][24]), "=r"(v[f][25]), "=r"(v[f][26]), "=r"(v[f][27]), "=r"(v[f][28]), "=r"(v[f][29]), "=r"(v[f][30]), "=r"(v[f][31])
                    : "r"(tm + col));
        }
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
        for (int f = 0; f < INFLIGHT; f++)
#pragma unroll
            for (int i = 0; i < C; i++) acc ^= v[f][i];
    }
    unsigned long long t1 = clock64();
    if ((threadIdx.x & 31) == 0) clk[blockIdx.x * 16 + warp] = t1 - t0;
    if (acc == 0x12345) sink[0] = acc;
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot) : "memory");
    }
}

template <int C, int INFLIGHT>
int run_tmem(int warps, int sms) {
    const int iters = 20000;
    unsigned long long* d; int* sink;
    CK(cudaMalloc(&d, sms * 16 * 8)); CK(cudaMalloc(&sink, 4));
    tmem_rd<C, INFLIGHT><<<sms, warps * 32>>>(100, d, sink);
    CK(cudaDeviceSynchronize());
    tmem_rd<C, INFLIGHT><<<sms, warps * 32>>>(iters, d, sink);
    CK(cudaDeviceSynchronize());
    unsigned long long h[148 * 16]; CK(cudaMemcpy(h, d, sms * 16 * 8, cudaMemcpyDeviceToHost));
    double mx = 0; for (int i = 0; i < sms; i++) for (int w = 0; w < warps; w++) mx = h[i * 16 + w] > mx ? h[i * 16 + w] : mx;
    const double bytes = (double)iters * INFLIGHT * warps * 32 * C * 4;
    printf("tmem read: %2d warps, x%d, %d in flight: %7.1f B/clk/SM  (%6.1f cycles per warp-load)\n", warps, C, INFLIGHT,
           bytes / mx, mx / iters / INFLIGHT);
    cudaFree(d); cudaFree(sink);
    return 0;
}

// Commit cost: groups of G i8 MMAs (128 x N x 32) each followed by tcgen05.commit to one of
// 4 mbarriers.  WAIT=0: nobody waits (throughput); WAIT=1: the issuing thread waits for
// every commit before the next group (issue-to-completion latency).
template <int WAIT>
__global__ void __launch_bounds__(128, 1) commit_k(int iters, int N, int G, unsigned long long* clk, int accmode = 0) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t bar[4];
    __shared__ uint32_t slot;
    for (int i = threadIdx.x; i < (128 + 256) * 128 / 16; i += blockDim.x)
        reinterpret_cast<uint4*>(sm)[i] = make_uint4(0x01010101u * (i & 3), 0, 0x01000100u, 0);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (threadIdx.x == 0) {
        for (int i = 0; i < 4; i++) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[i])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(&slot)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tm = slot;
    if (threadIdx.x == 0) {
        const uint32_t idesc = (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((128u >> 4) << 24);
        const uint32_t a0 = su32(sm), b0 = su32(sm + 128 * 128);
        unsigned long long t0 = clock64();
        for (int it = 0; it < iters; it++) {
            const int st = it & 3;
            for (int gI = 0; gI < G; gI++) {
                const uint64_t ad = desc(a0 + (gI & 3) * 256, 128, 1024, 0);
                const uint64_t bd = desc(b0 + (gI & 3) * 256, 128, 1024, 0);
                const uint32_t dcol = accmode == 0 ? (uint32_t)((it % (512 / N)) * N) : accmode == 1 ? 0u : (uint32_t)((it & 1) * 256);
                mma<0>(tm + dcol, ad, bd, idesc);
            }
            if (WAIT >= 0) asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar[st])) : "memory");
            if (WAIT == 1) {
                const uint32_t par = (uint32_t)(it >> 2) & 1u;
                asm volatile("{\n.reg .pred P1;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@!P1 bra W;\n}\n" ::"r"(su32(&bar[st])), "r"(par) : "memory");
            }
        }
        if (WAIT < 0) asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar[0])) : "memory");
        // drain: wait for the last commit of every barrier
        for (int st = 0; st < 4 && st < iters && WAIT >= 0; st++) {
            const int last = ((iters - 1 - st) / 4) * 4 + st;
            const uint32_t par = (uint32_t)(last >> 2) & 1u;
            asm volatile("{\n.reg .pred P1;\nW2:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@!P1 bra W2;\n}\n" ::"r"(su32(&bar[st])), "r"(par) : "memory");
        }
        if (WAIT < 0) asm volatile("{\n.reg .pred P1;\nW3:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n@!P1 bra W3;\n}\n" ::"r"(su32(&bar[0])) : "memory");
        unsigned long long t1 = clock64();
        clk[blockIdx.x] = t1 - t0;
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tm) : "memory");
    }
}

template <int WAIT>
int run_commit(int N, int G, int sms, int accmode = 0) {
    const int iters = WAIT ? 2000 : 20000;
    unsigned long long* d;
    CK(cudaMalloc(&d, sms * 8));
    const int smem = (128 + 256) * 128;
    CK(cudaFuncSetAttribute(commit_k<WAIT>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    commit_k<WAIT><<<sms, 128, smem>>>(100, N, G, d);
    CK(cudaDeviceSynchronize());
    commit_k<WAIT><<<sms, 128, smem>>>(iters, N, G, d, accmode);
    CK(cudaDeviceSynchronize());
    unsigned long long h[1024]; CK(cudaMemcpy(h, d, sms * 8, cudaMemcpyDeviceToHost));
    double avg = 0; for (int i = 0; i < sms; i++) avg += h[i]; avg /= sms;
    printf("acc%d i8 N=%3d, %2d MMA(K=32) per group, %-17s: %7.1f cycles per group (ideal %5.1f)\n", accmode, N, G,
           WAIT == 1 ? "commit+wait" : WAIT == 0 ? "commit, no wait" : "no commit", avg / iters, 128.0 * N * 32 * G / 8192.0);
    cudaFree(d);
    return 0;
}

int main() {
    int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int am : {0, 1, 2}) for (int G : {2, 4}) {
        run_commit<-1>(128, G, sms, am);
        run_commit<0>(128, G, sms, am);
    }
    run_commit<-1>(256, 2, sms);
    run_commit<0>(256, 2, sms);
    run_commit<1>(256, 2, sms);
    if (getenv("MB_ALL") == nullptr) return 0;
    run_tmem<32, 1>(4, sms);
    run_tmem<32, 2>(4, sms);
    run_tmem<32, 1>(8, sms);
    run_tmem<32, 2>(8, sms);
    run_tmem<32, 1>(16, sms);
    run_tmem<32, 2>(16, sms);
    for (int N : {128, 256}) {
        run<0, 0>("i8    no-swizzle", N, sms);
        run<0, 1>("i8    swizzle128", N, sms);
        run<1, 0>("bf16  no-swizzle", N, sms);
        run<1, 1>("bf16  swizzle128", N, sms);
        run<2, 0>("e4m3  no-swizzle", N, sms);
        run<2, 1>("e4m3  swizzle128", N, sms);
    }
    return 0;
}
