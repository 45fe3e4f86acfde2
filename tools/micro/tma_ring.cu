// Microbenchmark: per-CTA TMA ring (cp.async.bulk + mbarrier), persistent grid, to find the
// stage size / depth / copy count that streams HBM at full rate on B200.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_ring tma_ring.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned su(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(unsigned long long* b, unsigned c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su(b)), "r"(c) : "memory"); }
__device__ __forceinline__ void mb_tx(unsigned long long* b, unsigned n) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(b)), "r"(n) : "memory"); }
__device__ __forceinline__ void mb_arrive(unsigned long long* b) { asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su(b)) : "memory"); }
__device__ __forceinline__ void mb_wait(unsigned long long* b, unsigned ph) {
    asm volatile("{\n .reg .pred p;\n W%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W%=;\n}" ::"r"(su(b)), "r"(ph) : "memory");
}
__device__ __forceinline__ void bulk(void* d, const void* s, unsigned n, unsigned long long* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su(d)), "l"(s), "r"(n), "r"(su(b)) : "memory");
}

// mode 0: thread 0 refills after all warps consumed (empty barrier);  consumers sum one double per thread
__global__ void ring(const unsigned char* src, size_t per_cta, int nst, int sbytes, int ncopy, double* out, int lanes) {
    extern __shared__ __align__(16) unsigned char sm[];
    unsigned long long* full = reinterpret_cast<unsigned long long*>(sm + (size_t)nst * sbytes);
    unsigned long long* empty = full + nst;
    const int t = threadIdx.x;
    if (t == 0) { for (int s = 0; s < nst; ++s) { mb_init(&full[s], 1); mb_init(&empty[s], blockDim.x / 32); } asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
    __syncthreads();
    const unsigned char* base = src + (size_t)blockIdx.x * per_cta;
    const int ns = (int)(per_cta / sbytes);
    const unsigned cb = sbytes / ncopy;
    auto issue = [&](int k) {   // called by lanes [0, lanes) of warp 0
        int s = k % nst;
        if (t == 0) mb_tx(&full[s], sbytes);
        __syncwarp((1u << lanes) - 1);
        for (int c = t; c < ncopy; c += lanes) bulk(sm + (size_t)s * sbytes + c * cb, base + (size_t)k * sbytes + c * cb, cb, &full[s]);
    };
    if (t < lanes) for (int k = 0; k < nst && k < ns; ++k) issue(k);
    double acc = 0;
    for (int k = 0; k < ns; ++k) {
        int s = k % nst; unsigned ph = (k / nst) & 1;
        mb_wait(&full[s], ph);
        acc += reinterpret_cast<const double*>(sm + (size_t)s * sbytes)[t % (sbytes / 8)];
        __syncwarp();
        if ((t & 31) == 0) mb_arrive(&empty[s]);
        if (t < lanes && k + nst < ns) { mb_wait(&empty[s], ph); issue(k + nst); }
    }
    if (acc == 12345.678) out[0] = acc;
}


// cooperative cp.async (LDGSTS 16 B per thread) multistage ring with __syncthreads per stage
__global__ void ring_cpasync(const unsigned char* src, size_t per_cta, int nst, int sbytes, double* out) {
    extern __shared__ __align__(16) unsigned char sm[];
    const int t = threadIdx.x, B = blockDim.x;
    const unsigned char* base = src + (size_t)blockIdx.x * per_cta;
    const int ns = (int)(per_cta / sbytes);
    auto issue = [&](int k) {
        int s = k % nst;
        for (int o = t * 16; o < sbytes; o += B * 16)
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su(sm + (size_t)s * sbytes + o)), "l"(base + (size_t)k * sbytes + o) : "memory");
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    for (int k = 0; k < nst - 1; ++k) issue(k);
    double acc = 0;
    for (int k = 0; k < ns; ++k) {
        if (k + nst - 1 < ns) issue(k + nst - 1); else asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group 2;" :: : "memory");   // conservative; replaced below
        __syncthreads();
        acc += reinterpret_cast<const double*>(sm + (size_t)(k % nst) * sbytes)[t % (sbytes / 8)];
        __syncthreads();
    }
    if (acc == 12345.678) out[0] = acc;
}
int main() {
    int G = 148, B = 512;
    size_t per_cta = 64ull << 20 >> 4;   // 4 MiB per CTA -> 592 MiB total
    unsigned char* src; double* out;
    cudaMalloc(&src, per_cta * G); cudaMalloc(&out, 8);
    cudaMemset(src, 1, per_cta * G);
    cudaFuncSetAttribute(ring, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
    int cfg[][3] = {{2, 16384, 1}, {4, 16384, 1}, {8, 16384, 1}, {4, 32768, 1}, {6, 32768, 1}, {3, 65536, 1},
                    {4, 16384, 4}, {4, 16384, 8}, {8, 16384, 8}, {6, 32768, 8}, {12, 16384, 1}, {12, 16384, 8}, {24, 8192, 4}};
    for (int lanes : {1, 8})
    for (auto& c : cfg) {
        int nst = c[0], sb = c[1], nc = c[2];
        if (lanes > 1 && nc < 4) continue;
        size_t smem = (size_t)nst * sb + 16 * nst;
        if (smem > 220 * 1024) continue;
        cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
        for (int r = 0; r < 2; ++r) ring<<<G, B, smem>>>(src, per_cta, nst, sb, nc, out, lanes);
        cudaEventRecord(a);
        for (int r = 0; r < 5; ++r) ring<<<G, B, smem>>>(src, per_cta, nst, sb, nc, out, lanes);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        printf("lanes=%d nst=%2d stage=%6d copies=%d in-flight=%4zu KB: %7.1f GB/s  (%s)\n", (size_t)nst * sb / 1024,
               5.0 * per_cta * G / (ms / 1e3) / 1e9, cudaGetErrorString(cudaGetLastError()));
    }
    cudaFuncSetAttribute(ring_cpasync, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
    for (int nst : {3, 4, 6}) for (int sb : {16384, 32768}) {
        size_t smem = (size_t)nst * sb; if (smem > 220 * 1024) continue;
        cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
        ring_cpasync<<<G, B, smem>>>(src, per_cta, nst, sb, out);
        cudaEventRecord(a);
        for (int r = 0; r < 5; ++r) ring_cpasync<<<G, B, smem>>>(src, per_cta, nst, sb, out);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        printf("cp.async nst=%d stage=%d: %7.1f GB/s (%s)\n", nst, sb, 5.0 * per_cta * G / (ms / 1e3) / 1e9, cudaGetErrorString(cudaGetLastError()));
    }
    return 0;
}
