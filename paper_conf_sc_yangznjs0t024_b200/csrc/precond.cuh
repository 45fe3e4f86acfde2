// precond.cuh -- ILU(0) factors on the device and the sync-free triangular solve.
#pragma once

#include <vector>

#include "mf_internal.cuh"

namespace mf {

struct TriCSR {
    int64_t* rp = nullptr;
    int32_t* ci = nullptr;
    double* v = nullptr;
};

// Recursive block SpTRSV (the algorithm of [41]; oracle rb_lower / rb_upper, reading R27):
// the triangle of rows [lo, hi) splits at mid = lo + 16 * floor((hi - lo) / 32) into two triangles
// and one square block, down to `depth` levels (or fewer than 32 rows).  The nodes are stored in
// execution order: lower  = solve(lo, mid), square rows [mid, hi) x cols [lo, mid), solve(mid, hi);
// upper = solve(mid, hi), square rows [lo, mid) x cols [mid, hi), solve(lo, mid).  Each node owns a
// CSR slice of the factor: a leaf the entries with both row and column inside it (columns stored
// relative to r0, so the leaf is a standalone triangular solve), a square the entries of its
// rectangle (global columns).
struct RbNode {
    int64_t r0, r1;      // rows [r0, r1)
    int64_t rp_off;      // first of the node's (r1 - r0 + 1) row pointers in the tree's rp array
    int32_t leaf;        // 1 triangle, 0 square block
    int32_t leaf_idx;    // leaves: ordinal among the tree's leaves; squares: -1
};
struct RbTree {
    RbNode* nodes = nullptr;       // device copy
    std::vector<RbNode> h;         // host copy (execution order)
    int64_t* rp = nullptr;
    int32_t* ci = nullptr;
    double* v = nullptr;
    int nleaves = 0;
};

struct Precond {
    int64_t n = 0;
    int rb_depth = 0;             // 0: sync-free substitution; > 0: recursive block SpTRSV
    RbTree Lrb, Urb;
    TriCSR L, U;                  // L: strict lower part (unit diagonal implied); U: strict upper part
    double* udiag = nullptr;      // u_ii
    unsigned* flags = nullptr;    // [n+1] row-ready epochs (forward 2e+1, backward 2e+2)
    unsigned long long* ctr = nullptr;   // chunk-grab counters
    double *y = nullptr, *z = nullptr;   // workspace of mf_precond_apply / the solvers
    int64_t nnz_l = 0, nnz_u = 0;
    unsigned epoch = 0;           // applies issued so far (host side bookkeeping)
    unsigned long long grabs = 0;
    cudaStream_t owner_stream = nullptr;
};

mf_status build_precond(const TileMatrix& A, int rb_depth, cudaStream_t s, Precond* P);
void destroy_precond(Precond* P);
mf_status run_precond_apply(Precond& P, const double* r, double* z, cudaStream_t s);

}  // namespace mf

struct mf_precond {
    mf::Precond p;
};

namespace mfk {

__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u32(unsigned* p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Sync-free chunked triangular solve, called by all threads of a CTA (any number of CTAs).
//   FWD:  out_i = in_i - sum_{k<i} T_ik out_k                 rows ascending
//   !FWD: out_i = (in_i - sum_{k>i} T_ik out_k) / diag_i       rows descending
// Chunks of blockDim.x consecutive rows (in solve order) are grabbed with one atomicAdd on
// *ctr (values base, base+1, ...), so a chunk only waits on chunks grabbed earlier or on
// earlier rows of its own chunk: deadlock-free without co-residency.  Inside a chunk a row
// waits on a shared-memory flag; across chunks on the global row flag.
// Flag values are epochs that only grow (forward 2e+1 < backward 2e+2 < next forward ...), so
// every wait is ">=": a row whose flag already moved on to a later solve of the same apply (the
// backward solve of a nonsymmetric pattern can finish row k before a forward row that reads it)
// never blocks a reader.  wait_val != 0: row i additionally waits for flags[i] >= wait_val
// before reading in_i (the backward solve waits for the forward solve of the same row).
// OUTPV: out is in the PV layout (kernels.cuh) -- the SpMV input of the preconditioned solvers.
// Every spin has a watchdog: after timeout_ns (or when another CTA raised *abort_flag) the
// thread stops waiting, raises *abort_flag and the caller reports MF_ERR_DEADLOCK.
// Every CTA performs exactly one failing grab, so one solve consumes ceil(n/B) + (number of
// CTAs) counter values.
__device__ __forceinline__ unsigned long long sp_timer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// spin until *f >= v; false on watchdog / abort
__device__ __forceinline__ bool sp_wait_flag(const unsigned* f, unsigned v, int* abort_flag, unsigned long long t0,
                                             unsigned long long timeout_ns) {
    if (ld_acquire_u32(f) >= v) return true;
    for (unsigned k = 0;; ++k) {
        if (ld_acquire_u32(f) >= v) return true;
        if ((k & 63u) == 63u) {
            if (*(volatile int*)abort_flag) return false;
            if (sp_timer() - t0 > timeout_ns) { atomicExch(abort_flag, 1); return false; }
        }
    }
}
template <bool FWD, bool OUTPV>
__device__ void sptrsv_chunked(const int64_t* __restrict__ rp, const int32_t* __restrict__ ci,
                               const double* __restrict__ val, const double* __restrict__ diag, int64_t n,
                               const double* in, double* out, unsigned* flags, unsigned flag_val, unsigned wait_val,
                               unsigned long long* ctr, unsigned long long base, double* ys, volatile int* ready,
                               long long* s_chunk, int* abort_flag, unsigned long long timeout_ns) {
    const int B = blockDim.x, t = threadIdx.x;
    const int64_t nchunks = (n + B - 1) / B;
    const unsigned long long t0 = sp_timer();
    auto oidx = [](int64_t i) -> int64_t { return OUTPV ? ((i >> 4) * 18 + (i & 15)) : i; };
    while (true) {
        __syncthreads();
        if (t == 0) *s_chunk = (long long)(atomicAdd(ctr, 1ull) - base);
        ready[t] = 0;
        __syncthreads();
        const int64_t c = *s_chunk;
        if (c >= nchunks) break;
        const int64_t pos = c * B + t;                 // position in solve order
        if (pos < n) {
            const int64_t i = FWD ? pos : n - 1 - pos;
            if (wait_val) sp_wait_flag(&flags[i], wait_val, abort_flag, t0, timeout_ns);
            double acc = __ldcg(in + i);
            const int64_t lo = rp[i], hi = rp[i + 1];
            for (int64_t q = lo; q < hi; ++q) {
                const int64_t k = ci[q];
                const int64_t pk = FWD ? k : n - 1 - k;     // position of k in solve order (< pos)
                double xk;
                if (pk >= c * B) {
                    const int lk = (int)(pk - c * B);
                    for (unsigned sp = 0; ready[lk] == 0; ++sp)
                        if ((sp & 255u) == 255u && (*(volatile int*)abort_flag || sp_timer() - t0 > timeout_ns)) {
                            atomicExch(abort_flag, 1);
                            break;
                        }
                    xk = ((volatile double*)ys)[lk];
                } else {
                    sp_wait_flag(&flags[k], flag_val, abort_flag, t0, timeout_ns);
                    xk = __ldcg(out + oidx(k));
                }
                acc = __fma_rn(-val[q], xk, acc);
            }
            if (!FWD) acc = __ddiv_rn(acc, diag[i]);
            ys[t] = acc;
            out[oidx(i)] = acc;
            __threadfence();
            ready[t] = 1;
            st_release_u32(&flags[i], flag_val);
        }
    }
}

// Square block of the recursive block SpTRSV ("SpMV is applied to the square blocks"): rows
// [r0, r1) of the node, one thread per row: s = sum_k t_ik v_k (one fma chain from +0, ascending k),
// then v_i = v_i - s (in place on the solve's vector).  Rows i = r0 + first + k*stride.
__device__ __forceinline__ void rb_square_rows(const int64_t* __restrict__ rp, const int32_t* __restrict__ ci,
                                               const double* __restrict__ val, int64_t r0, int64_t r1, double* v,
                                               int64_t first, int64_t stride) {
    for (int64_t i = r0 + first; i < r1; i += stride) {
        const int64_t lo = rp[i - r0], hi = rp[i - r0 + 1];
        if (lo == hi) continue;                   // v_i - (+0) == v_i
        double sacc = 0.0;
        for (int64_t q = lo; q < hi; ++q) sacc = __fma_rn(val[q], __ldcg(v + ci[q]), sacc);
        v[i] = __dsub_rn(__ldcg(v + i), sacc);
    }
}

}  // namespace mfk
