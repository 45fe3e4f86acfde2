// solver.cu -- the single-kernel CG and BiCGSTAB of Mille-feuille on sm_100a
// (Section III-C, Alg. 3; mixed precision Section III-D).
//
// One cooperative persistent launch runs the whole solve.  CTA g owns the contiguous tile
// rows [plan_tr[g], plan_tr[g+1]) (the task distribution of P:130-132, balanced on nnz and
// tiles) and does every vector operation for its rows.  The paper's dependency
// counters d_s / d_d / d_a become:
//   * a monotone-epoch grid barrier (one atomic per CTA, acquire-spin) at each dot product,
//     carrying the per-CTA partial sums in fixed slots -> deterministic reductions;
//   * per-CTA "p ready" epoch flags: before an SpMV a CTA waits only for the CTAs owning the
//     column segments it gathers (the generalisation of d_s), not for the whole grid.
// The SpMV output mu (and theta) stays in shared memory of the owner CTA across the barrier
// (spilled to HBM only for rows beyond the smem capacity).  The convergent-element retrieval
// (Alg. 4) is fused into whoever writes the SpMV input: the level of a 16-element segment is
// the min over the half-warp that produced it.
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "kernels.cuh"
#include "mf_internal.cuh"
#include "precond.cuh"

namespace mf {
namespace {

using mfk::Counts;
using mfk::Mat;
using mfk::Thresh;

constexpr int NSLOT = 4;    // doubles reduced per barrier (max)
constexpr int NPHASE = 12;  // timed phases per CTA

struct SolveArgs {
    Mat A;
    int32_t G;
    const int32_t* __restrict__ plan_tr;
    const int32_t* __restrict__ dep_lo;
    const int32_t* __restrict__ dep_hi;
    const int32_t* __restrict__ seg_lo;
    const int32_t* __restrict__ seg_hi;
    int64_t n;
    const double* __restrict__ b;
    double* x;
    double* r;
    double* p;
    double* mu_g;      // spill of mu beyond mu_cap rows per CTA [n]
    uint8_t* lev_p;
    double* rh;        // BiCGSTAB r0*
    double* s;
    double* th_g;      // spill of theta
    uint8_t* lev_s;
    double* slots;     // [2][NSLOT][G]
    unsigned* bar;     // grid barrier counter
    unsigned* flags;   // [G] ready epochs
    int* abort_flag;
    unsigned long long* bar_ns;   // [G] time spent spinning
    unsigned long long* phase_ns; // [G][NPHASE] time per phase (thread 0's view)
    double* hist;
    int64_t hist_cap;
    unsigned long long* lcounts;  // [lc_cap][10]: tiles[5], nnz[5] per SpMV
    int64_t lc_cap;
    double* out;       // [8]: iterations, converged, relres, status
    double tol, switch_eps;
    int switch_abs, range_guard;
    int64_t max_iter;
    int mu_cap;
    unsigned long long timeout_ns;
    // ILU(0) preconditioner (PCG / right-preconditioned PBiCGSTAB); null when unpreconditioned
    const int64_t* Lrp; const int32_t* Lci; const double* Lv;
    const int64_t* Urp; const int32_t* Uci; const double* Uv; const double* Ud;
    unsigned* pflags;            // per-row ready epochs of the triangular solves
    unsigned long long* pctr;    // [2] chunk counters (forward, backward)
    double* py;                  // forward-solve output
    double* pz;                  // PCG: z; PBiCGSTAB: p^
    double* ps;                  // PBiCGSTAB: s^
    unsigned pe0;                // epoch of the first apply of this solve
};

__device__ __forceinline__ unsigned ld_acquire(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(unsigned* p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

struct Ctx {
    unsigned bar_target = 0;
    int parity = 0;
    int spmv = 0;
};

__device__ __forceinline__ void red_release_add(unsigned* p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// ---- synchronisation.  Stall time is accumulated in shared memory (spin_ns), not in global
// memory, so the barrier's critical path is: release-add, acquire-spin, fence.
__device__ unsigned long long* spin_ns_smem() {
    __shared__ unsigned long long spin_ns;
    return &spin_ns;
}

__device__ __forceinline__ bool grid_barrier(const SolveArgs& a, Ctx& c) {
    __shared__ int s_abort;
    c.bar_target += (unsigned)a.G;
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned long long t0 = gtimer();
        red_release_add(a.bar, 1u);       // cumulative release: this CTA's writes (ordered by bar.sync)
        int ab = 0;
        while (ld_acquire(a.bar) < c.bar_target) {
            if (*(volatile int*)a.abort_flag) { ab = 1; break; }
            if (gtimer() - t0 > a.timeout_ns) { atomicExch(a.abort_flag, 1); ab = 1; break; }
        }
        __threadfence();
        *spin_ns_smem() += gtimer() - t0;
        s_abort = ab;
    }
    __syncthreads();
    return s_abort == 0;
}

__device__ __forceinline__ void publish(const SolveArgs& a, unsigned epoch) {
    __syncthreads();
    if (threadIdx.x == 0) st_release(&a.flags[blockIdx.x], epoch);   // cumulative release (CTA writes via bar.sync)
}

__device__ __forceinline__ bool wait_deps(const SolveArgs& a, unsigned epoch) {
    __shared__ int s_abort;
    const int lo = a.dep_lo[blockIdx.x], hi = a.dep_hi[blockIdx.x];
    if (threadIdx.x == 0) s_abort = 0;
    __syncthreads();
    const unsigned long long t0 = gtimer();
    for (int h = lo + (int)threadIdx.x; h <= hi; h += blockDim.x) {
        while (ld_acquire(&a.flags[h]) < epoch) {
            if (*(volatile int*)a.abort_flag) { s_abort = 1; break; }
            if (gtimer() - t0 > a.timeout_ns) { atomicExch(a.abort_flag, 1); s_abort = 1; break; }
        }
    }
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) *spin_ns_smem() += gtimer() - t0;
    return s_abort == 0;
}

// K doubles: thread fma chains -> warp butterfly -> tree32 over warps -> slot -> barrier ->
// tree32 over CTAs.  Every thread returns the grid totals.
template <int K>
__device__ __forceinline__ bool grid_reduce(double (&v)[K], const SolveArgs& a, Ctx& c, double* red) {
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31, W = blockDim.x >> 5;
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const double wt = mfk::butterfly32(v[k]);
        if (l == 0) red[k * 32 + w] = wt;
    }
    __syncthreads();
    if (w == 0) {
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const double ct = mfk::tree32(red + k * 32, W);
            if (l == 0) a.slots[((size_t)c.parity * NSLOT + k) * a.G + blockIdx.x] = ct;
        }
    }
    const bool ok = grid_barrier(a, c);
    if (w == 0) {
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const double gt = mfk::tree32(a.slots + ((size_t)c.parity * NSLOT + k) * a.G, a.G);
            if (l == 0) red[128 + k] = gt;
        }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < K; ++k) v[k] = red[128 + k];
    __syncthreads();
    c.parity ^= 1;
    return ok;
}

template <bool COUNT>
__device__ __forceinline__ void flush_counts(const SolveArgs& a, Ctx& c, Counts& cnt, int* ired) {
    if (!COUNT) return;
    if (threadIdx.x < 10) ired[threadIdx.x] = 0;
    __syncthreads();
#pragma unroll
    for (int q = 0; q < 5; ++q) {
        int tv = cnt.tiles(q), nv = cnt.nnz(q);
        for (int o = 16; o >= 1; o >>= 1) { tv += __shfl_xor_sync(0xffffffffu, tv, o); nv += __shfl_xor_sync(0xffffffffu, nv, o); }
        if ((threadIdx.x & 31) == 0) { atomicAdd(&ired[q], tv); atomicAdd(&ired[5 + q], nv); }
    }
    __syncthreads();
    if (threadIdx.x < 10 && c.spmv < a.lc_cap && ired[threadIdx.x])
        atomicAdd(&a.lcounts[(size_t)c.spmv * 10 + threadIdx.x], (unsigned long long)ired[threadIdx.x]);
    cnt.zero();
    c.spmv++;
}

__device__ __forceinline__ Thresh make_thresh(const SolveArgs& a, double v0norm) {
    // reading R8: tau = eps * ||v0||_2 (P:174 threshold in the units of the SpMV input, P:264 relative stop test)
    const double tau = a.switch_abs ? a.switch_eps : __dmul_rn(a.switch_eps, v0norm);
    return Thresh{__dmul_rn(tau, 1e-3), __dmul_rn(tau, 1e-2), __dmul_rn(tau, 1e-1), tau};
}

struct Smem {
    double* mu;      // [mu_cap]
    double* th;      // [mu_cap] (BiCGSTAB)
    double* tys;     // [B] triangular-solve chunk values (preconditioned)
    int* tready;     // [B]
    long long* tchunk;
    double* red;     // [4*32 + 8]
    int* ired;       // [16]
    unsigned long long* timer;   // [NPHASE + 1]
    mfk::WinSmem win;
    mfk::TsSmem ts;
};

__host__ __device__ constexpr size_t fixed_smem_bytes() {
    return (4 * 32 + 8) * sizeof(double) + 16 * sizeof(int) + (NPHASE + 1) * 8 + mfk::SPMV_SMEM_BYTES + 96;
}

__device__ __forceinline__ Smem carve(const SolveArgs& a, int nvec) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    Smem s;
    double* d = reinterpret_cast<double*>(smem_raw);
    s.red = d;
    s.ired = reinterpret_cast<int*>(d + 4 * 32 + 8);
    s.timer = reinterpret_cast<unsigned long long*>(s.ired + 16);
    // alignment by offsets from smem_raw (never through an integer cast of the pointer): the
    // compiler keeps the shared address space and emits LDS/STS with 32-bit addresses
    unsigned char* p = smem_raw + mfk::pipe_r16((int)(reinterpret_cast<unsigned char*>(s.timer + NPHASE + 1) - smem_raw));
    mfk::carve_spmv(p, s.win, s.ts);
    mfk::pipe_init(s.ts);      // ordered before the first SpMV by the caller's __syncthreads (Timer::start)
    p += mfk::SPMV_SMEM_BYTES;
    p = smem_raw + mfk::pipe_r16((int)(p - smem_raw));
    s.mu = reinterpret_cast<double*>(p);
    s.th = s.mu + a.mu_cap;
    s.tys = s.mu + (size_t)nvec * a.mu_cap;
    s.tready = reinterpret_cast<int*>(s.tys + blockDim.x);
    s.tchunk = reinterpret_cast<long long*>(s.tready + blockDim.x + 2);
    return s;
}

// phase timer: thread 0 accumulates %globaltimer deltas per phase (barrier-stall share)
struct Timer {
    unsigned long long* acc;   // smem [NPHASE + 1]; acc[NPHASE] = last timestamp
    __device__ void start(unsigned long long* sm) {
        acc = sm;
        if (threadIdx.x == 0) {
            for (int k = 0; k < NPHASE; ++k) acc[k] = 0;
            acc[NPHASE] = gtimer();
            *spin_ns_smem() = 0;
        }
        __syncthreads();
    }
    __device__ void tick(int k) {
        if (threadIdx.x == 0) { const unsigned long long now = gtimer(); acc[k] += now - acc[NPHASE]; acc[NPHASE] = now; }
    }
    __device__ void flush(const SolveArgs& a) {
        if (threadIdx.x == 0) {
            for (int k = 0; k < NPHASE; ++k) a.phase_ns[(size_t)blockIdx.x * NPHASE + k] = acc[k];
            a.bar_ns[blockIdx.x] = *spin_ns_smem();
        }
    }
};

// -------------------------------------------------------------------------- CG (Alg. 1 / Alg. 3)
// Phases: 0 wait for SpMV inputs, 1 SpMV + (mu,p), 2 reduce sigma, 3 x/r update + (r,r),
//         4 reduce rho', 5 p update + levels + publish, 6 init
template <bool DYN, bool COUNT, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) cg_persistent(SolveArgs a) {
    constexpr int PF = MAXT >= 1024 ? 4 : 8;
    Smem sm = carve(a, 1);
    Ctx c;
    Counts cnt;
    cnt.zero();
    Timer tm;
    tm.start(sm.timer);
    const int t = threadIdx.x, B = blockDim.x, H = B >> 4, h = t >> 4, lane = t & 15;
    const unsigned m = mfk::hw_mask();
    const int64_t tr0 = a.plan_tr[blockIdx.x], tr1 = a.plan_tr[blockIdx.x + 1];
    const int64_t R0 = tr0 * 16, Rend = min(tr1 * 16, a.n);
    const int64_t n = a.n, nr = Rend - R0;
    const int mu_cap = a.mu_cap;
    double* __restrict__ X = a.x;
    double* __restrict__ Rv = a.r;
    double* __restrict__ P = a.p;
    double* __restrict__ MUg = a.mu_g;
    double* __restrict__ MUs = sm.mu;

    // init: r = b - A~ x0 at TilePrec; p = r; partial (b,b), (r,r)
    double v2[2] = {0.0, 0.0};
    mfk::spmv_cta<false, false, PF>(a.A, tr0, tr1, X, nullptr, 0, sm.win, sm.ts, nullptr, 0, -1, a.b,
                                [&](int64_t TR, int ln, double ax, double bi) {
                                    const int64_t i = TR * 16 + ln;
                                    if (i < n) {
                                        const double ri = __dsub_rn(bi, ax);
                                        Rv[i] = ri;
                                        P[i] = ri;
                                        v2[0] = __fma_rn(bi, bi, v2[0]);
                                        v2[1] = __fma_rn(ri, ri, v2[1]);
                                    }
                                });
    bool ok = grid_reduce<2>(v2, a, c, sm.red);
    const double nb = sqrt(v2[0]);
    double rho = v2[1];
    int64_t j = 0;
    int converged = 0, status = ok ? MF_OK : MF_ERR_DEADLOCK;
    if (ok && nb == 0.0) {
        for (int64_t i = R0 + t; i < Rend; i += B) X[i] = 0.0;
        converged = 1;
        if (blockIdx.x == 0 && t == 0 && a.hist_cap > 0) a.hist[0] = 0.0;
    } else if (ok) {
        const Thresh th = make_thresh(a, sqrt(rho));
        if (DYN) {
            for (int64_t TR = tr0 + h; TR < tr1; TR += H) {
                const int64_t i = TR * 16 + lane;
                const int lv = mfk::hw_min_i(i < n ? mfk::level_of(P[i], th) : 4, m);
                if (lane == 0) a.lev_p[TR] = (uint8_t)lv;
            }
        }
        publish(a, 1);
        tm.tick(6);
        for (;; ++j) {
            const double relres = __ddiv_rn(sqrt(rho), nb);
            if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = relres; a.out[2] = relres; }
            if (relres < a.tol) { converged = 1; break; }
            if (j == a.max_iter) break;
            if (!wait_deps(a, (unsigned)(j + 1))) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(0);
            // step A: mu = A~_j p_j (own tile rows) with the fused partial (mu, p)
            double sg[1] = {0.0};
            mfk::spmv_cta<DYN, COUNT, PF>(a.A, tr0, tr1, P, a.lev_p, a.range_guard, sm.win, sm.ts, &cnt, a.seg_lo[blockIdx.x], a.seg_hi[blockIdx.x], P,
                                      [&](int64_t TR, int ln, double mv, double ov) {
                                          const int64_t i = TR * 16 + ln;
                                          if (i < n) {
                                              const int64_t li = i - R0;
                                              if (li < mu_cap) MUs[li] = mv; else MUg[i] = mv;
                                              sg[0] = __fma_rn(mv, ov, sg[0]);
                                          }
                                      });
            flush_counts<COUNT>(a, c, cnt, sm.ired);
            __syncthreads();
            tm.tick(1);
            // step B: sigma = (mu, p) over the grid -> alpha
            if (!grid_reduce<1>(sg, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(2);
            const double sigma = sg[0];
            if (!(sigma > 0.0) || !isfinite(sigma)) { status = MF_ERR_BREAKDOWN; break; }
            const double alpha = __ddiv_rn(rho, sigma);
            // step C: x += alpha p, r -= alpha mu, partial (r, r); 4 rows in flight per thread
            double rr[1] = {0.0};
            for (int64_t l0 = t; l0 < nr; l0 += 4 * (int64_t)B) {
                double pv[4], xv[4], rv[4], mv[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t li = l0 + q * B;
                    if (li < nr) {
                        const int64_t i = R0 + li;
                        pv[q] = P[i]; xv[q] = X[i]; rv[q] = Rv[i];
                        mv[q] = li < mu_cap ? MUs[li] : MUg[i];
                    }
                }
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t li = l0 + q * B;
                    if (li < nr) {
                        const int64_t i = R0 + li;
                        X[i] = __fma_rn(alpha, pv[q], xv[q]);
                        const double ri = __fma_rn(-alpha, mv[q], rv[q]);
                        Rv[i] = ri;
                        rr[0] = __fma_rn(ri, ri, rr[0]);
                    }
                }
            }
            tm.tick(3);
            if (!grid_reduce<1>(rr, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(4);
            const double beta = __ddiv_rn(rr[0], rho);
            rho = rr[0];
            // step D: p = r + beta p (own rows) and the levels of its segments (Alg. 4)
            for (int64_t TR0 = tr0 + h; TR0 < tr1; TR0 += 4 * (int64_t)H) {
                double pv[4], rv[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t i = (TR0 + q * H) * 16 + lane;
                    pv[q] = 0.0; rv[q] = 0.0;
                    if (TR0 + q * H < tr1 && i < n) { pv[q] = P[i]; rv[q] = Rv[i]; }
                }
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t TR = TR0 + q * H;
                    if (TR < tr1) {                            // uniform per half-warp
                        const int64_t i = TR * 16 + lane;
                        double pn = 0.0;
                        if (i < n) { pn = __fma_rn(beta, pv[q], rv[q]); P[i] = pn; }
                        if (DYN) {
                            const int lv = mfk::hw_min_i(i < n ? mfk::level_of(pn, th) : 4, m);
                            if (lane == 0) a.lev_p[TR] = (uint8_t)lv;
                        }
                    }
                }
            }
            publish(a, (unsigned)(j + 2));
            tm.tick(5);
        }
    }
    if (blockIdx.x == 0 && t == 0) {
        a.out[0] = (double)j;
        a.out[1] = converged;
        a.out[3] = status;
    }
    tm.flush(a);
    if (status == MF_ERR_DEADLOCK && t == 0) atomicExch(a.abort_flag, 1);
}

// -------------------------------------------------------------------------- BiCGSTAB (Alg. 2)
// Phases: 0 wait p, 1 SpMV mu, 2 reduce eta, 3 s update, 4 wait s, 5 SpMV theta, 6 reduce tt,
//         7 x/r update, 8 reduce rho', 9 p update + publish, 10 init
template <bool DYN, bool COUNT, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) bicgstab_persistent(SolveArgs a) {
    constexpr int PF = MAXT >= 1024 ? 4 : 8;
    Smem sm = carve(a, 2);
    Ctx c;
    Counts cnt;
    cnt.zero();
    Timer tm;
    tm.start(sm.timer);
    const int t = threadIdx.x, B = blockDim.x, H = B >> 4, h = t >> 4, lane = t & 15;
    const unsigned m = mfk::hw_mask();
    const int64_t tr0 = a.plan_tr[blockIdx.x], tr1 = a.plan_tr[blockIdx.x + 1];
    const int64_t R0 = tr0 * 16, Rend = min(tr1 * 16, a.n);
    const int64_t n = a.n, nr = Rend - R0;
    const int mu_cap = a.mu_cap;
    double* __restrict__ X = a.x;
    double* __restrict__ Rv = a.r;
    double* __restrict__ P = a.p;
    double* __restrict__ S = a.s;
    const double* RH = a.rh;   // written at init in this kernel: no read-only (.nc) loads
    double* __restrict__ MUs = sm.mu;
    double* __restrict__ THs = sm.th;
    auto mu_at = [&](int64_t li) -> double& { return li < mu_cap ? MUs[li] : a.mu_g[R0 + li]; };
    auto th_at = [&](int64_t li) -> double& { return li < mu_cap ? THs[li] : a.th_g[R0 + li]; };

    // init: r = b - A~ x0; r0* = r; p = r; partial (b,b), (r,r), (r,r0*)
    double v3[3] = {0.0, 0.0, 0.0};
    mfk::spmv_cta<false, false, PF>(a.A, tr0, tr1, X, nullptr, 0, sm.win, sm.ts, nullptr, 0, -1, a.b,
                                [&](int64_t TR, int ln, double ax, double bi) {
                                    const int64_t i = TR * 16 + ln;
                                    if (i < n) {
                                        const double ri = __dsub_rn(bi, ax);
                                        Rv[i] = ri; a.rh[i] = ri; P[i] = ri;
                                        v3[0] = __fma_rn(bi, bi, v3[0]);
                                        v3[1] = __fma_rn(ri, ri, v3[1]);
                                        v3[2] = __fma_rn(ri, ri, v3[2]);
                                    }
                                });
    bool ok = grid_reduce<3>(v3, a, c, sm.red);
    const double nb = sqrt(v3[0]);
    double rr = v3[1], rho = v3[2];
    int64_t j = 0;
    int converged = 0, status = ok ? MF_OK : MF_ERR_DEADLOCK;
    unsigned epoch = 0;
    if (ok && nb == 0.0) {
        for (int64_t i = R0 + t; i < Rend; i += B) X[i] = 0.0;
        converged = 1;
        if (blockIdx.x == 0 && t == 0 && a.hist_cap > 0) a.hist[0] = 0.0;
    } else if (ok) {
        const Thresh th = make_thresh(a, sqrt(rr));
        if (DYN) {
            for (int64_t TR = tr0 + h; TR < tr1; TR += H) {
                const int64_t i = TR * 16 + lane;
                const int lv = mfk::hw_min_i(i < n ? mfk::level_of(P[i], th) : 4, m);
                if (lane == 0) a.lev_p[TR] = (uint8_t)lv;
            }
        }
        publish(a, ++epoch);
        tm.tick(10);
        for (;; ++j) {
            const double relres = __ddiv_rn(sqrt(rr), nb);
            if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = relres; a.out[2] = relres; }
            if (relres < a.tol) { converged = 1; break; }
            if (j == a.max_iter) break;
            if (!wait_deps(a, epoch)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(0);
            // mu = A~ p ; partial (mu, r0*)
            double eta[1] = {0.0};
            mfk::spmv_cta<DYN, COUNT, PF>(a.A, tr0, tr1, P, a.lev_p, a.range_guard, sm.win, sm.ts, &cnt, a.seg_lo[blockIdx.x], a.seg_hi[blockIdx.x], RH,
                                      [&](int64_t TR, int ln, double mv, double ov) {
                                          const int64_t i = TR * 16 + ln;
                                          if (i < n) { mu_at(i - R0) = mv; eta[0] = __fma_rn(mv, ov, eta[0]); }
                                      });
            flush_counts<COUNT>(a, c, cnt, sm.ired);
            __syncthreads();
            tm.tick(1);
            if (!grid_reduce<1>(eta, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(2);
            if (eta[0] == 0.0 || !isfinite(eta[0])) { status = MF_ERR_BREAKDOWN; break; }
            const double alpha = __ddiv_rn(rho, eta[0]);
            // s = r - alpha mu (own rows) + levels of s
            for (int64_t TR = tr0 + h; TR < tr1; TR += H) {
                const int64_t i = TR * 16 + lane;
                double si = 0.0;
                if (i < n) { si = __fma_rn(-alpha, mu_at(i - R0), Rv[i]); S[i] = si; }
                if (DYN) {
                    const int lv = mfk::hw_min_i(i < n ? mfk::level_of(si, th) : 4, m);
                    if (lane == 0) a.lev_s[TR] = (uint8_t)lv;
                }
            }
            publish(a, ++epoch);
            tm.tick(3);
            if (!wait_deps(a, epoch)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(4);
            // theta = A~ s ; partial (theta, theta), (theta, s)
            double tt[2] = {0.0, 0.0};
            mfk::spmv_cta<DYN, COUNT, PF>(a.A, tr0, tr1, S, a.lev_s, a.range_guard, sm.win, sm.ts, &cnt, a.seg_lo[blockIdx.x], a.seg_hi[blockIdx.x], S,
                                      [&](int64_t TR, int ln, double tv, double ov) {
                                          const int64_t i = TR * 16 + ln;
                                          if (i < n) {
                                              th_at(i - R0) = tv;
                                              tt[0] = __fma_rn(tv, tv, tt[0]);
                                              tt[1] = __fma_rn(tv, ov, tt[1]);
                                          }
                                      });
            flush_counts<COUNT>(a, c, cnt, sm.ired);
            __syncthreads();
            tm.tick(5);
            if (!grid_reduce<2>(tt, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(6);
            if (tt[0] == 0.0) {
                // theta == 0: take the half step x += alpha p, r = s, and stop (reading R14)
                double r2[1] = {0.0};
                for (int64_t li = t; li < nr; li += B) {
                    const int64_t i = R0 + li;
                    X[i] = __fma_rn(alpha, P[i], X[i]);
                    const double si = S[i];
                    Rv[i] = si;
                    r2[0] = __fma_rn(si, si, r2[0]);
                }
                if (!grid_reduce<1>(r2, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
                ++j;
                const double rl = __ddiv_rn(sqrt(r2[0]), nb);
                if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = rl; a.out[2] = rl; }
                if (rl < a.tol) converged = 1; else status = MF_ERR_BREAKDOWN;
                break;
            }
            const double omega = __ddiv_rn(tt[1], tt[0]);
            if (omega == 0.0 || !isfinite(omega)) { status = MF_ERR_BREAKDOWN; break; }
            // x += alpha p + omega s ; r = s - omega theta ; partial (r, r0*), (r, r)
            double rv[2] = {0.0, 0.0};
            for (int64_t l0 = t; l0 < nr; l0 += 2 * (int64_t)B) {
                double sv[2], pv[2], xv[2], tv[2], hv[2];
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                    const int64_t li = l0 + q * B;
                    if (li < nr) {
                        const int64_t i = R0 + li;
                        sv[q] = S[i]; pv[q] = P[i]; xv[q] = X[i]; hv[q] = RH[i];
                        tv[q] = th_at(li);
                    }
                }
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                    const int64_t li = l0 + q * B;
                    if (li < nr) {
                        const int64_t i = R0 + li;
                        X[i] = __fma_rn(omega, sv[q], __fma_rn(alpha, pv[q], xv[q]));
                        const double ri = __fma_rn(-omega, tv[q], sv[q]);
                        Rv[i] = ri;
                        rv[0] = __fma_rn(ri, hv[q], rv[0]);
                        rv[1] = __fma_rn(ri, ri, rv[1]);
                    }
                }
            }
            tm.tick(7);
            if (!grid_reduce<2>(rv, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(8);
            rr = rv[1];
            if (rv[0] == 0.0 || !isfinite(rv[0])) {
                ++j;
                const double rl = __ddiv_rn(sqrt(rr), nb);
                if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = rl; a.out[2] = rl; }
                if (rl < a.tol) converged = 1; else status = MF_ERR_BREAKDOWN;
                break;
            }
            const double beta = __dmul_rn(__ddiv_rn(rv[0], rho), __ddiv_rn(alpha, omega));
            rho = rv[0];
            // p = r + beta (p - omega mu) (own rows) + levels of p
            for (int64_t TR = tr0 + h; TR < tr1; TR += H) {
                const int64_t i = TR * 16 + lane;
                double pn = 0.0;
                if (i < n) { pn = __fma_rn(beta, __fma_rn(-omega, mu_at(i - R0), P[i]), Rv[i]); P[i] = pn; }
                if (DYN) {
                    const int lv = mfk::hw_min_i(i < n ? mfk::level_of(pn, th) : 4, m);
                    if (lane == 0) a.lev_p[TR] = (uint8_t)lv;
                }
            }
            publish(a, ++epoch);
            tm.tick(9);
        }
    }
    if (blockIdx.x == 0 && t == 0) {
        a.out[0] = (double)j;
        a.out[1] = converged;
        a.out[3] = status;
    }
    tm.flush(a);
    if (status == MF_ERR_DEADLOCK && t == 0) atomicExch(a.abort_flag, 1);
}

// -------------------------------------------------------------------------- preconditioned solvers
// z = M^-1 v with M = ILU(0): forward then backward sync-free chunked solves (all CTAs
// grab chunks; co-residency of the persistent grid makes the in-order grabbing deadlock-free).
// On return every thread has seen its own rows of `out` complete (row flags) and fenced.
struct PcState {
    unsigned long long base_f = 0, base_b = 0;
    unsigned apply = 0;
};

__device__ __forceinline__ bool precond_apply(const SolveArgs& a, PcState& ps, const Smem& sm, const double* in, double* out,
                              int64_t R0, int64_t Rend) {
    const unsigned e = a.pe0 + ps.apply++;
    const unsigned vf = 2 * e + 1, vb = 2 * e + 2;
    const int64_t nch = (a.n + blockDim.x - 1) / blockDim.x;
    mfk::sptrsv_chunked<true>(a.Lrp, a.Lci, a.Lv, nullptr, a.n, in, a.py, a.pflags, vf, 0u, a.pctr, ps.base_f,
                              sm.tys, sm.tready, sm.tchunk);
    ps.base_f += (unsigned long long)(nch + a.G);
    mfk::sptrsv_chunked<false>(a.Urp, a.Uci, a.Uv, a.Ud, a.n, a.py, out, a.pflags, vb, vf, a.pctr + 1, ps.base_b,
                               sm.tys, sm.tready, sm.tchunk);
    ps.base_b += (unsigned long long)(nch + a.G);
    const unsigned long long t0 = gtimer();
    bool ok = true;
    for (int64_t i = R0 + threadIdx.x; i < Rend; i += blockDim.x)
        while (mfk::ld_acquire_u32(&a.pflags[i]) != vb) {
            if (gtimer() - t0 > a.timeout_ns) { atomicExch(a.abort_flag, 1); ok = false; break; }
        }
    __threadfence();
    __syncthreads();
    return ok;
}

// levels of the own segments of v (Alg. 4), one half-warp per tile row
template <bool DYN>
__device__ __forceinline__ void own_levels(const SolveArgs& a, const double* v, uint8_t* lev, int64_t tr0, int64_t tr1, const Thresh& th) {
    if (!DYN) return;
    const int H = blockDim.x >> 4, h = threadIdx.x >> 4, lane = threadIdx.x & 15;
    const unsigned m = mfk::hw_mask();
    for (int64_t TR = tr0 + h; TR < tr1; TR += H) {
        const int64_t i = TR * 16 + lane;
        const int lv = mfk::hw_min_i(i < a.n ? mfk::level_of(__ldcg(v + i), th) : 4, m);
        if (lane == 0) lev[TR] = (uint8_t)lv;
    }
}

// PCG (SURVEY c-6): z = M^-1 r, rho = (r,z), p = z + beta p; stop on ||r||/||b||.
// Phases: 0 wait p, 1 SpMV, 2 reduce sigma, 3 x/r update, 4 reduce rr, 5 M^-1 r, 6 reduce rho,
//         7 p update + publish, 10 init
template <bool DYN, bool COUNT, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) pcg_persistent(SolveArgs a) {
    constexpr int PF = MAXT >= 1024 ? 4 : 8;
    Smem sm = carve(a, 1);
    Ctx c;
    Counts cnt;
    cnt.zero();
    Timer tm;
    tm.start(sm.timer);
    PcState pcs;
    const int t = threadIdx.x, B = blockDim.x, H = B >> 4, h = t >> 4, lane = t & 15;
    const int64_t tr0 = a.plan_tr[blockIdx.x], tr1 = a.plan_tr[blockIdx.x + 1];
    const int64_t R0 = tr0 * 16, Rend = min(tr1 * 16, a.n);
    const int64_t n = a.n, nr = Rend - R0;
    const int mu_cap = a.mu_cap;
    double* __restrict__ X = a.x;
    double* __restrict__ Rv = a.r;
    double* __restrict__ P = a.p;
    double* Z = a.pz;
    double* __restrict__ MUs = sm.mu;
    (void)H;
    (void)lane;
    (void)h;

    double v2[2] = {0.0, 0.0};
    mfk::spmv_cta<false, false, PF>(a.A, tr0, tr1, X, nullptr, 0, sm.win, sm.ts, nullptr, 0, -1, a.b,
                                    [&](int64_t TR, int ln, double ax, double bi) {
                                        const int64_t i = TR * 16 + ln;
                                        if (i < n) {
                                            const double ri = __dsub_rn(bi, ax);
                                            Rv[i] = ri;
                                            v2[0] = __fma_rn(bi, bi, v2[0]);
                                            v2[1] = __fma_rn(ri, ri, v2[1]);
                                        }
                                    });
    bool ok = grid_reduce<2>(v2, a, c, sm.red);   // also: r complete on every CTA
    const double nb = sqrt(v2[0]);
    double rr = v2[1], rho = 0.0;
    int64_t j = 0;
    int converged = 0, status = ok ? MF_OK : MF_ERR_DEADLOCK;
    if (ok && nb == 0.0) {
        for (int64_t i = R0 + t; i < Rend; i += B) X[i] = 0.0;
        converged = 1;
        if (blockIdx.x == 0 && t == 0 && a.hist_cap > 0) a.hist[0] = 0.0;
    } else if (ok) {
        if (!precond_apply(a, pcs, sm, Rv, Z, R0, Rend)) status = MF_ERR_DEADLOCK;
        double v3[2] = {0.0, 0.0};
        for (int64_t li = t; li < nr; li += B) {
            const int64_t i = R0 + li;
            const double zi = Z[i];
            P[i] = zi;
            v3[0] = __fma_rn(Rv[i], zi, v3[0]);
            v3[1] = __fma_rn(zi, zi, v3[1]);
        }
        if (status == MF_OK && !grid_reduce<2>(v3, a, c, sm.red)) status = MF_ERR_DEADLOCK;
        rho = v3[0];
        const Thresh th = make_thresh(a, sqrt(v3[1]));
        own_levels<DYN>(a, P, a.lev_p, tr0, tr1, th);
        publish(a, 1);
        tm.tick(10);
        for (; status == MF_OK; ++j) {
            const double relres = __ddiv_rn(sqrt(rr), nb);
            if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = relres; a.out[2] = relres; }
            if (relres < a.tol) { converged = 1; break; }
            if (j == a.max_iter) break;
            if (!wait_deps(a, (unsigned)(j + 1))) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(0);
            double sg[1] = {0.0};
            mfk::spmv_cta<DYN, COUNT, PF>(a.A, tr0, tr1, P, a.lev_p, a.range_guard, sm.win, sm.ts, &cnt, a.seg_lo[blockIdx.x], a.seg_hi[blockIdx.x], P,
                                          [&](int64_t TR, int ln, double mv, double ov) {
                                              const int64_t i = TR * 16 + ln;
                                              if (i < n) {
                                                  const int64_t li = i - R0;
                                                  if (li < mu_cap) MUs[li] = mv; else a.mu_g[i] = mv;
                                                  sg[0] = __fma_rn(mv, ov, sg[0]);
                                              }
                                          });
            flush_counts<COUNT>(a, c, cnt, sm.ired);
            __syncthreads();
            tm.tick(1);
            if (!grid_reduce<1>(sg, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(2);
            const double sigma = sg[0];
            if (!(sigma > 0.0) || !isfinite(sigma)) { status = MF_ERR_BREAKDOWN; break; }
            const double alpha = __ddiv_rn(rho, sigma);
            double r1[1] = {0.0};
            for (int64_t li = t; li < nr; li += B) {
                const int64_t i = R0 + li;
                X[i] = __fma_rn(alpha, P[i], X[i]);
                const double ri = __fma_rn(-alpha, li < mu_cap ? MUs[li] : a.mu_g[i], Rv[i]);
                Rv[i] = ri;
                r1[0] = __fma_rn(ri, ri, r1[0]);
            }
            tm.tick(3);
            if (!grid_reduce<1>(r1, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }   // r complete too
            rr = r1[0];
            tm.tick(4);
            if (!precond_apply(a, pcs, sm, Rv, Z, R0, Rend)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(5);
            double rz[1] = {0.0};
            for (int64_t li = t; li < nr; li += B) {
                const int64_t i = R0 + li;
                rz[0] = __fma_rn(Rv[i], Z[i], rz[0]);
            }
            if (!grid_reduce<1>(rz, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(6);
            const double beta = __ddiv_rn(rz[0], rho);
            rho = rz[0];
            for (int64_t li = t; li < nr; li += B) {
                const int64_t i = R0 + li;
                P[i] = __fma_rn(beta, P[i], Z[i]);
            }
            __syncthreads();
            own_levels<DYN>(a, P, a.lev_p, tr0, tr1, th);
            publish(a, (unsigned)(j + 2));
            tm.tick(7);
        }
    }
    if (blockIdx.x == 0 && t == 0) {
        a.out[0] = (double)j;
        a.out[1] = converged;
        a.out[3] = status;
    }
    tm.flush(a);
    if (status == MF_ERR_DEADLOCK && t == 0) atomicExch(a.abort_flag, 1);
}

// Right-preconditioned PBiCGSTAB (SURVEY c-6): p^ = M^-1 p, s^ = M^-1 s, x += alpha p^ + omega s^.
// Phases: 0 M^-1 p + levels, 1 SpMV mu, 2 reduce eta, 3 s update + barrier, 4 M^-1 s + levels,
//         5 SpMV theta, 6 reduce tt, 7 x/r update + reduce, 8 p update + barrier, 10 init
template <bool DYN, bool COUNT, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) pbicgstab_persistent(SolveArgs a) {
    constexpr int PF = MAXT >= 1024 ? 4 : 8;
    Smem sm = carve(a, 2);
    Ctx c;
    Counts cnt;
    cnt.zero();
    Timer tm;
    tm.start(sm.timer);
    PcState pcs;
    const int t = threadIdx.x, B = blockDim.x;
    const int64_t tr0 = a.plan_tr[blockIdx.x], tr1 = a.plan_tr[blockIdx.x + 1];
    const int64_t R0 = tr0 * 16, Rend = min(tr1 * 16, a.n);
    const int64_t n = a.n, nr = Rend - R0;
    const int mu_cap = a.mu_cap;
    double* __restrict__ X = a.x;
    double* __restrict__ Rv = a.r;
    double* __restrict__ P = a.p;
    double* __restrict__ S = a.s;
    double* PH = a.pz;
    double* SH = a.ps;
    const double* RH = a.rh;   // written at init in this kernel: no read-only (.nc) loads
    double* __restrict__ MUs = sm.mu;
    double* __restrict__ THs = sm.th;
    auto mu_at = [&](int64_t li) -> double& { return li < mu_cap ? MUs[li] : a.mu_g[R0 + li]; };
    auto th_at = [&](int64_t li) -> double& { return li < mu_cap ? THs[li] : a.th_g[R0 + li]; };

    double v3[3] = {0.0, 0.0, 0.0};
    mfk::spmv_cta<false, false, PF>(a.A, tr0, tr1, X, nullptr, 0, sm.win, sm.ts, nullptr, 0, -1, a.b,
                                    [&](int64_t TR, int ln, double ax, double bi) {
                                        const int64_t i = TR * 16 + ln;
                                        if (i < n) {
                                            const double ri = __dsub_rn(bi, ax);
                                            Rv[i] = ri; a.rh[i] = ri; P[i] = ri;
                                            v3[0] = __fma_rn(bi, bi, v3[0]);
                                            v3[1] = __fma_rn(ri, ri, v3[1]);
                                            v3[2] = __fma_rn(ri, ri, v3[2]);
                                        }
                                    });
    bool ok = grid_reduce<3>(v3, a, c, sm.red);
    const double nb = sqrt(v3[0]);
    double rr = v3[1], rho = v3[2];
    int64_t j = 0;
    int converged = 0, status = ok ? MF_OK : MF_ERR_DEADLOCK;
    unsigned epoch = 0;
    Thresh th{0, 0, 0, 0};
    if (ok && nb == 0.0) {
        for (int64_t i = R0 + t; i < Rend; i += B) X[i] = 0.0;
        converged = 1;
        if (blockIdx.x == 0 && t == 0 && a.hist_cap > 0) a.hist[0] = 0.0;
    } else if (ok) {
        for (;; ++j) {
            const double relres = __ddiv_rn(sqrt(rr), nb);
            if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = relres; a.out[2] = relres; }
            if (relres < a.tol) { converged = 1; break; }
            if (j == a.max_iter) break;
            // p^ = M^-1 p (p complete: the previous grid reduction / the init reduction)
            if (!precond_apply(a, pcs, sm, P, PH, R0, Rend)) { status = MF_ERR_DEADLOCK; break; }
            if (j == 0) {          // tau from ||p^_0|| (the first SpMV input)
                double pp[1] = {0.0};
                for (int64_t li = t; li < nr; li += B) { const double v = PH[R0 + li]; pp[0] = __fma_rn(v, v, pp[0]); }
                if (!grid_reduce<1>(pp, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
                th = make_thresh(a, sqrt(pp[0]));
            }
            own_levels<DYN>(a, PH, a.lev_p, tr0, tr1, th);
            publish(a, ++epoch);
            if (!wait_deps(a, epoch)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(0);
            double eta[1] = {0.0};
            mfk::spmv_cta<DYN, COUNT, PF>(a.A, tr0, tr1, PH, a.lev_p, a.range_guard, sm.win, sm.ts, &cnt, a.seg_lo[blockIdx.x], a.seg_hi[blockIdx.x], RH,
                                          [&](int64_t TR, int ln, double mv, double ov) {
                                              const int64_t i = TR * 16 + ln;
                                              if (i < n) { mu_at(i - R0) = mv; eta[0] = __fma_rn(mv, ov, eta[0]); }
                                          });
            flush_counts<COUNT>(a, c, cnt, sm.ired);
            __syncthreads();
            tm.tick(1);
            if (!grid_reduce<1>(eta, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(2);
            if (eta[0] == 0.0 || !isfinite(eta[0])) { status = MF_ERR_BREAKDOWN; break; }
            const double alpha = __ddiv_rn(rho, eta[0]);
            for (int64_t li = t; li < nr; li += B) {
                const int64_t i = R0 + li;
                S[i] = __fma_rn(-alpha, mu_at(li), Rv[i]);
            }
            if (!grid_barrier(a, c)) { status = MF_ERR_DEADLOCK; break; }    // s complete
            tm.tick(3);
            if (!precond_apply(a, pcs, sm, S, SH, R0, Rend)) { status = MF_ERR_DEADLOCK; break; }
            own_levels<DYN>(a, SH, a.lev_s, tr0, tr1, th);
            publish(a, ++epoch);
            if (!wait_deps(a, epoch)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(4);
            double tt[2] = {0.0, 0.0};
            mfk::spmv_cta<DYN, COUNT, PF>(a.A, tr0, tr1, SH, a.lev_s, a.range_guard, sm.win, sm.ts, &cnt, a.seg_lo[blockIdx.x], a.seg_hi[blockIdx.x], S,
                                          [&](int64_t TR, int ln, double tv, double ov) {
                                              const int64_t i = TR * 16 + ln;
                                              if (i < n) {
                                                  th_at(i - R0) = tv;
                                                  tt[0] = __fma_rn(tv, tv, tt[0]);
                                                  tt[1] = __fma_rn(tv, ov, tt[1]);
                                              }
                                          });
            flush_counts<COUNT>(a, c, cnt, sm.ired);
            __syncthreads();
            tm.tick(5);
            if (!grid_reduce<2>(tt, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(6);
            if (tt[0] == 0.0) {
                double r2[1] = {0.0};
                for (int64_t li = t; li < nr; li += B) {
                    const int64_t i = R0 + li;
                    X[i] = __fma_rn(alpha, PH[i], X[i]);
                    const double si = S[i];
                    Rv[i] = si;
                    r2[0] = __fma_rn(si, si, r2[0]);
                }
                if (!grid_reduce<1>(r2, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
                ++j;
                const double rl = __ddiv_rn(sqrt(r2[0]), nb);
                if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = rl; a.out[2] = rl; }
                if (rl < a.tol) converged = 1; else status = MF_ERR_BREAKDOWN;
                break;
            }
            const double omega = __ddiv_rn(tt[1], tt[0]);
            if (omega == 0.0 || !isfinite(omega)) { status = MF_ERR_BREAKDOWN; break; }
            double rv[2] = {0.0, 0.0};
            for (int64_t li = t; li < nr; li += B) {
                const int64_t i = R0 + li;
                const double si = S[i];
                X[i] = __fma_rn(omega, SH[i], __fma_rn(alpha, PH[i], X[i]));
                const double ri = __fma_rn(-omega, th_at(li), si);
                Rv[i] = ri;
                rv[0] = __fma_rn(ri, RH[i], rv[0]);
                rv[1] = __fma_rn(ri, ri, rv[1]);
            }
            if (!grid_reduce<2>(rv, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(7);
            rr = rv[1];
            if (rv[0] == 0.0 || !isfinite(rv[0])) {
                ++j;
                const double rl = __ddiv_rn(sqrt(rr), nb);
                if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = rl; a.out[2] = rl; }
                if (rl < a.tol) converged = 1; else status = MF_ERR_BREAKDOWN;
                break;
            }
            const double beta = __dmul_rn(__ddiv_rn(rv[0], rho), __ddiv_rn(alpha, omega));
            rho = rv[0];
            for (int64_t li = t; li < nr; li += B) {
                const int64_t i = R0 + li;
                P[i] = __fma_rn(beta, __fma_rn(-omega, mu_at(li), P[i]), Rv[i]);
            }
            if (!grid_barrier(a, c)) { status = MF_ERR_DEADLOCK; break; }    // p complete
            tm.tick(8);
        }
    }
    if (blockIdx.x == 0 && t == 0) {
        a.out[0] = (double)j;
        a.out[1] = converged;
        a.out[3] = status;
    }
    tm.flush(a);
    if (status == MF_ERR_DEADLOCK && t == 0) atomicExch(a.abort_flag, 1);
}

// -------------------------------------------------------------------------- standalone kernels
// mf_spmv: the same windowed SpMV as the solver, one block per CTA of the launch plan
template <bool DYN, bool COUNT>
__global__ void __launch_bounds__(1024) spmv_kernel(Mat A, const int32_t* __restrict__ plan_tr, const int32_t* __restrict__ seg_lo,
                                                    const int32_t* __restrict__ seg_hi, const double* __restrict__ x,
                                                    double* __restrict__ y, const uint8_t* __restrict__ level,
                                                    int range_guard, unsigned long long* counts) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    int* ired = reinterpret_cast<int*>(smem_raw);
    mfk::WinSmem w;
    mfk::TsSmem tsm;
    mfk::carve_spmv(smem_raw + 64, w, tsm);
    mfk::pipe_init(tsm);
    __syncthreads();
    Counts cnt;
    cnt.zero();
    if (COUNT && threadIdx.x < 10) ired[threadIdx.x] = 0;
    const int64_t tr0 = plan_tr[blockIdx.x], tr1 = plan_tr[blockIdx.x + 1];
    const int64_t n = A.n_rows;
    mfk::spmv_cta<DYN, COUNT, 4>(A, tr0, tr1, x, level, range_guard, w, tsm, &cnt, seg_lo[blockIdx.x], seg_hi[blockIdx.x], nullptr,
                                 [&](int64_t TR, int ln, double v, double) {
        const int64_t i = TR * 16 + ln;
        if (i < n) y[i] = v;
    });
    if (COUNT) {
        __syncthreads();
#pragma unroll
        for (int q = 0; q < 5; ++q) {
            if (cnt.tiles(q)) atomicAdd(&ired[q], cnt.tiles(q));
            if (cnt.nnz(q)) atomicAdd(&ired[5 + q], cnt.nnz(q));
        }
        __syncthreads();
        if (threadIdx.x < 10 && ired[threadIdx.x]) atomicAdd(&counts[threadIdx.x], (unsigned long long)ired[threadIdx.x]);
    }
}

__global__ void levels_kernel(const double* __restrict__ v, int64_t n, Thresh th, uint8_t* level) {
    const unsigned m = mfk::hw_mask();
    const int lane = threadIdx.x & 15;
    const int64_t nseg = (n + 15) / 16;
    const int64_t H = (int64_t)gridDim.x * (blockDim.x >> 4);
    for (int64_t J = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 4; J < nseg; J += H) {
        const int64_t i = J * 16 + lane;
        const int lv = mfk::hw_min_i(i < n ? mfk::level_of(v[i], th) : 4, m);
        if (lane == 0) level[J] = (uint8_t)lv;
    }
}

// dot with the plan's tree: block g = CTA g of the plan, B threads
__global__ void dot_partial_kernel(const int32_t* __restrict__ plan_tr, int64_t n, const double* __restrict__ u,
                                   const double* __restrict__ v, double* slots) {
    __shared__ double red[32];
    const int64_t R0 = (int64_t)plan_tr[blockIdx.x] * 16, Rend = min((int64_t)plan_tr[blockIdx.x + 1] * 16, n);
    double acc = 0.0;
    for (int64_t i = R0 + threadIdx.x; i < Rend; i += blockDim.x) acc = __fma_rn(u[i], v[i], acc);
    const double wt = mfk::butterfly32(acc);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = wt;
    __syncthreads();
    if (threadIdx.x < 32) {
        const double ct = mfk::tree32(red, blockDim.x >> 5);
        if (threadIdx.x == 0) slots[blockIdx.x] = ct;
    }
}
// CG vector steps for the row-block multi-GPU driver (same plan tree as the persistent kernel):
//   xr: x += alpha p, r = fma(-alpha, mu, r), partial (r, r);   p: p = fma(beta, p, r)
__global__ void cg_xr_kernel(const int32_t* __restrict__ plan_tr, int64_t n, double alpha, const double* p, const double* mu,
                             double* x, double* r, double* slots) {
    __shared__ double red[32];
    const int64_t R0 = (int64_t)plan_tr[blockIdx.x] * 16, Rend = min((int64_t)plan_tr[blockIdx.x + 1] * 16, n);
    double acc = 0.0;
    for (int64_t i = R0 + threadIdx.x; i < Rend; i += blockDim.x) {
        x[i] = __fma_rn(alpha, p[i], x[i]);
        const double ri = __fma_rn(-alpha, mu[i], r[i]);
        r[i] = ri;
        acc = __fma_rn(ri, ri, acc);
    }
    const double wt = mfk::butterfly32(acc);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = wt;
    __syncthreads();
    if (threadIdx.x < 32) {
        const double ct = mfk::tree32(red, blockDim.x >> 5);
        if (threadIdx.x == 0) slots[blockIdx.x] = ct;
    }
}
__global__ void cg_p_kernel(int64_t n, double beta, const double* r, double* p) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = __fma_rn(beta, p[i], r[i]);
}

__global__ void dot_final_kernel(const double* __restrict__ slots, int G, double* out) {
    const double gt = mfk::tree32(slots, G);
    if (threadIdx.x == 0) *out = gt;
}

template <int MAXT>
void* pick_kernel(bool bicg, bool dyn, bool count, bool pre) {
    if (pre && bicg)
        return dyn ? (count ? (void*)pbicgstab_persistent<true, true, MAXT> : (void*)pbicgstab_persistent<true, false, MAXT>)
                   : (count ? (void*)pbicgstab_persistent<false, true, MAXT> : (void*)pbicgstab_persistent<false, false, MAXT>);
    if (pre)
        return dyn ? (count ? (void*)pcg_persistent<true, true, MAXT> : (void*)pcg_persistent<true, false, MAXT>)
                   : (count ? (void*)pcg_persistent<false, true, MAXT> : (void*)pcg_persistent<false, false, MAXT>);
    if (bicg) return dyn ? (count ? (void*)bicgstab_persistent<true, true, MAXT> : (void*)bicgstab_persistent<true, false, MAXT>)
                         : (count ? (void*)bicgstab_persistent<false, true, MAXT> : (void*)bicgstab_persistent<false, false, MAXT>);
    return dyn ? (count ? (void*)cg_persistent<true, true, MAXT> : (void*)cg_persistent<true, false, MAXT>)
               : (count ? (void*)cg_persistent<false, true, MAXT> : (void*)cg_persistent<false, false, MAXT>);
}

Mat mat_view(const TileMatrix& A) {
    return Mat{A.n_rows, A.n_cols, A.ntr, A.tr_slot, A.TileRowPtr, A.tile_info, A.sidx, A.blob,
               reinterpret_cast<const mfk::PipeStage*>(A.stg), A.stg_ptr, A.TileNnz, A.ts, (int)A.max_w,
               A.plane64, A.plane32, A.plane16, A.plane8, nullptr};
}

}  // namespace

// ------------------------------------------------------------------------------- host side
mf_status run_spmv(const TileMatrix& A, const double* x, double* y, const uint8_t* level, int range_guard,
                   int64_t* counts_host, cudaStream_t s) {
    if (A.ntr == 0) return MF_OK;
    Mat M = mat_view(A);
    unsigned long long* dcnt = nullptr;
    if (counts_host) {
        MF_TRY(alloc(&dcnt, 10, s));
        MF_CUDA(cudaMemsetAsync(dcnt, 0, 10 * sizeof(unsigned long long), s));
    }
    const size_t smem = 64 + mfk::SPMV_SMEM_BYTES;
    void* fn;
    if (level) fn = counts_host ? (void*)spmv_kernel<true, true> : (void*)spmv_kernel<true, false>;
    else fn = counts_host ? (void*)spmv_kernel<false, true> : (void*)spmv_kernel<false, false>;
    MF_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const int32_t* plan = A.plan_tr;
    const int32_t* slo = A.seg_lo;
    const int32_t* shi = A.seg_hi;
    void* args[] = {&M, (void*)&plan, (void*)&slo, (void*)&shi, (void*)&x, (void*)&y, (void*)&level, &range_guard, &dcnt};
    MF_CUDA(cudaLaunchKernel(fn, dim3(A.G), dim3(A.B), args, smem, s));
    if (counts_host) {
        unsigned long long h[10];
        MF_CUDA(cudaMemcpyAsync(h, dcnt, sizeof(h), cudaMemcpyDeviceToHost, s));
        MF_CUDA(cudaStreamSynchronize(s));
        for (int q = 0; q < 5; ++q) counts_host[q] = (int64_t)h[q];
        dev_free(dcnt, s);
    }
    return MF_OK;
}

mf_status run_levels(const double* v, int64_t n, const double* th, uint8_t* level, cudaStream_t s) {
    if (n == 0) return MF_OK;
    Thresh t{th[0], th[1], th[2], th[3]};
    int64_t nseg = (n + 15) / 16;
    int blocks = (int)std::min<int64_t>((nseg + 15) / 16, 148 * 16);
    levels_kernel<<<blocks, 256, 0, s>>>(v, n, t, level);
    MF_CUDA(cudaGetLastError());
    return MF_OK;
}

mf_status run_dot(const TileMatrix& A, const double* u, const double* v, double* out_host, cudaStream_t s) {
    double* slots = nullptr;
    MF_TRY(alloc(&slots, A.G + 1, s));
    dot_partial_kernel<<<A.G, A.B, 0, s>>>(A.plan_tr, A.n_rows, u, v, slots);
    dot_final_kernel<<<1, 32, 0, s>>>(slots, A.G, slots + A.G);
    MF_CUDA(cudaGetLastError());
    MF_CUDA(cudaMemcpyAsync(out_host, slots + A.G, sizeof(double), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    dev_free(slots, s);
    return MF_OK;
}

mf_status run_cg_xr(const TileMatrix& A, double alpha, const double* p, const double* mu, double* x, double* r,
                    double* rr_host, cudaStream_t s) {
    double* slots = nullptr;
    MF_TRY(alloc(&slots, A.G + 1, s));
    cg_xr_kernel<<<A.G, A.B, 0, s>>>(A.plan_tr, A.n_rows, alpha, p, mu, x, r, slots);
    dot_final_kernel<<<1, 32, 0, s>>>(slots, A.G, slots + A.G);
    MF_CUDA(cudaGetLastError());
    MF_CUDA(cudaMemcpyAsync(rr_host, slots + A.G, sizeof(double), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    dev_free(slots, s);
    return MF_OK;
}

mf_status run_cg_p(const TileMatrix& A, double beta, const double* r, double* p, cudaStream_t s) {
    if (A.n_rows == 0) return MF_OK;
    const int blocks = (int)std::min<int64_t>((A.n_rows + 255) / 256, 148 * 8);
    cg_p_kernel<<<blocks, 256, 0, s>>>(A.n_rows, beta, r, p);
    MF_CUDA(cudaGetLastError());
    return MF_OK;
}

// byte model per SpMV: values at e_t + 0.5 B/nnz + 1 B per non-empty
// tile row + 8 B per tile, non-bypassed tiles only (index bytes of bypassed tiles excluded)
static double spmv_model_bytes(const TileMatrix& A, const unsigned long long* c10) {
    static const double vb[4] = {8, 4, 2, 1};
    double bytes = 0;
    double tiles_nb = 0, nnz_nb = 0;
    for (int q = 0; q < 4; ++q) { bytes += vb[q] * (double)c10[5 + q]; tiles_nb += (double)c10[q]; nnz_nb += (double)c10[5 + q]; }
    const double tiles_all = tiles_nb + (double)c10[4];
    const double rows_frac = tiles_all > 0 ? tiles_nb / tiles_all : 0;
    return bytes + 0.5 * nnz_nb + (double)A.rownum * rows_frac + 8.0 * tiles_nb;
}

mf_status run_solve(const TileMatrix& A, bool bicg, const double* b, double* x, const mf_solve_opts& o,
                    mf_solve_info* info, cudaStream_t s) {
    if (A.n_rows != A.n_cols) return fail(MF_ERR_INVALID_ARG, "solve needs a square matrix");
    // sticky variant (P:237 literal): dynamic mode only (as in the oracle), tile-synchronous layout
    const bool sticky = o.sticky && o.mode == MF_MODE_DYNAMIC_MIXED;
    if (sticky && !A.ts && (A.n_cols + 15) / 16 > ((int64_t)1 << 24))
        return fail(MF_ERR_NOT_IMPLEMENTED, "sticky downgrade, compact layout: more than 2^24 tile columns");
    if (sticky && (o.tile_level_counts != nullptr || o.collect_stats))
        return fail(MF_ERR_NOT_IMPLEMENTED, "sticky downgrade does not collect per-SpMV level statistics");
    Precond* P = o.M ? const_cast<Precond*>(&o.M->p) : nullptr;
    const bool pre = P != nullptr;
    if (pre && P->n != A.n_rows) return fail(MF_ERR_INVALID_ARG, "preconditioner built for another matrix size");
    int dev = 0, sms = 0, smem_optin = 0;
    MF_CUDA(cudaGetDevice(&dev));
    MF_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    MF_CUDA(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    const int64_t n = A.n_rows;
    const int G = A.G, B = A.B, H = B / 16;
    const bool dyn = o.mode == MF_MODE_DYNAMIC_MIXED;
    const int nvec = bicg ? 2 : 1;
    // per-SpMV level statistics (tile_level_counts, exact dynamic byte model) cost ALU in the
    // SpMV loop: collected only on request
    const bool count = o.tile_level_counts != nullptr || o.collect_stats;
    int64_t max_rows = 0;
    for (int g = 0; g < G; ++g) max_rows = std::max(max_rows, A.plan_rows_host[g + 1] - A.plan_rows_host[g]);
    const size_t fixed = fixed_smem_bytes();
    (void)H;
    int64_t cap = ((int64_t)smem_optin - (int64_t)fixed - 64) / (8 * nvec);
    cap = std::max<int64_t>(0, std::min(cap, max_rows));
    // the TMA pipeline (tile-synchronous layout) spends shared memory on stages in flight; the SpMV
    // outputs then live in global memory (L2-resident: the matrix streams with evict_first)
    if (A.ts) cap = 0;
    if (const char* ev = getenv("MF_MU_ONCHIP")) if (atoi(ev) == 0) cap = 0;   // tuning: trade smem for L1
    const size_t pre_smem = pre ? (size_t)B * 12 + 32 : 0;
    cap = std::max<int64_t>(0, std::min<int64_t>(cap, ((int64_t)smem_optin - (int64_t)fixed - (int64_t)pre_smem - 64) / (8 * nvec)));
    const size_t smem = fixed + (size_t)cap * 8 * nvec + pre_smem;

    // workspace
    double *r = nullptr, *p = nullptr, *mu_g = nullptr, *rh = nullptr, *sv = nullptr, *th_g = nullptr;
    double *slots = nullptr, *hist = nullptr, *out = nullptr;
    uint8_t *lev_p = nullptr, *lev_s = nullptr;
    unsigned* sync = nullptr;
    unsigned long long *lcounts = nullptr, *bar_ns = nullptr, *phase_ns = nullptr;
    const bool spill = cap < max_rows;
    const int64_t hist_cap = o.max_iter + 2;
    const int64_t lc_cap = (bicg ? 2 : 1) * (o.max_iter + 1);
    MF_TRY(alloc(&r, n, s));
    MF_TRY(alloc(&p, n, s));
    if (spill) MF_TRY(alloc(&mu_g, n, s));
    MF_TRY(alloc(&lev_p, A.ntr + 1, s));
    if (bicg) {
        MF_TRY(alloc(&rh, n, s));
        MF_TRY(alloc(&sv, n, s));
        MF_TRY(alloc(&lev_s, A.ntr + 1, s));
        if (spill) MF_TRY(alloc(&th_g, n, s));
    }
    MF_TRY(alloc(&slots, (size_t)2 * NSLOT * G, s));
    MF_TRY(alloc(&hist, hist_cap, s));
    MF_TRY(alloc(&out, 8, s));
    MF_TRY(alloc(&sync, (size_t)G + 2, s));
    MF_TRY(alloc(&bar_ns, G, s));
    MF_TRY(alloc(&phase_ns, (size_t)G * NPHASE, s));
    MF_CUDA(cudaMemsetAsync(phase_ns, 0, (size_t)G * NPHASE * sizeof(unsigned long long), s));
    if (count) MF_TRY(alloc(&lcounts, (size_t)lc_cap * 10, s));
    MF_CUDA(cudaMemsetAsync(sync, 0, (G + 2) * sizeof(unsigned), s));
    MF_CUDA(cudaMemsetAsync(bar_ns, 0, G * sizeof(unsigned long long), s));
    MF_CUDA(cudaMemsetAsync(out, 0, 8 * sizeof(double), s));
    if (count) MF_CUDA(cudaMemsetAsync(lcounts, 0, (size_t)lc_cap * 10 * sizeof(unsigned long long), s));

    uint8_t* stk = nullptr;
    if (sticky) {
        const size_t nst = (size_t)(A.ts ? A.slots : A.tilenum) + 1;   // per slice column (TS) / per tile (compact)
        MF_TRY(alloc(&stk, nst, s));
        MF_CUDA(cudaMemsetAsync(stk, 0, nst, s));
    }
    SolveArgs a{};
    a.A = mat_view(A);
    a.A.stk = stk;
    a.G = G; a.plan_tr = A.plan_tr; a.dep_lo = A.dep_lo; a.dep_hi = A.dep_hi; a.seg_lo = A.seg_lo; a.seg_hi = A.seg_hi;
    a.n = n; a.b = b; a.x = x; a.r = r; a.p = p; a.mu_g = mu_g; a.lev_p = lev_p;
    a.rh = rh; a.s = sv; a.th_g = th_g; a.lev_s = lev_s;
    a.slots = slots; a.bar = sync; a.abort_flag = reinterpret_cast<int*>(sync + 1); a.flags = sync + 2;
    a.bar_ns = bar_ns; a.phase_ns = phase_ns; a.hist = hist; a.hist_cap = hist_cap; a.lcounts = lcounts; a.lc_cap = count ? lc_cap : 0;
    a.out = out; a.tol = o.tol; a.switch_eps = o.switch_eps < 0 ? o.tol : o.switch_eps;   // reading R8: eps = tol
    a.switch_abs = o.switch_absolute; a.range_guard = o.range_guard; a.max_iter = o.max_iter;
    a.mu_cap = (int)cap; a.timeout_ns = 60ull * 1000000000ull;
    double *pz = nullptr, *psh = nullptr;
    if (pre) {
        MF_TRY(alloc(&pz, n, s));
        if (bicg) MF_TRY(alloc(&psh, n, s));
        const unsigned reserve = (unsigned)std::min<int64_t>((bicg ? 2 : 1) * (o.max_iter + 2) + 2, 0x3FFFFFFF);
        if ((uint64_t)P->epoch + reserve >= 0x7FFFFFF0ull) {
            MF_CUDA(cudaMemsetAsync(P->flags, 0, (P->n + 1) * sizeof(unsigned), s));
            P->epoch = 0;
        }
        a.pe0 = P->epoch + 1;
        P->epoch += reserve;
        MF_CUDA(cudaMemsetAsync(P->ctr, 0, 2 * sizeof(unsigned long long), s));
        a.Lrp = P->L.rp; a.Lci = P->L.ci; a.Lv = P->L.v;
        a.Urp = P->U.rp; a.Uci = P->U.ci; a.Uv = P->U.v; a.Ud = P->udiag;
        a.pflags = P->flags; a.pctr = P->ctr; a.py = P->y; a.pz = pz; a.ps = psh;
    }

    void* kfn = B > 512 ? pick_kernel<1024>(bicg, dyn, count, pre) : pick_kernel<512>(bicg, dyn, count, pre);
    MF_CUDA(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int per_sm = 0;
    MF_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kfn, B, smem));
    if (per_sm * sms < G) return fail(MF_ERR_INVALID_ARG, "plan G exceeds co-resident CTAs for this launch");

    cudaEvent_t e0, e1;
    MF_CUDA(cudaEventCreate(&e0));
    MF_CUDA(cudaEventCreate(&e1));
    void* args[] = {&a};
    MF_CUDA(cudaEventRecord(e0, s));
    MF_CUDA(cudaLaunchCooperativeKernel(kfn, dim3(G), dim3(B), args, smem, s));
    MF_CUDA(cudaEventRecord(e1, s));
    double hout[8];
    MF_CUDA(cudaMemcpyAsync(hout, out, sizeof(hout), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    float ms = 0;
    MF_CUDA(cudaEventElapsedTime(&ms, e0, e1));
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    const int64_t iters = (int64_t)hout[0];
    info->iterations = iters;
    info->converged = (int)hout[1];
    info->rel_residual = hout[2];
    info->status = (mf_status)(int)hout[3];
    info->kernel_ms = ms;
    info->launches = 1;
    const int64_t nspmv = (bicg ? 2 : 1) * iters;
    info->n_spmv = nspmv;
    if (o.residual_history && o.history_cap > 0) {
        const int64_t k = std::min<int64_t>(o.history_cap, std::min<int64_t>(iters + 1, hist_cap));
        MF_CUDA(cudaMemcpyAsync(o.residual_history, hist, k * sizeof(double), cudaMemcpyDeviceToHost, s));
    }
    std::vector<unsigned long long> ph((size_t)G * NPHASE), bns(G);
    MF_CUDA(cudaMemcpyAsync(ph.data(), phase_ns, ph.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaMemcpyAsync(bns.data(), bar_ns, bns.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
    std::vector<unsigned long long> lc;
    if (count) {
        const int64_t k = std::min<int64_t>(lc_cap, nspmv + 2);
        lc.resize((size_t)k * 10);
        MF_CUDA(cudaMemcpyAsync(lc.data(), lcounts, lc.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
    }
    MF_CUDA(cudaStreamSynchronize(s));
    double model = 0;
    if (!count) {   // every tile at TilePrec, nothing bypassed (static / FP64 modes)
        unsigned long long c10[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
        for (int q = 0; q < 4; ++q) { c10[q] = (unsigned long long)A.tiles_per_prec[q]; c10[5 + q] = (unsigned long long)A.nval[q]; }
        model = dyn ? 0.0 : spmv_model_bytes(A, c10) * (double)nspmv;
    } else {
        const int64_t k = (int64_t)lc.size() / 10;
        for (int64_t q = 0; q < k; ++q) {
            unsigned long long tot = 0;
            for (int e = 0; e < 5; ++e) tot += lc[q * 10 + e];
            if (tot == 0) continue;
            model += spmv_model_bytes(A, &lc[q * 10]);
            if (o.tile_level_counts && q < o.level_counts_cap)
                for (int e = 0; e < 5; ++e) o.tile_level_counts[q * 5 + e] = (int64_t)lc[q * 10 + e];
        }
    }
    // vectors: CG 48n per iteration (read p,x,r; write x,r,p); BiCGSTAB 72n (read p,x,r,r0*,s;
    // write s,x,r,p); + 16n per SpMV output that cannot stay on chip (capacity rule)
    const double vec = bicg ? 72.0 : 48.0;
    // capacity rule: the SpMV outputs count as HBM traffic only when they cannot fit
    // the GPU's shared memory, whatever this launch chose to do with them
    int smem_sm = 0;
    MF_CUDA(cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev));
    const bool over_cap = 8.0 * (double)n * (double)nvec > (double)sms * (double)smem_sm;
    const double spill_b = over_cap ? (bicg ? 32.0 : 16.0) : 0.0;
    info->model_bytes = model + (vec + spill_b) * (double)n * (double)iters;
    if (pre) {   // per apply: L and U values + column indices, row pointers, the vectors in/y/out
        const double apply_b = 12.0 * (double)(P->nnz_l + P->nnz_u) + 16.0 * (double)n + 8.0 * n + 32.0 * (double)n;
        info->model_bytes += apply_b * (double)((bicg ? 2 : 1) * iters + 1);
    }
    for (int k = 0; k < NPHASE && k < 12; ++k) {
        double sum = 0;
        for (int g = 0; g < G; ++g) sum += (double)ph[(size_t)g * NPHASE + k];
        info->phase_ms[k] = sum / G / 1e6;
    }
    if (getenv("MF_PHASE_DUMP")) {   // diagnostics: per-phase min / mean / max over CTAs (ms)
        for (int k = 0; k < NPHASE; ++k) {
            double mn = 1e300, mx = 0, sum = 0;
            for (int g = 0; g < G; ++g) { const double v = (double)ph[(size_t)g * NPHASE + k] / 1e6; mn = std::min(mn, v); mx = std::max(mx, v); sum += v; }
            if (mx > 0) fprintf(stderr, "phase %2d: min %.3f mean %.3f max %.3f ms\n", k, mn, sum / G, mx);
        }
        fprintf(stderr, "spmv per CTA:");
        for (int g = 0; g < G; ++g) fprintf(stderr, " %.2f", (double)ph[(size_t)g * NPHASE + 1] / 1e6);
        fprintf(stderr, "\nrows per CTA:");
        for (int g = 0; g < G; ++g) fprintf(stderr, " %lld", (long long)(A.plan_rows_host[g + 1] - A.plan_rows_host[g]));
        fprintf(stderr, "\n");
    }
    {
        double sum = 0;
        for (int g = 0; g < G; ++g) sum += (double)bns[g];
        info->barrier_ms = sum / G / 1e6;   // mean over CTAs of time spent spinning (barriers + ready flags)
    }
    mf_status st = info->status;
    dev_free(r, s); dev_free(p, s); dev_free(mu_g, s); dev_free(lev_p, s); dev_free(rh, s); dev_free(sv, s);
    dev_free(lev_s, s); dev_free(th_g, s); dev_free(slots, s); dev_free(hist, s); dev_free(out, s);
    dev_free(sync, s); dev_free(bar_ns, s); dev_free(phase_ns, s); dev_free(lcounts, s);
    dev_free(pz, s); dev_free(psh, s); dev_free(stk, s);
    if (st == MF_ERR_BREAKDOWN) return fail(st, "numerical breakdown");
    if (st == MF_ERR_DEADLOCK) return fail(st, "grid-barrier watchdog expired");
    return st;
}

}  // namespace mf
