// dist.cu -- the row-block multi-GPU path (SURVEY.md 8(b) mf_comm_* / *_dist, 8(e)).
//
// The paper's solver is single-GPU; for matrices too large for one GPU (C5) the rows are
// partitioned into contiguous blocks of whole tile rows, one block per GPU (one process per
// GPU, NCCL over NVLink).  Rank k owns rows [row_begin, row_end) and converts them as a local
// n_local x n_ext tile matrix whose columns are its own 16-element segments followed by the
// HALO segments it gathers from other ranks (sorted by global segment, so the halo of each peer
// is one contiguous block).  Segments map one-to-one, so tiles, TilePrec, the range floor and
// the dynamic levels of Alg. 4 are those of the global matrix.
//
// Per CG iteration (Alg. 1), every step on the device, stream-ordered, no host sync:
//   halo exchange of the SpMV input in the PV layout (values + level bytes; one grouped
//   ncclSend/ncclRecv per peer) -> staged SpMV of the local tiles with the fused per-CTA partial
//   (mu, p) (plan tree) -> rank partial -> ncclAllGather -> every rank sums the partials in rank
//   order from +0 and derives alpha (device scalars) -> r -= alpha mu, partial (r, r) -> same
//   reduction -> beta, relres, stop test -> x += alpha p, p = r + beta p with the levels.
// With ONE rank every reduction is the single kernel's tree plus "+0": the solve is bit-identical
// to mf_cg_solve and to the oracle's kernel-order emulation.  Iterations are enqueued in chunks
// captured once as a CUDA graph; a device "done" flag turns the iterations after the stop into
// no-ops, the host polls it once per chunk.
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <vector>

#include <chrono>
#include <condition_variable>
#include <memory>
#include <mutex>
#include <nccl_device.h>

#include "kernels.cuh"
#include "mf_internal.cuh"

namespace mf {

#define MF_NCCL(call)                                                                        \
    do {                                                                                     \
        ncclResult_t r_ = (call);                                                            \
        if (r_ != ncclSuccess) return ::mf::fail(MF_ERR_NCCL, std::string(#call) + ": " + ncclGetErrorString(r_)); \
    } while (0)

struct LocalGroup;
struct Comm {
    ncclComm_t nccl = nullptr;
    int nranks = 0, rank = 0;
    LocalGroup* local = nullptr;     // in-process rank group (ranks emulated on one device)
};

namespace {

using mfk::PVS;
using mfk::pv_idx;
using mfk::Thresh;

constexpr int DS_DONE = 0, DS_STATUS = 1, DS_CONV = 2;            // int state
// double scalars
enum { S_NB = 0, S_RHO, S_RR, S_ALPHA, S_BETA, S_OMEGA, S_RELRES, S_ETA, S_TH0, S_TH1, S_TH2, S_TH3, S_NSC };

struct DistArgs {
    mfk::Mat A;
    int32_t G;
    const int32_t* plan_tr;
    int64_t n;                  // local rows
    int64_t nown_seg;           // own segments (ceil(n / 16))
    const double* b;
    double* x;
    double* r;
    double* pv;                 // PV layout over own + halo segments (CG: p; BiCGSTAB: p)
    double* sv;                 // BiCGSTAB: s (PV)
    double* rh;                 // BiCGSTAB: r0*
    double* mu;                 // [n]
    double* th;                 // [n] BiCGSTAB theta
    double* slots;              // [4][G] per-CTA partials
    double* part;               // [4] rank partials (allgather send)
    double* gath;               // [4 * P] allgather receive
    int P;
    double* sc;                 // [S_NSC] device scalars
    int* st;                    // [4] device state: done, status, converged
    int64_t* iter;              // [1] iterations done
    double* hist;               // [hist_cap]
    int64_t hist_cap, max_iter;
    double tol, switch_eps;
    int switch_abs, range_guard, dyn;
    int nst, slot_bytes, blob_cap, ecap;
};

__device__ __forceinline__ bool is_done(const DistArgs& a) { return *(volatile int*)&a.st[DS_DONE] != 0; }

// per-CTA K partials of the plan tree (thread fma chains -> butterfly -> tree32 over warps)
template <int K>
__device__ __forceinline__ void cta_partials(double (&v)[K], double* slots, int G) {
    __shared__ double red[4 * 32];
    const int w = threadIdx.x >> 5, l = threadIdx.x & 31, W = blockDim.x >> 5;
#pragma unroll
    for (int k = 0; k < K; ++k) {
        const double wt = mfk::butterfly32(v[k]);
        if (l == 0) red[k * 32 + w] = wt;
    }
    __syncthreads();
    if (w == 0)
#pragma unroll
        for (int k = 0; k < K; ++k) {
            const double ct = mfk::tree32(red + k * 32, W);
            if (l == 0) slots[(size_t)k * G + blockIdx.x] = ct;
        }
}

// one block of 32: the rank partials (tree32 over the G CTA slots of each of k sums)
__global__ void k_rank_partial(DistArgs a, int k) {
    if (is_done(a)) return;
    for (int q = 0; q < k; ++q) {
        const double t = mfk::tree32(a.slots + (size_t)q * a.G, a.G);
        if (threadIdx.x == 0) a.part[q] = t;
    }
}
// rank-order sum of an all-gathered partial (layout [rank][k]) from +0
__device__ __forceinline__ double rank_sum(const DistArgs& a, int k, int K) {
    double s = 0.0;
    for (int r = 0; r < a.P; ++r) s = __dadd_rn(s, a.gath[r * K + k]);
    return s;
}

__device__ __forceinline__ void record(const DistArgs& a, int64_t j, double relres) {
    if (j < a.hist_cap) a.hist[j] = relres;
    a.sc[S_RELRES] = relres;
}
__device__ __forceinline__ void finish(const DistArgs& a, int status, int conv) {
    a.st[DS_STATUS] = status;
    a.st[DS_CONV] = conv;
    a.st[DS_DONE] = 1;
}

// x0 -> own PV segments (level FP64), padding rows zero
__global__ void k_stage_x0(DistArgs a, double* pv) {
    const int64_t nown = a.nown_seg * 16;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nown; i += (int64_t)gridDim.x * blockDim.x) {
        pv[pv_idx(i)] = i < a.n ? a.x[i] : 0.0;
        if ((i & 15) == 0) { pv[(i >> 4) * PVS + 16] = 0.0; pv[(i >> 4) * PVS + 17] = 0.0; }
    }
}

// gather my PV segments that peers need into the send buffer
__global__ void k_pack(const double* __restrict__ pv, const int32_t* __restrict__ idx, int64_t nseg, double* buf,
                       const int* st) {
    if (*(volatile const int*)&st[DS_DONE]) return;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nseg * PVS; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t s = k / PVS, e = k - s * PVS;
        buf[k] = pv[(int64_t)idx[s] * PVS + e];
    }
}

// SpMV of the local tiles over the extended PV vector.  MODE 0: init r = b - A x0, partials
// (b,b), (r,r); MODE 1: CG mu = A p, partial (mu, p); MODE 2: BiCGSTAB mu = A p, partial
// (mu, r0*); MODE 3: BiCGSTAB theta = A s, partials (theta, theta), (theta, s).
template <bool DYN, int MODE, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) k_spmv(DistArgs a, const double* in) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    if (MODE != 0 && is_done(a)) return;
    mfk::SpmvSmem sp;
    mfk::carve_spmv(smem_raw + 128, a.nst, a.slot_bytes, a.blob_cap, a.ecap, sp);
    mfk::ts_init(sp.ts);
    __syncthreads();
    const int64_t tr0 = a.plan_tr[blockIdx.x], tr1 = a.plan_tr[blockIdx.x + 1];
    const int64_t n = a.n;
    double v[2] = {0.0, 0.0};
    const int own_mode = MODE == 1 || MODE == 3 ? 1 : (MODE == 2 ? 2 : 0);
    mfk::spmv_cta<DYN, false, MAXT >= 1024 ? 4 : 8>(a.A, tr0, tr1, in, a.range_guard, sp, own_mode, a.rh,
        [&](int64_t TR, int ln, double y, double ov) {
            const int64_t i = TR * 16 + ln;
            if (i >= n) return;
            if (MODE == 0) {
                const double bi = a.b[i], ri = __dsub_rn(bi, y);
                a.r[i] = ri;
                v[0] = __fma_rn(bi, bi, v[0]);
                v[1] = __fma_rn(ri, ri, v[1]);
            } else if (MODE == 1 || MODE == 2) {
                a.mu[i] = y;
                v[0] = __fma_rn(y, ov, v[0]);
            } else {
                a.th[i] = y;
                v[0] = __fma_rn(y, y, v[0]);
                v[1] = __fma_rn(y, ov, v[1]);
            }
        });
    cta_partials<2>(v, a.slots, a.G);
}

// levels of the own segments of a PV vector (Alg. 4) from the device thresholds
__device__ __forceinline__ void own_level_store(const DistArgs& a, double* pv, int64_t i, double val, bool valid,
                                                const Thresh& th, unsigned m) {
    int lv = 0;
    if (a.dyn) lv = mfk::hw_min_i(valid ? mfk::level_of(val, th) : 4, m);
    if ((i & 15) == 0) mfk::pv_set_level(pv, i >> 4, lv);
}
__device__ __forceinline__ Thresh dev_thresh(const DistArgs& a) {
    return Thresh{a.sc[S_TH0], a.sc[S_TH1], a.sc[S_TH2], a.sc[S_TH3]};
}

// ---------------------------------------------------------------------------------- CG
// after the init reduction: nb, rho, tau / thresholds; stop test at j = 0
__global__ void k_cg_init_scalars(DistArgs a) {
    const double nb = sqrt(rank_sum(a, 0, 2)), rr = rank_sum(a, 1, 2);
    a.sc[S_NB] = nb;
    a.sc[S_RHO] = rr;
    const double tau = a.switch_abs ? a.switch_eps : __dmul_rn(a.switch_eps, sqrt(rr));   // reading R8
    a.sc[S_TH0] = __dmul_rn(tau, 1e-3); a.sc[S_TH1] = __dmul_rn(tau, 1e-2); a.sc[S_TH2] = __dmul_rn(tau, 1e-1); a.sc[S_TH3] = tau;
    *a.iter = 0;
    if (nb == 0.0) { record(a, 0, 0.0); finish(a, MF_OK, 1); return; }
    const double relres = __ddiv_rn(sqrt(rr), nb);
    record(a, 0, relres);
    if (relres < a.tol) finish(a, MF_OK, 1);
    else if (a.max_iter == 0) finish(a, MF_OK, 0);
}
// p0 = r0 (PV, own rows) + levels
__global__ void k_cg_p0(DistArgs a) {
    if (is_done(a)) return;
    const Thresh th = dev_thresh(a);
    const unsigned m = mfk::hw_mask();
    const int64_t R0 = (int64_t)a.plan_tr[blockIdx.x] * 16, R1 = (int64_t)a.plan_tr[blockIdx.x + 1] * 16;
    for (int64_t i = R0 + threadIdx.x; i < R1; i += blockDim.x) {
        const bool valid = i < a.n;
        const double pv = valid ? a.r[i] : 0.0;
        a.pv[pv_idx(i)] = pv;
        own_level_store(a, a.pv, i, pv, valid, th, m);
    }
}
// sigma -> alpha (breakdown test)
__global__ void k_cg_alpha(DistArgs a) {
    if (is_done(a)) return;
    const double sigma = rank_sum(a, 0, 2);
    if (!(sigma > 0.0) || !isfinite(sigma)) { finish(a, MF_ERR_BREAKDOWN, 0); return; }
    a.sc[S_ALPHA] = __ddiv_rn(a.sc[S_RHO], sigma);
}
// r -= alpha mu, partial (r, r)
__global__ void k_cg_r(DistArgs a) {
    if (is_done(a)) return;
    const double alpha = a.sc[S_ALPHA];
    const int64_t R0 = (int64_t)a.plan_tr[blockIdx.x] * 16, R1 = min((int64_t)a.plan_tr[blockIdx.x + 1] * 16, a.n);
    double v[1] = {0.0};
    for (int64_t i = R0 + threadIdx.x; i < R1; i += blockDim.x) {
        const double ri = __fma_rn(-alpha, a.mu[i], a.r[i]);
        a.r[i] = ri;
        v[0] = __fma_rn(ri, ri, v[0]);
    }
    cta_partials<1>(v, a.slots, a.G);
}
// rr -> beta, rho; iteration count, relres, stop test
__global__ void k_cg_beta(DistArgs a) {
    if (is_done(a)) return;
    const double rr = rank_sum(a, 0, 1);
    a.sc[S_BETA] = __ddiv_rn(rr, a.sc[S_RHO]);
    a.sc[S_RHO] = rr;
    const int64_t j = ++*a.iter;
    const double relres = __ddiv_rn(sqrt(rr), a.sc[S_NB]);
    record(a, j, relres);
    // the p update below still runs (as the single kernel's step D does before its stop test)
    if (relres < a.tol) a.st[DS_CONV] = 1;
}
// x += alpha p ; p = r + beta p (PV) + levels; then the stop decision
__global__ void k_cg_xp(DistArgs a) {
    if (is_done(a)) return;
    const double alpha = a.sc[S_ALPHA], beta = a.sc[S_BETA];
    const Thresh th = dev_thresh(a);
    const unsigned m = mfk::hw_mask();
    const int64_t R0 = (int64_t)a.plan_tr[blockIdx.x] * 16, R1 = (int64_t)a.plan_tr[blockIdx.x + 1] * 16;
    for (int64_t i = R0 + threadIdx.x; i < R1; i += blockDim.x) {
        const bool valid = i < a.n;
        double pn = 0.0;
        if (valid) {
            const double pv = a.pv[pv_idx(i)];
            a.x[i] = __fma_rn(alpha, pv, a.x[i]);
            pn = __fma_rn(beta, pv, a.r[i]);
            a.pv[pv_idx(i)] = pn;
        }
        own_level_store(a, a.pv, i, pn, valid, th, m);
    }
}
__global__ void k_cg_stop(DistArgs a) {
    if (is_done(a)) return;
    if (a.st[DS_CONV]) finish(a, MF_OK, 1);
    else if (*a.iter >= a.max_iter) finish(a, MF_OK, 0);
}

// ---------------------------------------------------------------------------------- BiCGSTAB
__global__ void k_bicg_init_scalars(DistArgs a) {
    const double nb = sqrt(rank_sum(a, 0, 2)), rr = rank_sum(a, 1, 2);
    a.sc[S_NB] = nb;
    a.sc[S_RR] = rr;
    a.sc[S_RHO] = rr;                  // (r0, r0*) with r0* = r0
    const double tau = a.switch_abs ? a.switch_eps : __dmul_rn(a.switch_eps, sqrt(rr));
    a.sc[S_TH0] = __dmul_rn(tau, 1e-3); a.sc[S_TH1] = __dmul_rn(tau, 1e-2); a.sc[S_TH2] = __dmul_rn(tau, 1e-1); a.sc[S_TH3] = tau;
    *a.iter = 0;
    if (nb == 0.0) { record(a, 0, 0.0); finish(a, MF_OK, 1); return; }
    const double relres = __ddiv_rn(sqrt(rr), nb);
    record(a, 0, relres);
    if (relres < a.tol) finish(a, MF_OK, 1);
    else if (a.max_iter == 0) finish(a, MF_OK, 0);
}
// r0* = r0, p0 = r0 (PV) + levels
__global__ void k_bicg_p0(DistArgs a) {
    if (is_done(a)) return;
    const Thresh th = dev_thresh(a);
    const unsigned m = mfk::hw_mask();
    const int64_t R0 = (int64_t)a.plan_tr[blockIdx.x] * 16, R1 = (int64_t)a.plan_tr[blockIdx.x + 1] * 16;
    for (int64_t i = R0 + threadIdx.x; i < R1; i += blockDim.x) {
        const bool valid = i < a.n;
        const double ri = valid ? a.r[i] : 0.0;
        if (valid) a.rh[i] = ri;
        a.pv[pv_idx(i)] = ri;
        own_level_store(a, a.pv, i, ri, valid, th, m);
    }
}
// eta -> alpha ; s = r - alpha mu (PV) + levels
__global__ void k_bicg_s(DistArgs a) {
    if (is_done(a)) return;
    const double eta = rank_sum(a, 0, 2);
    if (eta == 0.0 || !isfinite(eta)) {
        if (threadIdx.x == 0 && blockIdx.x == 0) finish(a, MF_ERR_BREAKDOWN, 0);
        return;
    }
    const double alpha = __ddiv_rn(a.sc[S_RHO], eta);
    if (threadIdx.x == 0 && blockIdx.x == 0) a.sc[S_ALPHA] = alpha;
    const Thresh th = dev_thresh(a);
    const unsigned m = mfk::hw_mask();
    const int64_t R0 = (int64_t)a.plan_tr[blockIdx.x] * 16, R1 = (int64_t)a.plan_tr[blockIdx.x + 1] * 16;
    for (int64_t i = R0 + threadIdx.x; i < R1; i += blockDim.x) {
        const bool valid = i < a.n;
        double si = 0.0;
        if (valid) { si = __fma_rn(-alpha, a.mu[i], a.r[i]); a.sv[pv_idx(i)] = si; }
        own_level_store(a, a.sv, i, si, valid, th, m);
    }
}
// tt, ts -> omega; x += alpha p + omega s; r = s - omega theta; partials (r, r0*), (r, r).
// theta == 0 (reading R14): the half step x += alpha p, r = s, partial (s, s); k_bicg_beta ends.
__global__ void k_bicg_xr(DistArgs a) {
    if (is_done(a)) return;
    const double tt = rank_sum(a, 0, 2), ts = rank_sum(a, 1, 2);
    const double alpha = a.sc[S_ALPHA];
    const int64_t R0 = (int64_t)a.plan_tr[blockIdx.x] * 16, R1 = min((int64_t)a.plan_tr[blockIdx.x + 1] * 16, a.n);
    double v[2] = {0.0, 0.0};
    if (tt == 0.0) {
        if (threadIdx.x == 0 && blockIdx.x == 0) a.st[3] = 1;
        for (int64_t i = R0 + threadIdx.x; i < R1; i += blockDim.x) {
            a.x[i] = __fma_rn(alpha, a.pv[pv_idx(i)], a.x[i]);
            const double si = a.sv[pv_idx(i)];
            a.r[i] = si;
            v[1] = __fma_rn(si, si, v[1]);
        }
    } else {
        const double omega = __ddiv_rn(ts, tt);
        if (omega == 0.0 || !isfinite(omega)) {
            if (threadIdx.x == 0 && blockIdx.x == 0) finish(a, MF_ERR_BREAKDOWN, 0);
            return;
        }
        if (threadIdx.x == 0 && blockIdx.x == 0) a.sc[S_OMEGA] = omega;
        for (int64_t i = R0 + threadIdx.x; i < R1; i += blockDim.x) {
            const double si = a.sv[pv_idx(i)];
            a.x[i] = __fma_rn(omega, si, __fma_rn(alpha, a.pv[pv_idx(i)], a.x[i]));
            const double ri = __fma_rn(-omega, a.th[i], si);
            a.r[i] = ri;
            v[0] = __fma_rn(ri, a.rh[i], v[0]);
            v[1] = __fma_rn(ri, ri, v[1]);
        }
    }
    cta_partials<2>(v, a.slots, a.G);
}
// rho', rr -> beta; iteration count, relres, stop decision (breakdowns as the single kernel)
__global__ void k_bicg_beta(DistArgs a) {
    if (is_done(a)) return;
    const double rho1 = rank_sum(a, 0, 2), rr = rank_sum(a, 1, 2);
    const int64_t j = ++*a.iter;
    const double relres = __ddiv_rn(sqrt(rr), a.sc[S_NB]);
    record(a, j, relres);
    a.sc[S_RR] = rr;
    if (a.st[3] || rho1 == 0.0 || !isfinite(rho1)) {      // half step taken, or rho breakdown
        if (relres < a.tol) finish(a, MF_OK, 1); else finish(a, MF_ERR_BREAKDOWN, 0);
        return;
    }
    a.sc[S_BETA] = __dmul_rn(__ddiv_rn(rho1, a.sc[S_RHO]), __ddiv_rn(a.sc[S_ALPHA], a.sc[S_OMEGA]));
    a.sc[S_RHO] = rho1;
    if (relres < a.tol) a.st[DS_CONV] = 1;
}
// p = r + beta (p - omega mu) (PV) + levels
__global__ void k_bicg_p(DistArgs a) {
    if (is_done(a)) return;
    const double beta = a.sc[S_BETA], omega = a.sc[S_OMEGA];
    const Thresh th = dev_thresh(a);
    const unsigned m = mfk::hw_mask();
    const int64_t R0 = (int64_t)a.plan_tr[blockIdx.x] * 16, R1 = (int64_t)a.plan_tr[blockIdx.x + 1] * 16;
    for (int64_t i = R0 + threadIdx.x; i < R1; i += blockDim.x) {
        const bool valid = i < a.n;
        double pn = 0.0;
        if (valid) {
            pn = __fma_rn(beta, __fma_rn(-omega, a.mu[i], a.pv[pv_idx(i)]), a.r[i]);
            a.pv[pv_idx(i)] = pn;
        }
        own_level_store(a, a.pv, i, pn, valid, th, m);
    }
}

template <bool DYN, int MODE>
void* spmv_fn(int maxt) {
    return maxt > 512 ? (void*)k_spmv<DYN, MODE, 1024> : (void*)k_spmv<DYN, MODE, 512>;
}

// device buffers of one distributed solve (released by the destructor)
struct DistWs {
    cudaStream_t s;
    std::vector<void*> ptrs;
    explicit DistWs(cudaStream_t st) : s(st) {}
    ~DistWs() { for (void* p : ptrs) if (p) dev_free(p, s); }
    template <class T>
    mf_status get(T** p, size_t count) {
        MF_TRY(alloc(p, std::max<size_t>(count, 1), s));
        ptrs.push_back((void*)*p);
        return MF_OK;
    }
};

}  // namespace

// ------------------------------------------------------------------------------------ host
// In-process rank group: P host threads of one process drive P ranks emulated on ONE device
// (same-device windows instead of NVLink peers).  Only the device-initiated kernel runs on it;
// it verifies the multi-rank exchange logic where only one GPU is available.
struct LocalGroup {
    int P = 0;
    std::mutex mu;
    std::condition_variable cv;
    int arrived = 0;
    uint64_t gen = 0;
    std::vector<std::vector<char>> slot;                 // [rank] all-gather payloads
    std::vector<std::vector<std::vector<int32_t>>> mail; // [src][dst] exchange payloads
    bool barrier() {
        std::unique_lock<std::mutex> lk(mu);
        const uint64_t g = gen;
        if (++arrived == P) {
            arrived = 0;
            ++gen;
            cv.notify_all();
            return true;
        }
        return cv.wait_for(lk, std::chrono::seconds(300), [&] { return gen != g; });
    }
};

struct DistInfo {
    Comm* comm = nullptr;
    int64_t n_global = 0, row_begin = 0, row_end = 0, nown_seg = 0, nhalo = 0;
    int64_t nlo = 0;                         // halo segments of lower ranks (they precede the own ones)
    std::vector<int64_t> rank_rows;          // [P + 1] row boundaries of every rank
    std::vector<int64_t> recv_off;           // [P + 1] halo segments per peer (prefix)
    std::vector<int64_t> send_off;           // [P + 1] my segments each peer needs (prefix)
    int32_t* send_idx = nullptr;             // device: my local segment ids, per peer
    // device-initiated kernel (f1)
    MgArgs mg{};                             // everything but seg_lo / seg_hi (from the tile matrix)
    char* win = nullptr;                     // my window
    size_t win_bytes = 0;
    bool win_nccl = false;                   // ncclMemAlloc + registered window
    ncclWindow_t nwin = nullptr;
    void* dev_arrays = nullptr;              // send lists (one allocation)
    int* bar_scratch = nullptr;              // stream-ordered cross-rank barrier (ncclAllReduce)
    cudaStream_t owner = nullptr;
    ~DistInfo() {
        if (send_idx) dev_free(send_idx, owner);
        if (dev_arrays) dev_free(dev_arrays, owner);
        if (bar_scratch) dev_free(bar_scratch, owner);
        if (win) {
            if (win_nccl) {
                cudaStreamSynchronize(owner);
                if (nwin) ncclCommWindowDeregister(comm->nccl, nwin);
                ncclMemFree(win);
            } else {
                dev_free(win, owner);
            }
        }
    }
};

namespace {

__global__ void k_mark_halo(const int32_t* __restrict__ colidx, int64_t nnz, int64_t seg_lo, int64_t seg_hi, int64_t* flag) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nnz; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t sgm = colidx[k] >> 4;
        if (sgm < seg_lo || sgm >= seg_hi) flag[sgm] = 1;
    }
}
__global__ void k_halo_list(const int64_t* __restrict__ flag, const int64_t* __restrict__ pre, int64_t nseg, int32_t* list) {
    for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < nseg; g += (int64_t)gridDim.x * blockDim.x)
        if (flag[g]) list[pre[g]] = (int32_t)g;
}
// Local columns that keep the global order: [halo of lower ranks][own][halo of higher ranks],
// each part ascending by global segment.  A row's fma chain then visits its tiles in the same
// order as on one GPU, so every rank's SpMV rows equal the global SpMV rows bit for bit.
__global__ void k_remap(const int32_t* __restrict__ colidx, int64_t nnz, int64_t row_begin, int64_t seg_lo, int64_t seg_hi,
                        int64_t nown_seg, int64_t nlo, const int64_t* __restrict__ pre, int32_t* out) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nnz; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = colidx[k], sgm = c >> 4;
        int64_t o;
        if (sgm >= seg_lo && sgm < seg_hi) o = c - row_begin + nlo * 16;
        else {
            const int64_t h = pre[sgm];
            o = (h < nlo ? h : nown_seg + h) * 16 + (c & 15);
        }
        out[k] = (int32_t)o;
    }
}
__global__ void k_peer_ptrs(ncclWindow_t w, int P, unsigned long long* out) {
    if ((int)threadIdx.x < P) out[threadIdx.x] = (unsigned long long)ncclGetPeerPointer(w, 0, (int)threadIdx.x);
}

// extended segment of a halo block received from rank q (order-preserving layout)
inline int64_t halo_base(const DistInfo& D, int q) {
    return q < D.comm->rank ? D.recv_off[q] : D.nown_seg + D.recv_off[q];
}

mf_status exchange(const DistInfo& D, const double* pv, double* sendbuf, double* pv_own, const int* st, cudaStream_t s) {
    const int P = D.comm->nranks;
    const int64_t nsend = D.send_off[P];
    if (nsend > 0) {
        const int blocks = (int)std::min<int64_t>((nsend * PVS + 255) / 256, 148 * 8);
        k_pack<<<blocks, 256, 0, s>>>(pv, D.send_idx, nsend, sendbuf, st);
        MF_CUDA(cudaGetLastError());
    }
    double* ext = pv_own - D.nlo * PVS;
    MF_NCCL(ncclGroupStart());
    for (int q = 0; q < P; ++q) {
        if (q == D.comm->rank) continue;
        const int64_t ns = D.send_off[q + 1] - D.send_off[q], nr = D.recv_off[q + 1] - D.recv_off[q];
        if (ns) MF_NCCL(ncclSend(sendbuf + D.send_off[q] * PVS, (size_t)(ns * PVS), ncclDouble, q, D.comm->nccl, s));
        if (nr) MF_NCCL(ncclRecv(ext + halo_base(D, q) * PVS, (size_t)(nr * PVS), ncclDouble, q, D.comm->nccl, s));
    }
    MF_NCCL(ncclGroupEnd());
    return MF_OK;
}

mf_status allgather(const DistInfo& D, const double* part, double* gath, int k, cudaStream_t s) {
    MF_NCCL(ncclAllGather(part, gath, (size_t)k, ncclDouble, D.comm->nccl, s));
    return MF_OK;
}

// ---- setup collectives over either backend (host buffers, synchronous)
mf_status comm_allgather(Comm* c, const void* mine, size_t bytes, void* all, cudaStream_t s) {
    const int P = c->nranks;
    if (c->local) {
        LocalGroup& g = *c->local;
        g.slot[c->rank].assign((const char*)mine, (const char*)mine + bytes);
        if (!g.barrier()) return fail(MF_ERR_DEADLOCK, "local rank group: barrier timed out");
        for (int q = 0; q < P; ++q) std::memcpy((char*)all + q * bytes, g.slot[q].data(), bytes);
        if (!g.barrier()) return fail(MF_ERR_DEADLOCK, "local rank group: barrier timed out");
        return MF_OK;
    }
    char *d_in = nullptr, *d_all = nullptr;
    DistWs ws(s);
    MF_TRY(ws.get(&d_in, bytes));
    MF_TRY(ws.get(&d_all, bytes * P));
    MF_CUDA(cudaMemcpyAsync(d_in, mine, bytes, cudaMemcpyHostToDevice, s));
    MF_NCCL(ncclAllGather(d_in, d_all, bytes, ncclChar, c->nccl, s));
    MF_CUDA(cudaMemcpyAsync(all, d_all, bytes * P, cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    return MF_OK;
}
// to[q] -> rank q; from[q] (pre-sized by the caller) <- rank q
mf_status comm_exchange_i32(Comm* c, const std::vector<std::vector<int32_t>>& to, std::vector<std::vector<int32_t>>& from,
                            cudaStream_t s) {
    const int P = c->nranks, me = c->rank;
    if (c->local) {
        LocalGroup& g = *c->local;
        for (int q = 0; q < P; ++q) g.mail[me][q] = to[q];
        if (!g.barrier()) return fail(MF_ERR_DEADLOCK, "local rank group: barrier timed out");
        for (int q = 0; q < P; ++q) from[q] = g.mail[q][me];
        if (!g.barrier()) return fail(MF_ERR_DEADLOCK, "local rank group: barrier timed out");
        return MF_OK;
    }
    size_t nt = 0, nf = 0;
    for (int q = 0; q < P; ++q) { nt += to[q].size(); nf += from[q].size(); }
    int32_t *dt = nullptr, *df = nullptr;
    DistWs ws(s);
    MF_TRY(ws.get(&dt, nt));
    MF_TRY(ws.get(&df, nf));
    size_t o = 0;
    for (int q = 0; q < P; ++q) {
        if (!to[q].empty()) MF_CUDA(cudaMemcpyAsync(dt + o, to[q].data(), to[q].size() * 4, cudaMemcpyHostToDevice, s));
        o += to[q].size();
    }
    MF_NCCL(ncclGroupStart());
    size_t ot = 0, of = 0;
    for (int q = 0; q < P; ++q) {
        if (q != me && !to[q].empty()) MF_NCCL(ncclSend(dt + ot, to[q].size(), ncclInt32, q, c->nccl, s));
        if (q != me && !from[q].empty()) MF_NCCL(ncclRecv(df + of, from[q].size(), ncclInt32, q, c->nccl, s));
        ot += to[q].size();
        of += from[q].size();
    }
    MF_NCCL(ncclGroupEnd());
    of = 0;
    for (int q = 0; q < P; ++q) {
        if (q != me && !from[q].empty()) MF_CUDA(cudaMemcpyAsync(from[q].data(), df + of, from[q].size() * 4, cudaMemcpyDeviceToHost, s));
        of += from[q].size();
    }
    MF_CUDA(cudaStreamSynchronize(s));
    return MF_OK;
}

// window layout (bytes): tags u32 [2][P] | counters u64 [P] | reduction slots f64 [2][P][4] | PV
constexpr int64_t WIN_TAG = 0, WIN_CNT = 64, WIN_RED = 128, WIN_PV = 1024;

// f1 setup: the CTA-ordered store lists, the arrival counts, my halo ranges, the windows
mf_status mg_setup(DistInfo& D, const TileMatrix& A, const std::vector<int32_t>& req_local, cudaStream_t s) {
    Comm* c = D.comm;
    const int P = c->nranks, me = c->rank;
    if (P > MG_PMAX) return MF_OK;           // only the host-orchestrated path (dist_mode 1)
    MgArgs& m = D.mg;
    m.P = P;
    m.me = me;
    // my base in every rank's extended vector (all-gathered P x P: row q = rank q's bases)
    std::vector<int64_t> base(P, 0), base_all((size_t)P * P);
    for (int r = 0; r < P; ++r) base[r] = r == me ? 0 : halo_base(D, r);
    MF_TRY(comm_allgather(c, base.data(), P * sizeof(int64_t), base_all.data(), s));
    // entries (cta, peer, src, dst) in CTA order, peers ascending inside a CTA
    const int G = A.G;
    struct E { int32_t cta, peer, src, dst; };
    std::vector<E> ent;
    ent.reserve(req_local.size());
    std::vector<int64_t> tr_end(G);
    for (int g = 0; g < G; ++g) tr_end[g] = (A.plan_rows_host[g + 1] + 15) / 16;
    for (int q = 0; q < P; ++q) {
        if (q == me) continue;
        for (int64_t k = D.send_off[q]; k < D.send_off[q + 1]; ++k) {
            const int32_t sg = req_local[k];
            const int g = (int)(std::upper_bound(tr_end.begin(), tr_end.end(), (int64_t)sg) - tr_end.begin());
            if (g >= G) return fail(MF_ERR_INVALID_ARG, "requested segment outside the own rows");
            ent.push_back(E{g, q, sg, (int32_t)(base_all[(size_t)q * P + me] + (k - D.send_off[q]))});
        }
    }
    std::stable_sort(ent.begin(), ent.end(), [](const E& x, const E& y) { return x.cta != y.cta ? x.cta < y.cta : x.peer < y.peer; });
    const size_t ne = ent.size();
    std::vector<int32_t> sptr(G + 1, 0), ssrc(ne), sdst(ne);
    std::vector<int8_t> speer(ne);
    std::vector<uint8_t> smask(G, 0);
    for (size_t k = 0; k < ne; ++k) {
        sptr[ent[k].cta + 1]++;
        ssrc[k] = ent[k].src; sdst[k] = ent[k].dst; speer[k] = (int8_t)ent[k].peer;
        smask[ent[k].cta] |= (uint8_t)(1u << ent[k].peer);
    }
    for (int g = 0; g < G; ++g) sptr[g + 1] += sptr[g];
    std::vector<int64_t> nprod_to(P, 0), nprod_all((size_t)P * P);
    for (int g = 0; g < G; ++g)
        for (int r = 0; r < P; ++r) nprod_to[r] += (smask[g] >> r) & 1u;
    MF_TRY(comm_allgather(c, nprod_to.data(), P * sizeof(int64_t), nprod_all.data(), s));
    for (int r = 0; r < MG_PMAX; ++r) { m.nprod[r] = 0; m.hlo[r] = 0; m.hhi[r] = 0; m.win[r] = nullptr; }
    for (int r = 0; r < P; ++r) {
        m.nprod[r] = r == me ? 0 : (int)nprod_all[(size_t)r * P + me];
        if (r != me) {
            m.hlo[r] = (int32_t)halo_base(D, r);
            m.hhi[r] = (int32_t)(halo_base(D, r) + D.recv_off[r + 1] - D.recv_off[r]);
        }
    }
    // device copies of the lists (one allocation: ptr | src | dst | peer | mask)
    const size_t bytes = (size_t)(G + 1) * 4 + ne * 4 * 2 + ne + (size_t)G + 64;
    char* d = nullptr;
    MF_TRY(alloc(&d, bytes, s));
    D.dev_arrays = d;
    size_t o = 0;
    auto put = [&](const void* h, size_t nb) -> char* {
        char* p = d + o;
        if (nb) cudaMemcpyAsync(p, h, nb, cudaMemcpyHostToDevice, s);
        o += (nb + 15) / 16 * 16;
        return p;
    };
    m.send_ptr = reinterpret_cast<const int32_t*>(put(sptr.data(), sptr.size() * 4));
    m.send_src = reinterpret_cast<const int32_t*>(put(ssrc.data(), ne * 4));
    m.send_dst = reinterpret_cast<const int32_t*>(put(sdst.data(), ne * 4));
    m.send_peer = reinterpret_cast<const int8_t*>(put(speer.data(), ne));
    m.send_mask = reinterpret_cast<const uint8_t*>(put(smask.data(), (size_t)G));
    if (o > bytes + 64) return fail(MF_ERR_INVALID_ARG, "internal: send list layout");
    MF_CUDA(cudaGetLastError());
    // windows: the extended PV vector and the sync words, same size on every rank
    const int64_t n_ext_seg = D.nown_seg + D.nhalo + 1;
    int64_t wb = WIN_PV + n_ext_seg * PVS * 8;
    wb = (wb + 4095) / 4096 * 4096;
    std::vector<int64_t> wall(P);
    MF_TRY(comm_allgather(c, &wb, sizeof(wb), wall.data(), s));
    for (int r = 0; r < P; ++r) wb = std::max(wb, wall[r]);
    D.win_bytes = (size_t)wb;
    m.off_tag = WIN_TAG; m.off_cnt = WIN_CNT; m.off_red = WIN_RED; m.off_pv = WIN_PV;
    if (c->local || P == 1) {
        MF_TRY(alloc(&D.win, D.win_bytes, s));
        MF_CUDA(cudaMemsetAsync(D.win, 0, D.win_bytes, s));
        MF_CUDA(cudaStreamSynchronize(s));
        std::vector<unsigned long long> ptrs(P);
        const unsigned long long mine = (unsigned long long)D.win;
        if (c->local) MF_TRY(comm_allgather(c, &mine, sizeof(mine), ptrs.data(), s));
        else ptrs[0] = mine;
        for (int r = 0; r < P; ++r) m.win[r] = (char*)ptrs[r];
    } else {
        // NVLink peers: an NCCL symmetric window, the peers' mappings from the device API
        const ncclTeam_t lsa = ncclTeamLsa(c->nccl);
        if (lsa.nRanks != P) return fail(MF_ERR_UNSUPPORTED, "device-initiated kernel needs every rank in one NVLink domain");
        void* wp = nullptr;
        MF_NCCL(ncclMemAlloc(&wp, D.win_bytes));
        D.win = (char*)wp;
        D.win_nccl = true;
        MF_NCCL(ncclCommWindowRegister(c->nccl, wp, D.win_bytes, &D.nwin, NCCL_WIN_COLL_SYMMETRIC));
        MF_CUDA(cudaMemsetAsync(D.win, 0, D.win_bytes, s));
        unsigned long long* dptr = nullptr;
        DistWs ws(s);
        MF_TRY(ws.get(&dptr, (size_t)P));
        k_peer_ptrs<<<1, 32, 0, s>>>(D.nwin, P, dptr);
        MF_CUDA(cudaGetLastError());
        std::vector<unsigned long long> ptrs(P);
        MF_CUDA(cudaMemcpyAsync(ptrs.data(), dptr, P * 8, cudaMemcpyDeviceToHost, s));
        MF_CUDA(cudaStreamSynchronize(s));
        for (int r = 0; r < P; ++r) m.win[r] = (char*)ptrs[r];
        MF_TRY(alloc(&D.bar_scratch, 1, s));
    }
    return MF_OK;
}

}  // namespace

mf_status dist_create(Comm* comm, int64_t n_global, int64_t row_begin, int64_t row_end, int64_t nnz, const int64_t* rowptr,
                      const int32_t* colidx, const double* vals, const mf_convert_opts& o, cudaStream_t s, TileMatrix* A,
                      DistInfo** out) {
    const int P = comm->nranks, me = comm->rank;
    const int64_t n_local = row_end - row_begin;
    if (row_begin % 16 != 0 || (row_end % 16 != 0 && row_end != n_global))
        return fail(MF_ERR_INVALID_ARG, "row blocks must be aligned to 16-row tile rows");
    DistWs ws(s);
    // every rank's row range (the owners of the halo segments)
    const int64_t mine[2] = {row_begin, row_end};
    std::vector<int64_t> rr(2 * (size_t)P);
    MF_TRY(comm_allgather(comm, mine, sizeof(mine), rr.data(), s));
    std::unique_ptr<DistInfo> D(new DistInfo());
    D->comm = comm; D->n_global = n_global; D->row_begin = row_begin; D->row_end = row_end; D->owner = s;
    D->rank_rows.resize(P + 1);
    for (int q = 0; q < P; ++q) {
        D->rank_rows[q] = rr[2 * q];
        if (q > 0 && rr[2 * q] != rr[2 * q - 1]) return fail(MF_ERR_INVALID_ARG, "rank row blocks must be contiguous and in rank order");
    }
    D->rank_rows[P] = rr[2 * P - 1];
    if (D->rank_rows[0] != 0 || D->rank_rows[P] != n_global) return fail(MF_ERR_INVALID_ARG, "rank row blocks must cover the matrix");
    // halo segments: global segments my rows gather outside my own range, ascending
    const int64_t nseg = (n_global + 15) / 16, seg_lo = row_begin / 16, seg_hi = (row_end + 15) / 16;
    D->nown_seg = seg_hi - seg_lo;
    int64_t *flag = nullptr, *pre = nullptr, *tmp = nullptr;
    MF_TRY(ws.get(&flag, (size_t)nseg));
    MF_TRY(ws.get(&pre, (size_t)nseg + 1));
    MF_TRY(ws.get(&tmp, (size_t)nseg / 2048 + 2));
    MF_CUDA(cudaMemsetAsync(flag, 0, nseg * 8, s));
    if (nnz > 0) k_mark_halo<<<(unsigned)std::min<int64_t>((nnz + 255) / 256, 148 * 16), 256, 0, s>>>(colidx, nnz, seg_lo, seg_hi, flag);
    MF_TRY(scan_excl_i64(flag, nseg, pre, tmp, s));
    int64_t cnt2[2] = {0, 0};   // halo segments in total, below my block
    MF_CUDA(cudaMemcpyAsync(&cnt2[0], pre + nseg, 8, cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaMemcpyAsync(&cnt2[1], pre + seg_lo, 8, cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    D->nhalo = cnt2[0];
    D->nlo = cnt2[1];
    int32_t *hlist = nullptr, *col2 = nullptr;
    MF_TRY(ws.get(&hlist, (size_t)D->nhalo));
    MF_TRY(ws.get(&col2, (size_t)nnz));
    k_halo_list<<<(unsigned)std::min<int64_t>((nseg + 255) / 256, 148 * 16), 256, 0, s>>>(flag, pre, nseg, hlist);
    if (nnz > 0)
        k_remap<<<(unsigned)std::min<int64_t>((nnz + 255) / 256, 148 * 16), 256, 0, s>>>(colidx, nnz, row_begin, seg_lo, seg_hi,
                                                                                    D->nown_seg, D->nlo, pre, col2);
    MF_CUDA(cudaGetLastError());
    std::vector<int32_t> hl((size_t)D->nhalo);
    if (D->nhalo) MF_CUDA(cudaMemcpyAsync(hl.data(), hlist, hl.size() * 4, cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    // halo block of each peer (the owners' ranges are contiguous and ascending)
    D->recv_off.assign(P + 1, 0);
    {
        int q = 0;
        for (int64_t k = 0; k < D->nhalo; ++k) {
            const int64_t row = (int64_t)hl[k] * 16;
            while (q + 1 <= P && D->rank_rows[q + 1] <= row) ++q;
            if (q == me || q >= P) return fail(MF_ERR_INVALID_ARG, "halo segment without an owner");
            D->recv_off[q + 1]++;
        }
        for (int q2 = 0; q2 < P; ++q2) D->recv_off[q2 + 1] += D->recv_off[q2];
    }
    if (D->recv_off[me] != D->nlo) return fail(MF_ERR_INVALID_ARG, "internal: halo order");
    // tell every owner which of its segments I need: counts (all-gathered P x P), then the lists
    std::vector<int64_t> cnt_me(P), cnt_all((size_t)P * P);
    for (int q = 0; q < P; ++q) cnt_me[q] = D->recv_off[q + 1] - D->recv_off[q];
    MF_TRY(comm_allgather(comm, cnt_me.data(), P * sizeof(int64_t), cnt_all.data(), s));
    D->send_off.assign(P + 1, 0);
    for (int q = 0; q < P; ++q) D->send_off[q + 1] = D->send_off[q] + (q == me ? 0 : cnt_all[(size_t)q * P + me]);
    std::vector<std::vector<int32_t>> to(P), from(P);
    for (int q = 0; q < P; ++q) {
        if (q == me) continue;
        to[q].assign(hl.begin() + D->recv_off[q], hl.begin() + D->recv_off[q + 1]);
        from[q].resize((size_t)(D->send_off[q + 1] - D->send_off[q]));
    }
    MF_TRY(comm_exchange_i32(comm, to, from, s));
    std::vector<int32_t> rq((size_t)D->send_off[P]);
    for (int q = 0; q < P; ++q)
        for (size_t k = 0; k < from[q].size(); ++k) rq[(size_t)D->send_off[q] + k] = (int32_t)(from[q][k] - seg_lo);   // my local segment ids
    for (auto g : rq)
        if (g < 0 || g >= D->nown_seg) return fail(MF_ERR_INVALID_ARG, "peer requested a segment I do not own");
    MF_TRY(alloc(&D->send_idx, std::max<size_t>(rq.size(), 1), s));
    if (!rq.empty()) MF_CUDA(cudaMemcpyAsync(D->send_idx, rq.data(), rq.size() * 4, cudaMemcpyHostToDevice, s));
    // the local matrix: columns [lower halo | own | upper halo]
    const int64_t n_ext = (D->nown_seg + D->nhalo) * 16;
    if (n_ext > INT32_MAX) return fail(MF_ERR_UNSUPPORTED, "local extended vector exceeds 2^31 columns");
    A->coff = D->nlo;
    MF_TRY(convert_csr(n_local, n_ext, nnz, rowptr, col2, vals, o, s, A));
    MF_CUDA(cudaStreamSynchronize(s));
    MF_TRY(mg_setup(*D, *A, rq, s));
    *out = D.release();
    return MF_OK;
}

void dist_destroy(DistInfo* D) { delete D; }

namespace {
struct MgCtx {
    DistInfo* D;
};
// before every device-initiated solve: clear my window (sync words, extended vector), then a
// cross-rank barrier so that no peer stores into a window that is still being cleared
mf_status mg_prelaunch(void* ctx, cudaStream_t s) {
    DistInfo& D = *static_cast<MgCtx*>(ctx)->D;
    MF_CUDA(cudaMemsetAsync(D.win, 0, D.win_bytes, s));
    Comm* c = D.comm;
    if (c->nranks == 1) return MF_OK;
    if (c->local) {
        MF_CUDA(cudaStreamSynchronize(s));
        if (!c->local->barrier()) return fail(MF_ERR_DEADLOCK, "local rank group: barrier timed out");
        return MF_OK;
    }
    MF_NCCL(ncclAllReduce(D.bar_scratch, D.bar_scratch, 1, ncclInt32, ncclSum, c->nccl, s));   // stream-ordered barrier
    return MF_OK;
}
// local group: every rank thread has enqueued its kernel (see MgLaunch::postlaunch)
mf_status mg_postlaunch(void* ctx) {
    DistInfo& D = *static_cast<MgCtx*>(ctx)->D;
    Comm* c = D.comm;
    if (c->local && c->nranks > 1 && !c->local->barrier()) return fail(MF_ERR_DEADLOCK, "local rank group: barrier timed out");
    return MF_OK;
}
}  // namespace

mf_status mg_solve(const TileMatrix& A, DistInfo& D, const double* b, double* x, const mf_solve_opts& o, mf_solve_info* info,
                   cudaStream_t s) {
    if (D.mg.P == 0 || !D.win) return fail(MF_ERR_UNSUPPORTED, "device-initiated kernel: more ranks than one NVLink domain");
    MgCtx ctx{&D};
    MgLaunch L;
    L.args = D.mg;
    L.pv_own = reinterpret_cast<double*>(D.win + D.mg.off_pv) + D.nlo * PVS;
    L.prelaunch = mg_prelaunch;
    L.ctx = &ctx;
    L.plain_launch = D.comm->local != nullptr;
    L.postlaunch = mg_postlaunch;
    return run_solve(A, false, b, x, o, info, s, &L);
}

mf_status dist_solve(const TileMatrix& A, const DistInfo& D, bool bicg, const double* b, double* x, const mf_solve_opts& o,
                     mf_solve_info* info, cudaStream_t s) {
    if (o.M) return fail(MF_ERR_NOT_IMPLEMENTED, "distributed preconditioned solves");
    if (o.sticky || o.tile_level_counts || o.collect_stats)
        return fail(MF_ERR_NOT_IMPLEMENTED, "distributed solve: sticky variant / level statistics");
    if (D.comm->local) return fail(MF_ERR_NOT_IMPLEMENTED, "local rank groups run the device-initiated kernel only");
    const int P = D.comm->nranks;
    const int64_t n = A.n_rows;
    int dev = 0, smem_optin = 0;
    MF_CUDA(cudaGetDevice(&dev));
    MF_CUDA(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    const bool dyn = o.mode == MF_MODE_DYNAMIC_MIXED;
    const int G = A.G, B = A.B;
    DistWs ws(s);
    DistArgs a{};
    a.A = mfk::Mat{A.n_rows, A.n_cols, A.ntr, A.tr_slot, A.TileRowPtr, A.tile_info, A.sidx, A.blob,
                   reinterpret_cast<const mfk::TsStage*>(A.stg), A.stg_ptr, A.TileNnz, A.ts, (int)A.max_w,
                   A.plane64, A.plane32, A.plane16, A.plane8, nullptr, A.coff};
    a.G = G; a.plan_tr = A.plan_tr; a.n = n; a.nown_seg = D.nown_seg; a.b = b; a.x = x; a.P = P;
    // extended PV vectors [lower halo | own | upper halo]; the kernels address the own part
    const int64_t npv = (D.nown_seg + D.nhalo + 1) * PVS;
    double *pv_ext = nullptr, *sv_ext = nullptr;
    MF_TRY(ws.get(&a.r, (size_t)n));
    MF_TRY(ws.get(&pv_ext, (size_t)npv));
    MF_TRY(ws.get(&a.mu, (size_t)n));
    if (bicg) {
        MF_TRY(ws.get(&sv_ext, (size_t)npv));
        MF_TRY(ws.get(&a.rh, (size_t)n));
        MF_TRY(ws.get(&a.th, (size_t)n));
        MF_CUDA(cudaMemsetAsync(sv_ext, 0, npv * 8, s));
        a.sv = sv_ext + D.nlo * PVS;
    }
    MF_CUDA(cudaMemsetAsync(pv_ext, 0, npv * 8, s));
    a.pv = pv_ext + D.nlo * PVS;
    MF_TRY(ws.get(&a.slots, (size_t)4 * G));
    MF_TRY(ws.get(&a.part, 4));
    MF_TRY(ws.get(&a.gath, (size_t)4 * P));
    MF_TRY(ws.get(&a.sc, S_NSC));
    MF_TRY(ws.get(&a.st, 4));
    MF_TRY(ws.get(&a.iter, 1));
    a.hist_cap = std::min<int64_t>(o.max_iter + 2, std::max<int64_t>(o.history_cap, 2) + 2);
    MF_TRY(ws.get(&a.hist, (size_t)a.hist_cap));
    MF_CUDA(cudaMemsetAsync(a.st, 0, 4 * sizeof(int), s));
    MF_CUDA(cudaMemsetAsync(a.slots, 0, 4 * G * sizeof(double), s));
    double* sendbuf = nullptr;
    MF_TRY(ws.get(&sendbuf, (size_t)(D.send_off[P] * PVS)));
    a.max_iter = o.max_iter; a.tol = o.tol; a.switch_eps = o.switch_eps < 0 ? o.tol : o.switch_eps;
    a.switch_abs = o.switch_absolute; a.range_guard = o.range_guard; a.dyn = dyn;
    const int64_t ebytes = A.ts ? (int64_t)(B / 32) * A.ecap * 128 : 0;
    int64_t k = A.ts ? ((int64_t)smem_optin - 128 - 256 - (int64_t)mfk::TS_CTRL_BYTES - ebytes) / std::max<int32_t>(A.slot_bytes, 128) : 1;
    a.nst = (int)std::max<int64_t>(1, std::min<int64_t>(k, mfk::TS_NSTMAX));
    a.slot_bytes = A.slot_bytes; a.blob_cap = A.blob_cap; a.ecap = A.ecap;
    const size_t smem = 128 + mfk::spmv_smem_bytes(A.ts, a.nst, A.slot_bytes, A.ecap, B / 32);
    void* f_init = spmv_fn<false, 0>(B);
    void* f_mu = dyn ? (bicg ? spmv_fn<true, 2>(B) : spmv_fn<true, 1>(B)) : (bicg ? spmv_fn<false, 2>(B) : spmv_fn<false, 1>(B));
    void* f_th = dyn ? spmv_fn<true, 3>(B) : spmv_fn<false, 3>(B);
    for (void* f : {f_init, f_mu, f_th}) MF_TRY(set_max_dyn_smem(f, smem_optin));
    cudaStream_t q = s;   // the stream the iteration is enqueued on (a private one while capturing)
    auto launch_spmv = [&](void* f, const double* in) -> mf_status {
        void* args[] = {&a, (void*)&in};
        MF_CUDA(cudaLaunchKernel(f, dim3(G), dim3(B), args, smem, q));
        return MF_OK;
    };
    cudaEvent_t e0, e1;
    MF_CUDA(cudaEventCreate(&e0));
    MF_CUDA(cudaEventCreate(&e1));
    MF_CUDA(cudaEventRecord(e0, s));
    // init: r0 = b - A~ x0 (x0 staged in the PV layout, halo exchanged), partials (b,b), (r,r)
    k_stage_x0<<<148, 256, 0, s>>>(a, a.pv);
    MF_TRY(exchange(D, a.pv, sendbuf, a.pv, a.st, s));
    MF_TRY(launch_spmv(f_init, a.pv));
    k_rank_partial<<<1, 32, 0, s>>>(a, 2);
    MF_TRY(allgather(D, a.part, a.gath, 2, s));
    if (bicg) {
        k_bicg_init_scalars<<<1, 1, 0, s>>>(a);
        k_bicg_p0<<<G, B, 0, s>>>(a);
    } else {
        k_cg_init_scalars<<<1, 1, 0, s>>>(a);
        k_cg_p0<<<G, B, 0, s>>>(a);
    }
    MF_CUDA(cudaGetLastError());
    // one iteration, enqueued as a chunk captured in a CUDA graph
    auto one_iter = [&]() -> mf_status {
        MF_TRY(exchange(D, a.pv, sendbuf, a.pv, a.st, q));
        MF_TRY(launch_spmv(f_mu, a.pv));
        k_rank_partial<<<1, 32, 0, q>>>(a, bicg ? 2 : 2);
        MF_TRY(allgather(D, a.part, a.gath, 2, q));
        if (bicg) {
            k_bicg_s<<<G, B, 0, q>>>(a);
            MF_TRY(exchange(D, a.sv, sendbuf, a.sv, a.st, q));
            MF_TRY(launch_spmv(f_th, a.sv));
            k_rank_partial<<<1, 32, 0, q>>>(a, 2);
            MF_TRY(allgather(D, a.part, a.gath, 2, q));
            k_bicg_xr<<<G, B, 0, q>>>(a);
            k_rank_partial<<<1, 32, 0, q>>>(a, 2);
            MF_TRY(allgather(D, a.part, a.gath, 2, q));
            k_bicg_beta<<<1, 1, 0, q>>>(a);
            k_bicg_p<<<G, B, 0, q>>>(a);
        } else {
            k_cg_alpha<<<1, 1, 0, q>>>(a);
            k_cg_r<<<G, B, 0, q>>>(a);
            k_rank_partial<<<1, 32, 0, q>>>(a, 1);
            MF_TRY(allgather(D, a.part, a.gath, 1, q));
            k_cg_beta<<<1, 1, 0, q>>>(a);
            k_cg_xp<<<G, B, 0, q>>>(a);
        }
        k_cg_stop<<<1, 1, 0, q>>>(a);
        if (q == s) MF_CUDA(cudaGetLastError());   // while capturing, errors surface at instantiation
        return MF_OK;
    };
    constexpr int CHUNK = 8;
    cudaGraph_t graph = nullptr;
    cudaGraphExec_t gexec = nullptr;
    bool graphed = getenv("MF_DIST_NO_GRAPH") == nullptr;
    // the chunk is captured on a private stream (the caller's may be the legacy stream, which
    // cannot capture) and launched on the caller's stream
    cudaStream_t cap = nullptr;
    if (graphed && cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking) != cudaSuccess) graphed = false;
    if (graphed) {
        if (cudaStreamBeginCapture(cap, cudaStreamCaptureModeRelaxed) != cudaSuccess) graphed = false;
        else {
            q = cap;
            mf_status cs = MF_OK;
            for (int c = 0; c < CHUNK && cs == MF_OK; ++c) cs = one_iter();
            q = s;
            const cudaError_t ce = cudaStreamEndCapture(cap, &graph);
            if (cs != MF_OK || ce != cudaSuccess || cudaGraphInstantiate(&gexec, graph, 0) != cudaSuccess) {
                if (graph) cudaGraphDestroy(graph);
                graph = nullptr;
                gexec = nullptr;
                graphed = false;
            }
        }
        cudaGetLastError();   // a refused capture leaves its error behind; the fallback is the eager chunk
    }
    if (cap) cudaStreamDestroy(cap);
    int hst[4] = {0, 0, 0, 0};
    int* pin = nullptr;
    MF_CUDA(cudaMallocHost(&pin, 4 * sizeof(int)));
    int64_t launched = 0;
    mf_status st = MF_OK;
    while (true) {
        MF_CUDA(cudaMemcpyAsync(pin, a.st, 4 * sizeof(int), cudaMemcpyDeviceToHost, s));
        cudaEvent_t ev;
        MF_CUDA(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
        MF_CUDA(cudaEventRecord(ev, s));
        // one chunk in flight while the host reads the previous done flag
        if (launched < o.max_iter + CHUNK) {
            if (graphed) MF_CUDA(cudaGraphLaunch(gexec, s));
            else for (int c = 0; c < CHUNK; ++c) MF_TRY(one_iter());
            launched += CHUNK;
        }
        MF_CUDA(cudaEventSynchronize(ev));
        cudaEventDestroy(ev);
        std::memcpy(hst, pin, sizeof(hst));
        if (hst[DS_DONE] || launched >= o.max_iter + 2 * CHUNK) break;
    }
    MF_CUDA(cudaStreamSynchronize(s));
    MF_CUDA(cudaMemcpy(hst, a.st, sizeof(hst), cudaMemcpyDeviceToHost));
    MF_CUDA(cudaEventRecord(e1, s));
    MF_CUDA(cudaEventSynchronize(e1));
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFreeHost(pin);
    if (gexec) cudaGraphExecDestroy(gexec);
    if (graph) cudaGraphDestroy(graph);
    int64_t iters = 0;
    double sc[S_NSC];
    MF_CUDA(cudaMemcpy(&iters, a.iter, 8, cudaMemcpyDeviceToHost));
    MF_CUDA(cudaMemcpy(sc, a.sc, sizeof(sc), cudaMemcpyDeviceToHost));
    if (o.residual_history && o.history_cap > 0) {
        const int64_t kk = std::min<int64_t>(o.history_cap, std::min<int64_t>(iters + 1, a.hist_cap));
        MF_CUDA(cudaMemcpy(o.residual_history, a.hist, kk * 8, cudaMemcpyDeviceToHost));
    }
    std::memset(info, 0, sizeof(*info));
    info->iterations = iters;
    info->converged = hst[DS_CONV];
    info->status = (mf_status)hst[DS_STATUS];
    info->rel_residual = sc[S_RELRES];
    info->kernel_ms = ms;
    info->n_spmv = (bicg ? 2 : 1) * iters;
    info->launches = (int64_t)((bicg ? 16 : 11) * launched + 6);
    st = info->status;
    if (st == MF_ERR_BREAKDOWN) return fail(st, "numerical breakdown");
    return st;
}

}  // namespace mf

// ------------------------------------------------------------------------------------ C ABI
struct mf_comm {
    mf::Comm c;
};

extern "C" {

mf_status mf_nccl_unique_id(void* out) {
    if (!out) return mf::fail(MF_ERR_INVALID_ARG, "out is NULL");
    ncclUniqueId id;
    MF_NCCL(ncclGetUniqueId(&id));
    std::memcpy(out, &id, sizeof(id));
    return MF_OK;
}

mf_status mf_comm_create(const void* nccl_unique_id, int32_t nranks, int32_t rank, mf_comm** out) {
    if (!out || !nccl_unique_id) return mf::fail(MF_ERR_INVALID_ARG, "NULL argument");
    *out = nullptr;
    if (nranks < 1 || rank < 0 || rank >= nranks) return mf::fail(MF_ERR_INVALID_ARG, "bad rank / nranks");
    int sms = 0;
    MF_TRY(mf::check_device(&sms));
    mf_comm* c = new (std::nothrow) mf_comm();
    if (!c) return mf::fail(MF_ERR_OOM, "host allocation failed");
    ncclUniqueId id;
    std::memcpy(&id, nccl_unique_id, sizeof(id));
    const ncclResult_t r = ncclCommInitRank(&c->c.nccl, nranks, id, rank);
    if (r != ncclSuccess) {
        delete c;
        return mf::fail(MF_ERR_NCCL, std::string("ncclCommInitRank: ") + ncclGetErrorString(r));
    }
    c->c.nranks = nranks;
    c->c.rank = rank;
    *out = c;
    return MF_OK;
}

mf_status mf_comm_destroy(mf_comm* c) {
    if (!c) return MF_OK;
    if (c->c.nccl) ncclCommDestroy(c->c.nccl);
    delete c;
    return MF_OK;
}

struct mf_local_group {
    mf::LocalGroup g;
};

mf_status mf_local_group_create(int32_t nranks, mf_local_group** out) {
    if (!out || nranks < 1 || nranks > mf::MG_PMAX) return mf::fail(MF_ERR_INVALID_ARG, "nranks must be in [1, 8]");
    mf_local_group* g = new (std::nothrow) mf_local_group();
    if (!g) return mf::fail(MF_ERR_OOM, "host allocation failed");
    g->g.P = nranks;
    g->g.slot.resize(nranks);
    g->g.mail.assign(nranks, std::vector<std::vector<int32_t>>(nranks));
    *out = g;
    return MF_OK;
}

mf_status mf_local_group_destroy(mf_local_group* g) {
    delete g;
    return MF_OK;
}

mf_status mf_comm_create_local(mf_local_group* g, int32_t rank, mf_comm** out) {
    if (!g || !out || rank < 0 || rank >= g->g.P) return mf::fail(MF_ERR_INVALID_ARG, "bad group / rank");
    int sms = 0;
    MF_TRY(mf::check_device(&sms));
    mf_comm* c = new (std::nothrow) mf_comm();
    if (!c) return mf::fail(MF_ERR_OOM, "host allocation failed");
    c->c.nranks = g->g.P;
    c->c.rank = rank;
    c->c.local = &g->g;
    *out = c;
    return MF_OK;
}

mf_status mf_comm_info(const mf_comm* c, int32_t* nranks, int32_t* rank) {
    if (!c) return mf::fail(MF_ERR_INVALID_ARG, "comm is NULL");
    if (nranks) *nranks = c->c.nranks;
    if (rank) *rank = c->c.rank;
    return MF_OK;
}

mf_status mf_tile_matrix_from_csr_dist(mf_comm* comm, int64_t n_global, int64_t row_begin, int64_t row_end, int64_t nnz_local,
                                       const int64_t* rowptr, const int32_t* colidx, const double* vals,
                                       const mf_convert_opts* opts, mf_stream stream, mf_tile_matrix** out) {
    if (!out || !comm) return mf::fail(MF_ERR_INVALID_ARG, "NULL argument");
    *out = nullptr;
    if (n_global < 0 || row_begin < 0 || row_end < row_begin || row_end > n_global || nnz_local < 0 || n_global > INT32_MAX)
        return mf::fail(MF_ERR_INVALID_ARG, "bad sizes");
    if (!rowptr || (nnz_local > 0 && (!colidx || !vals))) return mf::fail(MF_ERR_INVALID_ARG, "NULL CSR array");
    mf_convert_opts o;
    mf_default_convert_opts(&o);
    if (opts) o = *opts;
    mf_tile_matrix* h = new (std::nothrow) mf_tile_matrix();
    if (!h) return mf::fail(MF_ERR_OOM, "host allocation failed");
    mf::DistInfo* D = nullptr;
    const mf_status st = mf::dist_create(&comm->c, n_global, row_begin, row_end, nnz_local, rowptr, colidx, vals, o,
                                         (cudaStream_t)stream, &h->m, &D);
    if (st != MF_OK) {
        mf::destroy_tiles(&h->m);
        delete h;
        return st;
    }
    h->dist = D;
    *out = h;
    return MF_OK;
}

static mf_status solve_dist(const mf_tile_matrix* A, bool bicg, const double* b, double* x, const mf_solve_opts* opts,
                            mf_solve_info* info, mf_stream stream) {
    if (!A || !A->dist || !info) return mf::fail(MF_ERR_INVALID_ARG, "need a distributed matrix and info");
    if (A->m.n_rows > 0 && (!b || !x)) return mf::fail(MF_ERR_INVALID_ARG, "b / x is NULL");
    mf_solve_opts o;
    mf_default_solve_opts(&o);
    if (opts) o = *opts;
    if (!(o.tol >= 0) || o.max_iter < 0) return mf::fail(MF_ERR_INVALID_ARG, "bad tol / max_iter");
    if (o.dist_mode < 0 || o.dist_mode > 2) return mf::fail(MF_ERR_INVALID_ARG, "dist_mode must be 0, 1 or 2");
    const bool device_initiated = o.dist_mode == 2 || (o.dist_mode == 0 && !bicg && !o.M && !o.sticky &&
                                                       !o.tile_level_counts && !o.collect_stats && A->dist->mg.P > 0);
    if (device_initiated) {
        if (bicg) return mf::fail(MF_ERR_NOT_IMPLEMENTED, "device-initiated multi-GPU kernel: BiCGSTAB");
        return mf::mg_solve(A->m, *A->dist, b, x, o, info, (cudaStream_t)stream);
    }
    return mf::dist_solve(A->m, *A->dist, bicg, b, x, o, info, (cudaStream_t)stream);
}

mf_status mf_cg_solve_dist(const mf_tile_matrix* A, const double* b, double* x, const mf_solve_opts* opts, mf_solve_info* info,
                           mf_stream stream) {
    return solve_dist(A, false, b, x, opts, info, stream);
}

mf_status mf_bicgstab_solve_dist(const mf_tile_matrix* A, const double* b, double* x, const mf_solve_opts* opts,
                                 mf_solve_info* info, mf_stream stream) {
    return solve_dist(A, true, b, x, opts, info, stream);
}

// Host-only halo planner (the same plan dist_create builds on the device): the global
// 16-element segments rank `rank`'s rows gather outside its own block, ascending, and how many
// of them each peer owns.  No GPU needed (the multi-process CPU tests drive it).
mf_status mf_dist_plan(int64_t n_global, int32_t nranks, const int64_t* rank_rows, int32_t rank, int64_t nnz,
                       const int32_t* colidx, int64_t* recv_counts, int32_t* halo_segments, int64_t halo_cap, int64_t* nhalo) {
    if (!rank_rows || !recv_counts || !nhalo || nranks < 1 || rank < 0 || rank >= nranks || (nnz > 0 && !colidx))
        return mf::fail(MF_ERR_INVALID_ARG, "bad arguments");
    for (int q = 0; q < nranks; ++q)
        if (rank_rows[q] > rank_rows[q + 1] || (q > 0 && rank_rows[q] % 16))
            return mf::fail(MF_ERR_INVALID_ARG, "rank row blocks must be ascending and tile aligned");
    if (rank_rows[0] != 0 || rank_rows[nranks] != n_global) return mf::fail(MF_ERR_INVALID_ARG, "rank blocks must cover the matrix");
    const int64_t seg_lo = rank_rows[rank] / 16, seg_hi = (rank_rows[rank + 1] + 15) / 16;
    std::vector<int32_t> segs;
    segs.reserve((size_t)std::min<int64_t>(nnz, 1 << 20));
    for (int64_t k = 0; k < nnz; ++k) {
        if (colidx[k] < 0 || colidx[k] >= n_global) return mf::fail(MF_ERR_INVALID_ARG, "column out of range");
        const int64_t g = colidx[k] >> 4;
        if (g < seg_lo || g >= seg_hi) segs.push_back((int32_t)g);
    }
    std::sort(segs.begin(), segs.end());
    segs.erase(std::unique(segs.begin(), segs.end()), segs.end());
    *nhalo = (int64_t)segs.size();
    for (int q = 0; q < nranks; ++q) recv_counts[q] = 0;
    int q = 0;
    for (size_t k = 0; k < segs.size(); ++k) {
        while (q + 1 <= nranks && rank_rows[q + 1] <= (int64_t)segs[k] * 16) ++q;
        recv_counts[q]++;
        if (halo_segments && (int64_t)k < halo_cap) halo_segments[k] = segs[k];
    }
    return MF_OK;
}

mf_status mf_dist_info(const mf_tile_matrix* A, int64_t* row_begin, int64_t* row_end, int64_t* halo_segments,
                       int64_t* send_segments) {
    if (!A || !A->dist) return mf::fail(MF_ERR_INVALID_ARG, "not a distributed matrix");
    const int P = A->dist->comm->nranks;
    if (row_begin) *row_begin = A->dist->row_begin;
    if (row_end) *row_end = A->dist->row_end;
    if (halo_segments) *halo_segments = A->dist->nhalo;
    if (send_segments) *send_segments = A->dist->send_off[P];
    return MF_OK;
}

}  // extern "C"
