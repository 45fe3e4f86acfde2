// solver.cu -- host side of the single-kernel solvers (run_solve: workspace, shared-memory plan,
// cooperative launch, byte model, instrumentation) and the standalone kernels behind mf_spmv /
// mf_levels / mf_dot / the per-rank update calls.  The persistent kernels themselves are in
// solver_kernels.cuh, instantiated by solver_inst_*.cu.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "solver_kernels.cuh"

namespace mf {
namespace {

using mfk::Counts;
using mfk::Mat;
using mfk::Thresh;
using mfk::PVS;
using mfk::pv_idx;

// -------------------------------------------------------------------------- standalone kernels
// x (+ optional level array) -> PV layout (the SpMV input of mf_spmv / the per-rank SpMV)
__global__ void pack_pv_kernel(const double* __restrict__ x, int64_t n, const uint8_t* __restrict__ level, double* pv) {
    const int64_t nseg = (n + 15) / 16;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nseg * PVS; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t J = k / PVS, e = k - J * PVS, i = J * 16 + e;
        double v = 0.0;
        if (e < 16) v = i < n ? x[i] : 0.0;
        pv[k] = v;
        if (e == 16) mfk::pv_set_level(pv, J, level ? level[J] : 0);
    }
}

// mf_spmv: the same staged SpMV as the solver, one block per CTA of the launch plan
template <bool DYN, bool COUNT, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) spmv_kernel(Mat A, const int32_t* __restrict__ plan_tr, const double* pv,
                                                    double* __restrict__ y, int range_guard, unsigned long long* counts,
                                                    int nst, int slot_bytes, int blob_cap, int ecap) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    int* ired = reinterpret_cast<int*>(smem_raw);
    mfk::SpmvSmem sp;
    mfk::carve_spmv(smem_raw + 128, nst, slot_bytes, blob_cap, ecap, sp);
    mfk::ts_init(sp.ts);
    __syncthreads();
    const int64_t tr0 = plan_tr[blockIdx.x], tr1 = plan_tr[blockIdx.x + 1];
    const int64_t n = A.n_rows;
    mfk::spmv_cta<DYN, false, 4>(A, tr0, tr1, pv, range_guard, sp, 0, nullptr, [&](int64_t TR, int ln, double v, double) {
        const int64_t i = TR * 16 + ln;
        if (i < n) y[i] = v;
    });
    if (COUNT) {
        Counts cnt;
        cnt.zero();
        mfk::count_levels<DYN>(A, tr0, tr1, pv, range_guard, &cnt);
        if (threadIdx.x < 10) ired[threadIdx.x] = 0;
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

void* pick_kernel(int maxt, bool bicg, bool dyn, bool count, bool sticky, bool pre, bool sr = false) {
    if (sr) return maxt > 512 ? pick_cgsr_1024(dyn, count, sticky) : pick_cgsr_512(dyn, count, sticky);
    if (maxt > 512) {
        if (pre && bicg) return pick_pbicgstab_1024(dyn, count, sticky);
        if (pre) return pick_pcg_1024(dyn, count, sticky);
        return bicg ? pick_bicgstab_1024(dyn, count, sticky) : pick_cg_1024(dyn, count, sticky);
    }
    if (pre && bicg) return pick_pbicgstab_512(dyn, count, sticky);
    if (pre) return pick_pcg_512(dyn, count, sticky);
    return bicg ? pick_bicgstab_512(dyn, count, sticky) : pick_cg_512(dyn, count, sticky);
}

Mat mat_view(const TileMatrix& A) {
    return Mat{A.n_rows, A.n_cols, A.ntr, A.tr_slot, A.TileRowPtr, A.tile_info, A.sidx, A.blob,
               reinterpret_cast<const mfk::TsStage*>(A.stg), A.stg_ptr, A.TileNnz, A.ts, (int)A.max_w,
               A.plane64, A.plane32, A.plane16, A.plane8, nullptr, A.coff};
}

// Ring depth of the TMA pipeline for a shared-memory budget (bytes available to the ring)
int ring_depth(const TileMatrix& A, int64_t budget) {
    if (!A.ts) return 0;
    int64_t k = budget / std::max<int32_t>(A.slot_bytes, 128);
    if (const char* ev = getenv("MF_NST")) k = std::min<int64_t>(k, atoi(ev));
    return (int)std::max<int64_t>(0, std::min<int64_t>(k, mfk::TS_NSTMAX));
}

int64_t pv_doubles(int64_t n) { return ((n + 15) / 16) * PVS + PVS; }

}  // namespace

// ------------------------------------------------------------------------------- host side
namespace {
// device workspace released on every return path (scope guard)
struct Ws {
    cudaStream_t s;
    std::vector<void*> ptrs;
    explicit Ws(cudaStream_t st) : s(st) {}
    ~Ws() { for (void* p : ptrs) if (p) dev_free(p, s); }
    template <class T>
    mf_status get(T** p, size_t count) {
        MF_TRY(alloc(p, count, s));
        ptrs.push_back((void*)*p);
        return MF_OK;
    }
};
struct Events {
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    ~Events() { if (e0) cudaEventDestroy(e0); if (e1) cudaEventDestroy(e1); }
};
}  // namespace

mf_status run_spmv(const TileMatrix& A, const double* x, double* y, const uint8_t* level, int range_guard,
                   int64_t* counts_host, cudaStream_t s) {
    if (A.ntr == 0) return MF_OK;
    if (!A.ts && (A.n_cols + 15) / 16 > ((int64_t)1 << 28))
        return fail(MF_ERR_UNSUPPORTED, "compact layout: more than 2^28 tile columns");
    int dev = 0, smem_optin = 0;
    MF_CUDA(cudaGetDevice(&dev));
    MF_CUDA(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    Mat M = mat_view(A);
    Ws ws(s);
    unsigned long long* dcnt = nullptr;
    if (counts_host) {
        MF_TRY(ws.get(&dcnt, 10));
        MF_CUDA(cudaMemsetAsync(dcnt, 0, 10 * sizeof(unsigned long long), s));
    }
    double* pv = nullptr;
    const int64_t npv = pv_doubles(A.n_cols);
    MF_TRY(ws.get(&pv, (size_t)npv));
    MF_CUDA(cudaMemsetAsync(pv, 0, npv * sizeof(double), s));
    {
        const int blocks = (int)std::min<int64_t>((npv + 255) / 256, 148 * 16);
        pack_pv_kernel<<<blocks, 256, 0, s>>>(x, A.n_cols, level, pv);
        MF_CUDA(cudaGetLastError());
    }
    const int64_t ebytes = (int64_t)(A.B / 32) * A.ecap * 128;
    const int nst = std::max(1, ring_depth(A, (int64_t)smem_optin - 128 - 256 - (int64_t)mfk::TS_CTRL_BYTES - ebytes));
    const size_t smem = 128 + mfk::spmv_smem_bytes(A.ts, nst, A.slot_bytes, A.ecap, A.B / 32);
    void* fn;
    if (A.B > 512) {
        if (level) fn = counts_host ? (void*)spmv_kernel<true, true, 1024> : (void*)spmv_kernel<true, false, 1024>;
        else fn = counts_host ? (void*)spmv_kernel<false, true, 1024> : (void*)spmv_kernel<false, false, 1024>;
    } else {
        if (level) fn = counts_host ? (void*)spmv_kernel<true, true, 512> : (void*)spmv_kernel<true, false, 512>;
        else fn = counts_host ? (void*)spmv_kernel<false, true, 512> : (void*)spmv_kernel<false, false, 512>;
    }
    MF_TRY(set_max_dyn_smem(fn, smem_optin));
    const int32_t* plan = A.plan_tr;
    int slot_bytes = A.slot_bytes, blob_cap = A.blob_cap, nst_a = nst, ecap = A.ecap;
    void* args[] = {&M, (void*)&plan, (void*)&pv, (void*)&y, &range_guard, &dcnt, &nst_a, &slot_bytes, &blob_cap, &ecap};
    // diagnostics: MF_SPMV_REPS = launches of the SpMV kernel alone (timed with CUDA events,
    // reported on stderr with the warp-1 breakdown when MF_PHASE_DUMP is set)
    const int reps = getenv("MF_SPMV_REPS") ? std::max(1, atoi(getenv("MF_SPMV_REPS"))) : 1;
    Events ev;
    if (reps > 1) {
        MF_CUDA(cudaEventCreate(&ev.e0));
        MF_CUDA(cudaEventCreate(&ev.e1));
        MF_CUDA(cudaLaunchKernel(fn, dim3(A.G), dim3(A.B), args, smem, s));   // warm-up
        MF_CUDA(cudaEventRecord(ev.e0, s));
    }
    for (int k = 0; k < reps; ++k) MF_CUDA(cudaLaunchKernel(fn, dim3(A.G), dim3(A.B), args, smem, s));
    if (reps > 1) {
        MF_CUDA(cudaEventRecord(ev.e1, s));
        MF_CUDA(cudaEventSynchronize(ev.e1));
        float ms = 0;
        MF_CUDA(cudaEventElapsedTime(&ms, ev.e0, ev.e1));
        fprintf(stderr, "mf_spmv kernel: %.2f us per launch (%d launches, ring %d x %d B, decode %d cols/warp)\n",
                ms * 1e3 / reps, reps, nst, A.slot_bytes, A.ecap);
    }
    if (counts_host) {
        unsigned long long h[10];
        MF_CUDA(cudaMemcpyAsync(h, dcnt, sizeof(h), cudaMemcpyDeviceToHost, s));
        MF_CUDA(cudaStreamSynchronize(s));
        for (int q = 0; q < 5; ++q) counts_host[q] = (int64_t)h[q];
    }
    return MF_OK;
}

mf_status run_levels(const double* v, int64_t n, const double* th, uint8_t* level, cudaStream_t s) {
    if (!(th[0] <= th[1] && th[1] <= th[2] && th[2] <= th[3]))
        return fail(MF_ERR_INVALID_ARG, "mf_levels: thresholds must be non-decreasing");
    if (n == 0) return MF_OK;
    Thresh t{th[0], th[1], th[2], th[3]};
    int64_t nseg = (n + 15) / 16;
    int blocks = (int)std::min<int64_t>((nseg + 15) / 16, 148 * 16);
    levels_kernel<<<blocks, 256, 0, s>>>(v, n, t, level);
    MF_CUDA(cudaGetLastError());
    return MF_OK;
}

mf_status run_dot(const TileMatrix& A, const double* u, const double* v, double* out_host, cudaStream_t s) {
    Ws ws(s);
    double* slots = nullptr;
    MF_TRY(ws.get(&slots, A.G + 1));
    dot_partial_kernel<<<A.G, A.B, 0, s>>>(A.plan_tr, A.n_rows, u, v, slots);
    dot_final_kernel<<<1, 32, 0, s>>>(slots, A.G, slots + A.G);
    MF_CUDA(cudaGetLastError());
    MF_CUDA(cudaMemcpyAsync(out_host, slots + A.G, sizeof(double), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    return MF_OK;
}

mf_status run_cg_xr(const TileMatrix& A, double alpha, const double* p, const double* mu, double* x, double* r,
                    double* rr_host, cudaStream_t s) {
    Ws ws(s);
    double* slots = nullptr;
    MF_TRY(ws.get(&slots, A.G + 1));
    cg_xr_kernel<<<A.G, A.B, 0, s>>>(A.plan_tr, A.n_rows, alpha, p, mu, x, r, slots);
    dot_final_kernel<<<1, 32, 0, s>>>(slots, A.G, slots + A.G);
    MF_CUDA(cudaGetLastError());
    MF_CUDA(cudaMemcpyAsync(rr_host, slots + A.G, sizeof(double), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
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
                    mf_solve_info* info, cudaStream_t s, const MgLaunch* mgl) {
    if (A.n_rows != A.n_cols && !mgl) return fail(MF_ERR_INVALID_ARG, "solve needs a square matrix");
    if (mgl && (bicg || o.M || o.sticky || o.cg_variant || o.tile_level_counts || o.collect_stats))
        return fail(MF_ERR_NOT_IMPLEMENTED, "device-initiated multi-GPU kernel: CG without preconditioner, sticky variant or statistics");
    if (o.max_iter < 0 || o.max_iter > ((int64_t)1 << 40)) return fail(MF_ERR_INVALID_ARG, "max_iter out of range");
    // sticky variant (P:237 literal): dynamic mode only (as in the oracle)
    const bool sticky = o.sticky && o.mode == MF_MODE_DYNAMIC_MIXED;
    if (sticky && !A.ts && (A.n_cols + 15) / 16 > ((int64_t)1 << 24))
        return fail(MF_ERR_NOT_IMPLEMENTED, "sticky downgrade, compact layout: more than 2^24 tile columns");
    if (!A.ts && (A.n_cols + 15) / 16 > ((int64_t)1 << 28))
        return fail(MF_ERR_UNSUPPORTED, "compact layout: more than 2^28 tile columns");
    if (sticky && (o.tile_level_counts != nullptr || o.collect_stats))
        return fail(MF_ERR_NOT_IMPLEMENTED, "sticky downgrade does not collect per-SpMV level statistics");
    Precond* P = o.M ? const_cast<Precond*>(&o.M->p) : nullptr;
    const bool pre = P != nullptr;
    const bool sr = !bicg && o.cg_variant == 1;       // single-reduction CG
    if (sr && pre) return fail(MF_ERR_NOT_IMPLEMENTED, "single-reduction CG with a preconditioner");
    if (o.cg_variant != 0 && o.cg_variant != 1) return fail(MF_ERR_INVALID_ARG, "cg_variant must be 0 or 1");
    if (pre && P->n != A.n_rows) return fail(MF_ERR_INVALID_ARG, "preconditioner built for another matrix size");
    int dev = 0, sms = 0, smem_optin = 0;
    MF_CUDA(cudaGetDevice(&dev));
    MF_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    MF_CUDA(cudaDeviceGetAttribute(&smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    const int64_t n = A.n_rows;
    const int G = A.G, B = A.B;
    const bool dyn = o.mode == MF_MODE_DYNAMIC_MIXED;
    const int nvec = bicg ? 2 : 1;
    // per-SpMV level statistics (tile_level_counts, exact dynamic byte model): on request
    const bool count = o.tile_level_counts != nullptr || o.collect_stats;
    int64_t max_rows = 0;
    for (int g = 0; g < G; ++g) max_rows = std::max(max_rows, A.plan_rows_host[g + 1] - A.plan_rows_host[g]);
    // shared memory: fixed + SpMV region (TMA ring or compact buffers) + mu (and theta) + SpTRSV
    const size_t fixed = fixed_smem_bytes();
    const int64_t pre_smem = pre ? (int64_t)B * 12 + 32 + (P->sweep ? (int64_t)mfk::sweep_smem_bytes() + 32 : 0) : 0;
    const int64_t ebytes = A.ts ? (int64_t)(B / 32) * A.ecap * 128 : 0;
    // - 256: the carve's alignment padding and the +64 slack of `smem` below
    const int64_t avail = (int64_t)smem_optin - (int64_t)fixed - pre_smem - 128 - (int64_t)mfk::TS_CTRL_BYTES - ebytes - 256;
    int64_t cap = 0;
    int nst = 1;
    bool mu_onchip = true;
    if (const char* ev = getenv("MF_MU_ONCHIP")) mu_onchip = atoi(ev) != 0;   // tuning: trade smem for ring depth
    if (A.ts) {
        // mu on chip only when the ring still gets >= 3 slots (TMA latency cover)
        const int64_t need_mu = max_rows * 8 * nvec;
        // a 2-deep TMA ring already hides the stage loads once mu stays on chip (r02 sweep on C2:
        // ring 2 + mu on chip 73.0 us/it, ring 5 + mu in HBM 74.6)
        int min_ring = 2;
        if (const char* ev = getenv("MF_MU_MINRING")) min_ring = std::max(1, atoi(ev));   // tuning knob
        if (mu_onchip && ring_depth(A, avail - need_mu) >= min_ring) cap = max_rows;
        nst = ring_depth(A, avail - cap * 8 * nvec);
        if (nst < 1) return fail(MF_ERR_UNSUPPORTED, "TMA ring does not fit shared memory");
    } else {
        cap = mu_onchip ? std::max<int64_t>(0, std::min<int64_t>(max_rows, (avail - (int64_t)mfk::WIN_SMEM_BYTES - 16) / (8 * nvec))) : 0;
    }
    const size_t smem = fixed + mfk::spmv_smem_bytes(A.ts, nst, A.slot_bytes, A.ecap, B / 32) + (size_t)cap * 8 * nvec + (size_t)pre_smem + 64;
    if ((int64_t)smem > smem_optin) return fail(MF_ERR_UNSUPPORTED, "shared-memory plan exceeds the device limit");

    void* kfn = mgl ? pick_cgmg(B, dyn) : pick_kernel(B, bicg, dyn, count, sticky, pre, sr);
    // the opt-in maximum, not this launch's size: concurrent solves (rank threads of a local group,
    // other streams) share the function attribute, and a smaller value set by one would make
    // another's larger launch invalid
    MF_TRY(set_max_dyn_smem(kfn, smem_optin));
    int per_sm = 0;
    MF_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kfn, B, smem));
    if (per_sm * sms < G) return fail(MF_ERR_INVALID_ARG, "plan G exceeds co-resident CTAs for this launch");

    // workspace (released by the scope guard on every path)
    Ws ws(s);
    const bool spill = cap < max_rows;
    const int64_t hist_cap = std::min<int64_t>(o.max_iter + 2, std::max<int64_t>(o.history_cap, 2) + 2);
    const int64_t lc_cap = count ? (bicg ? 2 : 1) * (o.max_iter + 1) : 0;
    const int64_t npv = pv_doubles(n);
    double *r = nullptr, *p = nullptr, *mu_g = nullptr, *rh = nullptr, *sv = nullptr, *th_g = nullptr;
    double *slots = nullptr, *hist = nullptr, *out = nullptr, *pz = nullptr, *psh = nullptr;
    unsigned* sync = nullptr;
    unsigned long long *lcounts = nullptr, *bar_ns = nullptr, *phase_ns = nullptr;
    const bool pbicg = pre && bicg;
    MF_TRY(ws.get(&r, n));
    if (mgl) p = mgl->pv_own;             // the window's extended vector (cleared by prelaunch)
    else MF_TRY(ws.get(&p, pbicg ? n : npv));
    if (spill) MF_TRY(ws.get(&mu_g, n));
    if (bicg) {
        MF_TRY(ws.get(&rh, n));
        MF_TRY(ws.get(&sv, pbicg ? n : npv));
        if (spill) MF_TRY(ws.get(&th_g, n));
    }
    if (sr) {    // p and s of the single-reduction CG (start at 0)
        MF_TRY(ws.get(&rh, n));
        MF_TRY(ws.get(&sv, n));
        MF_CUDA(cudaMemsetAsync(rh, 0, n * sizeof(double), s));
        MF_CUDA(cudaMemsetAsync(sv, 0, n * sizeof(double), s));
    }
    if (pre) {
        MF_TRY(ws.get(&pz, bicg ? npv : n));
        if (bicg) MF_TRY(ws.get(&psh, npv));
    }
    // PV vectors: padding rows / slots stay zero
    if (!pbicg && !mgl) MF_CUDA(cudaMemsetAsync(p, 0, npv * sizeof(double), s));
    if (sv && !pbicg && !sr) MF_CUDA(cudaMemsetAsync(sv, 0, npv * sizeof(double), s));
    if (pz && bicg) MF_CUDA(cudaMemsetAsync(pz, 0, npv * sizeof(double), s));
    if (psh) MF_CUDA(cudaMemsetAsync(psh, 0, npv * sizeof(double), s));
    MF_TRY(ws.get(&slots, (size_t)2 * NSLOT * G));
    MF_TRY(ws.get(&hist, hist_cap));
    MF_TRY(ws.get(&out, 8));
    MF_TRY(ws.get(&sync, (size_t)G + 2));
    MF_TRY(ws.get(&bar_ns, G));
    MF_TRY(ws.get(&phase_ns, (size_t)G * NPHASE));
    MF_CUDA(cudaMemsetAsync(phase_ns, 0, (size_t)G * NPHASE * sizeof(unsigned long long), s));
    if (count) MF_TRY(ws.get(&lcounts, (size_t)lc_cap * 10));
    MF_CUDA(cudaMemsetAsync(sync, 0, (G + 2) * sizeof(unsigned), s));
    MF_CUDA(cudaMemsetAsync(bar_ns, 0, G * sizeof(unsigned long long), s));
    MF_CUDA(cudaMemsetAsync(out, 0, 8 * sizeof(double), s));
    if (count) MF_CUDA(cudaMemsetAsync(lcounts, 0, (size_t)lc_cap * 10 * sizeof(unsigned long long), s));

    uint8_t* stk = nullptr;
    if (sticky) {
        const size_t nstk = (size_t)(A.ts ? A.slots : A.tilenum) + 1;   // per slice column (TS) / per tile (compact)
        MF_TRY(ws.get(&stk, nstk));
        MF_CUDA(cudaMemsetAsync(stk, 0, nstk, s));
    }
    SolveArgs a{};
    a.A = mat_view(A);
    a.A.stk = stk;
    a.G = G; a.plan_tr = A.plan_tr; a.dep_lo = A.dep_lo; a.dep_hi = A.dep_hi;
    a.n = n; a.b = b; a.x = x; a.r = r; a.p = p; a.mu_g = mu_g;
    a.rh = rh; a.s = sv; a.th_g = th_g;
    a.slots = slots; a.bar = sync; a.abort_flag = reinterpret_cast<int*>(sync + 1); a.flags = sync + 2;
    a.bar_ns = bar_ns; a.phase_ns = phase_ns; a.hist = hist; a.hist_cap = hist_cap; a.lcounts = lcounts; a.lc_cap = lc_cap;
    a.out = out; a.tol = o.tol; a.switch_eps = o.switch_eps < 0 ? o.tol : o.switch_eps;   // reading R8: eps = tol
    a.switch_abs = o.switch_absolute; a.range_guard = o.range_guard; a.max_iter = o.max_iter;
    a.mu_cap = (int)cap;
    a.nst = nst; a.slot_bytes = A.slot_bytes; a.blob_cap = A.blob_cap; a.ecap = A.ecap;
    a.stall_cta = -1;
    // one-cluster launches of small plans (barrier.cluster instead of the grid barrier) were tried
    // for C1 and withdrawn: the static-mode kernels faulted with the cluster paths compiled in
    // (profiles/r02_gpu3/bisect.log); the launch below keeps the field at 0
    a.cluster = 0;
    if (const char* ev = getenv("MF_DEBUG_STALL_CTA")) a.stall_cta = atoi(ev);   // watchdog test hook
    a.timeout_ns = (o.watchdog_ms > 0 ? (unsigned long long)o.watchdog_ms : 60000ull) * 1000000ull;
    if (pre) {
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
        a.psweep = P->sweep;
        if (P->rb_depth > 0) {
            a.rb = 1;
            a.Lnodes = P->Lrb.nodes; a.nLn = (int)P->Lrb.h.size(); a.Lbrp = P->Lrb.rp; a.Lbci = P->Lrb.ci; a.Lbv = P->Lrb.v;
            a.Unodes = P->Urb.nodes; a.nUn = (int)P->Urb.h.size(); a.Ubrp = P->Urb.rp; a.Ubci = P->Urb.ci; a.Ubv = P->Urb.v;
        }
    }

    if (mgl) {
        a.mg = mgl->args;
        a.mg.seg_lo = A.seg_lo;
        a.mg.seg_hi = A.seg_hi;
        MF_TRY(mgl->prelaunch(mgl->ctx, s));
    }
    Events ev;
    MF_CUDA(cudaEventCreate(&ev.e0));
    MF_CUDA(cudaEventCreate(&ev.e1));
    void* args[] = {&a};
    MF_CUDA(cudaEventRecord(ev.e0, s));
    if (mgl && mgl->plain_launch) {
        MF_CUDA(cudaLaunchKernel(kfn, dim3(G), dim3(B), args, smem, s));
    } else {
        MF_CUDA(cudaLaunchCooperativeKernel(kfn, dim3(G), dim3(B), args, smem, s));
    }
    if (mgl && mgl->postlaunch) MF_TRY(mgl->postlaunch(mgl->ctx));
    MF_CUDA(cudaEventRecord(ev.e1, s));
    double hout[8];
    MF_CUDA(cudaMemcpyAsync(hout, out, sizeof(hout), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    float ms = 0;
    MF_CUDA(cudaEventElapsedTime(&ms, ev.e0, ev.e1));
    const int64_t iters = (int64_t)hout[0];
    info->iterations = iters;
    info->converged = (int)hout[1];
    info->rel_residual = hout[2];
    info->status = (mf_status)(int)hout[3];
    info->kernel_ms = ms;
    info->launches = 1;
    const int64_t nspmv = (bicg ? 2 : 1) * iters + (sr && iters > 0 ? 1 : 0);
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
    // write s,x,r,p); + 16n per SpMV output that cannot stay on chip (capacity rule, SURVEY 8(d):
    // counted when the outputs do not fit the GPU's shared memory, whatever this launch did)
    const double vec = bicg ? 72.0 : (sr ? 72.0 : 48.0);   // single-reduction CG: read p,s,x,r,w; write p,s,x,r
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
        fprintf(stderr, "smem %zu B: ring %d x %d B (blob cap %d, window cap %d segs), decode %d cols/warp, mu_cap %lld of %lld rows\n",
                smem, nst, A.slot_bytes, A.blob_cap, A.wcap, A.ecap, (long long)cap, (long long)max_rows);
    }
    {
        double sum = 0;
        for (int g = 0; g < G; ++g) sum += (double)bns[g];
        info->barrier_ms = sum / G / 1e6;   // mean over CTAs of time spent spinning (barriers + ready flags)
    }
    info->ring_slots = nst;
    info->mu_onchip = cap >= max_rows ? 1 : 0;
    const mf_status st = info->status;
    if (st == MF_ERR_BREAKDOWN) return fail(st, "numerical breakdown");
    if (st == MF_ERR_DEADLOCK) return fail(st, "grid-barrier watchdog expired");
    return st;
}

}  // namespace mf
