// solver_kernels.cuh -- the single-kernel CG and BiCGSTAB of Mille-feuille on sm_100a
// (Section III-C, Alg. 3; mixed precision Section III-D).
//
// One cooperative persistent launch runs the whole solve.  CTA g owns the contiguous tile
// rows [plan_tr[g], plan_tr[g+1]) (the task distribution of P:130-132, balanced on nnz and
// tiles) and does every vector operation for its rows.  The paper's dependency
// counters d_s / d_d / d_a become:
//   * a monotone-epoch grid barrier (one atomic per CTA, acquire-spin) at each dot product,
//     carrying the per-CTA partial sums in fixed slots -> deterministic reductions;
//   * per-CTA "ready" epoch flags: before an SpMV a CTA waits only for the CTAs owning the
//     column segments it gathers (the generalisation of d_s), not for the whole grid.
// The SpMV input (p, s, p^, s^) lives in the PV layout (kernels.cuh): its producer writes the
// level of every 16-element segment (Alg. 4, the convergent-element retrieval: the min over the
// half-warp that produced the segment) next to the values, and the SpMV stages values and levels
// together by TMA.  The SpMV output mu (and theta) stays in shared memory of the owner CTA across
// the barrier when it fits (the CG residual then reuses mu's slot), else it spills to global.
#pragma once
#include <cuda_runtime.h>

#include "kernels.cuh"
#include "mf_internal.cuh"
#include "precond.cuh"

namespace mf {
namespace {

using mfk::Counts;
using mfk::Mat;
using mfk::Thresh;
using mfk::PVS;
using mfk::pv_idx;

constexpr int NSLOT = 4;    // doubles reduced per barrier (max)
constexpr int NPHASE = 12;  // timed phases per CTA

struct SolveArgs {
    Mat A;
    int32_t G;
    const int32_t* __restrict__ plan_tr;
    const int32_t* __restrict__ dep_lo;
    const int32_t* __restrict__ dep_hi;
    int64_t n;
    const double* __restrict__ b;
    double* x;
    double* r;
    double* p;         // PV layout (CG, PCG, BiCGSTAB); normal (PBiCGSTAB)
    double* mu_g;      // spill of mu beyond mu_cap rows per CTA [n]
    double* rh;        // BiCGSTAB r0*
    double* s;         // PV layout (BiCGSTAB); normal (PBiCGSTAB)
    double* th_g;      // spill of theta
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
    int nst, slot_bytes, blob_cap, ecap;   // TMA ring + decode buffers of the SpMV (tile-synchronous layout)
    int stall_cta;                   // test hook: this CTA never publishes (-1: none)
    int cluster;                     // reserved (0): one-cluster launch of small plans, not enabled
    unsigned long long timeout_ns;
    // ILU(0) preconditioner (PCG / right-preconditioned PBiCGSTAB); null when unpreconditioned
    const int64_t* Lrp; const int32_t* Lci; const double* Lv;
    const int64_t* Urp; const int32_t* Uci; const double* Uv; const double* Ud;
    unsigned* pflags;            // per-row ready epochs of the triangular solves
    unsigned long long* pctr;    // [2] chunk counters (forward, backward)
    double* py;                  // forward-solve output
    double* pz;                  // PCG: z (normal); PBiCGSTAB: p^ (PV)
    double* ps;                  // PBiCGSTAB: s^ (PV)
    unsigned pe0;                // epoch of the first apply of this solve
    // recursive block SpTRSV (rb == 0: sync-free substitution over the whole factor)
    int rb;
    int psweep;                  // 1: triangular solves by the one-CTA sweep (deep dependency DAGs)
    const RbNode* Lnodes; int nLn; const int64_t* Lbrp; const int32_t* Lbci; const double* Lbv;
    const RbNode* Unodes; int nUn; const int64_t* Ubrp; const int32_t* Ubci; const double* Ubv;
    MgArgs mg;                   // multi-GPU single kernel (P == 0: off)
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
    unsigned nred = 0;           // cross-rank reductions so far (multi-GPU kernel)
};

__device__ __forceinline__ void red_release_add(unsigned* p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// generic-proxy writes of a PV vector -> later bulk copies (async proxy) of other CTAs / this CTA
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
// system scope (peer GPUs over NVLink)
__device__ __forceinline__ unsigned ld_acquire_sys(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long ld_acquire_sys64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ double ld_relaxed_sys_f64(const double* p) {
    double v;
    asm volatile("ld.relaxed.sys.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(unsigned* p, unsigned v) {
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_release_sys_add64(unsigned long long* p, unsigned long long v) {
    asm volatile("red.release.sys.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
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
    if (a.G == 1) return true;            // one CTA (small matrices): the CTA barrier orders everything
    if (threadIdx.x == 0) {
        const unsigned long long t0 = gtimer();
        red_release_add(a.bar, 1u);       // cumulative release: this CTA's writes (ordered by bar.sync)
        int ab = 0;
        while (ld_acquire(a.bar) < c.bar_target) {
            if (*(volatile int*)a.abort_flag) { ab = 1; break; }
            const unsigned long long dt = gtimer() - t0;
            if (dt > a.timeout_ns) { atomicExch(a.abort_flag, 1); ab = 1; break; }
            // long waits (one CTA at work, e.g. the triangular-solve sweep): back off, so that
            // 147 pollers do not keep the L2 line and the memory system busy
            if (dt > 20000ull) __nanosleep(1000);
        }
        __threadfence();
        *spin_ns_smem() += gtimer() - t0;
        s_abort = ab;
    }
    __syncthreads();
    return s_abort == 0;
}

// Multi-GPU kernel: store this CTA's own segments that peers gather (values + level byte, 144 B
// each) into the peers' extended vectors, then count the CTA as arrived at each such peer (one
// system-scope release-add per peer after the CTA barrier and a system fence).
__device__ __forceinline__ void mg_push(const SolveArgs& a, const double* own) {
    const MgArgs& m = a.mg;
    const int e0 = m.send_ptr[blockIdx.x], e1 = m.send_ptr[blockIdx.x + 1];
    if (e1 == e0) return;
    for (int k = threadIdx.x; k < (e1 - e0) * PVS; k += blockDim.x) {
        const int e = e0 + k / PVS, d = k - (k / PVS) * PVS;
        const double v = __ldcg(own + (int64_t)m.send_src[e] * PVS + d);
        double* dst = reinterpret_cast<double*>(m.win[m.send_peer[e]] + m.off_pv) + (int64_t)m.send_dst[e] * PVS + d;
        __stcg(dst, v);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence_system();
        const unsigned mask = m.send_mask[blockIdx.x];
        for (int r = 0; r < m.P; ++r)
            if (mask & (1u << r))
                red_release_sys_add64(reinterpret_cast<unsigned long long*>(m.win[r] + m.off_cnt) + m.me, 1ull);
    }
}

// all threads: the CTA's writes of the SpMV input are complete -> ready flag `epoch`
template <bool MG = false>
__device__ __forceinline__ void publish(const SolveArgs& a, unsigned epoch, const double* own = nullptr) {
    fence_proxy_async();
    __syncthreads();
    if (MG && a.mg.P > 1) mg_push(a, own);
    if (threadIdx.x == 0 && (int)blockIdx.x != a.stall_cta) st_release(&a.flags[blockIdx.x], epoch);
}

// Multi-GPU kernel: the halo segments this CTA gathers from rank r are complete once all nprod[r]
// storing CTAs of r arrived for this epoch (counters are monotone: epoch * nprod[r]).
__device__ __forceinline__ bool mg_wait_halo(const SolveArgs& a, unsigned epoch, unsigned long long t0) {
    const MgArgs& m = a.mg;
    bool ok = true;
    const int r = threadIdx.x;
    if (r < m.P && r != m.me && m.nprod[r] > 0 && m.hlo[r] < m.hhi[r]) {
        const int slo = m.seg_lo[blockIdx.x], shi = m.seg_hi[blockIdx.x];
        if (shi >= m.hlo[r] && slo < m.hhi[r]) {
            const unsigned long long* cnt = reinterpret_cast<const unsigned long long*>(m.win[m.me] + m.off_cnt) + r;
            const unsigned long long target = (unsigned long long)epoch * (unsigned long long)m.nprod[r];
            while (ld_acquire_sys64(cnt) < target) {
                if (*(volatile int*)a.abort_flag) { ok = false; break; }
                if (gtimer() - t0 > a.timeout_ns) { atomicExch(a.abort_flag, 1); ok = false; break; }
            }
        }
    }
    fence_proxy_async();     // peer (generic-proxy) stores -> this CTA's bulk copies of the halo
    return ok;
}

template <bool MG = false>
__device__ __forceinline__ bool wait_deps(const SolveArgs& a, unsigned epoch) {
    __shared__ int s_abort;
    if (a.G == 1 && a.stall_cta < 0 && !(MG && a.mg.P > 1)) {   // one CTA: its own writes, ordered by the CTA barrier
        __syncthreads();
        return true;
    }
    const int lo = a.dep_lo[blockIdx.x], hi = a.dep_hi[blockIdx.x];
    if (threadIdx.x == 0) s_abort = 0;
    __syncthreads();
    const unsigned long long t0 = gtimer();
    if (MG && a.mg.P > 1 && !mg_wait_halo(a, epoch, t0)) s_abort = 1;
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
//
// Multi-GPU kernel (MG, P ranks): the CTA totals of this rank give the rank partial (tree32 over
// the rank's CTAs); CTA 0 stores it, tagged with the reduction number, into slot [parity][me] of
// every rank's window; every CTA of every rank then sums the P rank partials in rank order from
// +0 (identical on all ranks: the oracle's rank-partitioned plan).  Slots alternate parities: a
// rank can only publish reduction k+2 after every rank published k+1, i.e. after every CTA of
// every rank read k.
template <int K, bool MG = false>
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
    bool ok = grid_barrier(a, c);
    if (!MG || a.mg.P <= 1) {
        if (w == 0) {
#pragma unroll
            for (int k = 0; k < K; ++k) {
                const double gt = mfk::tree32(a.slots + ((size_t)c.parity * NSLOT + k) * a.G, a.G);
                if (l == 0) red[128 + k] = (MG && a.mg.P == 1) ? __dadd_rn(0.0, gt) : gt;
            }
        }
    } else {
        const MgArgs& m = a.mg;
        const unsigned tag = ++c.nred;
        const int par = (int)(tag & 1u);
        if (blockIdx.x == 0 && w == 0) {
            double gt[K];
#pragma unroll
            for (int k = 0; k < K; ++k) gt[k] = mfk::tree32(a.slots + ((size_t)c.parity * NSLOT + k) * a.G, a.G);
            if (l < m.P) {
                double* dst = reinterpret_cast<double*>(m.win[l] + m.off_red) + ((size_t)par * m.P + m.me) * 4;
#pragma unroll
                for (int k = 0; k < K; ++k) __stcg(dst + k, gt[k]);
                st_release_sys(reinterpret_cast<unsigned*>(m.win[l] + m.off_tag) + par * m.P + m.me, tag);
            }
        }
        __shared__ int s_ab;
        if (threadIdx.x == 0) s_ab = 0;
        __syncthreads();
        if ((int)threadIdx.x < m.P) {
            const unsigned* tg = reinterpret_cast<const unsigned*>(m.win[m.me] + m.off_tag) + par * m.P + threadIdx.x;
            const unsigned long long t0 = gtimer();
            while ((int)(ld_acquire_sys(tg) - tag) < 0) {
                if (*(volatile int*)a.abort_flag) { s_ab = 1; break; }
                if (gtimer() - t0 > a.timeout_ns) { atomicExch(a.abort_flag, 1); s_ab = 1; break; }
            }
        }
        __syncthreads();
        if (s_ab) ok = false;
        if (threadIdx.x == 0) {
            const double* sl = reinterpret_cast<const double*>(m.win[m.me] + m.off_red) + (size_t)par * m.P * 4;
#pragma unroll
            for (int k = 0; k < K; ++k) {
                double t = 0.0;
                for (int r = 0; r < m.P; ++r) t = __dadd_rn(t, ld_relaxed_sys_f64(sl + r * 4 + k));
                red[128 + k] = t;
            }
        }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < K; ++k) v[k] = red[128 + k];
    __syncthreads();
    c.parity ^= 1;
    return ok;
}

// per-SpMV level statistics (stats mode): one pass over the CTA's tiles, then per-CTA sums
template <bool COUNT, bool DYN>
__device__ __forceinline__ void spmv_counts(const SolveArgs& a, Ctx& c, int64_t tr0, int64_t tr1, const double* pv, int* ired) {
    if (!COUNT) return;
    Counts cnt;
    cnt.zero();
    mfk::count_levels<DYN>(a.A, tr0, tr1, pv, a.range_guard, &cnt);
    __syncthreads();
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
    unsigned char* sweep;   // sweep triangular solve buffers (precond.cuh sweep_smem_bytes), CTA 0
    double* red;     // [4*32 + 8]
    int* ired;       // [16]
    unsigned long long* timer;   // [NPHASE + 1]
    mfk::SpmvSmem sp;
};

__host__ __device__ constexpr size_t fixed_smem_bytes() {
    return (4 * 32 + 8) * sizeof(double) + 16 * sizeof(int) + (NPHASE + 1) * 8 + 256;
}

__device__ __forceinline__ Smem carve(const SolveArgs& a, int nvec) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    Smem s;
    double* d = reinterpret_cast<double*>(smem_raw);
    s.red = d;
    s.ired = reinterpret_cast<int*>(d + 4 * 32 + 8);
    s.timer = reinterpret_cast<unsigned long long*>(s.ired + 16);
    // alignment by offsets from smem_raw (never through an integer cast of the pointer): the
    // compiler keeps the shared address space and emits LDS/STS with 32-bit addresses
    unsigned char* p = smem_raw + ((int)(reinterpret_cast<unsigned char*>(s.timer + NPHASE + 1) - smem_raw) + 127) / 128 * 128;
    mfk::carve_spmv(p, a.nst, a.slot_bytes, a.blob_cap, a.ecap, s.sp);
    mfk::ts_init(s.sp.ts);     // ordered before the first SpMV by the caller's __syncthreads (Timer::start)
    p += mfk::spmv_smem_bytes(a.A.ts, a.nst, a.slot_bytes, a.ecap, blockDim.x >> 5);
    p = smem_raw + mfk::ts_r16((int)(p - smem_raw));
    s.mu = reinterpret_cast<double*>(p);
    s.th = s.mu + a.mu_cap;
    s.tys = s.mu + (size_t)nvec * a.mu_cap;
    s.tready = reinterpret_cast<int*>(s.tys + blockDim.x);
    s.tchunk = reinterpret_cast<long long*>(s.tready + blockDim.x + 2);
    s.sweep = smem_raw + mfk::ts_r16((int)(reinterpret_cast<unsigned char*>(s.tchunk + 2) - smem_raw));
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

// The SpMV input of the init phase: x0 in the PV layout (own rows, level FP64), published with
// epoch 1 and awaited, so that r0 = b - A~ x0 runs through the same staged SpMV.
template <bool MG = false>
__device__ __forceinline__ bool stage_x0(const SolveArgs& a, double* PV, int64_t R0, int64_t Rend) {
    for (int64_t i = R0 + threadIdx.x; i < Rend; i += blockDim.x) {
        PV[pv_idx(i)] = a.x[i];
        if ((i & 15) == 0) {
            PV[(i >> 4) * PVS + 16] = 0.0;                 // level FP64 (static SpMV)
            PV[(i >> 4) * PVS + 17] = 0.0;
        }
    }
    // padding rows of the last segment (rows >= n) stay 0 (workspace cleared by the host)
    publish<MG>(a, 1, PV);
    return wait_deps<MG>(a, 1);
}

// levels of the own segments of a PV vector (Alg. 4): one half-warp per tile row
template <bool DYN>
__device__ __forceinline__ void pv_levels(const SolveArgs& a, double* PV, int64_t tr0, int64_t tr1, const Thresh& th) {
    const int H = blockDim.x >> 4, h = threadIdx.x >> 4, lane = threadIdx.x & 15;
    const unsigned m = mfk::hw_mask();
    for (int64_t TR = tr0 + h; TR < tr1; TR += H) {
        const int64_t i = TR * 16 + lane;
        int lv = 0;
        if (DYN) lv = mfk::hw_min_i(i < a.n ? mfk::level_of(__ldcg(PV + TR * PVS + lane), th) : 4, m);
        if (lane == 0) mfk::pv_set_level(PV, TR, lv);
    }
}

// -------------------------------------------------------------------------- CG (Alg. 1 / Alg. 3)
// Phases: 0 wait for SpMV inputs, 1 SpMV + (mu,p), 2 reduce sigma, 3 r update + (r,r),
//         4 reduce rho', 5 x and p update + levels + publish, 6 init
// Row mapping of every vector phase: thread t takes rows R0 + t + kB (the plan tree); r_{j+1}
// replaces mu in shared memory, x_{j+1} = x_j + alpha p_j is applied with the p update.
template <bool DYN, bool COUNT, bool STK, int MAXT, bool MG = false>
__global__ void __launch_bounds__(MAXT, 1) cg_persistent(SolveArgs a) {
    constexpr int PF = MAXT >= 1024 ? 4 : 8;
    Smem sm = carve(a, 1);
    Ctx c;
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
    double* P = a.p;                 // PV layout
    double* __restrict__ MUg = a.mu_g;
    double* __restrict__ MUs = sm.mu;
    (void)H; (void)h; (void)lane;

    // init: r = b - A~ x0 at TilePrec; partial (b,b), (r,r)
    double v2[2] = {0.0, 0.0};
    bool ok = stage_x0<MG>(a, P, R0, Rend);
    mfk::spmv_cta<false, false, PF>(a.A, tr0, tr1, P, 0, sm.sp, 0, nullptr,
                                    [&](int64_t TR, int ln, double ax, double) {
                                        const int64_t i = TR * 16 + ln;
                                        if (i < n) {
                                            const double bi = a.b[i];
                                            const double ri = __dsub_rn(bi, ax);
                                            Rv[i] = ri;
                                            v2[0] = __fma_rn(bi, bi, v2[0]);
                                            v2[1] = __fma_rn(ri, ri, v2[1]);
                                        }
                                    });
    ok = grid_reduce<2, MG>(v2, a, c, sm.red) && ok;     // every CTA's init SpMV is done: P may be overwritten
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
        // p0 = r0 (PV) + levels
        for (int64_t l0 = t; l0 < (tr1 - tr0) * 16; l0 += B) {
            const int64_t i = R0 + l0;
            const double pv = i < n ? Rv[i] : 0.0;
            P[pv_idx(i)] = pv;
            int lv = 0;
            if (DYN) lv = mfk::hw_min_i(i < n ? mfk::level_of(pv, th) : 4, m);
            if ((i & 15) == 0) mfk::pv_set_level(P, i >> 4, lv);
        }
        publish<MG>(a, 2, P);
        tm.tick(6);
        for (;; ++j) {
            const double relres = __ddiv_rn(sqrt(rho), nb);
            if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = relres; a.out[2] = relres; }
            if (relres < a.tol) { converged = 1; break; }
            if (j == a.max_iter) break;
            if (!wait_deps<MG>(a, (unsigned)(j + 2))) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(0);
            // step A: mu = A~_j p_j (own tile rows) with the fused partial (mu, p)
            double sg[1] = {0.0};
            mfk::spmv_cta<DYN, STK, PF>(a.A, tr0, tr1, P, a.range_guard, sm.sp, 1, nullptr,
                                        [&](int64_t TR, int ln, double mv, double ov) {
                                            const int64_t i = TR * 16 + ln;
                                            if (i < n) {
                                                const int64_t li = i - R0;
                                                if (li < mu_cap) MUs[li] = mv; else MUg[i] = mv;
                                                sg[0] = __fma_rn(mv, ov, sg[0]);
                                            }
                                        });
            spmv_counts<COUNT, DYN>(a, c, tr0, tr1, P, sm.ired);
            tm.tick(1);
            // step B: sigma = (mu, p) over the grid -> alpha
            if (!grid_reduce<1, MG>(sg, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(2);
            const double sigma = sg[0];
            if (!(sigma > 0.0) || !isfinite(sigma)) { status = MF_ERR_BREAKDOWN; break; }
            const double alpha = __ddiv_rn(rho, sigma);
            // step C: r -= alpha mu, partial (r, r); r_{j+1} replaces mu in shared memory.  The
            // loads of the next 4 rows per thread are issued before this chunk's arithmetic
            // (software pipeline: 8 rows of global loads in flight per thread)
            double rr[1] = {0.0};
            {
                double rv[4], rn[4];
                auto load_r = [&](int64_t l0, double (&d)[4]) {
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int64_t li = l0 + q * B;
                        d[q] = li < nr ? Rv[R0 + li] : 0.0;
                    }
                };
                load_r(t, rv);
                for (int64_t l0 = t; l0 < nr; l0 += 4 * (int64_t)B) {
                    if (l0 + 4 * (int64_t)B < nr) load_r(l0 + 4 * (int64_t)B, rn);
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int64_t li = l0 + q * B;
                        if (li < nr) {
                            const double mv = li < mu_cap ? MUs[li] : MUg[R0 + li];
                            const double ri = __fma_rn(-alpha, mv, rv[q]);
                            Rv[R0 + li] = ri;
                            if (li < mu_cap) MUs[li] = ri;
                            rr[0] = __fma_rn(ri, ri, rr[0]);
                        }
                    }
#pragma unroll
                    for (int q = 0; q < 4; ++q) rv[q] = rn[q];
                }
            }
            tm.tick(3);
            if (!grid_reduce<1, MG>(rr, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(4);
            const double beta = __ddiv_rn(rr[0], rho);
            rho = rr[0];
            // step D: x += alpha p_j ; p_{j+1} = r + beta p_j (own rows, PV) and the levels of its
            // segments (Alg. 4).  Rows l0 + qB of a half-warp form whole tile rows.
            {
                // software pipeline as in step C: p and x of the next 4 rows per thread in flight
                const int64_t L = (tr1 - tr0) * 16;
                double pv[4], xv[4], pn4[4], xn4[4];
                auto load_px = [&](int64_t l0, double (&pd)[4], double (&xd)[4]) {
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int64_t li = l0 + q * B, i = R0 + li;
                        pd[q] = li < nr ? P[pv_idx(i)] : 0.0;
                        xd[q] = li < nr ? X[i] : 0.0;
                    }
                };
                load_px(t, pv, xv);
                // warp-uniform trip count (the warp's first row decides), so that the levels are two
                // full-warp reductions; rows past the CTA's range are masked per lane
                const int64_t lane32 = t & 31;
                for (int64_t l0 = t; l0 - lane32 < L; l0 += 4 * (int64_t)B) {
                    if (l0 + 4 * (int64_t)B < L) load_px(l0 + 4 * (int64_t)B, pn4, xn4);
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int64_t li = l0 + q * B, i = R0 + li;
                        double pn = 0.0;
                        if (li < nr) {
                            const double rv = li < mu_cap ? MUs[li] : Rv[i];
                            X[i] = __fma_rn(alpha, pv[q], xv[q]);
                            pn = __fma_rn(beta, pv[q], rv);
                            P[pv_idx(i)] = pn;
                        }
                        if (DYN) {
                            const int lv = mfk::hw_min_level_full(li < nr ? mfk::level_of(pn, th) : 4);
                            if (li < L && (i & 15) == 0) mfk::pv_set_level(P, i >> 4, lv);
                        }
                    }
#pragma unroll
                    for (int q = 0; q < 4; ++q) { pv[q] = pn4[q]; xv[q] = xn4[q]; }
                }
            }
            publish<MG>(a, (unsigned)(j + 3), P);
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

// -------------------------------------------------------------------------- single-reduction CG
// the one-barrier variant of Alg. 1 (Chronopoulos & Gear; oracle
// orc_cg_single_reduction).  The SpMV input is r (PV layout, levels of r: "the input vector
// in SpMV"), w = A~ r; (r, r) is accumulated in the vector phase and (w, r) in the SpMV, and both go
// through ONE grid reduction per iteration.  p and s (= A~ p by recurrence) are plain vectors
// (a.rh, a.s).  Phases: 0 wait r, 1 SpMV + (w,r), 2 reduce, 3 vector update + (r,r) + publish, 6 init
template <bool DYN, bool COUNT, bool STK, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) cgsr_persistent(SolveArgs a) {
    constexpr int PF = MAXT >= 1024 ? 4 : 8;
    Smem sm = carve(a, 1);
    Ctx c;
    Timer tm;
    tm.start(sm.timer);
    const int t = threadIdx.x, B = blockDim.x;
    const unsigned m = mfk::hw_mask();
    const int64_t tr0 = a.plan_tr[blockIdx.x], tr1 = a.plan_tr[blockIdx.x + 1];
    const int64_t R0 = tr0 * 16, Rend = min(tr1 * 16, a.n);
    const int64_t n = a.n, nr = Rend - R0, nrp = (tr1 - tr0) * 16;
    const int mu_cap = a.mu_cap;
    double* __restrict__ X = a.x;
    double* RP = a.p;                 // r in the PV layout (the SpMV input)
    double* __restrict__ Pp = a.rh;   // p
    double* __restrict__ Ss = a.s;    // s
    double* __restrict__ Wg = a.mu_g;
    double* __restrict__ Ws = sm.mu;
    auto w_at = [&](int64_t li) -> double& { return li < mu_cap ? Ws[li] : Wg[R0 + li]; };

    double v2[2] = {0.0, 0.0};
    bool ok = stage_x0(a, RP, R0, Rend);
    mfk::spmv_cta<false, false, PF>(a.A, tr0, tr1, RP, 0, sm.sp, 0, nullptr,
                                    [&](int64_t TR, int ln, double ax, double) {
                                        const int64_t i = TR * 16 + ln;
                                        if (i < n) {
                                            const double bi = a.b[i];
                                            const double ri = __dsub_rn(bi, ax);
                                            a.r[i] = ri;
                                            v2[0] = __fma_rn(bi, bi, v2[0]);
                                            v2[1] = __fma_rn(ri, ri, v2[1]);
                                        }
                                    });
    ok = grid_reduce<2>(v2, a, c, sm.red) && ok;
    const double nb = sqrt(v2[0]);
    double gamma = v2[1], alpha = 0.0, beta = 0.0;
    int64_t j = 0;
    int converged = 0, status = ok ? MF_OK : MF_ERR_DEADLOCK;
    Thresh th{0, 0, 0, 0};
    if (ok && nb == 0.0) {
        for (int64_t i = R0 + t; i < Rend; i += B) X[i] = 0.0;
        converged = 1;
        if (blockIdx.x == 0 && t == 0 && a.hist_cap > 0) a.hist[0] = 0.0;
    } else if (ok) {
        th = make_thresh(a, sqrt(gamma));
        const double relres0 = __ddiv_rn(sqrt(gamma), nb);
        bool first = !(relres0 < a.tol) && a.max_iter > 0;
        if (first) {
            // r0 -> PV + levels; w0 = A~ r0 with the partial (w0, r0)
            for (int64_t li = t; li < nrp; li += B) {
                const int64_t i = R0 + li;
                const double rv = li < nr ? a.r[i] : 0.0;
                RP[pv_idx(i)] = rv;
                int lv = 0;
                if (DYN) lv = mfk::hw_min_i(li < nr ? mfk::level_of(rv, th) : 4, m);
                if ((i & 15) == 0) mfk::pv_set_level(RP, i >> 4, lv);
            }
            publish(a, 2);
            if (!wait_deps(a, 2)) status = MF_ERR_DEADLOCK;
            double d1[1] = {0.0};
            if (status == MF_OK) {
                mfk::spmv_cta<DYN, STK, PF>(a.A, tr0, tr1, RP, a.range_guard, sm.sp, 1, nullptr,
                                            [&](int64_t TR, int ln, double wv, double ov) {
                                                const int64_t i = TR * 16 + ln;
                                                if (i < n) { w_at(i - R0) = wv; d1[0] = __fma_rn(wv, ov, d1[0]); }
                                            });
                spmv_counts<COUNT, DYN>(a, c, tr0, tr1, RP, sm.ired);
                if (!grid_reduce<1>(d1, a, c, sm.red)) status = MF_ERR_DEADLOCK;
            }
            const double delta = d1[0];
            if (status == MF_OK && (!(delta > 0.0) || !isfinite(delta))) status = MF_ERR_BREAKDOWN;
            if (status == MF_OK) alpha = __ddiv_rn(gamma, delta);
            if (status != MF_OK && blockIdx.x == 0 && t == 0) {
                if (a.hist_cap > 0) a.hist[0] = relres0;
                a.out[2] = relres0;
            }
        }
        tm.tick(6);
        for (; status == MF_OK; ++j) {
            const double relres = __ddiv_rn(sqrt(gamma), nb);
            if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = relres; a.out[2] = relres; }
            if (relres < a.tol) { converged = 1; break; }
            if (j == a.max_iter) break;
            // p = r + beta p ; s = w + beta s ; x += alpha p ; r -= alpha s (own rows), r -> PV +
            // levels, partial (r, r)
            double v[2] = {0.0, 0.0};
            for (int64_t li = t; li < nrp; li += B) {
                const int64_t i = R0 + li;
                double rn = 0.0;
                if (li < nr) {
                    const double pi = __fma_rn(beta, Pp[i], RP[pv_idx(i)]);
                    const double si = __fma_rn(beta, Ss[i], w_at(li));
                    Pp[i] = pi;
                    Ss[i] = si;
                    X[i] = __fma_rn(alpha, pi, X[i]);
                    rn = __fma_rn(-alpha, si, RP[pv_idx(i)]);
                    RP[pv_idx(i)] = rn;
                    v[0] = __fma_rn(rn, rn, v[0]);
                }
                int lv = 0;
                if (DYN) lv = mfk::hw_min_i(li < nr ? mfk::level_of(rn, th) : 4, m);
                if ((i & 15) == 0) mfk::pv_set_level(RP, i >> 4, lv);
            }
            publish(a, (unsigned)(j + 3));
            tm.tick(3);
            if (!wait_deps(a, (unsigned)(j + 3))) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(0);
            mfk::spmv_cta<DYN, STK, PF>(a.A, tr0, tr1, RP, a.range_guard, sm.sp, 1, nullptr,
                                        [&](int64_t TR, int ln, double wv, double ov) {
                                            const int64_t i = TR * 16 + ln;
                                            if (i < n) { w_at(i - R0) = wv; v[1] = __fma_rn(wv, ov, v[1]); }
                                        });
            spmv_counts<COUNT, DYN>(a, c, tr0, tr1, RP, sm.ired);
            tm.tick(1);
            if (!grid_reduce<2>(v, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(2);
            const double gamma1 = v[0], delta1 = v[1];
            const double beta1 = __ddiv_rn(gamma1, gamma);
            const double tq = __ddiv_rn(__dmul_rn(beta1, gamma1), alpha);
            const double den = __dsub_rn(delta1, tq);
            if (!(den > 0.0) || !isfinite(den)) {
                ++j;
                const double rl = __ddiv_rn(sqrt(gamma1), nb);
                if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = rl; a.out[2] = rl; }
                if (rl < a.tol) converged = 1; else status = MF_ERR_BREAKDOWN;
                break;
            }
            alpha = __ddiv_rn(gamma1, den);
            beta = beta1;
            gamma = gamma1;
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
template <bool DYN, bool COUNT, bool STK, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) bicgstab_persistent(SolveArgs a) {
    constexpr int PF = MAXT >= 1024 ? 4 : 8;
    Smem sm = carve(a, 2);
    Ctx c;
    Timer tm;
    tm.start(sm.timer);
    const int t = threadIdx.x, B = blockDim.x;
    const unsigned m = mfk::hw_mask();
    const int64_t tr0 = a.plan_tr[blockIdx.x], tr1 = a.plan_tr[blockIdx.x + 1];
    const int64_t R0 = tr0 * 16, Rend = min(tr1 * 16, a.n);
    const int64_t n = a.n, nr = Rend - R0, nrp = (tr1 - tr0) * 16;
    const int mu_cap = a.mu_cap;
    double* __restrict__ X = a.x;
    double* __restrict__ Rv = a.r;
    double* P = a.p;       // PV
    double* S = a.s;       // PV
    const double* RH = a.rh;   // written at init in this kernel: no read-only (.nc) loads
    double* __restrict__ MUs = sm.mu;
    double* __restrict__ THs = sm.th;
    auto mu_at = [&](int64_t li) -> double& { return li < mu_cap ? MUs[li] : a.mu_g[R0 + li]; };
    auto th_at = [&](int64_t li) -> double& { return li < mu_cap ? THs[li] : a.th_g[R0 + li]; };

    // init: r = b - A~ x0; r0* = r; partial (b,b), (r,r), (r,r0*)
    double v3[3] = {0.0, 0.0, 0.0};
    bool ok = stage_x0(a, P, R0, Rend);
    mfk::spmv_cta<false, false, PF>(a.A, tr0, tr1, P, 0, sm.sp, 0, nullptr,
                                    [&](int64_t TR, int ln, double ax, double) {
                                        const int64_t i = TR * 16 + ln;
                                        if (i < n) {
                                            const double bi = a.b[i];
                                            const double ri = __dsub_rn(bi, ax);
                                            Rv[i] = ri; a.rh[i] = ri;
                                            v3[0] = __fma_rn(bi, bi, v3[0]);
                                            v3[1] = __fma_rn(ri, ri, v3[1]);
                                            v3[2] = __fma_rn(ri, ri, v3[2]);
                                        }
                                    });
    ok = grid_reduce<3>(v3, a, c, sm.red) && ok;
    const double nb = sqrt(v3[0]);
    double rr = v3[1], rho = v3[2];
    int64_t j = 0;
    int converged = 0, status = ok ? MF_OK : MF_ERR_DEADLOCK;
    unsigned epoch = 1;
    if (ok && nb == 0.0) {
        for (int64_t i = R0 + t; i < Rend; i += B) X[i] = 0.0;
        converged = 1;
        if (blockIdx.x == 0 && t == 0 && a.hist_cap > 0) a.hist[0] = 0.0;
    } else if (ok) {
        const Thresh th = make_thresh(a, sqrt(rr));
        for (int64_t li = t; li < nrp; li += B) {       // p0 = r0 (PV) + levels
            const int64_t i = R0 + li;
            const double pv = li < nr ? Rv[i] : 0.0;
            P[pv_idx(i)] = pv;
            int lv = 0;
            if (DYN) lv = mfk::hw_min_i(li < nr ? mfk::level_of(pv, th) : 4, m);
            if ((i & 15) == 0) mfk::pv_set_level(P, i >> 4, lv);
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
            mfk::spmv_cta<DYN, STK, PF>(a.A, tr0, tr1, P, a.range_guard, sm.sp, 2, RH,
                                        [&](int64_t TR, int ln, double mv, double ov) {
                                            const int64_t i = TR * 16 + ln;
                                            if (i < n) { mu_at(i - R0) = mv; eta[0] = __fma_rn(mv, ov, eta[0]); }
                                        });
            spmv_counts<COUNT, DYN>(a, c, tr0, tr1, P, sm.ired);
            tm.tick(1);
            if (!grid_reduce<1>(eta, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(2);
            if (eta[0] == 0.0 || !isfinite(eta[0])) { status = MF_ERR_BREAKDOWN; break; }
            const double alpha = __ddiv_rn(rho, eta[0]);
            // s = r - alpha mu (own rows, PV) + levels of s: 4 rows per thread with their loads
            // issued first, a warp-uniform trip count and full-warp level reductions
            for (int64_t l0 = t; l0 - (t & 31) < nrp; l0 += 4 * (int64_t)B) {
                double rv4[4], mv4[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t li = l0 + q * B;
                    rv4[q] = li < nr ? Rv[R0 + li] : 0.0;
                    mv4[q] = li < nr ? mu_at(li) : 0.0;
                }
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t li = l0 + q * B, i = R0 + li;
                    double si = 0.0;
                    if (li < nr) { si = __fma_rn(-alpha, mv4[q], rv4[q]); S[pv_idx(i)] = si; }
                    int lv = 0;
                    if (DYN) lv = mfk::hw_min_level_full(li < nr ? mfk::level_of(si, th) : 4);
                    if (li < nrp && (i & 15) == 0) mfk::pv_set_level(S, i >> 4, lv);
                }
            }
            publish(a, ++epoch);
            tm.tick(3);
            if (!wait_deps(a, epoch)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(4);
            // theta = A~ s ; partial (theta, theta), (theta, s)
            double tt[2] = {0.0, 0.0};
            mfk::spmv_cta<DYN, STK, PF>(a.A, tr0, tr1, S, a.range_guard, sm.sp, 1, nullptr,
                                        [&](int64_t TR, int ln, double tv, double ov) {
                                            const int64_t i = TR * 16 + ln;
                                            if (i < n) {
                                                th_at(i - R0) = tv;
                                                tt[0] = __fma_rn(tv, tv, tt[0]);
                                                tt[1] = __fma_rn(tv, ov, tt[1]);
                                            }
                                        });
            spmv_counts<COUNT, DYN>(a, c, tr0, tr1, S, sm.ired);
            tm.tick(5);
            if (!grid_reduce<2>(tt, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(6);
            if (tt[0] == 0.0) {
                // theta == 0: take the half step x += alpha p, r = s, and stop (reading R14)
                double r2[1] = {0.0};
                for (int64_t li = t; li < nr; li += B) {
                    const int64_t i = R0 + li;
                    X[i] = __fma_rn(alpha, P[pv_idx(i)], X[i]);
                    const double si = S[pv_idx(i)];
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
            for (int64_t l0 = t; l0 < nr; l0 += 4 * (int64_t)B) {
                double sv[4], pv[4], xv[4], tv[4], hv[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t li = l0 + q * B;
                    if (li < nr) {
                        const int64_t i = R0 + li;
                        sv[q] = S[pv_idx(i)]; pv[q] = P[pv_idx(i)]; xv[q] = X[i]; hv[q] = RH[i];
                        tv[q] = th_at(li);
                    }
                }
#pragma unroll
                for (int q = 0; q < 4; ++q) {
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
            // p = r + beta (p - omega mu) (own rows, PV) + levels of p (as the s update)
            for (int64_t l0 = t; l0 - (t & 31) < nrp; l0 += 4 * (int64_t)B) {
                double pv4[4], mv4[4], rv4[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t li = l0 + q * B, i = R0 + li;
                    pv4[q] = li < nr ? P[pv_idx(i)] : 0.0;
                    mv4[q] = li < nr ? mu_at(li) : 0.0;
                    rv4[q] = li < nr ? Rv[i] : 0.0;
                }
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int64_t li = l0 + q * B, i = R0 + li;
                    double pn = 0.0;
                    if (li < nr) { pn = __fma_rn(beta, __fma_rn(-omega, mv4[q], pv4[q]), rv4[q]); P[pv_idx(i)] = pn; }
                    int lv = 0;
                    if (DYN) lv = mfk::hw_min_level_full(li < nr ? mfk::level_of(pn, th) : 4);
                    if (li < nrp && (i & 15) == 0) mfk::pv_set_level(P, i >> 4, lv);
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

// Recursive block SpTRSV inside the persistent kernel: the node sequence of the
// precond.cuh trees in place on py (in copied to py first, py copied to out at the end); a leaf is
// the sync-free chunked solve of its rows (all CTAs grab chunks), a square block is spread over
// all CTAs' threads (one thread per row); a grid barrier separates consecutive nodes.
template <bool OUTPV>
__device__ __noinline__ bool precond_apply_rb(const SolveArgs& a, PcState& ps, const Smem& sm, Ctx& c, const double* in,
                                              double* out, int64_t R0, int64_t Rend) {
    const unsigned e = a.pe0 + ps.apply++;
    const unsigned vf = 2 * e + 1, vb = 2 * e + 2;
    const int B = blockDim.x;
    for (int64_t i = R0 + threadIdx.x; i < Rend; i += B) a.py[i] = in[i];
    bool ok = grid_barrier(a, c);
    for (int pass = 0; pass < 2 && ok; ++pass) {
        const RbNode* nodes = pass == 0 ? a.Lnodes : a.Unodes;
        const int nn = pass == 0 ? a.nLn : a.nUn;
        const int64_t* brp = pass == 0 ? a.Lbrp : a.Ubrp;
        const int32_t* bci = pass == 0 ? a.Lbci : a.Ubci;
        const double* bv = pass == 0 ? a.Lbv : a.Ubv;
        for (int k = 0; k < nn && ok; ++k) {
            const RbNode nd = nodes[k];
            const int64_t m = nd.r1 - nd.r0;
            if (nd.leaf && a.psweep) {
                if (blockIdx.x == 0) {
                    const bool sok = pass == 0
                        ? mfk::sweep_solve<true, false>(brp + nd.rp_off, bci, bv, nullptr, m, a.py + nd.r0, a.py + nd.r0,
                                                         sm.sweep, a.abort_flag, a.timeout_ns)
                        : mfk::sweep_solve<false, false>(brp + nd.rp_off, bci, bv, a.Ud + nd.r0, m, a.py + nd.r0,
                                                          a.py + nd.r0, sm.sweep, a.abort_flag, a.timeout_ns);
                    if (!sok && threadIdx.x == 0) atomicExch(a.abort_flag, 1);
                }
            } else if (nd.leaf) {
                const int64_t nch = (m + B - 1) / B;
                if (pass == 0) {
                    mfk::sptrsv_chunked<true, false>(brp + nd.rp_off, bci, bv, nullptr, m, a.py + nd.r0, a.py + nd.r0,
                                                     a.pflags + nd.r0, vf, 0u, a.pctr, ps.base_f, sm.tys, sm.tready, sm.tchunk,
                                                     a.abort_flag, a.timeout_ns);
                    ps.base_f += (unsigned long long)(nch + a.G);
                } else {
                    mfk::sptrsv_chunked<false, false>(brp + nd.rp_off, bci, bv, a.Ud + nd.r0, m, a.py + nd.r0, a.py + nd.r0,
                                                      a.pflags + nd.r0, vb, 0u, a.pctr + 1, ps.base_b, sm.tys, sm.tready,
                                                      sm.tchunk, a.abort_flag, a.timeout_ns);
                    ps.base_b += (unsigned long long)(nch + a.G);
                }
            } else {
                mfk::rb_square_rows(brp + nd.rp_off, bci, bv, nd.r0, nd.r1, a.py, (int64_t)blockIdx.x * B + threadIdx.x,
                                    (int64_t)a.G * B);
            }
            __threadfence();
            ok = grid_barrier(a, c) && *(volatile int*)a.abort_flag == 0;
        }
    }
    for (int64_t i = R0 + threadIdx.x; i < Rend; i += B) out[OUTPV ? pv_idx(i) : i] = __ldcg(a.py + i);
    __syncthreads();
    return ok;
}

template <bool OUTPV>
__device__ __forceinline__ bool precond_apply(const SolveArgs& a, PcState& ps, const Smem& sm, Ctx& c, const double* in,
                                              double* out, int64_t R0, int64_t Rend) {
    if (a.rb) return precond_apply_rb<OUTPV>(a, ps, sm, c, in, out, R0, Rend);
    if (a.psweep) {
        // one CTA sweeps L then U (the other CTAs wait in the grid barrier)
        ps.apply++;
        if (blockIdx.x == 0) {
            bool sok = mfk::sweep_solve<true, false>(a.Lrp, a.Lci, a.Lv, nullptr, a.n, in, a.py, sm.sweep, a.abort_flag,
                                                     a.timeout_ns);
            __syncthreads();
            if (sok)
                sok = mfk::sweep_solve<false, OUTPV>(a.Urp, a.Uci, a.Uv, a.Ud, a.n, a.py, out, sm.sweep, a.abort_flag,
                                                     a.timeout_ns);
            if (!sok && threadIdx.x == 0) atomicExch(a.abort_flag, 1);
        }
        __threadfence();
        return grid_barrier(a, c) && *(volatile int*)a.abort_flag == 0;
    }
    const unsigned e = a.pe0 + ps.apply++;
    const unsigned vf = 2 * e + 1, vb = 2 * e + 2;
    const int64_t nch = (a.n + blockDim.x - 1) / blockDim.x;
    mfk::sptrsv_chunked<true, false>(a.Lrp, a.Lci, a.Lv, nullptr, a.n, in, a.py, a.pflags, vf, 0u, a.pctr, ps.base_f,
                                     sm.tys, sm.tready, sm.tchunk, a.abort_flag, a.timeout_ns);
    ps.base_f += (unsigned long long)(nch + a.G);
    mfk::sptrsv_chunked<false, OUTPV>(a.Urp, a.Uci, a.Uv, a.Ud, a.n, a.py, out, a.pflags, vb, vf, a.pctr + 1, ps.base_b,
                                      sm.tys, sm.tready, sm.tchunk, a.abort_flag, a.timeout_ns);
    ps.base_b += (unsigned long long)(nch + a.G);
    const unsigned long long t0 = gtimer();
    for (int64_t i = R0 + threadIdx.x; i < Rend; i += blockDim.x)
        mfk::sp_wait_flag(&a.pflags[i], vb, a.abort_flag, t0, a.timeout_ns);
    __threadfence();
    __syncthreads();
    return *(volatile int*)a.abort_flag == 0;
}

// PCG (SURVEY c-6): z = M^-1 r, rho = (r,z), p = z + beta p; stop on ||r||/||b||.
// Phases: 0 wait p, 1 SpMV, 2 reduce sigma, 3 x/r update, 4 reduce rr, 5 M^-1 r, 6 reduce rho,
//         7 p update + publish, 10 init
template <bool DYN, bool COUNT, bool STK, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) pcg_persistent(SolveArgs a) {
    constexpr int PF = MAXT >= 1024 ? 4 : 8;
    Smem sm = carve(a, 1);
    Ctx c;
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
    double* P = a.p;    // PV
    double* Z = a.pz;
    double* __restrict__ MUs = sm.mu;

    double v2[2] = {0.0, 0.0};
    bool ok = stage_x0(a, P, R0, Rend);
    mfk::spmv_cta<false, false, PF>(a.A, tr0, tr1, P, 0, sm.sp, 0, nullptr,
                                    [&](int64_t TR, int ln, double ax, double) {
                                        const int64_t i = TR * 16 + ln;
                                        if (i < n) {
                                            const double bi = a.b[i];
                                            const double ri = __dsub_rn(bi, ax);
                                            Rv[i] = ri;
                                            v2[0] = __fma_rn(bi, bi, v2[0]);
                                            v2[1] = __fma_rn(ri, ri, v2[1]);
                                        }
                                    });
    ok = grid_reduce<2>(v2, a, c, sm.red) && ok;   // also: r complete on every CTA
    const double nb = sqrt(v2[0]);
    double rr = v2[1], rho = 0.0;
    int64_t j = 0;
    int converged = 0, status = ok ? MF_OK : MF_ERR_DEADLOCK;
    if (ok && nb == 0.0) {
        for (int64_t i = R0 + t; i < Rend; i += B) X[i] = 0.0;
        converged = 1;
        if (blockIdx.x == 0 && t == 0 && a.hist_cap > 0) a.hist[0] = 0.0;
    } else if (ok) {
        if (!precond_apply<false>(a, pcs, sm, c, Rv, Z, R0, Rend)) status = MF_ERR_DEADLOCK;
        double v3[2] = {0.0, 0.0};
        for (int64_t li = t; li < nr; li += B) {
            const int64_t i = R0 + li;
            const double zi = Z[i];
            P[pv_idx(i)] = zi;
            v3[0] = __fma_rn(Rv[i], zi, v3[0]);
            v3[1] = __fma_rn(zi, zi, v3[1]);
        }
        if (status == MF_OK && !grid_reduce<2>(v3, a, c, sm.red)) status = MF_ERR_DEADLOCK;
        rho = v3[0];
        const Thresh th = make_thresh(a, sqrt(v3[1]));
        __syncthreads();
        pv_levels<DYN>(a, P, tr0, tr1, th);
        publish(a, 2);
        tm.tick(10);
        for (; status == MF_OK; ++j) {
            const double relres = __ddiv_rn(sqrt(rr), nb);
            if (blockIdx.x == 0 && t == 0) { if (j < a.hist_cap) a.hist[j] = relres; a.out[2] = relres; }
            if (relres < a.tol) { converged = 1; break; }
            if (j == a.max_iter) break;
            if (!wait_deps(a, (unsigned)(j + 2))) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(0);
            double sg[1] = {0.0};
            mfk::spmv_cta<DYN, STK, PF>(a.A, tr0, tr1, P, a.range_guard, sm.sp, 1, nullptr,
                                        [&](int64_t TR, int ln, double mv, double ov) {
                                            const int64_t i = TR * 16 + ln;
                                            if (i < n) {
                                                const int64_t li = i - R0;
                                                if (li < mu_cap) MUs[li] = mv; else a.mu_g[i] = mv;
                                                sg[0] = __fma_rn(mv, ov, sg[0]);
                                            }
                                        });
            spmv_counts<COUNT, DYN>(a, c, tr0, tr1, P, sm.ired);
            tm.tick(1);
            if (!grid_reduce<1>(sg, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(2);
            const double sigma = sg[0];
            if (!(sigma > 0.0) || !isfinite(sigma)) { status = MF_ERR_BREAKDOWN; break; }
            const double alpha = __ddiv_rn(rho, sigma);
            double r1[1] = {0.0};
            for (int64_t li = t; li < nr; li += B) {
                const int64_t i = R0 + li;
                X[i] = __fma_rn(alpha, P[pv_idx(i)], X[i]);
                const double ri = __fma_rn(-alpha, li < mu_cap ? MUs[li] : a.mu_g[i], Rv[i]);
                Rv[i] = ri;
                r1[0] = __fma_rn(ri, ri, r1[0]);
            }
            tm.tick(3);
            if (!grid_reduce<1>(r1, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }   // r complete too
            rr = r1[0];
            tm.tick(4);
            if (!precond_apply<false>(a, pcs, sm, c, Rv, Z, R0, Rend)) { status = MF_ERR_DEADLOCK; break; }
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
                P[pv_idx(i)] = __fma_rn(beta, P[pv_idx(i)], Z[i]);
            }
            __syncthreads();
            pv_levels<DYN>(a, P, tr0, tr1, th);
            publish(a, (unsigned)(j + 3));
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
// p and s are plain vectors here; the SpMV inputs p^ and s^ are written in the PV layout by the
// backward triangular solve.
// Phases: 0 M^-1 p + levels, 1 SpMV mu, 2 reduce eta, 3 s update + barrier, 4 M^-1 s + levels,
//         5 SpMV theta, 6 reduce tt, 7 x/r update + reduce, 8 p update + barrier, 10 init
template <bool DYN, bool COUNT, bool STK, int MAXT>
__global__ void __launch_bounds__(MAXT, 1) pbicgstab_persistent(SolveArgs a) {
    constexpr int PF = MAXT >= 1024 ? 4 : 8;
    Smem sm = carve(a, 2);
    Ctx c;
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
    double* __restrict__ P = a.p;    // normal
    double* __restrict__ S = a.s;    // normal
    double* PH = a.pz;               // PV
    double* SH = a.ps;               // PV
    const double* RH = a.rh;   // written at init in this kernel: no read-only (.nc) loads
    double* __restrict__ MUs = sm.mu;
    double* __restrict__ THs = sm.th;
    auto mu_at = [&](int64_t li) -> double& { return li < mu_cap ? MUs[li] : a.mu_g[R0 + li]; };
    auto th_at = [&](int64_t li) -> double& { return li < mu_cap ? THs[li] : a.th_g[R0 + li]; };

    double v3[3] = {0.0, 0.0, 0.0};
    bool ok = stage_x0(a, PH, R0, Rend);
    mfk::spmv_cta<false, false, PF>(a.A, tr0, tr1, PH, 0, sm.sp, 0, nullptr,
                                    [&](int64_t TR, int ln, double ax, double) {
                                        const int64_t i = TR * 16 + ln;
                                        if (i < n) {
                                            const double bi = a.b[i];
                                            const double ri = __dsub_rn(bi, ax);
                                            Rv[i] = ri; a.rh[i] = ri; P[i] = ri;
                                            v3[0] = __fma_rn(bi, bi, v3[0]);
                                            v3[1] = __fma_rn(ri, ri, v3[1]);
                                            v3[2] = __fma_rn(ri, ri, v3[2]);
                                        }
                                    });
    ok = grid_reduce<3>(v3, a, c, sm.red) && ok;
    const double nb = sqrt(v3[0]);
    double rr = v3[1], rho = v3[2];
    int64_t j = 0;
    int converged = 0, status = ok ? MF_OK : MF_ERR_DEADLOCK;
    unsigned epoch = 1;
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
            if (!precond_apply<true>(a, pcs, sm, c, P, PH, R0, Rend)) { status = MF_ERR_DEADLOCK; break; }
            if (j == 0) {          // tau from ||p^_0|| (the first SpMV input)
                double pp[1] = {0.0};
                for (int64_t li = t; li < nr; li += B) { const double v = PH[pv_idx(R0 + li)]; pp[0] = __fma_rn(v, v, pp[0]); }
                if (!grid_reduce<1>(pp, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
                th = make_thresh(a, sqrt(pp[0]));
            }
            pv_levels<DYN>(a, PH, tr0, tr1, th);
            publish(a, ++epoch);
            if (!wait_deps(a, epoch)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(0);
            double eta[1] = {0.0};
            mfk::spmv_cta<DYN, STK, PF>(a.A, tr0, tr1, PH, a.range_guard, sm.sp, 2, RH,
                                        [&](int64_t TR, int ln, double mv, double ov) {
                                            const int64_t i = TR * 16 + ln;
                                            if (i < n) { mu_at(i - R0) = mv; eta[0] = __fma_rn(mv, ov, eta[0]); }
                                        });
            spmv_counts<COUNT, DYN>(a, c, tr0, tr1, PH, sm.ired);
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
            if (!precond_apply<true>(a, pcs, sm, c, S, SH, R0, Rend)) { status = MF_ERR_DEADLOCK; break; }
            pv_levels<DYN>(a, SH, tr0, tr1, th);
            publish(a, ++epoch);
            if (!wait_deps(a, epoch)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(4);
            double tt[2] = {0.0, 0.0};
            mfk::spmv_cta<DYN, STK, PF>(a.A, tr0, tr1, SH, a.range_guard, sm.sp, 2, S,
                                        [&](int64_t TR, int ln, double tv, double ov) {
                                            const int64_t i = TR * 16 + ln;
                                            if (i < n) {
                                                th_at(i - R0) = tv;
                                                tt[0] = __fma_rn(tv, tv, tt[0]);
                                                tt[1] = __fma_rn(tv, ov, tt[1]);
                                            }
                                        });
            spmv_counts<COUNT, DYN>(a, c, tr0, tr1, SH, sm.ired);
            tm.tick(5);
            if (!grid_reduce<2>(tt, a, c, sm.red)) { status = MF_ERR_DEADLOCK; break; }
            tm.tick(6);
            if (tt[0] == 0.0) {
                double r2[1] = {0.0};
                for (int64_t li = t; li < nr; li += B) {
                    const int64_t i = R0 + li;
                    X[i] = __fma_rn(alpha, PH[pv_idx(i)], X[i]);
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
                X[i] = __fma_rn(omega, SH[pv_idx(i)], __fma_rn(alpha, PH[pv_idx(i)], X[i]));
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

}  // namespace

// kernel selection, one translation unit per (solver, block-size bound) for parallel builds
// (solver_inst_*.cu): returns the __global__ function for the template flags
#define MF_DECLARE_PICK(NAME) void* NAME(bool dyn, bool count, bool sticky)
MF_DECLARE_PICK(pick_cg_512);
MF_DECLARE_PICK(pick_cg_1024);
MF_DECLARE_PICK(pick_bicgstab_512);
MF_DECLARE_PICK(pick_bicgstab_1024);
MF_DECLARE_PICK(pick_pcg_512);
MF_DECLARE_PICK(pick_pcg_1024);
MF_DECLARE_PICK(pick_pbicgstab_512);
MF_DECLARE_PICK(pick_pbicgstab_1024);
MF_DECLARE_PICK(pick_cgsr_512);
MF_DECLARE_PICK(pick_cgsr_1024);
// device-initiated multi-GPU CG (SolveArgs::mg set): no statistics, no sticky variant
void* pick_cgmg(int maxt, bool dyn);

#define MF_DEFINE_PICK(NAME, KERNEL, MAXT)                                                        \
    void* NAME(bool dyn, bool count, bool sticky) {                                               \
        if (dyn && sticky) return (void*)KERNEL<true, false, true, MAXT>;                         \
        if (dyn) return count ? (void*)KERNEL<true, true, false, MAXT> : (void*)KERNEL<true, false, false, MAXT>; \
        return count ? (void*)KERNEL<false, true, false, MAXT> : (void*)KERNEL<false, false, false, MAXT>;      \
    }

}  // namespace mf
