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
    int sweep = 0;                // 1: triangular solves (or rb leaves) by the one-CTA sweep (deep DAGs)
    int64_t depth_l = 0, depth_u = 0;   // levels of the L / U dependency DAGs
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
//   FWD:  out_i = in_i - sum_{k<i} T_ik out_k                 rows ascending, k ascending
//   !FWD: out_i = (in_i - sum_{k>i} T_ik out_k) / diag_i       rows descending, k descending
// (each fma chain in the order the substitution produces the unknowns, reading R20)
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
            // chain in solve order of the columns: forward ascending, backward descending (R20)
            for (int64_t qq = lo; qq < hi; ++qq) {
                const int64_t q = FWD ? qq : lo + hi - 1 - qq;
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

// ------------------------------------------------------------------------------------------
// Sweep triangular solve: ONE CTA (its first SW_WARPS warps), for factors whose dependency DAG is
// too deep for grid-wide parallelism (C4: 2^20 rows, 2.8e5 levels, ~4 rows per level -- a grid
// barrier or a cross-SM flag per level would cost microseconds per level).  Same arithmetic as
// sptrsv_chunked (and the oracle): position p in solve order is row i = FWD ? p : n-1-p; row i's
// chain runs over its entries in solve order of their columns; !FWD divides by diag_i last.
//
// Windows of 32 consecutive positions; warp w takes windows w, w + SW_WARPS, ...; lane l owns
// position 32*win + l.  Per window: (1) the warp stages the window's CSR range (contiguous: the
// rows of a window are consecutive) in its shared-memory buffer with coalesced loads; (2) entries
// whose column lies in an earlier window are consumed in chain order, the warp waiting (warp-
// uniform) until the window holding the column is complete -- most of this overlaps the previous
// window's sweep; (3) the in-window sweep: step s finalises lane s (all its remaining entries have
// earlier in-window positions, consumed at earlier steps) and broadcasts the value by shuffle to the
// lanes whose next entry is position 32*win + s.  Values of recent windows are kept in a shared
// ring; older ones are read back from `out`.  `done` counts completed windows (in order).
constexpr int SW_WARPS = 8;
constexpr int SW_CAP = 768;        // staged entries per warp and window (larger windows read global)
constexpr int SW_RING = 2048;      // recent solution values kept in shared memory (positions)
__host__ __device__ constexpr size_t sweep_smem_bytes() {
    return (size_t)SW_WARPS * SW_CAP * (8 + 4) + (size_t)SW_RING * 8 + 64;
}
__device__ __forceinline__ unsigned smem_u32_(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
// spin back-off of the waiting warps (ns, 0 = none): tuning knob of the standalone apply
static __device__ int g_sweep_sleep_ns = 0;
// diagnostics (standalone apply, MF_SWEEP_DBG): per window clock64 at sweep start / end / signal
static __device__ long long* g_sweep_dbg = nullptr;
template <bool FWD, bool OUTPV>
__device__ __noinline__ bool sweep_solve(const int64_t* __restrict__ rp, const int32_t* __restrict__ ci,
                                         const double* __restrict__ val, const double* __restrict__ diag, int64_t n,
                                         const double* in, double* out, unsigned char* smem, int* abort_flag,
                                         unsigned long long timeout_ns) {
    const int t = threadIdx.x, w = t >> 5, lane = t & 31;
    double* ring = reinterpret_cast<double*>(smem);
    double* sval = ring + SW_RING;
    int32_t* sci = reinterpret_cast<int32_t*>(sval + (size_t)SW_WARPS * SW_CAP);
    volatile int* done = reinterpret_cast<volatile int*>(sci + (size_t)SW_WARPS * SW_CAP);
    auto oidx = [](int64_t i) -> int64_t { return OUTPV ? ((i >> 4) * 18 + (i & 15)) : i; };
    if (t == 0) { done[0] = 0; done[1] = 0; }
    __syncthreads();
    const int NWS = min(SW_WARPS, (int)(blockDim.x >> 5));   // sweeping warps
    if (w >= NWS) return true;
    double* wv = sval + (size_t)w * SW_CAP;
    int32_t* wc = sci + (size_t)w * SW_CAP;
    const int64_t nwin = (n + 31) >> 5;
    const unsigned long long t0 = sp_timer();
    const unsigned FULL = 0xffffffffu;
    bool ok = true;
    int seen = 0;                      // windows known complete (this warp's last observation)
    // spin (warp-uniform) until at least `need` windows are complete; one CTA-scope acquire fence
    auto wait_done = [&](int64_t need) {
        if (seen >= need) return;
        int d = done[0];
        const int slp = g_sweep_sleep_ns;
        for (unsigned sp = 0; d < need; ++sp, d = done[0]) {
            if (slp) __nanosleep(slp);
            if ((sp & 1023u) == 1023u && (*(volatile int*)abort_flag || sp_timer() - t0 > timeout_ns)) {
                atomicExch(abort_flag, 1);
                ok = false;
                done[1] = 1;
                break;
            }
        }
        seen = __shfl_sync(FULL, d, 0);
        __threadfence_block();
    };
    for (int64_t win = w; win < nwin && ok && !done[1]; win += NWS) {
        const int64_t p0 = win << 5, p = p0 + lane;
        const bool valid = p < n;
        const int64_t i = FWD ? p : n - 1 - p;
        const int64_t lo = valid ? rp[i] : 0, hi = valid ? rp[i + 1] : 0;
        // (1) stage the window's CSR range (rows p0 .. p0+31 in solve order are consecutive rows)
        // with asynchronous global->shared copies (all in flight at once: one memory latency);
        // the right-hand side and the diagonal are loaded alongside
        const int64_t plast = min(p0 + 31, n - 1);
        const int64_t e0 = FWD ? rp[p0] : rp[n - 1 - plast];
        const int64_t e1 = FWD ? rp[plast + 1] : rp[n - p0];
        const double dg = (!FWD && valid) ? diag[i] : 1.0;
        double acc = valid ? __ldcg(in + i) : 0.0;
        const int ne = (int)(e1 - e0);
        const bool staged = ne <= SW_CAP;
        if (staged) {
            for (int j = lane; j < ne; j += 32) {
                asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32_(wc + j)), "l"(ci + e0 + j) : "memory");
                asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32_(wv + j)), "l"(val + e0 + j) : "memory");
            }
            asm volatile("cp.async.wait_all;" ::: "memory");
        }
        __syncwarp();
        const int cnt = (int)(hi - lo);
        int k = 0;
        int64_t pc = INT64_MAX;      // position (solve order) of the current entry's column
        double v = 0.0;
        int32_t col = 0;
        auto load_entry = [&]() {
            if (k < cnt) {
                const int64_t q = FWD ? lo + k : hi - 1 - k;
                col = staged ? wc[q - e0] : __ldg(ci + q);
                v = staged ? wv[q - e0] : __ldg(val + q);
                pc = FWD ? (int64_t)col : n - 1 - col;
            } else {
                pc = INT64_MAX;
            }
        };
        load_entry();
        // the chain's tail (computed before any wait): entries in this window (bit s of hm =
        // position p0 + s, from index kb) and in the previous window (bit s of pm = position
        // p0 - 32 + s, from index kp); the older entries precede them in chain order
        unsigned hm = 0, pm = 0;
        int kb = cnt, kp = cnt;
        for (int kk = cnt - 1; kk >= k; --kk) {
            const int64_t q = FWD ? lo + kk : hi - 1 - kk;
            const int32_t cc = staged ? wc[q - e0] : __ldg(ci + q);
            const int64_t pcc = FWD ? (int64_t)cc : n - 1 - cc;
            if (pcc >= p0) { hm |= 1u << (int)(pcc - p0); kb = kk; kp = kk; }
            else if (pcc >= p0 - 32) { pm |= 1u << (int)(pcc - (p0 - 32)); kp = kk; }
            else break;
        }
        const double yr = FWD ? 1.0 : __drcp_rn(dg);
        const bool dg_ok = FWD || (fabs(dg) >= 0x1p-960 && fabs(dg) <= 0x1p960);
        // (2a) entries older than the ring: their windows completed before any window in flight
        // started (ring distance > windows in flight), values from `out`
        const int64_t ring_lo = p0 - SW_RING + (int64_t)NWS * 32;
        if (__any_sync(FULL, pc < ring_lo)) {
            // the writer of a column stores `out` after its signal; its next window's fence (NWS
            // windows later) publishes it
            wait_done(max((int64_t)0, (ring_lo >> 5) + NWS));
            while (pc < ring_lo) {
                acc = __fma_rn(-v, __ldcg(out + oidx(col)), acc);
                ++k;
                load_entry();
            }
        }
        // (2b) entries in earlier windows inside the ring.  First every entry of a window already
        // complete (one read of the counter), in batches of 4 whose loads are all in flight
        // together (the fma chain is the only serial part); then the windows still in flight one
        // by one (a warp-uniform wait each); the previous window last, after its own wait.
        const int64_t pprev = p0 - 32;            // the previous window is handled after its wait
        if (staged) {
            const int dn = done[0];
            __threadfence_block();
            const int64_t lim = min((int64_t)dn, win - 1) << 5;
            while (__any_sync(FULL, pc < lim)) {
                double yv[4], vv[4];
                bool use[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int idx = k + u;
                    const int64_t q = FWD ? lo + idx : hi - 1 - idx;
                    const int qi = idx < cnt ? (int)(q - e0) : 0;
                    const int32_t cc = wc[qi];
                    const int64_t pcu = FWD ? (int64_t)cc : n - 1 - cc;
                    use[u] = idx < cnt && pcu < lim;
                    yv[u] = ring[use[u] ? (int)(pcu & (SW_RING - 1)) : 0];
                    vv[u] = wv[qi];
                }
                int used = 0;
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const bool go = use[u] && used == u;        // positions ascend: a prefix is used
                    const double na = __fma_rn(-vv[u], yv[u], acc);
                    acc = go ? na : acc;
                    used += go ? 1 : 0;
                }
                k += used;
                load_entry();
            }
        }
        int64_t nextw = pc < pprev ? (pc >> 5) : win;
        for (int o = 16; o >= 1; o >>= 1) nextw = min(nextw, (int64_t)__shfl_xor_sync(FULL, (long long)nextw, o));
        while (nextw < win - 1) {
            wait_done(nextw + 1);
            if (!ok) break;
            const int64_t wend = (nextw + 1) << 5;
            while (pc < wend) {
                acc = __fma_rn(-v, ring[pc & (SW_RING - 1)], acc);
                ++k;
                load_entry();
            }
            nextw = pc < pprev ? (pc >> 5) : win;
            for (int o = 16; o >= 1; o >>= 1) nextw = min(nextw, (int64_t)__shfl_xor_sync(FULL, (long long)nextw, o));
        }
        if (!ok) break;
        // previous window: positions known in advance (pm).  The first SW_PK entries' values and
        // ring slots are gathered into registers BEFORE the wait; after it, their ring values are
        // read together and the fma chain runs without per-entry address work; more entries (rare)
        // continue in a loop.
        constexpr int SW_PK = 8;
        double pvv[SW_PK];
        int pslot[SW_PK];
        unsigned mm = pm;
        const int npk = min(__popc(pm), SW_PK);
        const int wpk = __reduce_max_sync(FULL, (unsigned)npk);     // the warp's longest preloaded chain
#pragma unroll
        for (int u = 0; u < SW_PK; ++u) {
            const int sb = mm ? __ffs(mm) - 1 : 0;
            if (mm) mm &= mm - 1u;
            const int64_t q = FWD ? lo + kp + u : hi - 1 - (kp + u);
            pvv[u] = u < npk ? (staged ? wv[q - e0] : __ldg(val + q)) : 0.0;
            pslot[u] = (int)((pprev + sb) & (SW_RING - 1));
        }
        long long* dbg = g_sweep_dbg;
        if (dbg && lane == 0) dbg[win * 5] = clock64();
        if (win > 0) wait_done(win);
        if (!ok) break;
        if (dbg && lane == 0) dbg[win * 5 + 1] = clock64();
        {
            double ry[SW_PK];
#pragma unroll
            for (int u = 0; u < SW_PK; ++u) ry[u] = ring[pslot[u]];     // valid slots for every lane
#pragma unroll
            for (int u = 0; u < SW_PK; ++u) {
                if (u >= wpk) break;                                  // warp-uniform
                const double na = __fma_rn(-pvv[u], ry[u], acc);
                acc = u < npk ? na : acc;
            }
            int kk = kp + npk;
            while (mm) {                                              // entries beyond SW_PK
                const int sb = __ffs(mm) - 1;
                mm &= mm - 1u;
                const int64_t q = FWD ? lo + kk : hi - 1 - kk;
                const double vv = staged ? wv[q - e0] : __ldg(val + q);
                acc = __fma_rn(-vv, ring[(pprev + sb) & (SW_RING - 1)], acc);
                ++kk;
            }
            k = kb;
        }
        // (3) in-window sweep: the lane's remaining entries are in the window, ascending; hm has
        // bit s for an entry at position p0 + s, its value is entry kb + popc(hm below s).  Step s
        // broadcasts lane s's final value (all its entries precede position p0 + s); every step is
        // branch-free: a predicated fma, then the lane's value refreshed.  !FWD: the quotient by
        // diag_i with Markstein's correction of a*RN(1/d) (correctly rounded: RN(1/d) and a one-ulp
        // q0 give RN(a/d) for normal operands), IEEE division for zero or extreme operands.
        if (dbg && lane == 0) dbg[win * 5 + 2] = clock64();
        const double acc0 = acc;
        double fin = 0.0;
        bool slow = !staged;
        if (staged) {
            // fast path: every step branch-free (the value load uses a valid shared address for
            // every lane, masked afterwards), Markstein quotient; any lane with an operand outside
            // its validity range sends the whole window to the exact path below
            const int vb0 = FWD ? (int)(lo - e0) + kb : (int)(hi - 1 - e0) - kb;   // staged index of entry kb
            bool bad = false;
            auto mark = [&](double a) -> double {
                const double q0 = __dmul_rn(a, yr);
                const double q1 = __fma_rn(__fma_rn(-q0, dg, a), yr, q0);
                const double aq = fabs(q1);
                bad |= a == 0.0 || !(aq >= 0x1p-960 && aq <= 0x1p960);
                return q1;
            };
            fin = FWD ? acc : mark(acc);
#pragma unroll 8
            for (int sstep = 0; sstep < 32; ++sstep) {
                const bool hit = (hm >> sstep) & 1u;
                const int r = __popc(hm & ((1u << sstep) - 1u));
                const double vraw = wv[hit ? (FWD ? vb0 + r : vb0 - r) : 0];   // a valid address for every lane
                const double vv = hit ? vraw : 0.0;
                const double ys = __shfl_sync(FULL, fin, sstep);
                const double na = __fma_rn(-vv, ys, acc);
                acc = hit ? na : acc;
                if (FWD) fin = acc;
                else { const double nf = mark(acc); fin = hit ? nf : fin; }
            }
            if (!FWD) slow = __any_sync(FULL, bad || !dg_ok);
        }
        if (slow) {
            // exact path: IEEE division, values from the staged buffer or global memory
            acc = acc0;
            fin = FWD ? acc : __ddiv_rn(acc, dg);
            for (int sstep = 0; sstep < 32; ++sstep) {
                const bool hit = (hm >> sstep) & 1u;
                double vv = 0.0;
                if (hit) {
                    const int idx = kb + __popc(hm & ((1u << sstep) - 1u));
                    const int64_t q = FWD ? lo + idx : hi - 1 - idx;
                    vv = staged ? wv[q - e0] : __ldg(val + q);
                }
                const double ys = __shfl_sync(FULL, fin, sstep);
                const double na = __fma_rn(-vv, ys, acc);
                acc = hit ? na : acc;
                if (hit) fin = FWD ? acc : __ddiv_rn(acc, dg);
            }
        }
        if (dbg && lane == 0) dbg[win * 5 + 3] = clock64();
        if (valid) ring[p & (SW_RING - 1)] = fin;
        __threadfence_block();     // the ring values (shared memory) before the signal
        __syncwarp();
        wait_done(win);            // windows complete in order
        if (!ok) break;
        if (lane == 0) done[0] = (int)(win + 1);
        if (dbg && lane == 0) dbg[win * 5 + 4] = clock64();
        seen = (int)(win + 1);
        // the global copy after the signal: readers of `out` (columns older than the ring) start
        // at least SW_RING / 32 - NWS windows later, after this warp's later fences
        if (valid) out[oidx(i)] = fin;
        __syncwarp();
    }
    return ok;
}

}  // namespace mfk
