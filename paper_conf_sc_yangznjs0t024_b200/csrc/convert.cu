// convert.cu -- CSR -> two-level tile format on the GPU (Section III-B),
// per-nonzero precision criterion (Section II-A), per-tile precision, range floor,
// the SELL-16 kernel layout with lower-precision value planes ("convert once, reuse"),
// and the persistent-kernel launch plan (P:130-132 task distribution, balanced on nnz+tiles).
//
// One half-warp owns one tile row (16 matrix rows, lane r = row 16*TR + r) and merges its 16
// sorted rows tile column by tile column, so tiles come out in (row, col) order without a sort.
// Two passes with the same merge: COUNT (sizes per tile row) -> exclusive scans -> FILL.
#include <cuda_runtime.h>
#include <stdio.h>

#include <algorithm>
#include <cstdlib>
#include <vector>

#include "kernels.cuh"
#include "mf_internal.cuh"

namespace mf {
namespace {

constexpr int CNT_TILES = 0, CNT_ROWS = 1, CNT_WIDTH = 2, CNT_NNZP = 3 /*..6*/, CNT_TILEP = 7 /*..10*/;
constexpr int CNT_WTS = 11;   // tile-synchronous width: sum over tiles of the max entries per row
constexpr int CNT_VB = 12;    // tile-synchronous value bytes: sum over tiles of width * 16 * size(TilePrec)
constexpr int NCNT = 13;
constexpr int THREADS = 256;

__device__ __forceinline__ unsigned hw_mask() { return (threadIdx.x & 16) ? 0xFFFF0000u : 0x0000FFFFu; }

template <class T>
__device__ __forceinline__ T hw_min(T v, unsigned m) {
    for (int o = 8; o >= 1; o >>= 1) { T u = __shfl_xor_sync(m, v, o); v = u < v ? u : v; }
    return v;
}
template <class T>
__device__ __forceinline__ T hw_max(T v, unsigned m) {
    for (int o = 8; o >= 1; o >>= 1) { T u = __shfl_xor_sync(m, v, o); v = u > v ? u : v; }
    return v;
}
template <class T>
__device__ __forceinline__ T hw_sum(T v, unsigned m) {
    for (int o = 8; o >= 1; o >>= 1) v += __shfl_xor_sync(m, v, o);
    return v;
}
// exclusive prefix sum over the 16 lanes of the half-warp
template <class T>
__device__ __forceinline__ T hw_excl_scan(T v, unsigned m, int lane16) {
    T incl = v;
    for (int o = 1; o < 16; o <<= 1) {
        T u = __shfl_up_sync(m, incl, o, 16);
        if (lane16 >= o) incl += u;
    }
    return incl - v;
}

// Per-nonzero class: lowest of {FP8, FP16, FP32} whose single-RNE rounding loses less
// than loss_tol*|v| (relative reading); v == 0 -> FP8.  No contraction: explicit _rn ops.
__device__ __forceinline__ int classify(double v, double loss_tol) {
    if (v == 0.0) return 3;
    double thr = __dmul_rn(loss_tol, fabs(v));
    if (fabs(__dsub_rn(v, mfk::e4m3_to_d(mfk::to_e4m3(v)))) < thr) return 3;
    if (fabs(__dsub_rn(v, mfk::f16_to_d(mfk::to_f16(v)))) < thr) return 2;
    if (fabs(__dsub_rn(v, (double)mfk::to_f32(v))) < thr) return 1;
    return 0;
}

// lowest-precision format whose normal range holds |sv|; zeros are neutral (3)
__device__ __forceinline__ int range_class(double sv) {
    double a = fabs(sv);
    if (a == 0.0) return 3;
    if (a >= 0x1p-6 && a <= 448.0) return 3;
    if (a >= 0x1p-14 && a <= 65504.0) return 2;
    if (a >= 0x1p-126 && a <= 3.4028234663852886e38) return 1;
    return 0;
}

__global__ void validate_kernel(int64_t n_rows, int64_t n_cols, int64_t nnz, const int64_t* __restrict__ rowptr,
                                const int32_t* __restrict__ colidx, const double* __restrict__ vals, int* err) {
    int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_rows; i += stride) {
        int64_t a = rowptr[i], b = rowptr[i + 1];
        if ((i == 0 && a != 0) || (i == n_rows - 1 && b != nnz) || b < a || a < 0 || b > nnz) {
            atomicOr(err, 1);
            continue;
        }
        for (int64_t k = a; k < b; ++k) {
            int32_t c = colidx[k];
            if (c < 0 || c >= n_cols) atomicOr(err, 1);
            else if (k > a && c <= colidx[k - 1]) atomicOr(err, 2);
            if (!isfinite(vals[k])) atomicOr(err, 4);
        }
    }
}

struct Out {  // FILL-pass destinations (all device)
    int32_t *TileRowidx, *TileColidx;
    uint8_t *TilePrec, *Floor;
    int64_t *TileNnz, *Nonrow, *ValOff, *TileRowPtr;
    uint8_t *RowIndex, *CsrRowptr, *CsrColidx;
    double* Val64; float* Val32; uint16_t* Val16; uint8_t* Val8;
    uint32_t* tile_info; uint16_t* sidx; uint8_t* sslot; uint2* crec; int ts; uint8_t* vstream;
    double* p64; float* p32; __half* p16; uint8_t* p8;
    const int64_t* off;   // [NCNT][ntr+1] exclusive scans of the counts
    int64_t ntr;
};

// The merge of one tile row.  FILL == false: write counts; FILL == true: write the arrays.
template <bool FILL>
__global__ void __launch_bounds__(THREADS) tile_row_kernel(int64_t n_rows, int64_t ntr, const int64_t* __restrict__ rowptr,
                                                           const int32_t* __restrict__ colidx,
                                                           const double* __restrict__ vals, int classify_on,
                                                           double loss_tol, int64_t* cnt, int* err, Out o) {
    const unsigned m = hw_mask();
    const int lane = threadIdx.x & 15;
    const int64_t TR = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 4;
    if (TR >= ntr) return;                       // uniform per half-warp
    const int64_t row = TR * TS + lane;
    const bool valid = row < n_rows;
    const int64_t rstart = valid ? rowptr[row] : 0;
    const int64_t rend = valid ? rowptr[row + 1] : 0;
    int64_t ptr = rstart;
    int cur = ptr < rend ? (colidx[ptr] >> 4) : INT32_MAX;
    const int64_t width = hw_max<int64_t>(rend - rstart, m);

    int64_t j = 0, nz_run = 0, ri_run = 0, colbase = 0;
    int64_t pnnz[4] = {0, 0, 0, 0}, ptile[4] = {0, 0, 0, 0};
    int64_t tile0 = 0, row0 = 0, nnz0 = 0, slot0 = 0, voff[4] = {0, 0, 0, 0}, vb0 = 0, vb_run = 0;
    if (FILL) {
        const int64_t S = ntr + 1;
        tile0 = o.off[CNT_TILES * S + TR];
        row0 = o.off[CNT_ROWS * S + TR];
        slot0 = o.off[(o.ts ? CNT_WTS : CNT_WIDTH) * S + TR];
        vb0 = o.off[CNT_VB * S + TR];
        for (int q = 0; q < 4; ++q) voff[q] = o.off[(CNT_NNZP + q) * S + TR];
        nnz0 = rowptr[TR * TS];
        if (lane == 0) o.TileRowPtr[TR] = tile0;
        if (lane == 0 && TR == ntr - 1) o.TileRowPtr[ntr] = tile0 + o.off[CNT_TILES * S + ntr] - tile0;
    }
    while (true) {
        const int tc = hw_min<int>(cur, m);
        if (tc == INT32_MAX) break;
        const bool mine = (cur == tc);
        int64_t q = ptr;
        int cls = classify_on ? 3 : 0;
        if (mine) {
            while (q < rend && (colidx[q] >> 4) == tc) {
                if (classify_on) { int c = classify(vals[q], loss_tol); cls = c < cls ? c : cls; }
                ++q;
            }
        }
        const int cnt_r = (int)(q - ptr);
        const int best = hw_min<int>(mine ? cls : 3, m);        // TilePrec: highest needed precision
        int rc = 3;
        if (mine)
            for (int64_t k = ptr; k < q; ++k) { int c = range_class(mfk::round_to(vals[k], best)); rc = c < rc ? c : rc; }
        const int minrc = hw_min<int>(rc, m);
        const int floor_t = minrc > best ? minrc : best;
        const int tile_nz = hw_sum<int>(cnt_r, m);
        // tile-synchronous layout: one slice column per diagonal (local column - local row) that
        // holds an entry of the tile, diagonals ascending (so each row's entries stay in ascending
        // column order); compact layout: the row-packed width
        unsigned dmask = 0;
        if (mine)
            for (int64_t k = ptr; k < q; ++k) dmask |= 1u << ((colidx[k] & 15) - lane + 15);
        dmask = __reduce_or_sync(m, dmask);
        const int w_j = __popc(dmask);                      // slice columns of this tile (TS layout)
        const unsigned bal = __ballot_sync(m, mine) >> (threadIdx.x & 16);
        const int rows_in_tile = __popc(bal);
        if (FILL) {
            const int64_t t = tile0 + j;
            const int csr_off = hw_excl_scan<int>(cnt_r, m, lane);
            const int ri_loc = __popc(bal & ((1u << lane) - 1u));
            const int64_t vbase = voff[best] + pnnz[best];
            if (lane == 0) {
                o.TileRowidx[t] = (int32_t)TR;
                o.TileColidx[t] = tc;
                o.TilePrec[t] = (uint8_t)best;
                o.Floor[t] = (uint8_t)floor_t;
                o.TileNnz[t] = nnz0 + nz_run;
                o.Nonrow[t] = row0 + ri_run;
                o.ValOff[t] = vbase;
                o.tile_info[t] = ((uint32_t)tc << 4) | ((uint32_t)floor_t << 2) | (uint32_t)best;
            }
            if (mine) {
                const int64_t ri = row0 + ri_run + ri_loc;
                o.RowIndex[ri] = (uint8_t)lane;
                o.CsrRowptr[ri] = (uint8_t)csr_off;
                for (int64_t k = ptr; k < q; ++k) {
                    const int a = csr_off + (int)(k - ptr);
                    const double v = vals[k];
                    const int lc = colidx[k] & 15;
                    o.CsrColidx[nnz0 + nz_run + a] = (uint8_t)lc;
                    const int64_t vp = vbase + a;
                    double sv;
                    switch (best) {
                    case 0: o.Val64[vp] = v; sv = v; break;
                    case 1: { float f = mfk::to_f32(v); o.Val32[vp] = f; sv = (double)f; } break;
                    case 2: { __half h = mfk::to_f16(v); o.Val16[vp] = __half_as_ushort(h); sv = mfk::f16_to_d(h); } break;
                    default: { uint8_t b = mfk::to_e4m3(v); o.Val8[vp] = b; sv = mfk::e4m3_to_d(b); } break;
                    }
                    // kernel layout: compact slot (k - rstart) of this row, or tile-synchronous column
                    // colbase + (k - ptr); value planes RNE_q(stored) for q at or below TilePrec
                    const int di = __popc(dmask & ((1u << (lc - lane + 15)) - 1u));   // diagonal slice of the entry
                    const int64_t pos = o.ts ? (slot0 + colbase + di) * TS + lane
                                             : (slot0 + (k - rstart)) * TS + lane;
                    if (o.ts) {
                        // value stream: slice column (colbase + di) of the tile row, 16 * size(TilePrec) bytes
                        const int64_t vb = vb0 + vb_run + ((int64_t)di * 16 + lane) * (8 >> best);
                        switch (best) {
                        case 0: *reinterpret_cast<double*>(o.vstream + vb) = sv; break;
                        case 1: *reinterpret_cast<float*>(o.vstream + vb) = (float)sv; break;
                        case 2: *reinterpret_cast<__half*>(o.vstream + vb) = mfk::to_f16(sv); break;
                        default: o.vstream[vb] = mfk::to_e4m3(sv); break;
                        }
                    } else {
                        o.sidx[pos] = (uint16_t)((j << 4) | lc);
                    }
                    if (best <= 0 && o.p64) o.p64[pos] = sv;
                    if (best <= 1 && o.p32) o.p32[pos] = mfk::to_f32(sv);
                    if (best <= 2 && o.p16) o.p16[pos] = mfk::to_f16(sv);
                    if (o.p8) o.p8[pos] = mfk::to_e4m3(sv);
                }
            }
        }
        // static column record: word, value offset within the tile row (stage_kernel rebases it)
        if (FILL && o.ts && lane < w_j) {
            // slice `lane` of the tile: its diagonal (the lane-th set bit of dmask) in bits 24..28
            unsigned mm = dmask;
            for (int z = 0; z < lane; ++z) mm &= mm - 1u;
            const uint32_t dg = (uint32_t)(__ffs(mm) - 1);    // diagonal + 15
            o.crec[slot0 + colbase + lane] = make_uint2(((uint32_t)tc << 4) | ((uint32_t)floor_t << 2) | (uint32_t)best,
                                                        (uint32_t)(vb_run + (int64_t)lane * 16 * (8 >> best)) | (dg << 24));
        }
        if (mine) { ptr = q; cur = ptr < rend ? (colidx[ptr] >> 4) : INT32_MAX; }
        ++j;
        colbase += w_j;
        vb_run += (int64_t)w_j * 16 * (8 >> best);
        nz_run += tile_nz;
        ri_run += rows_in_tile;
        pnnz[best] += tile_nz;
        ptile[best] += 1;
    }
    if (FILL) {
        if (lane == 0 && TR == ntr - 1) {
            o.TileNnz[tile0 + j] = nnz0 + nz_run;
            o.Nonrow[tile0 + j] = row0 + ri_run;
        }
    } else if (lane == 0) {
        cnt[CNT_TILES * ntr + TR] = j;
        cnt[CNT_ROWS * ntr + TR] = ri_run;
        cnt[CNT_WIDTH * ntr + TR] = width;
        cnt[CNT_WTS * ntr + TR] = colbase;
        cnt[CNT_VB * ntr + TR] = vb_run;
        for (int q = 0; q < 4; ++q) {
            cnt[(CNT_NNZP + q) * ntr + TR] = pnnz[q];
            cnt[(CNT_TILEP + q) * ntr + TR] = ptile[q];
        }
        if (j > MAX_TILES_PER_TR) atomicOr(err, 8);
    }
}

// ------------------------------------------------------------------ exclusive scan (int64)
constexpr int SCAN_T = 1024, SCAN_CHUNK = 2 * SCAN_T;

__device__ int64_t block_incl_scan(int64_t v, int64_t* sh) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int o = 1; o < 32; o <<= 1) { int64_t u = __shfl_up_sync(0xffffffffu, v, o); if (lane >= o) v += u; }
    if (lane == 31) sh[w] = v;
    __syncthreads();
    if (w == 0) {
        int64_t s = lane < (int)(blockDim.x >> 5) ? sh[lane] : 0;
        for (int o = 1; o < 32; o <<= 1) { int64_t u = __shfl_up_sync(0xffffffffu, s, o); if (lane >= o) s += u; }
        sh[lane] = s;
    }
    __syncthreads();
    if (w > 0) v += sh[w - 1];
    __syncthreads();
    return v;
}

// Multi-array scans: blockIdx.y selects array y (in + y * istride, out + y * ostride, tmp + y * nb).
__global__ void scan_block_sums(const int64_t* __restrict__ in, int64_t n, int64_t* bsum, int64_t istride, int64_t nb) {
    __shared__ int64_t sh[32];
    in += blockIdx.y * istride;
    bsum += blockIdx.y * nb;
    int64_t base = (int64_t)blockIdx.x * SCAN_CHUNK;
    int64_t a = base + 2 * threadIdx.x;
    int64_t v = (a < n ? in[a] : 0) + (a + 1 < n ? in[a + 1] : 0);
    v = block_incl_scan(v, sh);
    if (threadIdx.x == blockDim.x - 1) bsum[blockIdx.x] = v;
}

__global__ void scan_sums_serial(int64_t* bsum, int64_t nb) {   // block y: exclusive scan of array y in place
    __shared__ int64_t sh[32];
    __shared__ int64_t carry;
    bsum += blockIdx.x * nb;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (int64_t c = 0; c < nb; c += blockDim.x) {
        int64_t i = c + threadIdx.x;
        int64_t v = i < nb ? bsum[i] : 0;
        int64_t incl = block_incl_scan(v, sh);
        int64_t cr = carry;
        if (i < nb) bsum[i] = cr + incl - v;
        __syncthreads();
        if (threadIdx.x == blockDim.x - 1) carry = cr + incl;
        __syncthreads();
    }
}

__global__ void scan_apply(const int64_t* __restrict__ in, int64_t n, const int64_t* __restrict__ bsum, int64_t* out,
                           int64_t istride, int64_t ostride, int64_t nb) {
    __shared__ int64_t sh[32];
    in += blockIdx.y * istride;
    out += blockIdx.y * ostride;
    bsum += blockIdx.y * nb;
    int64_t base = (int64_t)blockIdx.x * SCAN_CHUNK;
    int64_t a = base + 2 * threadIdx.x;
    int64_t x0 = a < n ? in[a] : 0, x1 = a + 1 < n ? in[a + 1] : 0;
    int64_t incl = block_incl_scan(x0 + x1, sh);
    int64_t excl = bsum[blockIdx.x] + incl - (x0 + x1);
    if (a < n) out[a] = excl;
    if (a + 1 < n) out[a + 1] = excl + x0;
    if (a + 1 == n - 1 || (a == n - 1)) out[n] = excl + x0 + x1;   // total
    if (n == 0 && blockIdx.x == 0 && threadIdx.x == 0) out[0] = 0;
}

// out[y][0..n] = exclusive scans of in[y][0..n) for narr arrays (out[y][n] = total): 3 launches
mf_status scan_excl_multi(const int64_t* in, int64_t n, int narr, int64_t istride, int64_t* out, int64_t ostride, int64_t* tmp,
                          cudaStream_t s) {
    if (n == 0) {
        for (int y = 0; y < narr; ++y) MF_CUDA(cudaMemsetAsync(out + y * ostride, 0, sizeof(int64_t), s));
        return MF_OK;
    }
    const int64_t nb = (n + SCAN_CHUNK - 1) / SCAN_CHUNK;
    scan_block_sums<<<dim3((unsigned)nb, narr), SCAN_T, 0, s>>>(in, n, tmp, istride, nb);
    scan_sums_serial<<<narr, SCAN_T, 0, s>>>(tmp, nb);
    scan_apply<<<dim3((unsigned)nb, narr), SCAN_T, 0, s>>>(in, n, tmp, out, istride, ostride, nb);
    MF_CUDA(cudaGetLastError());
    return MF_OK;
}
// out[0..n] = exclusive scan of in[0..n), out[n] = total
mf_status scan_excl(const int64_t* in, int64_t n, int64_t* out, int64_t* tmp, cudaStream_t s) {
    return scan_excl_multi(in, n, 1, 0, out, 0, tmp, s);
}

// ------------------------------------------------------------------ launch plan
// cost of a tile row: slice bytes (2 B index + ~2 B value per slot) + vector bytes (48 B per row)
__global__ void tr_cost_kernel(const int64_t* __restrict__ cnt, int64_t ntr, int64_t n_rows, int ts, int64_t* cost) {
    int64_t TR = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (TR >= ntr) return;
    int64_t rows = n_rows - TR * TS < TS ? n_rows - TR * TS : TS;
    cost[TR] = 4 * TS * cnt[(ts ? CNT_WTS : CNT_WIDTH) * ntr + TR] + 48 * rows + 1;
}

// plan_tr[g] = first tile row whose exclusive cost prefix reaches g*total/G
__global__ void plan_kernel(const int64_t* __restrict__ pre, int64_t ntr, int G, int32_t* plan_tr) {
    int g = blockIdx.x * blockDim.x + threadIdx.x;
    if (g > G) return;
    if (g == 0) { plan_tr[0] = 0; return; }
    if (g == G) { plan_tr[G] = (int32_t)ntr; return; }
    int64_t total = pre[ntr];
    int64_t target = (int64_t)((__int128)total * g / G);
    int64_t lo = 0, hi = ntr;            // first TR with pre[TR] >= target
    while (lo < hi) { int64_t mid = (lo + hi) / 2; if (pre[mid] >= target) hi = mid; else lo = mid + 1; }
    plan_tr[g] = (int32_t)lo;
}

__device__ int owner_of(const int32_t* plan_tr, int G, int64_t TR) {   // CTA owning tile row TR
    int lo = 0, hi = G - 1;
    while (lo < hi) { int mid = (lo + hi + 1) / 2; if (plan_tr[mid] <= TR) lo = mid; else hi = mid - 1; }
    return lo;
}

// dependency range: CTAs owning the column segments this CTA's tiles gather (square matrices)
__global__ void deps_kernel(const int32_t* __restrict__ plan_tr, int G, const int64_t* __restrict__ TileRowPtr,
                            const int32_t* __restrict__ TileColidx, int64_t n_seg_owned, int64_t coff, int32_t* dep_lo,
                            int32_t* dep_hi, int32_t* seg_lo, int32_t* seg_hi) {
    int g = blockIdx.x;
    __shared__ int smin, smax;
    if (threadIdx.x == 0) { smin = INT32_MAX; smax = -1; }
    __syncthreads();
    int lmin = INT32_MAX, lmax = -1;
    for (int64_t TR = plan_tr[g] + threadIdx.x; TR < plan_tr[g + 1]; TR += blockDim.x) {
        int64_t a = TileRowPtr[TR], b = TileRowPtr[TR + 1];
        if (b > a) { lmin = min(lmin, TileColidx[a]); lmax = max(lmax, TileColidx[b - 1]); }
    }
    atomicMin(&smin, lmin);
    atomicMax(&smax, lmax);
    __syncthreads();
    if (threadIdx.x == 0) {
        int lo = g, hi = g;
        if (smax >= 0) {
            // column segments outside the owned ones [coff, coff + n_seg_owned) (non-square / halo)
            // have no owner CTA
            const int64_t cmin = max((int64_t)smin, coff) - coff, cmax = min((int64_t)smax - coff, n_seg_owned - 1);
            if (cmin <= cmax) {
                lo = min(lo, owner_of(plan_tr, G, cmin));
                hi = max(hi, owner_of(plan_tr, G, cmax));
            }
        }
        dep_lo[g] = lo;
        dep_hi[g] = hi;
        seg_lo[g] = smax >= 0 ? smin : 0;     // column segments gathered by this CTA's tiles
        seg_hi[g] = smax;
    }
}

// max over tile rows of the tile-synchronous width and value bytes (stage-capacity check)
__global__ void max2_kernel(const int64_t* __restrict__ a, const int64_t* __restrict__ b, int64_t n, unsigned long long* out) {
    unsigned long long ma = 0, mb = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        ma = max(ma, (unsigned long long)a[i]);
        mb = max(mb, (unsigned long long)b[i]);
    }
    for (int o = 16; o >= 1; o >>= 1) {
        ma = max(ma, __shfl_xor_sync(0xffffffffu, ma, o));
        mb = max(mb, __shfl_xor_sync(0xffffffffu, mb, o));
    }
    if ((threadIdx.x & 31) == 0) { atomicMax(&out[0], ma); atomicMax(&out[1], mb); }
}

// Stages of the TMA pipeline (kernels.cuh): one warp per CTA of the plan walks its tile rows and
// cuts them greedily into stages within the caps (tile rows <= kcap, slice columns, value bytes),
// each a whole number of H-row groups when one fits, so that every half-warp gets the same number
// of tile rows per stage.  COUNT pass: stages per CTA; FILL pass: the records (tr0, tr1, nc).
template <bool FILL>
__global__ void stage_kernel(const int32_t* __restrict__ plan_tr, int G, int H, int kcap, const int64_t* __restrict__ tr_slot,
                             const int64_t* __restrict__ tr_vb, int32_t* nst, const int32_t* __restrict__ sptr,
                             mfk::TsStage* stg) {
    const int g = blockIdx.x;
    const int lane = threadIdx.x & 31;
    if (g >= G) return;
    const int64_t tr0 = plan_tr[g], tr1 = plan_tr[g + 1];
    const int64_t base = FILL ? sptr[g] : 0;
    int64_t S = tr0;
    int32_t k = 0;
    while (S < tr1) {
        const int64_t c0 = tr_slot[S], v0 = tr_vb[S];
        const int64_t lim = min(S + (int64_t)kcap, tr1);
        int64_t emax = S;
        for (int64_t e0 = S + 1; e0 <= lim; e0 += 32) {
            const int64_t E = e0 + lane;
            const bool fit = E <= lim && tr_slot[E] - c0 <= mfk::TS_CCAP && tr_vb[E] - v0 <= mfk::TS_VCAP;
            const int nfit = __popc(__ballot_sync(0xffffffffu, fit));     // fits are a prefix (monotone)
            if (nfit > 0) emax = e0 + nfit - 1;
            if (nfit < 32) break;
        }
        if (emax == S) emax = S + 1;          // oversize tile row: excluded by the host's capacity check
        const int64_t grp = tr0 + ((emax - tr0) / H) * H;
        const int64_t E = grp > S ? grp : emax;
        if (FILL && lane == 0) {
            mfk::TsStage st{};
            st.tr0 = (int32_t)S; st.tr1 = (int32_t)E;
            st.nc = (int32_t)(tr_slot[E] - c0);
            stg[base + k] = st;
        }
        ++k;
        S = E;
    }
    if (!FILL && lane == 0) nst[g] = k;
}

// Window runs of each stage: the distinct tile columns its tiles gather, sorted, cut into runs of
// consecutive column segments (gaps of <= RUN_GAP segments are bridged: one bulk copy instead of
// two), merged down to TS_RUNCAP runs by bridging the smallest gaps.  One block per stage.
constexpr int RUN_GAP = 2;
constexpr int RUNS_T = 1024;
__global__ void __launch_bounds__(RUNS_T) runs_kernel(mfk::TsStage* stg, const int64_t* __restrict__ TileRowPtr,
                                                      const int32_t* __restrict__ TileColidx, unsigned long long* maxw) {
    __shared__ int32_t key[RUNS_T];
    __shared__ int32_t rs[RUNS_T], rn[RUNS_T];
    const int t = threadIdx.x;
    mfk::TsStage st = stg[blockIdx.x];
    const int64_t a = TileRowPtr[st.tr0], b = TileRowPtr[st.tr1];
    const int nt = (int)(b - a);                          // <= TS_CCAP (a tile owns >= 1 slice column)
    key[t] = t < nt ? TileColidx[a + t] : INT32_MAX;
    __syncthreads();
    for (int k = 2; k <= RUNS_T; k <<= 1)                 // bitonic sort
        for (int j = k >> 1; j > 0; j >>= 1) {
            const int ix = t ^ j;
            if (ix > t) {
                const int32_t x = key[t], y = key[ix];
                if (((t & k) == 0) == (x > y)) { key[t] = y; key[ix] = x; }
            }
            __syncthreads();
        }
    if (t == 0) {
        int nr = 0;
        for (int i = 0; i < nt; ++i) {
            const int32_t c = key[i];
            if (nr > 0 && c <= rs[nr - 1] + rn[nr - 1] + RUN_GAP) {
                if (c >= rs[nr - 1] + rn[nr - 1]) rn[nr - 1] = c - rs[nr - 1] + 1;
            } else {
                rs[nr] = c; rn[nr] = 1; ++nr;
            }
        }
        while (nr > mfk::TS_RUNCAP) {                     // bridge the smallest gap
            int best = 0;
            int64_t bg = INT64_MAX;
            for (int i = 0; i + 1 < nr; ++i) {
                const int64_t gp = (int64_t)rs[i + 1] - (rs[i] + rn[i]);
                if (gp < bg) { bg = gp; best = i; }
            }
            rn[best] = rs[best + 1] + rn[best + 1] - rs[best];
            for (int i = best + 1; i + 1 < nr; ++i) { rs[i] = rs[i + 1]; rn[i] = rn[i + 1]; }
            --nr;
        }
        int64_t w = 0;
        for (int i = 0; i < mfk::TS_RUNCAP; ++i) {
            st.run_s[i] = i < nr ? rs[i] : 0;
            st.run_n[i] = i < nr ? rn[i] : 0;
            st.run_w[i] = (int32_t)w;
            if (i < nr) w += rn[i];
        }
        st.nrun = nr;
        st.wseg = (int32_t)(w < (int64_t)INT32_MAX ? w : (int64_t)INT32_MAX);
        stg[blockIdx.x] = st;
        atomicMax(maxw, (unsigned long long)w);
    }
}

// Blob of each stage (layout in kernels.cuh): its byte size, then, after an exclusive scan of the
// sizes, its contents.  One block of TS_CCAP threads per stage: thread c owns column c.
struct BlobLayout {
    int off_desc, off_wl, off_gd, off_val, bytes;
};
__host__ __device__ __forceinline__ BlobLayout blob_layout(int K, int64_t nc, int64_t nv, int NW) {
    BlobLayout L;
    L.off_desc = mfk::TS_HDR + mfk::ts_r16((K + 1) * 2);
    L.off_wl = L.off_desc + mfk::ts_r16(((int)nc + mfk::TS_DPAD) * 4);
    L.off_gd = L.off_wl + NW * 16;
    L.off_val = L.off_gd + mfk::ts_r16((int)nc * 4);
    L.bytes = L.off_val + (int)nv;
    return L;
}
__global__ void blob_size_kernel(const mfk::TsStage* __restrict__ stg, int64_t n, const int64_t* __restrict__ tr_vb, int NW,
                                 int64_t* sz) {
    const int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n) return;
    const mfk::TsStage st = stg[s];
    sz[s] = blob_layout(st.tr1 - st.tr0, st.nc, tr_vb[st.tr1] - tr_vb[st.tr0], NW).bytes;
}
__device__ int owner_cta(const int32_t* plan_tr, int G, int64_t TR) {
    int lo = 0, hi = G - 1;
    while (lo < hi) { const int mid = (lo + hi + 1) / 2; if (plan_tr[mid] <= TR) lo = mid; else hi = mid - 1; }
    return lo;
}
__global__ void __launch_bounds__(mfk::TS_CCAP) blob_fill_kernel(mfk::TsStage* stg, const int64_t* __restrict__ boff,
                                                                   const int64_t* __restrict__ tr_slot, const int64_t* __restrict__ tr_vb,
                                                                   const uint2* __restrict__ crec,
                                                                   const uint8_t* __restrict__ vstream, uint8_t* blob,
                                                                   const int32_t* __restrict__ plan_tr, int G, int H,
                                                                   int64_t coff, unsigned long long* maxb) {
    __shared__ int32_t hdr[mfk::TS_KCAP + 1];
    __shared__ int16_t cw[mfk::TS_KCAP];                 // warp of each tile row
    __shared__ uint8_t cq[mfk::TS_CCAP];                 // TilePrec of each column
    __shared__ int32_t cdst[mfk::TS_CCAP];               // value byte offset of each column (grouped order)
    __shared__ uint8_t cslot[mfk::TS_CCAP];              // decode-buffer slot of each column
    __shared__ int32_t wcol[33], wval[33];               // columns / value bytes per warp, exclusive prefixes
    const int64_t sidx = blockIdx.x;
    const mfk::TsStage st = stg[sidx];
    const int K = st.tr1 - st.tr0, c = threadIdx.x;
    const int nc = st.nc, NW = H / 2 > 1 ? H / 2 : 1;   // warps = B / 32 = H / 2
    const int64_t col0 = tr_slot[st.tr0];
    const int64_t vb0 = tr_vb[st.tr0], nv = tr_vb[st.tr1] - vb0;
    const BlobLayout L = blob_layout(K, nc, nv, NW);
    const int64_t tr0c = plan_tr[owner_cta(plan_tr, G, st.tr0)];
    uint8_t* b = blob + boff[sidx];
    for (int k = c; k <= K; k += blockDim.x) {
        hdr[k] = (int32_t)(tr_slot[st.tr0 + k] - col0);
        reinterpret_cast<int16_t*>(b + mfk::TS_HDR)[k] = (int16_t)hdr[k];
        if (k < K) cw[k] = (int16_t)((int)((st.tr0 + k - tr0c) % H) >> 1);
    }
    __shared__ uint8_t cfl[mfk::TS_CCAP];                // Floor of each column
    uint2 rc = make_uint2(0u, 0u);
    if (c < nc) {
        rc = crec[col0 + c];
        cq[c] = (uint8_t)(rc.x & 3u);
        cfl[c] = (uint8_t)((rc.x >> 2) & 3u);
    }
    __syncthreads();
    if (c < NW) {      // columns and value bytes of warp c (its rows: half-warps 2c, 2c+1)
        int nw = 0, vw = 0;
        for (int k = 0; k < K; ++k)
            if (cw[k] == c)
                for (int cc = hdr[k]; cc < hdr[k + 1]; ++cc) { ++nw; vw += 16 * (8 >> cq[cc]); }
        wcol[c + 1] = nw;
        wval[c + 1] = vw;
    }
    __syncthreads();
    if (c == 0) {
        // own window segment: column segment tr0 + coff if the stage's own segments lie inside one
        // run, else -1
        int own = -1;
        const int64_t oc0 = st.tr0 + coff, oc1 = st.tr1 + coff;
        for (int i = 0; i < st.nrun; ++i)
            if (st.run_s[i] <= oc0 && oc1 <= (int64_t)st.run_s[i] + st.run_n[i]) own = st.run_w[i] + (int)(oc0 - st.run_s[i]);
        int32_t* h = reinterpret_cast<int32_t*>(b);
        h[0] = st.tr0; h[1] = st.tr1; h[2] = nc; h[3] = L.off_desc; h[4] = 0; h[5] = L.off_val; h[6] = own;
        h[7] = (int32_t)(uint32_t)(uint64_t)col0; h[8] = (int32_t)(uint32_t)((uint64_t)col0 >> 32);
        h[9] = L.off_wl; h[10] = L.off_gd; h[11] = (int32_t)((st.tr0 - tr0c) % H);   // off0: half-warp of tile row tr0
        for (int k = 12; k < 16; ++k) h[k] = 0;
        wcol[0] = 0; wval[0] = 0;
        for (int w = 0; w < NW; ++w) { wcol[w + 1] += wcol[w]; wval[w + 1] += wval[w]; }
    }
    __syncthreads();
    if (c < NW) {
        // warp c: its columns grouped by TilePrec (FP64 | FP32 | FP16 | E4M3), ascending within a
        // group; the group order gives each column its decode-buffer slot and its value position
        const int w = c;
        uint32_t cnt = 0;
        int slot = 0, voff = wval[w];
        uint32_t* gd = reinterpret_cast<uint32_t*>(b + L.off_gd) + wcol[w];
        for (int q = 0; q < 4; ++q) {
            int nq = 0;
            for (int k = 0; k < K; ++k) {
                if (cw[k] != w) continue;
                for (int cc = hdr[k]; cc < hdr[k + 1]; ++cc)
                    if (cq[cc] == q) {
                        cslot[cc] = (uint8_t)slot;      // decode-buffer slot: rank in the warp's grouped order
                        cdst[cc] = voff;
                        gd[slot] = ((uint32_t)cfl[cc] << 16) | ((uint32_t)cc << 20);   // + window offset below
                        ++slot; ++nq;
                        voff += 16 * (8 >> q);
                    }
            }
            cnt |= (uint32_t)min(nq, 255) << (8 * q);
        }
        reinterpret_cast<uint4*>(b + L.off_wl)[w] = make_uint4(cnt, (uint32_t)wval[w], (uint32_t)wcol[w], 0u);
        atomicMax(maxb + 1, (unsigned long long)slot);
    }
    __syncthreads();
    if (c < nc) {
        const uint32_t tc = rc.x >> 4;
        int lo = 0, hi = K - 1;                              // tile row of column c
        while (lo < hi) { const int mid = (lo + hi + 1) / 2; if (hdr[mid] <= c) lo = mid; else hi = mid - 1; }
        int wseg = 0;
        for (int i = 0; i < st.nrun; ++i)
            if ((int64_t)tc >= st.run_s[i] && (int64_t)tc < (int64_t)st.run_s[i] + st.run_n[i]) wseg = st.run_w[i] + (int)(tc - st.run_s[i]);
        const uint32_t woff = (uint32_t)(wseg * mfk::PV_SEG_BYTES);
        const int dg = (int)((rc.y >> 24) & 31u) - 15;      // diagonal of the slice column
        // x of lane r is window element 16 * wseg + r + dg: byte offset from the window guard
        const uint32_t xoff = (uint32_t)(mfk::TS_GUARD + (int)woff + 8 * dg);
        reinterpret_cast<uint32_t*>(b + L.off_desc)[c] = xoff | ((uint32_t)cslot[c] << 16);
        reinterpret_cast<uint32_t*>(b + L.off_gd)[wcol[cw[lo]] + cslot[c]] |= woff;
        // values of column c (16 x size(TilePrec) bytes, column order in vstream) -> grouped position
        const int64_t src = tr_vb[st.tr0 + lo] + (rc.y & 0xFFFFFFu);
        const int n16 = 8 >> cq[c];
        const uint4* sp = reinterpret_cast<const uint4*>(vstream + src);
        uint4* dp = reinterpret_cast<uint4*>(b + L.off_val + cdst[c]);
        for (int k = 0; k < n16; ++k) dp[k] = sp[k];
    }
    if (c < mfk::TS_DPAD)                                  // padding read by short rows: x = guard, slot 0
        reinterpret_cast<uint32_t*>(b + L.off_desc)[nc + c] = (uint32_t)mfk::TS_GUARD;
    if (c == 0) {
        stg[sidx].boff_lo = (uint32_t)(uint64_t)boff[sidx];
        stg[sidx].boff_hi = (uint32_t)((uint64_t)boff[sidx] >> 32);
        stg[sidx].bbytes = L.bytes;
        atomicMax(maxb, (unsigned long long)L.bytes);
    }
}

}  // namespace

mf_status scan_excl_i64(const int64_t* in, int64_t n, int64_t* out, int64_t* tmp, cudaStream_t s) {
    return scan_excl(in, n, out, tmp, s);
}

void destroy_tiles(TileMatrix* A) {
    cudaStream_t s = A->owner_stream;
    void* ptrs[] = {A->TileRowidx, A->TileColidx, A->TilePrec, A->Floor, A->TileNnz, A->Nonrow, A->ValOff,
                    A->TileRowPtr, A->RowIndex, A->CsrRowptr, A->CsrColidx, A->Val64, A->Val32, A->Val16,
                    A->Val8, A->tr_slot, A->tile_info, A->sidx, A->sslot, A->crec, A->plane64, A->plane32, A->plane16,
                    A->plane8, A->plan_tr, A->dep_lo, A->dep_hi, A->seg_lo, A->seg_hi, A->tr_vb, A->vstream, A->stg,
                    A->stg_ptr, A->blob};
    for (void* p : ptrs) if (p) dev_free(p, s);
    delete[] A->plan_rows_host;
    *A = TileMatrix();
}

mf_status convert_csr(int64_t n_rows, int64_t n_cols, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                      const double* vals, const mf_convert_opts& o, cudaStream_t s, TileMatrix* A) {
    int sms = 0;
    MF_TRY(check_device(&sms));
    // launch-plan arguments are validated before any device work (nothing to release on failure)
    if (o.block_threads != 0 && (o.block_threads % 32 || o.block_threads > 1024 || o.block_threads < 32))
        return fail(MF_ERR_INVALID_ARG, "block_threads must be a multiple of 32 in [32, 1024]");
    A->n_rows = n_rows; A->n_cols = n_cols; A->nnz = nnz; A->owner_stream = s;
    A->ntr = (n_rows + TS - 1) / TS;
    const int64_t ntr = A->ntr;
    cudaEvent_t e0, e1;
    MF_CUDA(cudaEventCreate(&e0));
    MF_CUDA(cudaEventCreate(&e1));
    MF_CUDA(cudaEventRecord(e0, s));

    // 1. validation (before any other device work)
    int* d_err = nullptr;
    MF_TRY(alloc(&d_err, 1, s));
    MF_CUDA(cudaMemsetAsync(d_err, 0, sizeof(int), s));
    if (n_rows > 0) {
        int blocks = (int)std::min<int64_t>((n_rows + 255) / 256, 4 * 148 * 8);
        validate_kernel<<<blocks, 256, 0, s>>>(n_rows, n_cols, nnz, rowptr, colidx, vals, d_err);
        MF_CUDA(cudaGetLastError());
    }
    int h_err = 0;
    MF_CUDA(cudaMemcpyAsync(&h_err, d_err, sizeof(int), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    if (h_err & 1) { dev_free(d_err, s); return fail(MF_ERR_INVALID_ARG, "CSR rowptr/colidx out of range or not monotone"); }
    if (h_err & 2) { dev_free(d_err, s); return fail(MF_ERR_UNSORTED_CSR, "columns not strictly increasing within a row"); }
    if (h_err & 4) { dev_free(d_err, s); return fail(MF_ERR_NONFINITE, "non-finite matrix value"); }

    // 2. COUNT pass
    int64_t *cnt = nullptr, *off = nullptr, *tmp = nullptr;
    const int64_t S = ntr + 1;
    MF_TRY(alloc(&cnt, (size_t)NCNT * std::max<int64_t>(ntr, 1), s));
    MF_TRY(alloc(&off, (size_t)NCNT * S, s));
    MF_TRY(alloc(&tmp, (size_t)NCNT * (ntr / SCAN_CHUNK + 2), s));
    const int tr_per_block = THREADS / 16;
    const unsigned tblocks = (unsigned)std::max<int64_t>((ntr + tr_per_block - 1) / tr_per_block, 1);
    Out none{};
    none.ts = 0;
    if (ntr > 0) {
        tile_row_kernel<false><<<tblocks, THREADS, 0, s>>>(n_rows, ntr, rowptr, colidx, vals, o.classify, o.loss_tol,
                                                            cnt, d_err, none);
        MF_CUDA(cudaGetLastError());
    }
    MF_TRY(scan_excl_multi(cnt, ntr, NCNT, ntr, off, S, tmp, s));
    std::vector<int64_t> tot(NCNT);
    for (int c = 0; c < NCNT; ++c)
        MF_CUDA(cudaMemcpyAsync(&tot[c], off + c * S + ntr, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaMemcpyAsync(&h_err, d_err, sizeof(int), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    if (h_err & 8) {
        dev_free(d_err, s); dev_free(cnt, s); dev_free(off, s); dev_free(tmp, s);
        return fail(MF_ERR_UNSUPPORTED, "a tile row holds more than 4096 tiles");
    }
    A->tilenum = tot[CNT_TILES];
    A->rownum = tot[CNT_ROWS];
    // kernel layout: tile-synchronous slices (uniform tile per slice column, streamed by the TMA
    // pipeline) unless they cost more than 60% extra slots over the compact (row-packed) slices,
    // or one tile row exceeds a pipeline stage
    unsigned long long mx[4] = {0, 0, 0, 0};   // max over tile rows: TS width, TS value bytes, tiles, compact width
    if (ntr > 0) {
        unsigned long long* dmx = nullptr;
        MF_TRY(alloc(&dmx, 4, s));
        MF_CUDA(cudaMemsetAsync(dmx, 0, 4 * sizeof(unsigned long long), s));
        const unsigned mb = (unsigned)std::min<int64_t>((ntr + 255) / 256, 1184);
        max2_kernel<<<mb, 256, 0, s>>>(cnt + CNT_WTS * ntr, cnt + CNT_VB * ntr, ntr, dmx);
        max2_kernel<<<mb, 256, 0, s>>>(cnt + CNT_TILES * ntr, cnt + CNT_WIDTH * ntr, ntr, dmx + 2);
        MF_CUDA(cudaMemcpyAsync(mx, dmx, sizeof(mx), cudaMemcpyDeviceToHost, s));
        MF_CUDA(cudaStreamSynchronize(s));
        dev_free(dmx, s);
    }
    const bool ts_fits = mx[0] <= (unsigned long long)mfk::TS_CCAP && mx[1] <= (unsigned long long)mfk::TS_VCAP;
    if (o.layout == 1) A->ts = 0;
    else if (o.layout == 2) A->ts = ts_fits ? 1 : 0;
    else A->ts = ts_fits && (double)tot[CNT_WTS] <= 1.6 * (double)tot[CNT_WIDTH] ? 1 : 0;
    A->slots = A->ts ? tot[CNT_WTS] : tot[CNT_WIDTH];
    for (int q = 0; q < 4; ++q) { A->nval[q] = tot[CNT_NNZP + q]; A->tiles_per_prec[q] = tot[CNT_TILEP + q]; }

    // 3. allocate
    const int64_t nt = A->tilenum, nslot = A->slots * TS;
    MF_TRY(alloc(&A->TileRowidx, nt, s)); MF_TRY(alloc(&A->TileColidx, nt, s));
    MF_TRY(alloc(&A->TilePrec, nt, s)); MF_TRY(alloc(&A->Floor, nt, s));
    MF_TRY(alloc(&A->TileNnz, nt + 1, s)); MF_TRY(alloc(&A->Nonrow, nt + 1, s));
    MF_TRY(alloc(&A->ValOff, nt, s)); MF_TRY(alloc(&A->TileRowPtr, ntr + 1, s));
    MF_TRY(alloc(&A->RowIndex, A->rownum, s)); MF_TRY(alloc(&A->CsrRowptr, A->rownum, s));
    MF_TRY(alloc(&A->CsrColidx, nnz, s));
    MF_TRY(alloc(&A->Val64, A->nval[0], s)); MF_TRY(alloc(&A->Val32, A->nval[1], s));
    MF_TRY(alloc(&A->Val16, A->nval[2], s)); MF_TRY(alloc(&A->Val8, A->nval[3], s));
    MF_TRY(alloc(&A->tile_info, nt, s));
    A->vbytes = A->ts ? tot[CNT_VB] : 0;
    if (A->ts) {
        // padded so that the pipeline's 16-byte aligned bulk copies stay inside the arrays
        MF_TRY(alloc(&A->crec, A->slots + 8, s));
        MF_TRY(alloc(&A->vstream, A->vbytes + 64, s));
        MF_TRY(alloc(&A->tr_vb, ntr + 4, s));
        MF_CUDA(cudaMemsetAsync(A->crec, 0, (A->slots + 8) * sizeof(uint2), s));
        MF_CUDA(cudaMemsetAsync(A->vstream, 0, A->vbytes + 64, s));
        MF_CUDA(cudaMemsetAsync(A->tr_vb, 0, (ntr + 4) * sizeof(int64_t), s));
        MF_CUDA(cudaMemcpyAsync(A->tr_vb, off + CNT_VB * S, (ntr + 1) * sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
    } else {
        MF_TRY(alloc(&A->sidx, nslot, s));
    }
    // value planes (compact layout): plane q exists when some tile can compute at q (TilePrec <= q)
    bool need[4] = {false, false, false, false};
    if (!A->ts)
        for (int q = 0; q < 4; ++q)
            for (int p = 0; p <= q; ++p) if (A->tiles_per_prec[p] > 0) need[q] = true;
    // planes padded to whole 8-byte words: the SpMV fetches the aligned 8-byte word around a value
    if (need[0]) MF_TRY(alloc(&A->plane64, nslot + 1, s));
    if (need[1]) MF_TRY(alloc(&A->plane32, nslot + 2, s));
    if (need[2]) MF_TRY(alloc(&A->plane16, nslot + 4, s));
    if (need[3]) MF_TRY(alloc(&A->plane8, nslot + 8, s));
    if (nslot && A->sidx) MF_CUDA(cudaMemsetAsync(A->sidx, 0xFF, nslot * sizeof(uint16_t), s));
    if (nt == 0) {
        MF_CUDA(cudaMemsetAsync(A->TileNnz, 0, sizeof(int64_t), s));
        MF_CUDA(cudaMemsetAsync(A->Nonrow, 0, sizeof(int64_t), s));
    }
    MF_TRY(alloc(&A->tr_slot, ntr + 4, s));
    MF_CUDA(cudaMemsetAsync(A->tr_slot, 0, (ntr + 4) * sizeof(int64_t), s));
    MF_CUDA(cudaMemcpyAsync(A->tr_slot, off + (A->ts ? CNT_WTS : CNT_WIDTH) * S, (ntr + 1) * sizeof(int64_t),
                            cudaMemcpyDeviceToDevice, s));

    // 4. FILL pass
    Out fo{A->TileRowidx, A->TileColidx, A->TilePrec, A->Floor, A->TileNnz, A->Nonrow, A->ValOff, A->TileRowPtr,
           A->RowIndex, A->CsrRowptr, A->CsrColidx, A->Val64, A->Val32, A->Val16, A->Val8, A->tile_info, A->sidx,
           A->sslot, A->crec, A->ts, A->vstream, A->plane64, A->plane32, A->plane16, A->plane8, off, ntr};
    if (ntr > 0) {
        tile_row_kernel<true><<<tblocks, THREADS, 0, s>>>(n_rows, ntr, rowptr, colidx, vals, o.classify, o.loss_tol,
                                                           cnt, d_err, fo);
        MF_CUDA(cudaGetLastError());
    } else {
        MF_CUDA(cudaMemsetAsync(A->TileRowPtr, 0, sizeof(int64_t), s));
    }
    A->max_nt = (int64_t)mx[2];
    A->max_w = (int64_t)(A->ts ? mx[0] : mx[3]);

    // 5. launch plan
    int G = o.grid_ctas, B = o.block_threads;
    if (B <= 0) B = 512;
    if (B % 32 || B > 1024 || B < 32) {
        return fail(MF_ERR_INVALID_ARG, "block_threads must be a multiple of 32 in [32, 1024]");
    }
    // auto plan: one CTA per SM; small matrices get at least 8 tile rows per CTA (latency-bound:
    // more CTAs shorten the per-CTA chain more than the extra barrier participants cost)
    if (G <= 0) G = (int)std::max<int64_t>(1, std::min<int64_t>(sms, (ntr + 7) / 8));
    if (G > sms * 2) G = sms * 2;
    if (ntr > 0 && G > ntr) G = (int)ntr;
    if (G < 1) G = 1;
    A->G = G; A->B = B;
    int64_t* cost = nullptr;
    MF_TRY(alloc(&cost, std::max<int64_t>(ntr, 1), s));
    if (ntr) tr_cost_kernel<<<(unsigned)((ntr + 255) / 256), 256, 0, s>>>(cnt, ntr, n_rows, A->ts, cost);
    MF_TRY(scan_excl(cost, ntr, off, tmp, s));    // reuse off[0..ntr]
    MF_TRY(alloc(&A->plan_tr, G + 1, s));
    MF_TRY(alloc(&A->dep_lo, G, s));
    MF_TRY(alloc(&A->dep_hi, G, s));
    MF_TRY(alloc(&A->seg_lo, G, s));
    MF_TRY(alloc(&A->seg_hi, G, s));
    plan_kernel<<<(G + 1 + 127) / 128, 128, 0, s>>>(off, ntr, G, A->plan_tr);
    deps_kernel<<<G, 256, 0, s>>>(A->plan_tr, G, A->TileRowPtr, A->TileColidx, ntr, A->coff, A->dep_lo, A->dep_hi, A->seg_lo,
                                  A->seg_hi);
    MF_CUDA(cudaGetLastError());
    bool ts_failed = false;
    if (A->ts) {   // pipeline stages of every CTA (two passes: count, fill), their window runs
        int32_t* nst = nullptr;
        unsigned long long* dmax = nullptr;
        MF_TRY(alloc(&nst, G, s));
        MF_TRY(alloc(&dmax, 3, s));
        std::vector<int32_t> nst_h(G), sp_h(G + 1);
        // the window of a stage grows with its tile rows: halve the stage cap until every
        // stage's window fits TS_WCAP segments
        // two tile rows per half-warp per stage (K = 2H: two independent fma chains per lane), halved
        // until every stage window fits
        // 32 tile columns per stage measured best on C2 (r02 sweep: 73 us/it vs 81 at 64, 92 at 16)
        int kcap0 = std::min(32, std::max(1, B / 8));
        if (const char* ev = getenv("MF_KCAP"))   // tuning knob
            if (atoi(ev) > 0) kcap0 = std::min(mfk::TS_KCAP, atoi(ev));
        for (int kcap = kcap0;; kcap /= 2) {
            stage_kernel<false><<<G, 32, 0, s>>>(A->plan_tr, G, B / 16, kcap, A->tr_slot, A->tr_vb, nst, nullptr, nullptr);
            MF_CUDA(cudaGetLastError());
            MF_CUDA(cudaMemcpyAsync(nst_h.data(), nst, G * sizeof(int32_t), cudaMemcpyDeviceToHost, s));
            MF_CUDA(cudaStreamSynchronize(s));
            sp_h[0] = 0;
            for (int g = 0; g < G; ++g) sp_h[g + 1] = sp_h[g] + nst_h[g];
            A->nstg = sp_h[G];
            if (A->stg_ptr) dev_free(A->stg_ptr, s);
            if (A->stg) dev_free(A->stg, s);
            A->stg_ptr = nullptr; A->stg = nullptr;
            MF_TRY(alloc(&A->stg_ptr, G + 1, s));
            MF_CUDA(cudaMemcpyAsync(A->stg_ptr, sp_h.data(), (G + 1) * sizeof(int32_t), cudaMemcpyHostToDevice, s));
            mfk::TsStage* stg = nullptr;
            MF_TRY(alloc(&stg, std::max<int64_t>(A->nstg, 1), s));
            A->stg = stg;
            stage_kernel<true><<<G, 32, 0, s>>>(A->plan_tr, G, B / 16, kcap, A->tr_slot, A->tr_vb, nullptr, A->stg_ptr, stg);
            MF_CUDA(cudaMemsetAsync(dmax, 0, 3 * sizeof(unsigned long long), s));
            if (A->nstg > 0) runs_kernel<<<(unsigned)A->nstg, RUNS_T, 0, s>>>(stg, A->TileRowPtr, A->TileColidx, dmax);
            MF_CUDA(cudaGetLastError());
            unsigned long long mw = 0;
            MF_CUDA(cudaMemcpyAsync(&mw, dmax, sizeof(mw), cudaMemcpyDeviceToHost, s));
            MF_CUDA(cudaStreamSynchronize(s));   // sp_h (pageable) consumed
            A->wcap = (int32_t)std::min<unsigned long long>(mw, 1ull << 30);
            if (mw <= (unsigned long long)mfk::TS_WCAP) break;
            if (kcap == 1) { ts_failed = true; break; }
        }
        // blobs: sizes -> offsets -> contents; the per-column source arrays are then released
        if (!ts_failed && A->nstg > 0) {
            int64_t *bsz = nullptr, *boff = nullptr, *btmp = nullptr;
            MF_TRY(alloc(&bsz, A->nstg, s));
            MF_TRY(alloc(&boff, A->nstg + 1, s));
            MF_TRY(alloc(&btmp, A->nstg / 2048 + 2, s));
            blob_size_kernel<<<(unsigned)((A->nstg + 255) / 256), 256, 0, s>>>(static_cast<mfk::TsStage*>(A->stg), A->nstg, A->tr_vb,
                                                                              B / 32, bsz);
            MF_TRY(scan_excl(bsz, A->nstg, boff, btmp, s));
            MF_CUDA(cudaMemcpyAsync(&A->blob_bytes, boff + A->nstg, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
            MF_CUDA(cudaStreamSynchronize(s));
            MF_TRY(alloc(&A->blob, A->blob_bytes + 64, s));
            blob_fill_kernel<<<(unsigned)A->nstg, mfk::TS_CCAP, 0, s>>>(static_cast<mfk::TsStage*>(A->stg), boff, A->tr_slot, A->tr_vb, A->crec,
                                                                       A->vstream, A->blob, A->plan_tr, G, B / 16, A->coff, dmax + 1);
            MF_CUDA(cudaGetLastError());
            unsigned long long mb[2] = {0, 0};
            MF_CUDA(cudaMemcpyAsync(mb, dmax + 1, sizeof(mb), cudaMemcpyDeviceToHost, s));
            MF_CUDA(cudaStreamSynchronize(s));
            A->blob_cap = (int32_t)((mb[0] + 127) / 128 * 128);
            A->ecap = (int32_t)mb[1];
            // the warp-private decode buffers must leave room for the ring (TS_EBYTES of shared memory)
            if ((int64_t)A->ecap * 128 * (B / 32) > mfk::TS_EBYTES || A->ecap > 255) ts_failed = true;
            A->slot_bytes = (int32_t)((A->blob_cap + mfk::TS_GUARD + (int64_t)A->wcap * mfk::PV_SEG_BYTES + 127) / 128 * 128);
            dev_free(bsz, s); dev_free(boff, s); dev_free(btmp, s);
        }
        dev_free(nst, s);
        dev_free(dmax, s);
        dev_free(A->sslot, s); A->sslot = nullptr;
        dev_free(A->crec, s); A->crec = nullptr;
        dev_free(A->vstream, s); A->vstream = nullptr;
        dev_free(A->tr_vb, s); A->tr_vb = nullptr;
    }
    if (ts_failed) {
        // a stage of a single tile row gathers more than TS_WCAP column segments: this pattern
        // is not tile-synchronous enough -- convert again with the compact layout
        cudaEventDestroy(e0);
        cudaEventDestroy(e1);
        dev_free(cost, s); dev_free(cnt, s); dev_free(off, s); dev_free(tmp, s); dev_free(d_err, s);
        const int64_t coff = A->coff;
        destroy_tiles(A);
        A->coff = coff;
        mf_convert_opts o2 = o;
        o2.layout = 1;
        return convert_csr(n_rows, n_cols, nnz, rowptr, colidx, vals, o2, s, A);
    }
    std::vector<int32_t> ptr_h(G + 1);
    MF_CUDA(cudaMemcpyAsync(ptr_h.data(), A->plan_tr, (G + 1) * sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaEventRecord(e1, s));
    MF_CUDA(cudaStreamSynchronize(s));
    A->plan_rows_host = new int64_t[G + 1];
    for (int g = 0; g <= G; ++g) A->plan_rows_host[g] = std::min<int64_t>((int64_t)ptr_h[g] * TS, n_rows);
    float ms = 0;
    MF_CUDA(cudaEventElapsedTime(&ms, e0, e1));
    A->convert_ms = ms;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    dev_free(cost, s); dev_free(cnt, s); dev_free(off, s); dev_free(tmp, s); dev_free(d_err, s);

    // kernels launched: validate, COUNT, 12 scans x 3, FILL, cost, plan, deps
    A->convert_launches = (n_rows > 0 ? 1 : 0) + (ntr > 0 ? 2 + 1 : 0) + (NCNT + 1) * (ntr > 0 ? 3 : 0) + 2;
    A->canonical_bytes = nt * (4 + 4 + 1 + 1 + 8 + 8 + 8) + 16 + (ntr + 1) * 8 + A->rownum * 2 + nnz +
                         A->nval[0] * 8 + A->nval[1] * 4 + A->nval[2] * 2 + A->nval[3];
    A->kernel_bytes = (A->ts ? A->blob_bytes + A->nstg * (int64_t)sizeof(mfk::TsStage) : nslot * 2) +
                      (A->plane64 ? nslot * 8 : 0) + (A->plane32 ? nslot * 4 : 0) +
                      (A->plane16 ? nslot * 2 : 0) + (A->plane8 ? nslot : 0) + nt * 4 + (ntr + 1) * 8;
    return MF_OK;
}

}  // namespace mf
