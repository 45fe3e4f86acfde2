// precond.cu -- ILU(0) preconditioning (reading R20).
//
// Setup (host, C++, once per matrix: "preprocessing"): the stored (TilePrec) values are read
// back from the canonical tile arrays into a row-major CSR, factorised with ILU(0) in the IKJ
// order (a_ik /= a_kk, then a_ij -= a_ik * a_kj for the j > k present in row i, k ascending,
// each update one fma), and split into L (unit lower, strict part) and U (upper with
// diagonal).  Every a_ij receives its updates in ascending k, so the factors are bit-identical
// to any implementation of the same definition.
//
// Apply (device): z = U^-1 (L^-1 r) by sync-free triangular solves inside the persistent
// PCG / PBiCGSTAB kernels (solver.cu: sptrsv_chunked) or by mf_precond_apply.  Row i is one
// fma chain in ascending column order: y_i = r_i - sum l_ik y_k ; z_i = (y_i - sum u_ik z_k) / u_ii.
#include <cuda_runtime.h>
#include <string.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <vector>

#include "mf_internal.cuh"
#include "precond.cuh"

namespace mf {
namespace {

// exact decoders of the stored formats (host)
double half_bits_to_double(uint16_t b) {
    const int s = b >> 15, e = (b >> 10) & 0x1F, m = b & 0x3FF;
    double v;
    if (e == 0) v = std::ldexp((double)m, -24);
    else if (e == 31) v = m ? NAN : INFINITY;
    else v = std::ldexp((double)(m | 0x400), e - 25);
    return s ? -v : v;
}
double e4m3_bits_to_double(uint8_t b) {
    const int s = b >> 7, e = (b >> 3) & 0xF, m = b & 7;
    double v;
    if (e == 15 && m == 7) v = NAN;
    else if (e == 0) v = std::ldexp((double)m, -9);
    else v = std::ldexp((double)(m | 8), e - 10);
    return s ? -v : v;
}

struct HostCSR {
    int64_t n = 0;
    std::vector<int64_t> rp;
    std::vector<int32_t> ci;
    std::vector<double> v;
};

mf_status stored_csr(const TileMatrix& A, cudaStream_t s, HostCSR& out) {
    const int64_t nt = A.tilenum, nr = A.rownum;
    std::vector<int32_t> trow(nt), tcol(nt);
    std::vector<uint8_t> prec(nt), rowidx(nr), rowptr(nr), colidx(A.nnz);
    std::vector<int64_t> tnnz(nt + 1), nonrow(nt + 1), voff(nt);
    std::vector<double> v64(A.nval[0]);
    std::vector<float> v32(A.nval[1]);
    std::vector<uint16_t> v16(A.nval[2]);
    std::vector<uint8_t> v8(A.nval[3]);
    auto cp = [&](void* d, const void* src, size_t bytes) -> mf_status {
        if (bytes) MF_CUDA(cudaMemcpyAsync(d, src, bytes, cudaMemcpyDeviceToHost, s));
        return MF_OK;
    };
    MF_TRY(cp(trow.data(), A.TileRowidx, nt * 4));
    MF_TRY(cp(tcol.data(), A.TileColidx, nt * 4));
    MF_TRY(cp(prec.data(), A.TilePrec, nt));
    MF_TRY(cp(tnnz.data(), A.TileNnz, (nt + 1) * 8));
    MF_TRY(cp(nonrow.data(), A.Nonrow, (nt + 1) * 8));
    MF_TRY(cp(voff.data(), A.ValOff, nt * 8));
    MF_TRY(cp(rowidx.data(), A.RowIndex, nr));
    MF_TRY(cp(rowptr.data(), A.CsrRowptr, nr));
    MF_TRY(cp(colidx.data(), A.CsrColidx, A.nnz));
    MF_TRY(cp(v64.data(), A.Val64, A.nval[0] * 8));
    MF_TRY(cp(v32.data(), A.Val32, A.nval[1] * 4));
    MF_TRY(cp(v16.data(), A.Val16, A.nval[2] * 2));
    MF_TRY(cp(v8.data(), A.Val8, A.nval[3]));
    MF_CUDA(cudaStreamSynchronize(s));
    const int64_t n = A.n_rows;
    out.n = n;
    out.rp.assign(n + 1, 0);
    for (int64_t t = 0; t < nt; ++t)
        for (int64_t r = nonrow[t]; r < nonrow[t + 1]; ++r) {
            const int64_t end = (r + 1 < nonrow[t + 1]) ? rowptr[r + 1] : tnnz[t + 1] - tnnz[t];
            out.rp[(int64_t)trow[t] * TS + rowidx[r] + 1] += end - rowptr[r];
        }
    for (int64_t i = 0; i < n; ++i) out.rp[i + 1] += out.rp[i];
    out.ci.resize(A.nnz);
    out.v.resize(A.nnz);
    std::vector<int64_t> fill(out.rp.begin(), out.rp.end() - 1);
    // tiles of a tile row are in ascending column, entries of a row in a tile ascending:
    // appending in tile order yields ascending columns per row
    for (int64_t t = 0; t < nt; ++t)
        for (int64_t r = nonrow[t]; r < nonrow[t + 1]; ++r) {
            const int64_t row = (int64_t)trow[t] * TS + rowidx[r];
            const int64_t end = (r + 1 < nonrow[t + 1]) ? rowptr[r + 1] : tnnz[t + 1] - tnnz[t];
            for (int64_t a = rowptr[r]; a < end; ++a) {
                const int64_t o = voff[t] + a;
                double val;
                switch (prec[t]) {
                case 0: val = v64[o]; break;
                case 1: val = (double)v32[o]; break;
                case 2: val = half_bits_to_double(v16[o]); break;
                default: val = e4m3_bits_to_double(v8[o]); break;
                }
                out.ci[fill[row]] = tcol[t] * TS + colidx[tnnz[t] + a];
                out.v[fill[row]] = val;
                fill[row]++;
            }
        }
    return MF_OK;
}

// ILU(0), IKJ order with a column marker (see the file header)
mf_status ilu0(HostCSR& M, std::vector<int64_t>& diag) {
    const int64_t n = M.n;
    diag.assign(n, -1);
    for (int64_t i = 0; i < n; ++i)
        for (int64_t k = M.rp[i]; k < M.rp[i + 1]; ++k)
            if (M.ci[k] == i) diag[i] = k;
    for (int64_t i = 0; i < n; ++i)
        if (diag[i] < 0) return fail(MF_ERR_ZERO_PIVOT, "ILU(0): row " + std::to_string(i) + " has no diagonal entry");
    std::vector<int64_t> pos(n, -1);
    for (int64_t i = 0; i < n; ++i) {
        for (int64_t q = M.rp[i]; q < M.rp[i + 1]; ++q) pos[M.ci[q]] = q;
        for (int64_t kk = M.rp[i]; kk < M.rp[i + 1] && M.ci[kk] < i; ++kk) {
            const int64_t k = M.ci[kk];
            const double akk = M.v[diag[k]];
            if (akk == 0.0) return fail(MF_ERR_ZERO_PIVOT, "ILU(0): zero pivot in row " + std::to_string(k));
            M.v[kk] = M.v[kk] / akk;
            const double aik = M.v[kk];
            for (int64_t q = diag[k] + 1; q < M.rp[k + 1]; ++q) {
                const int64_t p = pos[M.ci[q]];
                if (p >= 0) M.v[p] = std::fma(-aik, M.v[q], M.v[p]);
            }
        }
        for (int64_t q = M.rp[i]; q < M.rp[i + 1]; ++q) pos[M.ci[q]] = -1;
        if (M.v[diag[i]] == 0.0) return fail(MF_ERR_ZERO_PIVOT, "ILU(0): zero pivot in row " + std::to_string(i));
    }
    return MF_OK;
}

// standalone apply: one sync-free triangular solve per launch (any grid size is deadlock-free)
template <bool FWD>
__global__ void __launch_bounds__(256) sptrsv_kernel(TriCSR T, const double* __restrict__ diag, int64_t n,
                                                     const double* in, double* out, unsigned* flags, unsigned flag_val,
                                                     unsigned wait_val, unsigned long long* ctr, int* abort_flag) {
    __shared__ double ys[256];
    __shared__ int ready[256];
    __shared__ long long chunk;
    mfk::sptrsv_chunked<FWD, false>(T.rp, T.ci, T.v, diag, n, in, out, flags, flag_val, wait_val, ctr, 0ull, ys, ready, &chunk,
                                    abort_flag, 20ull * 1000000000ull);
}

// one-CTA sweep triangular solve (precond.cuh sweep_solve): deep dependency DAGs
template <bool FWD>
__global__ void __launch_bounds__(32 * mfk::SW_WARPS) sweep_kernel(TriCSR T, const double* __restrict__ diag, int64_t n, const double* in,
                                                   double* out, int* abort_flag) {
    extern __shared__ __align__(16) unsigned char sw_smem[];
    if (!mfk::sweep_solve<FWD, false>(T.rp, T.ci, T.v, diag, n, in, out, sw_smem, abort_flag, 20ull * 1000000000ull) &&
        threadIdx.x == 0)
        atomicExch(abort_flag, 1);
}

// levels of the dependency DAG of a triangular factor (host): longest path, in solve order
int64_t dag_depth(int64_t n, const std::vector<int64_t>& rp, const std::vector<int32_t>& ci, bool fwd) {
    std::vector<int32_t> lev(n, 0);
    int64_t mx = n > 0 ? 1 : 0;
    for (int64_t p = 0; p < n; ++p) {
        const int64_t i = fwd ? p : n - 1 - p;
        int32_t l = 0;
        for (int64_t q = rp[i]; q < rp[i + 1]; ++q) l = std::max(l, lev[ci[q]] + 1);
        lev[i] = l;
        mx = std::max<int64_t>(mx, l + 1);
    }
    return mx;
}

__global__ void __launch_bounds__(256) rb_square_kernel(const int64_t* __restrict__ rp, const int32_t* __restrict__ ci,
                                                        const double* __restrict__ val, int64_t r0, int64_t r1, double* v) {
    mfk::rb_square_rows(rp, ci, val, r0, r1, v, (int64_t)blockIdx.x * blockDim.x + threadIdx.x, (int64_t)gridDim.x * blockDim.x);
}

// Recursive block partition of a factor (precond.cuh RbNode; oracle rb_lower / rb_upper).
// M: the ILU(0) factors in one CSR (columns ascending per row), diag[i] = position of a_ii.
struct RbHost {
    std::vector<RbNode> nodes;
    std::vector<int64_t> rp;
    std::vector<int32_t> ci;
    std::vector<double> v;
    int nleaves = 0;
};
int64_t rb_mid(int64_t lo, int64_t hi) { return lo + 16 * ((hi - lo) / 32); }
// one node: rows [r0, r1), entries of row i with column in [c0, c1) (and, for leaves, in the
// strict triangle), columns stored minus `cshift`
void rb_emit(RbHost& T, const HostCSR& M, const std::vector<int64_t>& diag, bool lower, bool leaf, int64_t r0, int64_t r1,
             int64_t c0, int64_t c1, int64_t cshift) {
    RbNode nd{r0, r1, (int64_t)T.rp.size(), leaf ? 1 : 0, leaf ? T.nleaves++ : -1};
    T.nodes.push_back(nd);
    for (int64_t i = r0; i < r1; ++i) {
        T.rp.push_back((int64_t)T.ci.size());
        const int64_t q0 = lower ? M.rp[i] : diag[i] + 1, q1 = lower ? diag[i] : M.rp[i + 1];
        for (int64_t q = q0; q < q1; ++q) {
            const int64_t c = M.ci[q];
            if (c >= c0 && c < c1) { T.ci.push_back((int32_t)(c - cshift)); T.v.push_back(M.v[q]); }
        }
    }
    T.rp.push_back((int64_t)T.ci.size());
}
void rb_lower(RbHost& T, const HostCSR& M, const std::vector<int64_t>& diag, int64_t lo, int64_t hi, int depth) {
    if (depth == 0 || hi - lo < 32) { rb_emit(T, M, diag, true, true, lo, hi, lo, hi, lo); return; }
    const int64_t mid = rb_mid(lo, hi);
    rb_lower(T, M, diag, lo, mid, depth - 1);
    rb_emit(T, M, diag, true, false, mid, hi, lo, mid, 0);
    rb_lower(T, M, diag, mid, hi, depth - 1);
}
void rb_upper(RbHost& T, const HostCSR& M, const std::vector<int64_t>& diag, int64_t lo, int64_t hi, int depth) {
    if (depth == 0 || hi - lo < 32) { rb_emit(T, M, diag, false, true, lo, hi, lo, hi, lo); return; }
    const int64_t mid = rb_mid(lo, hi);
    rb_upper(T, M, diag, mid, hi, depth - 1);
    rb_emit(T, M, diag, false, false, lo, mid, mid, hi, 0);
    rb_upper(T, M, diag, lo, mid, depth - 1);
}

template <class T>
mf_status upload(T** d, const std::vector<T>& h, cudaStream_t s) {
    MF_TRY(alloc(d, h.size(), s));
    if (!h.empty()) MF_CUDA(cudaMemcpyAsync(*d, h.data(), h.size() * sizeof(T), cudaMemcpyHostToDevice, s));
    return MF_OK;
}

}  // namespace

mf_status run_precond_apply(Precond& P, const double* r, double* z, cudaStream_t s) {
    if (P.n == 0) return MF_OK;
    int dev = 0, sms = 0;
    MF_CUDA(cudaGetDevice(&dev));
    MF_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    if (P.epoch >= 0x7FFFFFF0u) {   // flag values wrap: start over
        MF_CUDA(cudaMemsetAsync(P.flags, 0, (P.n + 1) * sizeof(unsigned), s));
        P.epoch = 0;
    }
    const unsigned e = ++P.epoch;
    const int blocks = (int)std::min<int64_t>((P.n + 255) / 256, (int64_t)sms * 8);
    if (P.rb_depth > 0) {
        // the multi-kernel recursive block SpTRSV: one launch per node, in place on y
        const int nctr = P.Lrb.nleaves + P.Urb.nleaves;
        MF_CUDA(cudaMemsetAsync(P.ctr, 0, (size_t)(nctr + 1) * sizeof(unsigned long long), s));
        int* abort_flag = reinterpret_cast<int*>(P.ctr + nctr);
        MF_CUDA(cudaMemcpyAsync(P.y, r, P.n * sizeof(double), cudaMemcpyDeviceToDevice, s));
        for (int pass = 0; pass < 2; ++pass) {
            const RbTree& T = pass == 0 ? P.Lrb : P.Urb;
            for (const RbNode& nd : T.h) {
                const int64_t m = nd.r1 - nd.r0;
                const int nb = (int)std::max<int64_t>(1, std::min<int64_t>((m + 255) / 256, (int64_t)sms * 8));
                if (nd.leaf && P.sweep) {
                    const size_t sb = mfk::sweep_smem_bytes();
                    if (pass == 0)
                        sweep_kernel<true><<<1, 32 * mfk::SW_WARPS, sb, s>>>(TriCSR{T.rp + nd.rp_off, T.ci, T.v}, nullptr, m, P.y + nd.r0,
                                                              P.y + nd.r0, abort_flag);
                    else
                        sweep_kernel<false><<<1, 32 * mfk::SW_WARPS, sb, s>>>(TriCSR{T.rp + nd.rp_off, T.ci, T.v}, P.udiag + nd.r0, m,
                                                               P.y + nd.r0, P.y + nd.r0, abort_flag);
                } else if (nd.leaf) {
                    unsigned long long* c = P.ctr + (pass == 0 ? 0 : P.Lrb.nleaves) + nd.leaf_idx;
                    if (pass == 0)
                        sptrsv_kernel<true><<<nb, 256, 0, s>>>(TriCSR{T.rp + nd.rp_off, T.ci, T.v}, nullptr, m, P.y + nd.r0,
                                                               P.y + nd.r0, P.flags + nd.r0, 2 * e + 1, 0u, c, abort_flag);
                    else
                        sptrsv_kernel<false><<<nb, 256, 0, s>>>(TriCSR{T.rp + nd.rp_off, T.ci, T.v}, P.udiag + nd.r0, m,
                                                                P.y + nd.r0, P.y + nd.r0, P.flags + nd.r0, 2 * e + 2, 0u, c,
                                                                abort_flag);
                } else {
                    rb_square_kernel<<<nb, 256, 0, s>>>(T.rp + nd.rp_off, T.ci, T.v, nd.r0, nd.r1, P.y);
                }
            }
        }
        MF_CUDA(cudaGetLastError());
        MF_CUDA(cudaMemcpyAsync(z, P.y, P.n * sizeof(double), cudaMemcpyDeviceToDevice, s));
        int ab = 0;
        MF_CUDA(cudaMemcpyAsync(&ab, abort_flag, sizeof(int), cudaMemcpyDeviceToHost, s));
        MF_CUDA(cudaStreamSynchronize(s));
        if (ab) return fail(MF_ERR_DEADLOCK, "triangular-solve watchdog expired");
        return MF_OK;
    }
    MF_CUDA(cudaMemsetAsync(P.ctr, 0, 3 * sizeof(unsigned long long), s));
    int* abort_flag = reinterpret_cast<int*>(P.ctr + 2);
    if (P.sweep) {
        const size_t sb = mfk::sweep_smem_bytes();
        int nthr = 32 * mfk::SW_WARPS;
        if (const char* ev = getenv("MF_SWEEP_WARPS")) nthr = 32 * std::max(1, std::min(mfk::SW_WARPS, atoi(ev)));
        if (const char* ev = getenv("MF_SWEEP_SLEEP")) {
            const int v = atoi(ev);
            MF_CUDA(cudaMemcpyToSymbolAsync(mfk::g_sweep_sleep_ns, &v, sizeof(int), 0, cudaMemcpyHostToDevice, s));
        }
        long long* dbg = nullptr;
        const int64_t nwin = (P.n + 31) / 32;
        const bool want_dbg = getenv("MF_SWEEP_DBG") != nullptr;
        if (want_dbg) {
            MF_CUDA(cudaMalloc(&dbg, (size_t)nwin * 5 * 8 * 2));
            MF_CUDA(cudaMemcpyToSymbolAsync(mfk::g_sweep_dbg, &dbg, sizeof(dbg), 0, cudaMemcpyHostToDevice, s));
        }
        sweep_kernel<true><<<1, nthr, sb, s>>>(P.L, nullptr, P.n, r, P.y, abort_flag);
        if (want_dbg) {
            long long* d2 = dbg + nwin * 5;
            MF_CUDA(cudaMemcpyToSymbolAsync(mfk::g_sweep_dbg, &d2, sizeof(d2), 0, cudaMemcpyHostToDevice, s));
        }
        sweep_kernel<false><<<1, nthr, sb, s>>>(P.U, P.udiag, P.n, P.y, z, abort_flag);
        if (want_dbg) {
            std::vector<long long> h((size_t)nwin * 10);
            MF_CUDA(cudaMemcpyAsync(h.data(), dbg, h.size() * 8, cudaMemcpyDeviceToHost, s));
            MF_CUDA(cudaStreamSynchronize(s));
            for (int tri = 0; tri < 2; ++tri) {
                const long long* d = h.data() + (size_t)tri * nwin * 5;
                // per window: [0] before the previous-window wait, [1] wait returned, [2] sweep start,
                // [3] sweep end, [4] signal
                double pre = 0, hand = 0, prev = 0, sw = 0, tail = 0, step = 0;
                int64_t cntw = 0;
                for (int64_t w = 1; w < nwin; ++w) {
                    const long long sig_prev = d[(w - 1) * 5 + 4];
                    hand += (double)(d[w * 5 + 1] - sig_prev);        // previous signal -> wait returns
                    pre += (double)(d[w * 5] > sig_prev ? d[w * 5] - sig_prev : 0);   // arrived late at the wait
                    prev += (double)(d[w * 5 + 2] - d[w * 5 + 1]);
                    sw += (double)(d[w * 5 + 3] - d[w * 5 + 2]);
                    tail += (double)(d[w * 5 + 4] - d[w * 5 + 3]);
                    step += (double)(d[w * 5 + 4] - sig_prev);
                    ++cntw;
                }
                fprintf(stderr, "sweep %s: cycles per window: signal-to-signal %.0f = signal->wait-return %.0f (of which the warp "
                        "arrived late %.0f) + previous-window entries %.0f + sweep %.0f + signalling %.0f\n",
                        tri ? "U" : "L", step / cntw, hand / cntw, pre / cntw, prev / cntw, sw / cntw, tail / cntw);
            }
            MF_CUDA(cudaFree(dbg));
            long long* z0 = nullptr;
            MF_CUDA(cudaMemcpyToSymbolAsync(mfk::g_sweep_dbg, &z0, sizeof(z0), 0, cudaMemcpyHostToDevice, s));
        }
        MF_CUDA(cudaGetLastError());
        int ab = 0;
        MF_CUDA(cudaMemcpyAsync(&ab, abort_flag, sizeof(int), cudaMemcpyDeviceToHost, s));
        MF_CUDA(cudaStreamSynchronize(s));
        if (ab) return fail(MF_ERR_DEADLOCK, "triangular-solve watchdog expired");
        return MF_OK;
    }
    sptrsv_kernel<true><<<blocks, 256, 0, s>>>(P.L, nullptr, P.n, r, P.y, P.flags, 2 * e + 1, 0u, P.ctr, abort_flag);
    sptrsv_kernel<false><<<blocks, 256, 0, s>>>(P.U, P.udiag, P.n, P.y, z, P.flags, 2 * e + 2, 2 * e + 1, P.ctr + 1, abort_flag);
    MF_CUDA(cudaGetLastError());
    int ab = 0;
    MF_CUDA(cudaMemcpyAsync(&ab, abort_flag, sizeof(int), cudaMemcpyDeviceToHost, s));
    MF_CUDA(cudaStreamSynchronize(s));
    if (ab) return fail(MF_ERR_DEADLOCK, "triangular-solve watchdog expired");
    return MF_OK;
}

void destroy_precond(Precond* P) {
    cudaStream_t s = P->owner_stream;
    void* ptrs[] = {P->L.rp, P->L.ci, P->L.v, P->U.rp, P->U.ci, P->U.v, P->udiag, P->flags, P->ctr, P->y, P->z,
                    P->Lrb.nodes, P->Lrb.rp, P->Lrb.ci, P->Lrb.v, P->Urb.nodes, P->Urb.rp, P->Urb.ci, P->Urb.v};
    for (void* p : ptrs) if (p) dev_free(p, s);
    *P = Precond();
}

mf_status build_precond(const TileMatrix& A, int rb_depth, cudaStream_t s, Precond* P) {
    if (A.n_rows != A.n_cols) return fail(MF_ERR_INVALID_ARG, "ILU(0) needs a square matrix");
    if (rb_depth < 0 || rb_depth > 24) return fail(MF_ERR_INVALID_ARG, "rb_depth must be in [0, 24]");
    P->owner_stream = s;
    P->n = A.n_rows;
    HostCSR M;
    MF_TRY(stored_csr(A, s, M));
    std::vector<int64_t> diag;
    MF_TRY(ilu0(M, diag));
    const int64_t n = M.n;
    std::vector<int64_t> lrp(n + 1, 0), urp(n + 1, 0);
    std::vector<int32_t> lci, uci;
    std::vector<double> lv, uv, ud(n);
    for (int64_t i = 0; i < n; ++i) {
        for (int64_t q = M.rp[i]; q < diag[i]; ++q) { lci.push_back(M.ci[q]); lv.push_back(M.v[q]); }
        for (int64_t q = diag[i] + 1; q < M.rp[i + 1]; ++q) { uci.push_back(M.ci[q]); uv.push_back(M.v[q]); }
        ud[i] = M.v[diag[i]];
        lrp[i + 1] = (int64_t)lci.size();
        urp[i + 1] = (int64_t)uci.size();
    }
    MF_TRY(upload(&P->L.rp, lrp, s)); MF_TRY(upload(&P->L.ci, lci, s)); MF_TRY(upload(&P->L.v, lv, s));
    MF_TRY(upload(&P->U.rp, urp, s)); MF_TRY(upload(&P->U.ci, uci, s)); MF_TRY(upload(&P->U.v, uv, s));
    MF_TRY(upload(&P->udiag, ud, s));
    int nctr = 4;
    P->rb_depth = rb_depth;
    // one-CTA sweep when the DAG is too deep for grid-wide parallelism (< 64 rows per level)
    P->depth_l = dag_depth(n, lrp, lci, true);
    P->depth_u = dag_depth(n, urp, uci, false);
    P->sweep = n > 0 && (double)n / (double)std::max(P->depth_l, P->depth_u) < 64.0 ? 1 : 0;
    if (const char* ev = getenv("MF_SPTRSV_SWEEP")) P->sweep = atoi(ev) != 0;   // experiments / tests
    if (P->sweep) {
        const int sb = (int)mfk::sweep_smem_bytes();
        MF_CUDA(cudaFuncSetAttribute((const void*)sweep_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sb));
        MF_CUDA(cudaFuncSetAttribute((const void*)sweep_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sb));
    }
    if (rb_depth > 0) {
        RbHost HL, HU;
        rb_lower(HL, M, diag, 0, n, rb_depth);
        rb_upper(HU, M, diag, 0, n, rb_depth);
        for (int k = 0; k < 2; ++k) {
            RbHost& H = k == 0 ? HL : HU;
            RbTree& T = k == 0 ? P->Lrb : P->Urb;
            MF_TRY(upload(&T.nodes, H.nodes, s));
            MF_TRY(upload(&T.rp, H.rp, s));
            MF_TRY(upload(&T.ci, H.ci, s));
            MF_TRY(upload(&T.v, H.v, s));
            T.h = H.nodes;
            T.nleaves = H.nleaves;
        }
        nctr = std::max(nctr, HL.nleaves + HU.nleaves + 1);
    }
    MF_TRY(alloc(&P->flags, (size_t)n + 1, s));
    MF_TRY(alloc(&P->ctr, (size_t)nctr, s));
    MF_TRY(alloc(&P->y, n, s));
    MF_TRY(alloc(&P->z, n, s));
    MF_CUDA(cudaMemsetAsync(P->flags, 0, (n + 1) * sizeof(unsigned), s));
    MF_CUDA(cudaMemsetAsync(P->ctr, 0, (size_t)nctr * sizeof(unsigned long long), s));
    MF_CUDA(cudaStreamSynchronize(s));
    P->nnz_l = (int64_t)lv.size();
    P->nnz_u = (int64_t)uv.size();
    P->epoch = 0;
    P->grabs = 0;
    return MF_OK;
}

}  // namespace mf

using namespace mf;

extern "C" {

mf_status mf_precond_create(const mf_tile_matrix* A, mf_precond_kind kind, mf_stream stream, mf_precond** out) {
    mf_precond_opts o{kind, 0, 0};
    return mf_precond_create_ex(A, &o, stream, out);
}

mf_status mf_precond_create_ex(const mf_tile_matrix* A, const mf_precond_opts* opts, mf_stream stream, mf_precond** out) {
    if (!A || !out || !opts) return fail(MF_ERR_INVALID_ARG, "NULL argument");
    *out = nullptr;
    const mf_precond_kind kind = opts->kind;
    if (kind != MF_PRECOND_ILU0) return fail(MF_ERR_INVALID_ARG, "only MF_PRECOND_ILU0 is defined (P:164)");
    if (opts->sptrsv != MF_SPTRSV_SYNC_FREE && opts->sptrsv != MF_SPTRSV_RECURSIVE_BLOCK)
        return fail(MF_ERR_INVALID_ARG, "sptrsv must be MF_SPTRSV_SYNC_FREE or MF_SPTRSV_RECURSIVE_BLOCK");
    int depth = 0;
    if (opts->sptrsv == MF_SPTRSV_RECURSIVE_BLOCK) {
        depth = opts->rb_depth;
        if (depth == 0) {   // auto: leaves of about 2^14 rows, at least one split
            depth = 1;
            while (depth < 12 && (A->m.n_rows >> (depth + 1)) >= 16384) ++depth;
        }
        if (depth < 1 || depth > 24) return fail(MF_ERR_INVALID_ARG, "rb_depth must be in [1, 24] (0 = auto)");
    }
    MF_TRY(check_device(nullptr));
    mf_precond* h = new (std::nothrow) mf_precond();
    if (!h) return fail(MF_ERR_OOM, "host allocation failed");
    mf_status st = build_precond(A->m, depth, (cudaStream_t)stream, &h->p);
    if (st != MF_OK) {
        destroy_precond(&h->p);
        delete h;
        return st;
    }
    *out = h;
    return MF_OK;
}

mf_status mf_precond_info(const mf_precond* M, mf_precond_stats* out) {
    if (!M || !out) return fail(MF_ERR_INVALID_ARG, "NULL argument");
    out->rb_depth = M->p.rb_depth;
    out->nodes_l = (int32_t)M->p.Lrb.h.size();
    out->nodes_u = (int32_t)M->p.Urb.h.size();
    out->sweep = M->p.sweep;
    out->depth_l = M->p.depth_l;
    out->depth_u = M->p.depth_u;
    out->nnz_l = M->p.nnz_l;
    out->nnz_u = M->p.nnz_u;
    return MF_OK;
}

mf_status mf_precond_destroy(mf_precond* M) {
    if (!M) return MF_OK;
    destroy_precond(&M->p);
    delete M;
    return MF_OK;
}

mf_status mf_precond_apply(const mf_precond* M, const double* r, double* z, mf_stream stream) {
    if (!M || (M->p.n > 0 && (!r || !z))) return fail(MF_ERR_INVALID_ARG, "NULL argument");
    return run_precond_apply(const_cast<Precond&>(M->p), r, z, (cudaStream_t)stream);
}

}  // extern "C"
