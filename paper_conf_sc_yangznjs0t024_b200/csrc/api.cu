// api.cu -- the C ABI of libmf (include/mf.h): argument checks, handles, allocator hook,
// error strings.  Every compute step runs in the kernels of convert.cu / solver.cu /
// precond.cu / dist.cu (the multi-GPU calls are defined in dist.cu).
#include <cuda_runtime.h>

#include <mutex>
#include <unordered_map>
#include <string>

#include "mf_internal.cuh"

namespace mf {

static thread_local std::string g_last_error;
static std::mutex g_alloc_mu;
static void* (*g_alloc)(size_t, mf_stream, void*) = nullptr;
static void (*g_dealloc)(void*, mf_stream, void*) = nullptr;
static void* g_alloc_ctx = nullptr;

void set_error(const std::string& msg) { g_last_error = msg; }
mf_status fail(mf_status s, const std::string& msg) {
    set_error(msg);
    return s;
}

// every block remembers which allocator produced it (the hook can change between an allocation
// and its release: a block is always returned to its own allocator)
static std::unordered_map<void*, std::pair<void (*)(void*, mf_stream, void*), void*>> g_hooked;

void* dev_alloc(size_t bytes, cudaStream_t s) {
    {
        std::lock_guard<std::mutex> lk(g_alloc_mu);
        if (g_alloc) {
            void* p = g_alloc(bytes, (mf_stream)s, g_alloc_ctx);
            if (p) g_hooked[p] = {g_dealloc, g_alloc_ctx};
            return p;
        }
    }
    // stream-ordered allocator: keep freed blocks in the device's default pool across
    // synchronisations (release threshold = max) so repeated conversions / solves reuse them
    // instead of re-mapping physical memory each time
    static thread_local int pool_dev = -1;
    int dev = 0;
    if (cudaGetDevice(&dev) == cudaSuccess && dev != pool_dev) {
        cudaMemPool_t pool;
        if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
            unsigned long long thr = ~0ull;
            cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
        }
        cudaGetLastError();
        pool_dev = dev;
    }
    void* p = nullptr;
    if (cudaMallocAsync(&p, bytes, s) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    return p;
}

void dev_free(void* p, cudaStream_t s) {
    if (!p) return;
    {
        std::lock_guard<std::mutex> lk(g_alloc_mu);
        auto it = g_hooked.find(p);
        if (it != g_hooked.end()) {
            const auto h = it->second;
            g_hooked.erase(it);
            h.first(p, (mf_stream)s, h.second);
            return;
        }
    }
    cudaFreeAsync(p, s);
}

mf_status check_device(int* sm_count) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return fail(MF_ERR_CUDA, std::string("cudaGetDevice: ") + cudaGetErrorString(e));
    int major = 0, minor = 0;
    cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
    cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
    if (major != 10 || minor != 0)
        return fail(MF_ERR_UNSUPPORTED_DEVICE, "libmf is built for sm_100a (B200); device is sm_" +
                                                   std::to_string(major) + std::to_string(minor));
    if (sm_count) cudaDeviceGetAttribute(sm_count, cudaDevAttrMultiProcessorCount, dev);
    return MF_OK;
}

}  // namespace mf

using namespace mf;

extern "C" {

int32_t mf_abi_version(void) { return 2; }

const char* mf_last_error(void) { return g_last_error.c_str(); }

const char* mf_status_string(mf_status s) {
    switch (s) {
    case MF_OK: return "MF_OK";
    case MF_ERR_INVALID_ARG: return "MF_ERR_INVALID_ARG";
    case MF_ERR_UNSORTED_CSR: return "MF_ERR_UNSORTED_CSR";
    case MF_ERR_NONFINITE: return "MF_ERR_NONFINITE";
    case MF_ERR_OOM: return "MF_ERR_OOM";
    case MF_ERR_CUDA: return "MF_ERR_CUDA";
    case MF_ERR_NCCL: return "MF_ERR_NCCL";
    case MF_ERR_BREAKDOWN: return "MF_ERR_BREAKDOWN";
    case MF_ERR_ZERO_PIVOT: return "MF_ERR_ZERO_PIVOT";
    case MF_ERR_DEADLOCK: return "MF_ERR_DEADLOCK";
    case MF_ERR_UNSUPPORTED_DEVICE: return "MF_ERR_UNSUPPORTED_DEVICE";
    case MF_ERR_NOT_IMPLEMENTED: return "MF_ERR_NOT_IMPLEMENTED";
    case MF_ERR_UNSUPPORTED: return "MF_ERR_UNSUPPORTED";
    }
    return "MF_ERR_UNKNOWN";
}

void mf_default_convert_opts(mf_convert_opts* o) {
    if (!o) return;
    o->classify = 1;
    o->loss_tol = 1e-15;
    o->grid_ctas = 0;
    o->block_threads = 0;
    o->layout = 0;
}

void mf_default_solve_opts(mf_solve_opts* o) {
    if (!o) return;
    o->tol = 1e-10;
    o->max_iter = 1000;
    o->mode = MF_MODE_DYNAMIC_MIXED;
    o->switch_eps = -1.0;
    o->switch_absolute = 0;
    o->sticky = 0;
    o->range_guard = 1;
    o->M = nullptr;
    o->residual_history = nullptr;
    o->history_cap = 0;
    o->tile_level_counts = nullptr;
    o->level_counts_cap = 0;
    o->collect_stats = 0;
    o->watchdog_ms = 0;
    o->cg_variant = 0;
    o->dist_mode = 0;
}

mf_status mf_set_allocator(void* (*alloc)(size_t, mf_stream, void*), void (*dealloc)(void*, mf_stream, void*),
                           void* ctx) {
    if ((alloc == nullptr) != (dealloc == nullptr)) return fail(MF_ERR_INVALID_ARG, "alloc and dealloc go together");
    std::lock_guard<std::mutex> lk(g_alloc_mu);
    g_alloc = alloc;
    g_dealloc = dealloc;
    g_alloc_ctx = ctx;
    return MF_OK;
}

mf_status mf_tile_matrix_from_csr(int64_t n_rows, int64_t n_cols, int64_t nnz, const int64_t* rowptr,
                                  const int32_t* colidx, const double* vals, const mf_convert_opts* opts,
                                  mf_stream stream, mf_tile_matrix** out) {
    if (!out) return fail(MF_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    if (n_rows < 0 || n_cols < 0 || nnz < 0 || n_cols > INT32_MAX) return fail(MF_ERR_INVALID_ARG, "bad sizes");
    if (!rowptr || (nnz > 0 && (!colidx || !vals))) return fail(MF_ERR_INVALID_ARG, "NULL CSR array");
    mf_convert_opts o;
    mf_default_convert_opts(&o);
    if (opts) o = *opts;
    if (!(o.loss_tol >= 0)) return fail(MF_ERR_INVALID_ARG, "loss_tol must be >= 0");
    mf_tile_matrix* h = new (std::nothrow) mf_tile_matrix();
    if (!h) return fail(MF_ERR_OOM, "host allocation failed");
    mf_status st = convert_csr(n_rows, n_cols, nnz, rowptr, colidx, vals, o, (cudaStream_t)stream, &h->m);
    if (st != MF_OK) {
        destroy_tiles(&h->m);
        delete h;
        return st;
    }
    *out = h;
    return MF_OK;
}

mf_status mf_tile_matrix_destroy(mf_tile_matrix* A) {
    if (!A) return MF_OK;
    if (A->dist) dist_destroy(A->dist);
    destroy_tiles(&A->m);
    delete A;
    return MF_OK;
}

mf_status mf_tile_matrix_info(const mf_tile_matrix* A, mf_tile_info* o) {
    if (!A || !o) return fail(MF_ERR_INVALID_ARG, "NULL argument");
    const TileMatrix& m = A->m;
    o->n_rows = m.n_rows; o->n_cols = m.n_cols; o->nnz = m.nnz; o->T = TS;
    o->tilenum = m.tilenum; o->rownum = m.rownum; o->n_tile_rows = m.ntr;
    for (int q = 0; q < 4; ++q) { o->tiles_per_prec[q] = m.tiles_per_prec[q]; o->nval[q] = m.nval[q]; }
    o->max_tiles_per_tile_row = m.max_nt;
    o->slots = m.slots * TS;
    o->canonical_bytes = m.canonical_bytes;
    o->csr_bytes = (m.n_rows + 1) * 8 + m.nnz * 12;
    o->kernel_bytes = m.kernel_bytes;
    o->plan_G = m.G; o->plan_B = m.B;
    o->convert_ms = m.convert_ms;
    o->convert_launches = m.convert_launches;
    o->layout = m.ts ? 2 : 1;
    return MF_OK;
}

mf_status mf_tile_matrix_export(const mf_tile_matrix* A, mf_tile_export* h, mf_stream stream) {
    if (!A || !h) return fail(MF_ERR_INVALID_ARG, "NULL argument");
    const TileMatrix& m = A->m;
    cudaStream_t s = (cudaStream_t)stream;
    auto cp = [&](void* dst, const void* src, size_t bytes) -> mf_status {
        if (dst && bytes) MF_CUDA(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, s));
        return MF_OK;
    };
    const size_t nt = (size_t)m.tilenum;
    MF_TRY(cp(h->TileRowidx, m.TileRowidx, nt * 4));
    MF_TRY(cp(h->TileColidx, m.TileColidx, nt * 4));
    MF_TRY(cp(h->TilePrec, m.TilePrec, nt));
    MF_TRY(cp(h->Floor, m.Floor, nt));
    MF_TRY(cp(h->TileNnz, m.TileNnz, (nt + 1) * 8));
    MF_TRY(cp(h->Nonrow, m.Nonrow, (nt + 1) * 8));
    MF_TRY(cp(h->ValOff, m.ValOff, nt * 8));
    MF_TRY(cp(h->TileRowPtr, m.TileRowPtr, (size_t)(m.ntr + 1) * 8));
    MF_TRY(cp(h->RowIndex, m.RowIndex, (size_t)m.rownum));
    MF_TRY(cp(h->CsrRowptr, m.CsrRowptr, (size_t)m.rownum));
    MF_TRY(cp(h->CsrColidx, m.CsrColidx, (size_t)m.nnz));
    MF_TRY(cp(h->Val64, m.Val64, (size_t)m.nval[0] * 8));
    MF_TRY(cp(h->Val32, m.Val32, (size_t)m.nval[1] * 4));
    MF_TRY(cp(h->Val16, m.Val16, (size_t)m.nval[2] * 2));
    MF_TRY(cp(h->Val8, m.Val8, (size_t)m.nval[3]));
    MF_CUDA(cudaStreamSynchronize(s));
    if (h->PlanRows)
        for (int g = 0; g <= m.G; ++g) h->PlanRows[g] = m.plan_rows_host[g];
    return MF_OK;
}

mf_status mf_spmv(const mf_tile_matrix* A, const double* x, double* y, const uint8_t* level, int32_t range_guard,
                  int64_t* counts, mf_stream stream) {
    if (!A || (A->m.n_rows > 0 && (!x || !y))) return fail(MF_ERR_INVALID_ARG, "NULL argument");
    return run_spmv(A->m, x, y, level, range_guard, counts, (cudaStream_t)stream);
}

mf_status mf_levels(const double* v, int64_t n, const double* th, uint8_t* level, mf_stream stream) {
    if (n < 0 || (n > 0 && (!v || !level)) || !th) return fail(MF_ERR_INVALID_ARG, "bad argument");
    MF_TRY(check_device(nullptr));
    return run_levels(v, n, th, level, (cudaStream_t)stream);
}

mf_status mf_dot(const mf_tile_matrix* A, const double* u, const double* v, double* out, mf_stream stream) {
    if (!A || !out || (A->m.n_rows > 0 && (!u || !v))) return fail(MF_ERR_INVALID_ARG, "NULL argument");
    return run_dot(A->m, u, v, out, (cudaStream_t)stream);
}

mf_status mf_cg_update_xr(const mf_tile_matrix* A, double alpha, const double* p, const double* mu, double* x, double* r,
                          double* rr, mf_stream stream) {
    if (!A || !rr || (A->m.n_rows > 0 && (!p || !mu || !x || !r))) return fail(MF_ERR_INVALID_ARG, "NULL argument");
    return run_cg_xr(A->m, alpha, p, mu, x, r, rr, (cudaStream_t)stream);
}

mf_status mf_cg_update_p(const mf_tile_matrix* A, double beta, const double* r, double* p, mf_stream stream) {
    if (!A || (A->m.n_rows > 0 && (!r || !p))) return fail(MF_ERR_INVALID_ARG, "NULL argument");
    return run_cg_p(A->m, beta, r, p, (cudaStream_t)stream);
}

static mf_status solve_common(const mf_tile_matrix* A, bool bicg, const double* b, double* x,
                              const mf_solve_opts* opts, mf_solve_info* info, mf_stream stream) {
    if (!A || !info || (A->m.n_rows > 0 && (!b || !x))) return fail(MF_ERR_INVALID_ARG, "NULL argument");
    mf_solve_opts o;
    mf_default_solve_opts(&o);
    if (opts) o = *opts;
    if (!(o.tol >= 0) || o.max_iter < 0) return fail(MF_ERR_INVALID_ARG, "tol must be >= 0 and max_iter >= 0");
    if (o.mode < MF_MODE_FP64 || o.mode > MF_MODE_DYNAMIC_MIXED) return fail(MF_ERR_INVALID_ARG, "bad mode");
    *info = mf_solve_info{};
    return run_solve(A->m, bicg, b, x, o, info, (cudaStream_t)stream);
}

mf_status mf_cg_solve(const mf_tile_matrix* A, const double* b, double* x, const mf_solve_opts* opts,
                      mf_solve_info* info, mf_stream stream) {
    return solve_common(A, false, b, x, opts, info, stream);
}

mf_status mf_bicgstab_solve(const mf_tile_matrix* A, const double* b, double* x, const mf_solve_opts* opts,
                            mf_solve_info* info, mf_stream stream) {
    return solve_common(A, true, b, x, opts, info, stream);
}

}  // extern "C"
