// mf_internal.cuh -- internal declarations of libmf (B200 / sm_100a).
// Nothing here is shared with oracle/; the two sides are independent implementations.
#pragma once

#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_fp8.h>
#include <stdint.h>

#include <string>

#include "mf.h"

namespace mf {

// ------------------------------------------------------------------ errors
void set_error(const std::string& msg);
mf_status fail(mf_status s, const std::string& msg);

#define MF_CUDA(call)                                                                   \
    do {                                                                                \
        cudaError_t e_ = (call);                                                        \
        if (e_ != cudaSuccess)                                                          \
            return ::mf::fail(MF_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
    } while (0)

#define MF_TRY(call)                                                                    \
    do {                                                                                \
        mf_status s_ = (call);                                                          \
        if (s_ != MF_OK) return s_;                                                     \
    } while (0)

// ------------------------------------------------------------------ memory
void* dev_alloc(size_t bytes, cudaStream_t s);
void dev_free(void* p, cudaStream_t s);

template <class T>
mf_status alloc(T** p, size_t count, cudaStream_t s) {
    *p = nullptr;
    if (count == 0) return MF_OK;
    if (count > SIZE_MAX / sizeof(T)) return fail(MF_ERR_OOM, "device allocation size overflows size_t");
    *p = static_cast<T*>(dev_alloc(count * sizeof(T), s));
    if (!*p) return fail(MF_ERR_OOM, "device allocation of " + std::to_string(count * sizeof(T)) + " bytes failed");
    return MF_OK;
}

mf_status check_device(int* sm_count);

// ------------------------------------------------------------------ the tile matrix handle
constexpr int TS = 16;               // tile size
constexpr int MAX_TILES_PER_TR = 4096;   // 12-bit tile index in the kernel-layout slot word
constexpr uint16_t SLOT_PAD = 0xFFFF;

struct TileMatrix {
    int64_t n_rows = 0, n_cols = 0, nnz = 0;
    int64_t tilenum = 0, rownum = 0, ntr = 0;
    int64_t nval[4] = {0, 0, 0, 0};
    int64_t tiles_per_prec[4] = {0, 0, 0, 0};
    int64_t slots = 0;               // slice columns (each 16 slots wide)
    int64_t max_nt = 0;              // max tiles in one tile row
    int64_t max_w = 0;               // max slice columns of one tile row (kernel layout)
    double convert_ms = 0;
    int64_t convert_launches = 0;
    // canonical arrays (device)
    int32_t *TileRowidx = nullptr, *TileColidx = nullptr;
    uint8_t *TilePrec = nullptr, *Floor = nullptr;
    int64_t *TileNnz = nullptr, *Nonrow = nullptr, *ValOff = nullptr, *TileRowPtr = nullptr;
    uint8_t *RowIndex = nullptr, *CsrRowptr = nullptr, *CsrColidx = nullptr;
    double* Val64 = nullptr;
    float* Val32 = nullptr;
    uint16_t* Val16 = nullptr;
    uint8_t* Val8 = nullptr;
    // kernel layout (device): SELL-16 slices, one per tile row, columns in ascending global
    // column per row; slot word = (tile index in tile row << 4) | local column.
    int64_t* tr_slot = nullptr;      // [ntr+1] first slice column of each tile row
    uint32_t* tile_info = nullptr;   // [tilenum] (TileColidx << 4) | (Floor << 2) | TilePrec
    int ts = 0;                      // 1: tile-synchronous slices
    uint16_t* sidx = nullptr;        // compact: [16*slots] (tile index in tile row << 4) | local column
    uint8_t* sslot = nullptr;        // tile-synchronous: [16*slots] local column (0 on padding)
    uint2* crec = nullptr;           // tile-synchronous: [slots] static column record (see kernels.cuh)
    int64_t* tr_vb = nullptr;        // tile-synchronous: [ntr+1] value-byte start of each tile row in vstream
    uint8_t* vstream = nullptr;      // tile-synchronous: values at TilePrec, 16*size(TilePrec) bytes per slice column
    int64_t vbytes = 0;              // bytes of vstream
    uint8_t* blob = nullptr;         // tile-synchronous: per-stage blobs streamed by the TMA pipeline
    int64_t blob_bytes = 0;
    void* stg = nullptr;             // tile-synchronous: mfk::TsStage per stage of every CTA
    int32_t* stg_ptr = nullptr;      // device [G+1]
    int64_t nstg = 0;
    int32_t blob_cap = 0;            // tile-synchronous: largest stage blob (bytes, 128-aligned)
    int32_t wcap = 0;                // tile-synchronous: largest stage window (column segments)
    int32_t slot_bytes = 0;          // tile-synchronous: ring slot = blob_cap + wcap * 144 (128-aligned)
    int32_t ecap = 0;                // tile-synchronous: most columns one warp decodes per stage
    // compact layout only: value planes RNE_q(stored value) per slot
    double* plane64 = nullptr;       // [16*slots] value at FP64 (tiles with TilePrec == FP64)
    float* plane32 = nullptr;        // value rounded to FP32 (tiles with TilePrec <= FP32)
    __half* plane16 = nullptr;       // ... FP16
    uint8_t* plane8 = nullptr;       // ... E4M3
    // launch plan: G CTAs x B threads, CTA g owns tile rows [plan_tr[g], plan_tr[g+1])
    int32_t G = 0, B = 0;
    int32_t* plan_tr = nullptr;      // device [G+1]
    int32_t* dep_lo = nullptr;       // device [G] first CTA whose rows this CTA's tiles gather
    int32_t* dep_hi = nullptr;       // device [G]
    int32_t* seg_lo = nullptr;       // device [G] first column segment gathered by CTA g
    int32_t* seg_hi = nullptr;       // device [G] last column segment gathered (-1: none)
    int64_t* plan_rows_host = nullptr;  // host [G+1]
    // byte bookkeeping
    int64_t canonical_bytes = 0, kernel_bytes = 0;
    // column segment of row segment 0: set by the caller before convert_csr (row-block ranks
    // whose lower-rank halo segments precede the own ones, dist.cu); 0 = square
    int64_t coff = 0;
    cudaStream_t owner_stream = nullptr;
};

constexpr int MG_PMAX = 8;  // ranks of the device-initiated multi-GPU kernel (one NVLink domain)

// Device-initiated multi-GPU solve (Finding 2, applied across GPUs): one
// persistent kernel per rank, every exchange done by the kernel itself through peer memory.
// Each rank exposes a window (an NCCL symmetric window over NVLink, or same-device buffers for
// ranks emulated on one GPU) holding: its extended PV vector (own + halo segments; peers store
// their boundary segments straight into it), the cross-rank reduction slots with their tags,
// and one arrival counter per peer.
struct MgArgs {
    int P = 0, me = 0;                 // P == 0: single-GPU kernel
    char* win[MG_PMAX];                // window base of every rank (this process's mapping)
    int64_t off_pv;                    // byte offset of the extended PV vector in each window
    int64_t off_red;                   // doubles [2 parities][P][4]
    int64_t off_tag;                   // u32 [2][P]: reduction number published with the slot
    int64_t off_cnt;                   // u64 [P]: halo stores completed by CTAs of rank r
    const int32_t* send_ptr;           // [G+1] entries of each CTA (sorted by CTA, then peer)
    const int32_t* send_src;           // own segment (relative to the own part)
    const int32_t* send_dst;           // segment of the peer's extended vector
    const int8_t* send_peer;
    const uint8_t* send_mask;          // [G] peers CTA g stores to (bit r)
    const int32_t* seg_lo;             // [G] extended column segments gathered by CTA g
    const int32_t* seg_hi;
    int nprod[MG_PMAX];                // CTAs of rank r that store into my window
    int32_t hlo[MG_PMAX], hhi[MG_PMAX];   // my extended segments received from rank r
};

// what run_solve needs to launch the multi-GPU kernel of one rank (dist.cu fills it)
struct MgLaunch {
    MgArgs args;
    double* pv_own;                                      // own part of the window's extended PV vector
    mf_status (*prelaunch)(void* ctx, cudaStream_t s);   // clear the window, cross-rank barrier
    void* ctx;
    // in-process rank group (all ranks on one device): a plain launch, because concurrent
    // cooperative launches of the ranks' kernels are refused / serialised by the driver, and the
    // ranks' grids must run side by side (co-residency is the caller's plan: G * nranks <= SMs)
    bool plain_launch = false;
    // after the launch call returned, before any blocking call (local group: a host barrier, so
    // every rank's kernel is enqueued before a thread blocks in the driver on its own kernel)
    mf_status (*postlaunch)(void* ctx) = nullptr;
};

// Dynamic shared memory limit of a kernel = the opt-in maximum minus its static shared memory.
// Set to the maximum (not to one launch's size): concurrent solves share the function attribute.
inline mf_status set_max_dyn_smem(const void* fn, int smem_optin) {
    cudaFuncAttributes fa;
    MF_CUDA(cudaFuncGetAttributes(&fa, fn));
    MF_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_optin - (int)fa.sharedSizeBytes));
    return MF_OK;
}

mf_status convert_csr(int64_t n_rows, int64_t n_cols, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                      const double* vals, const mf_convert_opts& o, cudaStream_t s, TileMatrix* A);
void destroy_tiles(TileMatrix* A);
// out[0..n] = exclusive scan of in[0..n) (out[n] = total); tmp: n / 2048 + 2 elements
mf_status scan_excl_i64(const int64_t* in, int64_t n, int64_t* out, int64_t* tmp, cudaStream_t s);

mf_status run_spmv(const TileMatrix& A, const double* x, double* y, const uint8_t* level, int range_guard,
                   int64_t* counts_host, cudaStream_t s);
mf_status run_levels(const double* v, int64_t n, const double* th, uint8_t* level, cudaStream_t s);
mf_status run_dot(const TileMatrix& A, const double* u, const double* v, double* out_host, cudaStream_t s);
mf_status run_cg_xr(const TileMatrix& A, double alpha, const double* p, const double* mu, double* x, double* r,
                    double* rr_host, cudaStream_t s);
mf_status run_cg_p(const TileMatrix& A, double beta, const double* r, double* p, cudaStream_t s);
mf_status run_solve(const TileMatrix& A, bool bicg, const double* b, double* x, const mf_solve_opts& o,
                    mf_solve_info* info, cudaStream_t s, const MgLaunch* mgl = nullptr);

}  // namespace mf

namespace mf {
struct DistInfo;      // dist.cu: the row block, halo plan and communicator of a distributed matrix
struct Comm;
void dist_destroy(DistInfo* D);
}  // namespace mf

struct mf_tile_matrix {
    mf::TileMatrix m;
    mf::DistInfo* dist = nullptr;       // set by mf_tile_matrix_from_csr_dist
};

// ------------------------------------------------------------------ device helpers
namespace mfk {

// binary64 -> binary32 with round-to-odd: RZ, then OR the sticky bit into the last place.
// Rounding this to a format with at least 2 fewer significand bits (FP16, E4M3) with RNE
// equals a single RNE from the binary64 value.
__device__ __forceinline__ float d2f_rto(double v) {
    float f = __double2float_rz(v);
    if ((double)f != v) f = __int_as_float(__float_as_int(f) | 1);
    return f;
}
__device__ __forceinline__ float to_f32(double v) { return __double2float_rn(v); }
__device__ __forceinline__ __half to_f16(double v) { return __float2half_rn(d2f_rto(v)); }
__device__ __forceinline__ uint8_t to_e4m3(double v) {
    return (uint8_t)__nv_cvt_float_to_fp8(d2f_rto(v), __NV_SATFINITE, __NV_E4M3);
}
__device__ __forceinline__ double f16_to_d(__half h) { return (double)__half2float(h); }
__device__ __forceinline__ double e4m3_to_d(uint8_t b) {
    __half_raw hr = __nv_cvt_fp8_to_halfraw((__nv_fp8_storage_t)b, __NV_E4M3);
    return (double)__half2float(__half(hr));
}
// value rounded to precision q (0..3) as binary64
__device__ __forceinline__ double round_to(double v, int q) {
    switch (q) {
    case 0: return v;
    case 1: return (double)to_f32(v);
    case 2: return f16_to_d(to_f16(v));
    default: return e4m3_to_d(to_e4m3(v));
    }
}

}  // namespace mfk
