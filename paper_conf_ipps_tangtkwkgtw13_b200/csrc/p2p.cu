// p2p.cu -- z-slab decomposition with the halo exchange FUSED into the sweep
// (north star (3) asks for an r-plane exchange per iteration).
//
// One process (or one plan) per GPU slab.  Each plan owns its two ping-pong
// grids; the neighbours' grids are mapped into this process through CUDA IPC
// (NVLink 5 / NVSwitch peer memory; on one device, plain device pointers).
// The in-plane PS kernel stores every completed boundary plane both into its
// own grid and into the neighbour's halo plane (inplane.cuh), so no exchange
// step, copy kernel or NCCL call exists.  Ordering is stream-side only:
//   before sweep e (e >= 2): wait until both neighbours have finished sweep
//     e-1 (cuStreamWaitValue32 GEQ on this rank's own flag words, which the
//     neighbours write) -- this covers RAW (our halos of grid[(e-1)%2] were
//     written by their sweep e-1) and WAR (their sweep e-1 no longer reads the
//     halo planes of grid[e%2] that our sweep e overwrites);
//   after sweep e: write e into the neighbours' flag words
//     (cuStreamWriteValue32, which orders the kernel's stores before the flag).
// No SM ever spins, so plans sharing one GPU cannot deadlock each other.
#include <algorithm>
#include <cstring>
#include <mutex>

#include <string>

#include "internal.h"

namespace {

typedef CUresult (*PFN_waitv32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
typedef CUresult (*PFN_writev32)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);

struct MemOps {
    PFN_waitv32 wait = nullptr;
    PFN_writev32 write = nullptr;
};

const MemOps& memops() {
    static MemOps m;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPointByVersion("cuStreamWaitValue32", &p, 12000, cudaEnableDefault, &q) ==
                cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            m.wait = reinterpret_cast<PFN_waitv32>(p);
        p = nullptr;
        if (cudaGetDriverEntryPointByVersion("cuStreamWriteValue32", &p, 12000, cudaEnableDefault, &q) ==
                cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            m.write = reinterpret_cast<PFN_writev32>(p);
    });
    return m;
}

constexpr unsigned kWaitGeq = 0x0;   // CU_STREAM_WAIT_VALUE_GEQ
// CU_STREAM_WAIT_VALUE_FLUSH: a peer's halo stores and its flag write are both REMOTE writes to this
// device, which may reorder remote writes internally; the flush after the wait makes every remote
// write that reached the device before the flag visible to the sweep that follows.  Used where the
// device reports cudaDevAttrCanFlushRemoteWrites.
constexpr unsigned kWaitFlush = 1u << 30;
constexpr unsigned kWriteDefault = 0x0;  // CU_STREAM_WRITE_VALUE_DEFAULT (memory barrier before the write)

}  // namespace

extern "C" stencil_status_t stencil_plan_init_internal(stencil_plan_t p, int64_t nx, int64_t ny, int64_t nz,
                                                       int radius, const double* coeffs, stencil_dtype_t dtype);
extern "C" stencil_status_t stencil_timing_mark_internal(stencil_plan_t p, cudaStream_t st);
extern "C" stencil_status_t stencil_residual_internal(stencil_plan_t p, const void* a, const void* b, cudaStream_t st,
                                                      double* res);
extern "C" stencil_status_t stencil_residual_launch_internal(stencil_plan_t p, const void* a, const void* b,
                                                             cudaStream_t st);
extern "C" stencil_status_t stencil_residual_read_internal(stencil_plan_t p, cudaStream_t st, double* res);

// Residual max across the slabs without any host-side collective: P-1 rounds of exchanging the
// running max with both neighbours through the same mapped flag buffers the sweeps use.  Flag
// buffer layout (256 bytes per plan, flags[] as u32): words 0 / 1 sweep epochs from rank-1 / rank+1;
// words 8 / 9 residual rounds from rank-1 / rank+1; u64 slots at byte 64 + 8*(2*parity + side) the
// neighbours' running max of a round (side 0 from rank-1, 1 from rank+1; double-buffered by round
// parity, so a neighbour one round ahead never overwrites a value not yet merged).
__global__ void res_send_kernel(const unsigned long long* __restrict__ mine, unsigned long long* lo_slot,
                                unsigned long long* hi_slot) {
    const unsigned long long v = *mine;
    if (lo_slot) *lo_slot = v;
    if (hi_slot) *hi_slot = v;
}

__global__ void res_merge_kernel(unsigned long long* mine, const unsigned long long* from_lo,
                                 const unsigned long long* from_hi) {
    unsigned long long v = *mine;
    if (from_lo && *from_lo > v) v = *from_lo;
    if (from_hi && *from_hi > v) v = *from_hi;
    *mine = v;
}

namespace stencil {

stencil_status_t p2p_destroy(stencil_plan_s* p) {
    if (!p->p2p) return STENCIL_SUCCESS;
    for (void* q : p->ipc_opened) cudaIpcCloseMemHandle(q);
    p->ipc_opened.clear();
    for (void*& g : p->grid)
        if (g) {
            cudaFree(g);
            g = nullptr;
        }
    if (p->flags) cudaFree(p->flags);
    p->flags = nullptr;
    return STENCIL_SUCCESS;
}

static stencil_status_t p2p_check(stencil_plan_s* p, const char* what) {
    if (!p) return fail(STENCIL_ERROR_INVALID_VALUE, std::string(what) + ": NULL plan");
    if (!p->p2p) return fail(STENCIL_ERROR_INVALID_VALUE, std::string(what) + ": not a p2p slab plan");
    return STENCIL_SUCCESS;
}

}  // namespace stencil

using namespace stencil;

extern "C" {

stencil_status_t stencil_p2p_targets(const stencil_layout_t* L, int64_t nz_global, int nranks, int rank,
                                     stencil_p2p_targets_t* out) {
    if (!L || !out) return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_targets: NULL argument");
    int64_t z0 = 0, nzl = 0, z0lo = 0, nzlo = 0;
    stencil_status_t rc = stencil_slab_partition(nz_global, nranks, rank, (int)L->radius, &z0, &nzl);
    if (rc != STENCIL_SUCCESS) return rc;
    if (nzl != L->nz) return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_targets: layout nz is not this rank's slab");
    if (rank > 0 && (rc = stencil_slab_partition(nz_global, nranks, rank - 1, (int)L->radius, &z0lo, &nzlo)) !=
                        STENCIL_SUCCESS)
        return rc;
    const int64_t plane = L->rows_y * L->pitch_x;
    stencil_p2p_targets_t t{};
    t.lo_rank = rank > 0 ? rank - 1 : -1;
    t.hi_rank = rank < nranks - 1 ? rank + 1 : -1;
    t.planes = (int32_t)L->radius;
    t.lo_delta = rank > 0 ? nzlo * plane : 0;          // our plane z -> its plane nz_lo + z
    t.hi_delta = rank < nranks - 1 ? -nzl * plane : 0;  // our plane z -> its plane z - nz
    *out = t;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_plan_create_p2p(stencil_plan_t* plan, int64_t nx, int64_t ny, int64_t nz_global, int radius,
                                         const double* coeffs, stencil_dtype_t dtype, int rank, int nranks) {
    if (!plan || !coeffs) return fail(STENCIL_ERROR_INVALID_VALUE, "create_p2p: NULL argument");
    *plan = nullptr;
    int64_t z0 = 0, nzl = 0, z0lo = 0, nzlo = 0;
    stencil_status_t rc = stencil_slab_partition(nz_global, nranks, rank, radius, &z0, &nzl);
    if (rc != STENCIL_SUCCESS) return rc;
    if (rank > 0 && (rc = stencil_slab_partition(nz_global, nranks, rank - 1, radius, &z0lo, &nzlo)) != STENCIL_SUCCESS)
        return rc;
    const MemOps& m = memops();
    if (!m.wait || !m.write)
        return fail(STENCIL_ERROR_NOT_SUPPORTED, "create_p2p: cuStreamWaitValue32 / cuStreamWriteValue32 unavailable");
    stencil_plan_t p = new (std::nothrow) stencil_plan_s();
    if (!p) return fail(STENCIL_ERROR_OUT_OF_MEMORY, "create_p2p: host allocation");
    rc = stencil_plan_init_internal(p, nx, ny, nzl, radius, coeffs, dtype);
    if (rc == STENCIL_SUCCESS) {
        p->p2p = true;
        p->rank = rank;
        p->nranks = nranks;
        p->nz_global = nz_global;
        p->z0_global = z0;
        p->nz_lo = nzlo;
        for (int i = 0; i < 2 && rc == STENCIL_SUCCESS; ++i) {
            cudaError_t e = cudaMalloc(&p->grid[i], (size_t)p->lay.bytes);
            if (e != cudaSuccess) rc = cuda_fail(e, "create_p2p: grid allocation");
            else if ((e = cudaMemset(p->grid[i], 0, (size_t)p->lay.bytes)) != cudaSuccess)
                rc = cuda_fail(e, "create_p2p: grid memset");
        }
        if (rc == STENCIL_SUCCESS) {
            int can_flush = 0;
            if (cudaDeviceGetAttribute(&can_flush, cudaDevAttrCanFlushRemoteWrites, p->device) == cudaSuccess &&
                can_flush)
                p->wait_flags = kWaitGeq | kWaitFlush;
            else
                p->wait_flags = kWaitGeq;
            cudaError_t e = cudaMalloc(&p->flags, 256);
            if (e == cudaSuccess) e = cudaMemset(p->flags, 0, 256);
            // the stop-criterion words now: an allocation during a run can wait for the device to go
            // idle, which a slab blocked on its neighbours' flags never does
            if (e == cudaSuccess) e = cudaMalloc(&p->d_res, sizeof(unsigned long long));
            if (e == cudaSuccess) e = cudaMallocHost(&p->h_res, sizeof(unsigned long long));
            if (e != cudaSuccess) rc = cuda_fail(e, "create_p2p: flag allocation");
        }
    }
    if (rc != STENCIL_SUCCESS) {
        stencil_destroy(p);
        return rc;
    }
    p->cfg = default_config(p, STENCIL_KERNEL_INPLANE);
    preload_kernels(p);
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, res_send_kernel);
    cudaFuncGetAttributes(&fa, res_merge_kernel);
    cudaGetLastError();
    *plan = p;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_p2p_endpoint(stencil_plan_t p, stencil_p2p_endpoint_t* out) {
    stencil_status_t rc = p2p_check(p, "p2p_endpoint");
    if (rc != STENCIL_SUCCESS) return rc;
    if (!out) return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_endpoint: NULL output");
    stencil_p2p_endpoint_t e{};
    e.grid[0] = p->grid[0];
    e.grid[1] = p->grid[1];
    e.flags = p->flags;
    e.rank = p->rank;
    e.nz_local = p->lay.nz;
    *out = e;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_p2p_connect(stencil_plan_t p, const stencil_p2p_endpoint_t* lo,
                                     const stencil_p2p_endpoint_t* hi) {
    stencil_status_t rc = p2p_check(p, "p2p_connect");
    if (rc != STENCIL_SUCCESS) return rc;
    if ((p->rank > 0) != (lo != nullptr) || (p->rank < p->nranks - 1) != (hi != nullptr))
        return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_connect: need exactly the existing neighbours (lo iff rank > 0, "
                                                 "hi iff rank < nranks-1)");
    if (lo && (lo->rank != p->rank - 1 || lo->nz_local != p->nz_lo || !lo->grid[0] || !lo->grid[1] || !lo->flags))
        return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_connect: lower endpoint does not match rank-1's slab");
    if (hi) {
        int64_t z0h = 0, nzh = 0;
        if ((rc = stencil_slab_partition(p->nz_global, p->nranks, p->rank + 1, p->r, &z0h, &nzh)) != STENCIL_SUCCESS)
            return rc;
        if (hi->rank != p->rank + 1 || hi->nz_local != nzh || !hi->grid[0] || !hi->grid[1] || !hi->flags)
            return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_connect: upper endpoint does not match rank+1's slab");
    }
    // the sweep kernel stores into the neighbours' grids and the stream writes their flag words: a
    // neighbour on another device needs peer access (one process driving several GPUs); without it
    // those stores would fault, so refuse the connection instead
    for (const stencil_p2p_endpoint_t* ep : {lo, hi}) {
        if (!ep) continue;
        cudaPointerAttributes at{};
        STENCIL_CUDA_TRY(cudaPointerGetAttributes(&at, ep->grid[0]));
        if (at.device != p->device) {
            int can = 0;
            STENCIL_CUDA_TRY(cudaDeviceCanAccessPeer(&can, p->device, at.device));
            if (!can)
                return fail(STENCIL_ERROR_NOT_SUPPORTED, "p2p_connect: neighbour grid on device " + std::to_string(at.device) +
                                                             " is not peer-accessible from device " + std::to_string(p->device));
            STENCIL_CUDA_TRY(cudaSetDevice(p->device));
            cudaError_t e = cudaDeviceEnablePeerAccess(at.device, 0);
            if (e == cudaErrorPeerAccessAlreadyEnabled)
                cudaGetLastError();
            else if (e != cudaSuccess)
                return cuda_fail(e, "cudaDeviceEnablePeerAccess");
        }
    }
    stencil_p2p_targets_t tg{};
    if ((rc = stencil_p2p_targets(&p->lay, p->nz_global, p->nranks, p->rank, &tg)) != STENCIL_SUCCESS) return rc;
    if (lo) {
        p->lo_grid[0] = lo->grid[0];
        p->lo_grid[1] = lo->grid[1];
        p->lo_flag = static_cast<unsigned*>(lo->flags) + 1;  // rank-1 hears from its upper neighbour in word 1
        p->lo_delta = tg.lo_delta;                           // our plane z -> its plane nz_lo + z
    }
    if (hi) {
        p->hi_grid[0] = hi->grid[0];
        p->hi_grid[1] = hi->grid[1];
        p->hi_flag = static_cast<unsigned*>(hi->flags) + 0;  // rank+1 hears from its lower neighbour in word 0
        p->hi_delta = tg.hi_delta;                           // our plane z -> its plane z - nz
    }
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_p2p_export(stencil_plan_t p, void* handles) {
    stencil_status_t rc = p2p_check(p, "p2p_export");
    if (rc != STENCIL_SUCCESS) return rc;
    if (!handles) return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_export: NULL output");
    cudaIpcMemHandle_t h[3];
    void* ptrs[3] = {p->grid[0], p->grid[1], p->flags};
    for (int i = 0; i < 3; ++i) STENCIL_CUDA_TRY(cudaIpcGetMemHandle(&h[i], ptrs[i]));
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
    memcpy(handles, h, sizeof h);
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_p2p_import(stencil_plan_t p, const void* lo_handles, const void* hi_handles) {
    stencil_status_t rc = p2p_check(p, "p2p_import");
    if (rc != STENCIL_SUCCESS) return rc;
    STENCIL_CUDA_TRY(cudaSetDevice(p->device));
    stencil_p2p_endpoint_t ep[2]{};
    const void* hs[2] = {lo_handles, hi_handles};
    for (int side = 0; side < 2; ++side) {
        if (!hs[side]) continue;
        cudaIpcMemHandle_t h[3];
        memcpy(h, hs[side], sizeof h);
        void* ptr[3] = {nullptr, nullptr, nullptr};
        for (int i = 0; i < 3; ++i) {
            cudaError_t e = cudaIpcOpenMemHandle(&ptr[i], h[i], cudaIpcMemLazyEnablePeerAccess);
            if (e != cudaSuccess) return cuda_fail(e, "p2p_import: cudaIpcOpenMemHandle");
            p->ipc_opened.push_back(ptr[i]);
        }
        const int nbr = side == 0 ? p->rank - 1 : p->rank + 1;
        int64_t z0n = 0, nzn = 0;
        if ((rc = stencil_slab_partition(p->nz_global, p->nranks, nbr, p->r, &z0n, &nzn)) != STENCIL_SUCCESS) return rc;
        ep[side].grid[0] = ptr[0];
        ep[side].grid[1] = ptr[1];
        ep[side].flags = ptr[2];
        ep[side].rank = nbr;
        ep[side].nz_local = nzn;
    }
    return stencil_p2p_connect(p, lo_handles ? &ep[0] : nullptr, hi_handles ? &ep[1] : nullptr);
}

stencil_status_t stencil_p2p_run(stencil_plan_t p, int iters, stencil_stream_t stream, int* current) {
    stencil_status_t rc = p2p_check(p, "p2p_run");
    if (rc != STENCIL_SUCCESS) return rc;
    if (iters < 0 || !current) return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_run: iters < 0 or NULL output");
    if ((p->rank > 0 && !p->lo_flag) || (p->rank < p->nranks - 1 && !p->hi_flag))
        return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_run: plan not connected to its neighbours");
    STENCIL_CUDA_TRY(cudaSetDevice(p->device));
    cudaStream_t st = (cudaStream_t)stream;
    const MemOps& m = memops();
    const size_t span0 = p->tev_used;
    if (p->timing && (rc = stencil_timing_mark_internal(p, st)) != STENCIL_SUCCESS) return rc;
    for (int t = 0; t < iters; ++t) {
        const unsigned e = p->epoch + 1;  // sweep e: grid[(e-1)%2] -> grid[e%2]
        if (e >= 2) {
            CUresult r = CUDA_SUCCESS;
            if (p->rank > 0) r = m.wait(st, (CUdeviceptr)(p->flags + 0), e - 1, p->wait_flags);
            if (r == CUDA_SUCCESS && p->rank < p->nranks - 1) r = m.wait(st, (CUdeviceptr)(p->flags + 1), e - 1, p->wait_flags);
            if (r != CUDA_SUCCESS) return fail(STENCIL_ERROR_CUDA, "p2p_run: cuStreamWaitValue32 failed");
        }
        p->sweep_peer_lo = p->rank > 0 ? p->lo_grid[e % 2] : nullptr;
        p->sweep_peer_hi = p->rank < p->nranks - 1 ? p->hi_grid[e % 2] : nullptr;
        SweepSegments all{0, 1, p->cfg.zsegs};
        rc = launch_sweep(p, p->cfg, p->grid[(e - 1) % 2], nullptr, p->grid[e % 2], all, (e % 2 == 1) ? 1 : -1, st);
        p->sweep_peer_lo = p->sweep_peer_hi = nullptr;
        if (rc != STENCIL_SUCCESS) return rc;
        CUresult r = CUDA_SUCCESS;
        if (p->rank > 0) r = m.write(st, (CUdeviceptr)p->lo_flag, e, kWriteDefault);
        if (r == CUDA_SUCCESS && p->rank < p->nranks - 1) r = m.write(st, (CUdeviceptr)p->hi_flag, e, kWriteDefault);
        if (r != CUDA_SUCCESS) return fail(STENCIL_ERROR_CUDA, "p2p_run: cuStreamWriteValue32 failed");
        p->epoch = e;
        if ((p->timing == 2 || (p->timing && t == iters - 1)) && (rc = stencil_timing_mark_internal(p, st)) != STENCIL_SUCCESS) return rc;
    }
    if (p->timing && iters > 0) p->spans.push_back({span0, p->tev_used - 1, iters});
    p->last_sweeps = iters;
    *current = (int)(p->epoch % 2);
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_p2p_quiesce(stencil_plan_t p, stencil_stream_t stream) {
    stencil_status_t rc = p2p_check(p, "p2p_quiesce");
    if (rc != STENCIL_SUCCESS) return rc;
    if (p->epoch == 0) return STENCIL_SUCCESS;
    const MemOps& m = memops();
    cudaStream_t st = (cudaStream_t)stream;
    CUresult r = CUDA_SUCCESS;
    if (p->rank > 0 && p->lo_flag) r = m.wait(st, (CUdeviceptr)(p->flags + 0), p->epoch, p->wait_flags);
    if (r == CUDA_SUCCESS && p->rank < p->nranks - 1 && p->hi_flag)
        r = m.wait(st, (CUdeviceptr)(p->flags + 1), p->epoch, p->wait_flags);
    if (r != CUDA_SUCCESS) return fail(STENCIL_ERROR_CUDA, "p2p_quiesce: cuStreamWaitValue32 failed");
    return STENCIL_SUCCESS;
}

static unsigned long long* res_slot(unsigned* flags_base, unsigned parity, int side) {
    return reinterpret_cast<unsigned long long*>(reinterpret_cast<char*>(flags_base) + 64 + 8 * (2 * parity + side));
}

// in-place max over all slabs of p->d_res (stream-ordered; every rank issues the same rounds)
static stencil_status_t p2p_allreduce_max(stencil_plan_s* p, cudaStream_t st) {
    const MemOps& m = memops();
    unsigned* lo_base = p->rank > 0 ? p->lo_flag - 1 : nullptr;  // rank-1's flag buffer (lo_flag = its word 1)
    unsigned* hi_base = p->rank < p->nranks - 1 ? p->hi_flag : nullptr;  // rank+1's (hi_flag = its word 0)
    for (int round = 1; round < p->nranks; ++round) {
        const unsigned seq = ++p->res_seq, par = seq & 1u;
        // our running max into rank-1's "from its upper neighbour" slot and rank+1's "from lower" slot
        res_send_kernel<<<1, 1, 0, st>>>(p->d_res, lo_base ? res_slot(lo_base, par, 1) : nullptr,
                                         hi_base ? res_slot(hi_base, par, 0) : nullptr);
        STENCIL_CUDA_TRY(cudaGetLastError());
        CUresult r = CUDA_SUCCESS;
        if (lo_base) r = m.write(st, (CUdeviceptr)(lo_base + 9), seq, kWriteDefault);
        if (r == CUDA_SUCCESS && hi_base) r = m.write(st, (CUdeviceptr)(hi_base + 8), seq, kWriteDefault);
        if (r == CUDA_SUCCESS && lo_base) r = m.wait(st, (CUdeviceptr)(p->flags + 8), seq, p->wait_flags);
        if (r == CUDA_SUCCESS && hi_base) r = m.wait(st, (CUdeviceptr)(p->flags + 9), seq, p->wait_flags);
        if (r != CUDA_SUCCESS) return fail(STENCIL_ERROR_CUDA, "p2p residual reduction: stream memory operation failed");
        res_merge_kernel<<<1, 1, 0, st>>>(p->d_res, lo_base ? res_slot(p->flags, par, 0) : nullptr,
                                          hi_base ? res_slot(p->flags, par, 1) : nullptr);
        STENCIL_CUDA_TRY(cudaGetLastError());
        p->aux_launches += 2;
    }
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_p2p_run_until(stencil_plan_t p, int max_iters, double tol, int check_every,
                                       stencil_stream_t stream, int* iters_done, double* residual) {
    stencil_status_t rc = p2p_check(p, "p2p_run_until");
    if (rc != STENCIL_SUCCESS) return rc;
    if (!iters_done || !residual) return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_run_until: NULL output");
    if (max_iters < 1 || check_every < 1 || !(tol >= 0.0))
        return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_run_until: max_iters, check_every >= 1 and tol >= 0 required");
    cudaStream_t st = (cudaStream_t)stream;
    int t = 0, cur = 0;
    double res = -1.0;
    while (t < max_iters) {
        const int n = std::min(check_every, max_iters - t);
        if ((rc = stencil_p2p_run(p, n, stream, &cur)) != STENCIL_SUCCESS) return rc;
        t += n;
        if ((rc = stencil_residual_launch_internal(p, p->grid[p->epoch % 2], p->grid[(p->epoch - 1) % 2], st)) !=
            STENCIL_SUCCESS)
            return rc;
        if ((rc = p2p_allreduce_max(p, st)) != STENCIL_SUCCESS) return rc;
        if ((rc = stencil_residual_read_internal(p, st, &res)) != STENCIL_SUCCESS) return rc;
        if (res <= tol) break;
    }
    *iters_done = t;
    *residual = res;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_p2p_residual(stencil_plan_t p, stencil_stream_t stream, double* residual) {
    stencil_status_t rc = p2p_check(p, "p2p_residual");
    if (rc != STENCIL_SUCCESS) return rc;
    if (!residual) return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_residual: NULL output");
    if (p->epoch == 0) return fail(STENCIL_ERROR_INVALID_VALUE, "p2p_residual: no sweep has run yet");
    // interior of u_e (grid[e%2]) against u_{e-1} (grid[(e-1)%2]); neighbours only ever write halo planes
    return stencil_residual_internal(p, p->grid[p->epoch % 2], p->grid[(p->epoch - 1) % 2], (cudaStream_t)stream,
                                     residual);
}

}  // extern "C"
