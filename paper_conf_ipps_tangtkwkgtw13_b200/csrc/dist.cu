// dist.cu -- z-slab decomposition over the GPUs of one box (north star (3);
// not in the paper).  One process per GPU; NCCL point-to-point over
// NVLink 5 / NVSwitch for the per-iteration r-plane halo exchange.
//
// NCCL is loaded at run time (dlopen "libnccl.so.2", or STENCIL_NCCL_LIB) so
// the library has no link-time NCCL dependency and the host-only helpers work
// on machines without NCCL or GPUs.
#include <dlfcn.h>

#include <cstring>
#include <mutex>
#include <string>

#include "internal.h"

namespace {

// Minimal NCCL ABI (stable since NCCL 2.0).
typedef struct { char internal[128]; } nccl_uid_t;
typedef void* nccl_comm_t;
typedef int nccl_result_t;
const int kNcclInt8 = 0;
const int kNcclUint64 = 5;  // ncclUint64
const int kNcclMax = 2;     // ncclMax

struct NcclApi {
    bool ok = false;
    std::string err;
    nccl_result_t (*GetUniqueId)(nccl_uid_t*) = nullptr;
    nccl_result_t (*CommInitRank)(nccl_comm_t*, int, nccl_uid_t, int) = nullptr;
    nccl_result_t (*CommDestroy)(nccl_comm_t) = nullptr;
    nccl_result_t (*Send)(const void*, size_t, int, int, nccl_comm_t, cudaStream_t) = nullptr;
    nccl_result_t (*Recv)(void*, size_t, int, int, nccl_comm_t, cudaStream_t) = nullptr;
    nccl_result_t (*AllReduce)(const void*, void*, size_t, int, int, nccl_comm_t, cudaStream_t) = nullptr;
    nccl_result_t (*GroupStart)() = nullptr;
    nccl_result_t (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(nccl_result_t) = nullptr;
};

NcclApi& nccl() {
    static NcclApi api;
    static std::once_flag once;
    std::call_once(once, [] {
        const char* env = getenv("STENCIL_NCCL_LIB");
        void* h = nullptr;
        if (env && *env) h = dlopen(env, RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) {
            api.err = std::string("dlopen libnccl.so.2 failed: ") + dlerror();
            return;
        }
        auto sym = [&](const char* n) { return dlsym(h, n); };
        api.GetUniqueId = (decltype(api.GetUniqueId))sym("ncclGetUniqueId");
        api.CommInitRank = (decltype(api.CommInitRank))sym("ncclCommInitRank");
        api.CommDestroy = (decltype(api.CommDestroy))sym("ncclCommDestroy");
        api.Send = (decltype(api.Send))sym("ncclSend");
        api.Recv = (decltype(api.Recv))sym("ncclRecv");
        api.AllReduce = (decltype(api.AllReduce))sym("ncclAllReduce");
        api.GroupStart = (decltype(api.GroupStart))sym("ncclGroupStart");
        api.GroupEnd = (decltype(api.GroupEnd))sym("ncclGroupEnd");
        api.GetErrorString = (decltype(api.GetErrorString))sym("ncclGetErrorString");
        api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.Send && api.Recv && api.AllReduce &&
                 api.GroupStart &&
                 api.GroupEnd && api.GetErrorString;
        if (!api.ok) api.err = "libnccl.so.2 lacks a required symbol";
    });
    return api;
}

stencil_status_t nccl_fail(nccl_result_t r, const char* what) {
    NcclApi& a = nccl();
    return stencil::fail(STENCIL_ERROR_NCCL, std::string(what) + ": " + (a.GetErrorString ? a.GetErrorString(r) : "?"));
}

}  // namespace

extern "C" stencil_status_t stencil_plan_init_internal(stencil_plan_t p, int64_t nx, int64_t ny, int64_t nz,
                                                       int radius, const double* coeffs, stencil_dtype_t dtype);

namespace stencil {

stencil_status_t dist_exchange(stencil_plan_s* p, void* buf, cudaStream_t st) {
    if (!p->dist || p->nranks < 2 || !buf) return STENCIL_SUCCESS;
    NcclApi& a = nccl();
    const stencil_exchange_plan_t& x = p->xplan;
    char* b = static_cast<char*>(buf);
    nccl_comm_t comm = p->comm;
    nccl_result_t r = a.GroupStart();
    if (r) return nccl_fail(r, "ncclGroupStart");
    if (x.peer_lo >= 0) {
        if ((r = a.Send(b + x.send_lo_off, (size_t)x.msg_bytes, kNcclInt8, x.peer_lo, comm, st))) return nccl_fail(r, "ncclSend lo");
        if ((r = a.Recv(b + x.recv_lo_off, (size_t)x.msg_bytes, kNcclInt8, x.peer_lo, comm, st))) return nccl_fail(r, "ncclRecv lo");
    }
    if (x.peer_hi >= 0) {
        if ((r = a.Send(b + x.send_hi_off, (size_t)x.msg_bytes, kNcclInt8, x.peer_hi, comm, st))) return nccl_fail(r, "ncclSend hi");
        if ((r = a.Recv(b + x.recv_hi_off, (size_t)x.msg_bytes, kNcclInt8, x.peer_hi, comm, st))) return nccl_fail(r, "ncclRecv hi");
    }
    if ((r = a.GroupEnd())) return nccl_fail(r, "ncclGroupEnd");
    return STENCIL_SUCCESS;
}

stencil_status_t dist_allreduce_max_u64(stencil_plan_s* p, unsigned long long* word, cudaStream_t st) {
    if (!p->dist || p->nranks < 2) return STENCIL_SUCCESS;
    NcclApi& a = nccl();
    nccl_result_t r = a.AllReduce(word, word, 1, kNcclUint64, kNcclMax, p->comm, st);
    if (r) return nccl_fail(r, "ncclAllReduce (residual max)");
    return STENCIL_SUCCESS;
}

stencil_status_t dist_destroy(stencil_plan_s* p) {
    if (!p->dist) return STENCIL_SUCCESS;
    if (p->comm) {
        NcclApi& a = nccl();
        if (a.ok) a.CommDestroy(p->comm);
        p->comm = nullptr;
    }
    if (p->s_comm) cudaStreamDestroy(p->s_comm);
    if (p->ev_bnd) cudaEventDestroy(p->ev_bnd);
    if (p->ev_xchg) cudaEventDestroy(p->ev_xchg);
    p->s_comm = nullptr;
    p->ev_bnd = p->ev_xchg = nullptr;
    return STENCIL_SUCCESS;
}

}  // namespace stencil

using namespace stencil;

extern "C" {

stencil_status_t stencil_slab_partition(int64_t nz_global, int nranks, int rank, int radius, int64_t* z0,
                                        int64_t* nz_local) {
    if (!z0 || !nz_local) return fail(STENCIL_ERROR_INVALID_VALUE, "slab_partition: NULL output");
    if (nranks < 1 || rank < 0 || rank >= nranks || nz_global < 1 || radius < 1)
        return fail(STENCIL_ERROR_INVALID_VALUE, "slab_partition: bad arguments");
    const int64_t base = nz_global / nranks, extra = nz_global % nranks;
    const int64_t n = base + (rank < extra ? 1 : 0);
    const int64_t start = rank * base + (rank < extra ? rank : extra);
    if (nranks > 1 && base < radius)
        return fail(STENCIL_ERROR_INVALID_VALUE, "slab_partition: every rank needs >= r planes");
    *z0 = start;
    *nz_local = n;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_exchange_plan(const stencil_layout_t* L, int nranks, int rank, stencil_exchange_plan_t* out) {
    if (!L || !out) return fail(STENCIL_ERROR_INVALID_VALUE, "exchange_plan: NULL argument");
    if (nranks < 1 || rank < 0 || rank >= nranks) return fail(STENCIL_ERROR_INVALID_VALUE, "exchange_plan: bad rank");
    const int r = L->radius;
    if (nranks > 1 && L->nz < r) return fail(STENCIL_ERROR_INVALID_VALUE, "exchange_plan: nz_local < r");
    const int64_t plane_bytes = L->rows_y * L->pitch_x * L->elem_size;
    stencil_exchange_plan_t x{};
    x.peer_lo = rank > 0 ? rank - 1 : -1;
    x.peer_hi = rank < nranks - 1 ? rank + 1 : -1;
    x.msg_bytes = (int64_t)r * plane_bytes;
    x.send_lo_off = (int64_t)r * plane_bytes;          // owned planes [0, r)      -> rank-1
    x.recv_lo_off = 0;                                 // halo planes  [-r, 0)     <- rank-1
    x.send_hi_off = L->nz * plane_bytes;               // owned planes [nz-r, nz)  -> rank+1
    x.recv_hi_off = (L->nz + r) * plane_bytes;         // halo planes  [nz, nz+r)  <- rank+1
    *out = x;
    return STENCIL_SUCCESS;
}

// ---------------------------------------------------------------------------
// In-process rank groups: P slab plans of one process
// with the DistPlan's exact split, events and exchange offsets, the transport a
// cudaMemcpyAsync into the neighbour's buffer.  Runs every rank's sweeps in
// lock step so the cross-rank events exist when they are waited on.
// ---------------------------------------------------------------------------
stencil_status_t stencil_plan_create_dist_local(stencil_plan_t* plans, int64_t nx, int64_t ny, int64_t nz_global,
                                                int radius, const double* coeffs, stencil_dtype_t dtype, int nranks) {
    if (!plans || !coeffs || nranks < 1) return fail(STENCIL_ERROR_INVALID_VALUE, "create_dist_local: bad argument");
    for (int k = 0; k < nranks; ++k) plans[k] = nullptr;
    auto group = std::make_shared<std::vector<stencil_plan_s*>>(nranks, nullptr);
    stencil_status_t rc = STENCIL_SUCCESS;
    for (int k = 0; k < nranks && rc == STENCIL_SUCCESS; ++k) {
        int64_t z0 = 0, nzl = 0;
        if ((rc = stencil_slab_partition(nz_global, nranks, k, radius, &z0, &nzl)) != STENCIL_SUCCESS) break;
        stencil_plan_t p = new (std::nothrow) stencil_plan_s();
        if (!p) {
            rc = fail(STENCIL_ERROR_OUT_OF_MEMORY, "create_dist_local: host allocation");
            break;
        }
        plans[k] = p;
        (*group)[k] = p;
        if ((rc = stencil_plan_init_internal(p, nx, ny, nzl, radius, coeffs, dtype)) != STENCIL_SUCCESS) break;
        p->dist = true;
        p->rank = k;
        p->nranks = nranks;
        p->nz_global = nz_global;
        p->z0_global = z0;
        p->local_group = group;
        if ((rc = stencil_exchange_plan(&p->lay, nranks, k, &p->xplan)) != STENCIL_SUCCESS) break;
        if (cudaStreamCreateWithFlags(&p->s_comm, cudaStreamNonBlocking) != cudaSuccess ||
            cudaEventCreateWithFlags(&p->ev_bnd, cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&p->ev_xchg, cudaEventDisableTiming) != cudaSuccess)
            rc = cuda_fail(cudaGetLastError(), "create_dist_local streams/events");
        if (rc == STENCIL_SUCCESS) p->cfg = default_config(p, STENCIL_KERNEL_INPLANE_WS);
    }
    if (rc != STENCIL_SUCCESS) {
        for (int k = 0; k < nranks; ++k) {
            stencil_destroy(plans[k]);
            plans[k] = nullptr;
        }
    }
    return rc;
}

stencil_status_t stencil_run_dist_local(stencil_plan_t* plans, int nranks, const void* const* in, void* const* out,
                                        int iters, const stencil_stream_t* streams) {
    if (!plans || !in || !out || !streams || nranks < 1 || iters < 0)
        return fail(STENCIL_ERROR_INVALID_VALUE, "run_dist_local: bad argument");
    std::vector<stencil_plan_s*>& G = *plans[0]->local_group;
    if (!plans[0]->local_group || (int)G.size() != nranks)
        return fail(STENCIL_ERROR_INVALID_VALUE, "run_dist_local: plans are not one in-process rank group");
    for (int k = 0; k < nranks; ++k) {
        stencil_plan_s* p = plans[k];
        if (!p || p->local_group != plans[0]->local_group || p->rank != k)
            return fail(STENCIL_ERROR_INVALID_VALUE, "run_dist_local: plans[k] must be rank k of the group");
        if (!in[k] || !out[k] || (((uintptr_t)in[k] | (uintptr_t)out[k]) & 127))
            return fail(STENCIL_ERROR_MISALIGNED, "run_dist_local: buffers must be non-NULL and 128-byte aligned");
    }
    STENCIL_CUDA_TRY(cudaSetDevice(plans[0]->device));
    stencil_status_t rc;
    auto st = [&](int k) { return (cudaStream_t)streams[k]; };
    if (iters == 0) {
        for (int k = 0; k < nranks; ++k)
            STENCIL_CUDA_TRY(cudaMemcpyAsync(out[k], in[k], (size_t)plans[k]->lay.bytes, cudaMemcpyDeviceToDevice, st(k)));
        return STENCIL_SUCCESS;
    }
    for (int k = 0; k < nranks; ++k) {
        stencil_plan_s* p = plans[k];
        if (iters >= 2 && (rc = stencil_plan_reserve(p)) != STENCIL_SUCCESS) return rc;
        if ((rc = launch_shell_copy(p, in[k], out[k], st(k))) != STENCIL_SUCCESS) return rc;
        if (iters >= 2 && (rc = launch_shell_copy(p, in[k], p->scratch, st(k))) != STENCIL_SUCCESS) return rc;
    }
    std::vector<const void*> src(in, in + nranks);
    std::vector<void*> dst(nranks);
    for (int t = 1; t <= iters; ++t) {
        const int dir = (t % 2 == 1) ? 1 : -1;
        for (int k = 0; k < nranks; ++k) dst[k] = ((iters - t) % 2 == 0) ? out[k] : plans[k]->scratch;
        // (1) boundary segments (they produce the planes that are exchanged), exactly as sweep_step
        std::vector<int> split(nranks);
        for (int k = 0; k < nranks; ++k) {
            stencil_plan_s* p = plans[k];
            const int zsegs = p->cfg.zsegs;
            split[k] = zsegs >= 2 && p->lay.nz / zsegs >= p->r;
            SweepSegments b = split[k] ? SweepSegments{0, zsegs - 1, 2} : SweepSegments{0, 1, zsegs};
            if ((rc = launch_sweep(p, p->cfg, src[k], nullptr, dst[k], b, dir, st(k))) != STENCIL_SUCCESS) return rc;
            STENCIL_CUDA_TRY(cudaEventRecord(p->ev_bnd, st(k)));
        }
        // (2) the exchange on each rank's comm stream: its first / last r owned planes into the
        // neighbours' halo planes of the same sweep's output (stencil_exchange_plan offsets), once its
        // own planes exist and the neighbour is done reading that buffer (its boundary event follows
        // its previous sweep in stream order)
        for (int k = 0; k < nranks; ++k) {
            stencil_plan_s* p = plans[k];
            const stencil_exchange_plan_t& x = p->xplan;
            STENCIL_CUDA_TRY(cudaStreamWaitEvent(p->s_comm, p->ev_bnd, 0));
            if (x.peer_lo >= 0) {
                stencil_plan_s* q = plans[x.peer_lo];
                STENCIL_CUDA_TRY(cudaStreamWaitEvent(p->s_comm, q->ev_bnd, 0));
                STENCIL_CUDA_TRY(cudaMemcpyAsync(static_cast<char*>(dst[x.peer_lo]) + q->xplan.recv_hi_off,
                                                 static_cast<const char*>(dst[k]) + x.send_lo_off, (size_t)x.msg_bytes,
                                                 cudaMemcpyDeviceToDevice, p->s_comm));
            }
            if (x.peer_hi >= 0) {
                stencil_plan_s* q = plans[x.peer_hi];
                STENCIL_CUDA_TRY(cudaStreamWaitEvent(p->s_comm, q->ev_bnd, 0));
                STENCIL_CUDA_TRY(cudaMemcpyAsync(static_cast<char*>(dst[x.peer_hi]) + q->xplan.recv_lo_off,
                                                 static_cast<const char*>(dst[k]) + x.send_hi_off, (size_t)x.msg_bytes,
                                                 cudaMemcpyDeviceToDevice, p->s_comm));
            }
            STENCIL_CUDA_TRY(cudaEventRecord(p->ev_xchg, p->s_comm));
        }
        // (3) interior segments overlap the exchange
        for (int k = 0; k < nranks; ++k) {
            stencil_plan_s* p = plans[k];
            if (!split[k]) continue;
            SweepSegments in_segs{1, 1, p->cfg.zsegs - 2};
            if ((rc = launch_sweep(p, p->cfg, src[k], nullptr, dst[k], in_segs, dir, st(k))) != STENCIL_SUCCESS) return rc;
        }
        // (4) the next sweep reads the halos the neighbours wrote and overwrites what our copies read
        for (int k = 0; k < nranks; ++k) {
            const stencil_exchange_plan_t& x = plans[k]->xplan;
            STENCIL_CUDA_TRY(cudaStreamWaitEvent(st(k), plans[k]->ev_xchg, 0));
            if (x.peer_lo >= 0) STENCIL_CUDA_TRY(cudaStreamWaitEvent(st(k), plans[x.peer_lo]->ev_xchg, 0));
            if (x.peer_hi >= 0) STENCIL_CUDA_TRY(cudaStreamWaitEvent(st(k), plans[x.peer_hi]->ev_xchg, 0));
            src[k] = dst[k];
        }
    }
    for (int k = 0; k < nranks; ++k) plans[k]->last_sweeps = iters;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_nccl_unique_id(void* uid128) {
    if (!uid128) return fail(STENCIL_ERROR_INVALID_VALUE, "nccl_unique_id: NULL output");
    NcclApi& a = nccl();
    if (!a.ok) return fail(STENCIL_ERROR_NCCL, a.err);
    nccl_uid_t id;
    nccl_result_t r = a.GetUniqueId(&id);
    if (r) return nccl_fail(r, "ncclGetUniqueId");
    memcpy(uid128, id.internal, 128);
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_plan_create_dist(stencil_plan_t* plan, int64_t nx, int64_t ny, int64_t nz_global, int radius,
                                          const double* coeffs, stencil_dtype_t dtype, const void* nccl_uid128,
                                          int rank, int nranks) {
    if (!plan || !coeffs || !nccl_uid128) return fail(STENCIL_ERROR_INVALID_VALUE, "create_dist: NULL argument");
    *plan = nullptr;
    int64_t z0 = 0, nzl = 0;
    stencil_status_t rc = stencil_slab_partition(nz_global, nranks, rank, radius, &z0, &nzl);
    if (rc != STENCIL_SUCCESS) return rc;
    stencil_plan_t p = new (std::nothrow) stencil_plan_s();
    if (!p) return fail(STENCIL_ERROR_OUT_OF_MEMORY, "create_dist: host allocation");
    rc = stencil_plan_init_internal(p, nx, ny, nzl, radius, coeffs, dtype);
    if (rc != STENCIL_SUCCESS) {
        stencil_destroy(p);
        return rc;
    }
    p->dist = true;
    p->rank = rank;
    p->nranks = nranks;
    p->nz_global = nz_global;
    p->z0_global = z0;
    rc = stencil_exchange_plan(&p->lay, nranks, rank, &p->xplan);
    if (rc == STENCIL_SUCCESS && nranks > 1) {
        NcclApi& a = nccl();
        if (!a.ok) {
            rc = fail(STENCIL_ERROR_NCCL, a.err);
        } else {
            nccl_uid_t id;
            memcpy(id.internal, nccl_uid128, 128);
            nccl_result_t r = a.CommInitRank(&p->comm, nranks, id, rank);
            if (r) rc = nccl_fail(r, "ncclCommInitRank");
        }
        if (rc == STENCIL_SUCCESS) {
            if (cudaStreamCreateWithFlags(&p->s_comm, cudaStreamNonBlocking) != cudaSuccess ||
                cudaEventCreateWithFlags(&p->ev_bnd, cudaEventDisableTiming) != cudaSuccess ||
                cudaEventCreateWithFlags(&p->ev_xchg, cudaEventDisableTiming) != cudaSuccess)
                rc = cuda_fail(cudaGetLastError(), "create_dist streams/events");
        }
    }
    if (rc != STENCIL_SUCCESS) {
        stencil_destroy(p);
        return rc;
    }
    p->cfg = default_config(p, STENCIL_KERNEL_INPLANE);
    *plan = p;
    return STENCIL_SUCCESS;
}

}  // extern "C"
