// internal.h -- host-side internals shared by plan.cu, tune.cu, dist.cu.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <string>
#include <deque>
#include <memory>
#include <vector>

#include "../../include/stencil.h"

namespace stencil {

// ---- errors -----------------------------------------------------------------
void set_error(const std::string& msg);
stencil_status_t fail(stencil_status_t st, const std::string& msg);
stencil_status_t cuda_fail(cudaError_t e, const char* what);
#define STENCIL_CUDA_TRY(expr)                                      \
    do {                                                            \
        cudaError_t _e = (expr);                                    \
        if (_e != cudaSuccess) return ::stencil::cuda_fail(_e, #expr); \
    } while (0)

// ---- kernel registry ------------------------------------------------------
struct LaunchArgs {
    dim3 grid, block;
    size_t smem;
    cudaStream_t stream;
    const CUtensorMap* tmap;  // in-plane only
    const CUtensorMap* tmap_g;  // in-plane with a second grid only (div: v)
    const CUtensorMap* tmap_h;  // div: w
    const void* in;           // forward only
    const void* g;            // forward with a second grid only
    void* out;
    void* out1;               // grad: gy
    void* out2;               // grad: gz
    const void* params;       // SweepParams<T>*
};

struct KernelEntry {
    int kernel;  // stencil_kernel_t
    int dtype;   // stencil_dtype_t
    int radius;
    int bx;      // threads along x (in-plane, compile time); 0 for forward
    int rxv;     // 16-byte vectors per thread along x (in-plane); 0 for forward
    int ry;      // rows per thread (in-plane); 1 for forward
    int source;  // 1: variant with a second, centre-only input grid (application stencils)
    int zb;      // warp-specialized in-plane: planes per TMA box (compile time); 0 otherwise
    const void* func;
    cudaError_t (*launch)(const LaunchArgs&);
};

const std::vector<KernelEntry>& kernel_registry();
// kernels that stage planes with TMA boxes (in-plane, warp-specialized in-plane, forward-plane + TMA):
// tile geometry from (tx, rx, ry), tensor maps, ytiles
inline bool tma_kernel(int k) {
    return k == STENCIL_KERNEL_INPLANE || k == STENCIL_KERNEL_INPLANE_WS || k == STENCIL_KERNEL_FP_TMA;
}
const KernelEntry* find_kernel(int kernel, int dtype, int radius, int bx, int rxv, int ry, int source = 0, int zb = 0);

// ---- geometry of a configuration -------------------------------------------
struct Geometry {
    int vec;         // elements per 16-byte vector
    int hx;          // x halo (padded) of the in-plane tile
    int W, H;        // tile extents
    int tiles_x, tiles_y;
    int threads;
    size_t smem;     // dynamic shared memory per block
    int smem_pitch;  // in-plane tile row pitch (elements)
    int stage_elems; // in-plane ring stage (elements)
    uint32_t box_bytes;  // bytes a stage receives (in-plane box + g box)
    int gstage_off;      // element offset of the g box in a stage (source plans)
};

// Validates cfg for a problem; fills g.  Returns SUCCESS or an error (detail set).
stencil_status_t config_geometry(const stencil_layout_t& lay, const stencil_config_t& cfg, Geometry* g,
                                 int source = 0);

// ---- launching one sweep ----------------------------------------------------
struct SweepSegments {
    int seg_base, seg_stride, count;
};

}  // namespace stencil

// ---- the plan -------------------------------------------------------------------
struct stencil_plan_s {
    int device = 0;
    int sm_count = 148;
    stencil_layout_t lay{};
    int r = 1;
    stencil_dtype_t dtype = STENCIL_F32;
    double coeffs[STENCIL_MAX_RADIUS + 1] = {};    // c0, c_m (isotropic) or cx_m (per-axis plans)
    double coeffs_y[STENCIL_MAX_RADIUS + 1] = {};  // per-axis plans: cy_m (isotropic: = coeffs)
    double coeffs_z[STENCIL_MAX_RADIUS + 1] = {};  // per-axis plans: cz_m (isotropic: = coeffs)
    bool axes = false;                             // created by stencil_plan_create_axes
    int app = STENCIL_APP_JACOBI;  // stencil_app_t
    double d = 0.0;                // coefficient of the second grid (SOURCE / WAVE), rounded to dtype
    stencil_config_t cfg{};
    void* scratch = nullptr;
    unsigned long long* d_res = nullptr;  // stencil_run_until: residual bits (device) ...
    unsigned long long* h_res = nullptr;  // ... and its pinned host copy

    // statistics / timing
    int64_t launches = 0, aux_launches = 0;
    int timing = 0;  // 0 off, 1 events around each run's sweeps, 2 an event after every sweep
    std::vector<cudaEvent_t> tev;            // event pool (reused after every stencil_plan_stats)
    size_t tev_used = 0;
    struct Span { size_t first, last; int sweeps; };  // events of one run: first .. last
    std::vector<Span> spans;                 // runs recorded since the last stats call
    int64_t acc_sweeps = 0;                  // totals since stencil_plan_set_timing
    double acc_ms = 0.0, acc_min = -1.0, acc_max = -1.0, last_ms = -1.0;
    int last_sweeps = 0;

    // tensor-map cache (in-plane): keyed by buffer pointer + geometry
    struct MapEntry {
        const void* ptr;
        int box0, box1, box2;
        CUtensorMap map;
    };
    std::deque<MapEntry> maps;  // deque: references stay valid across push_back / pop_front

    // distributed
    bool dist = false;
    int rank = 0, nranks = 1;
    int64_t nz_global = 0, z0_global = 0;
    void* comm = nullptr;
    cudaStream_t s_comm = nullptr, s_aux = nullptr;
    cudaEvent_t ev_bnd = nullptr, ev_xchg = nullptr, ev_fork = nullptr, ev_join = nullptr;
    stencil_exchange_plan_t xplan{};
    // in-process rank group (stencil_plan_create_dist_local): the ranks' plans, shared by all members;
    // the exchange is cudaMemcpyAsync into the neighbour's buffer instead of NCCL
    std::shared_ptr<std::vector<stencil_plan_s*>> local_group;
    unsigned res_seq = 0;  // p2p: residual-reduction rounds so far (flag values)

    // fused peer-store slab plans (p2p.cu): two plan-owned grids, this rank's
    // incoming flags (word 0 written by rank-1, word 1 by rank+1), the
    // neighbours' grids / flag words as mapped into this process
    bool p2p = false;
    void* grid[2] = {nullptr, nullptr};
    unsigned* flags = nullptr;
    unsigned wait_flags = 0;  // cuStreamWaitValue32 flags: GEQ, + FLUSH of remote writes where supported
    void* lo_grid[2] = {nullptr, nullptr};
    void* hi_grid[2] = {nullptr, nullptr};
    unsigned* lo_flag = nullptr;  // word of rank-1 that we write (its flags[1])
    unsigned* hi_flag = nullptr;  // word of rank+1 that we write (its flags[0])
    std::vector<void*> ipc_opened;  // peer allocations opened with cudaIpcOpenMemHandle
    int64_t nz_lo = 0;              // interior planes of rank-1
    unsigned epoch = 0;             // sweeps issued so far (flag values)
    // per-sweep peer targets read by fill_params (null outside p2p sweeps)
    void* sweep_peer_lo = nullptr;
    void* sweep_peer_hi = nullptr;
    long long lo_delta = 0, hi_delta = 0;

    // captured runs (run_jacobi_graph)
    struct GraphEntry {
        const void *in, *g;
        void* out;
        int iters;
        stencil_config_t cfg;
        cudaGraphExec_t exec;
        int64_t launches, aux_launches;
    };
    std::vector<GraphEntry> graphs;
    cudaStream_t s_capture = nullptr;

    // pipelined host-to-host runs (stencil_run_host)
    struct HostSlot {
        void *din = nullptr, *dout = nullptr;
        cudaEvent_t h2d_done = nullptr, comp_done = nullptr, d2h_done = nullptr;
    };
    HostSlot hslot[2];
    cudaStream_t hs_h2d = nullptr, hs_comp = nullptr, hs_d2h = nullptr;
    cudaEvent_t hs_fork = nullptr;
    int64_t host_calls = 0;

    // tuner results
    std::vector<stencil_tune_entry_t> tune_results;
};

namespace stencil {
// Kernel variant a plan runs (KernelEntry::source): 0 plain Eq. (1), 1 second grid, 2 per-axis.
inline int kernel_variant(const stencil_plan_s* p) {
    if (p->app == STENCIL_APP_DIV) return 4;
    if (p->app == STENCIL_APP_GRAD) return 5;
    return p->app != STENCIL_APP_JACOBI ? 1 : (p->axes ? 2 : (p->p2p ? 3 : 0));
}
stencil_status_t p2p_destroy(stencil_plan_s* p);
void preload_kernels(stencil_plan_s* p);

// One sweep src -> dst of the given segments, on stream st (counts launches).
stencil_status_t launch_sweep(stencil_plan_s* plan, const stencil_config_t& cfg, const void* src, const void* g, void* dst,
                              const SweepSegments& segs, int dir, cudaStream_t st);
// Copy the outer shell of src into dst (async).
stencil_status_t launch_shell_copy(stencil_plan_s* plan, const void* src, void* dst, cudaStream_t st);
// Exchange halos of `buf` after a sweep (distributed plans; dist.cu).
stencil_status_t dist_exchange(stencil_plan_s* plan, void* buf, cudaStream_t st);
stencil_status_t dist_destroy(stencil_plan_s* plan);
// In-place max over the ranks of one device u64 (NCCL all-reduce; distributed plans).
stencil_status_t dist_allreduce_max_u64(stencil_plan_s* plan, unsigned long long* word, cudaStream_t st);
// Default configuration chosen from the B200 model (tune.cu).
stencil_config_t default_config(stencil_plan_s* plan, int kernel);
void gpu_params(int device, stencil_gpu_params_t* g);
}  // namespace stencil
