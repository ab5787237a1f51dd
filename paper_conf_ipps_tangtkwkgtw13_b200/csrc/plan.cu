// plan.cu -- C ABI entry points (include/stencil.h): plans, layout, the
// iteration loop of Fig. 1, kernel registry and launches.
#include <cudaTypedefs.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <initializer_list>
#include <mutex>
#include <string>

#include "common.cuh"
#include "forward.cuh"
#include "internal.h"

namespace stencil {

// ============================================================================
// errors
// ============================================================================
static thread_local std::string g_err;

void set_error(const std::string& msg) { g_err = msg; }

stencil_status_t fail(stencil_status_t st, const std::string& msg) {
    g_err = msg;
    return st;
}

stencil_status_t cuda_fail(cudaError_t e, const char* what) {
    g_err = std::string(what) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")";
    return STENCIL_ERROR_CUDA;
}

// ============================================================================
// auxiliary kernels
// ============================================================================

// Copy the r-wide outer shell of src into dst.  One warp per outer row.
template <typename T>
__global__ void shell_copy_kernel(const T* __restrict__ src, T* __restrict__ dst, int nx, int ny, int nz, int r,
                                  long long pitch, int rows, int x_origin) {
    const long long nrows = (long long)rows * (nz + 2 * r);
    const int lane = threadIdx.x & 31;
    const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    for (long long row = warp; row < nrows; row += nwarps) {
        const int z = (int)(row / rows), y = (int)(row % rows);
        const long long base = row * pitch + x_origin;
        const bool full = (z < r) || (z >= nz + r) || (y < r) || (y >= ny + r);
        if (full) {
            for (int x = lane; x < nx + 2 * r; x += 32) dst[base + x] = src[base + x];
        } else if (lane < 2 * r) {
            const int x = lane < r ? lane : nx + lane;  // [0, r) and [nx + r, nx + 2r)
            dst[base + x] = src[base + x];
        }
    }
}

// Stop criterion of Fig. 1 (reading R5b): max over interior points of
// |a - b| in T, as the bit pattern of a non-negative T (ordered like the
// value; a NaN compares above +inf, so it never passes a tolerance).  One warp
// per interior row, warp max by shuffle, one atomicMax per warp.
template <typename T>
__global__ void residual_kernel(const T* __restrict__ a, const T* __restrict__ b, int nx, int ny, int nz, int r,
                                long long pitch, int rows, int x0, unsigned long long* __restrict__ res) {
    const long long nrows = (long long)ny * nz;
    const int lane = threadIdx.x & 31;
    const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
    T m = T(0);
    for (long long row = warp; row < nrows; row += nwarps) {
        const int z = (int)(row / ny), y = (int)(row % ny);
        const long long base = ((long long)(z + r) * rows + (y + r)) * pitch + x0;
        for (int x = lane; x < nx; x += 32) {
            const T d = fabs(a[base + x] - b[base + x]);
            m = (d > m || d != d) ? d : m;
        }
    }
    unsigned long long bits = sizeof(T) == 4 ? (unsigned long long)__float_as_uint((float)m)
                                             : (unsigned long long)__double_as_longlong((double)m);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long other = __shfl_xor_sync(0xffffffffu, bits, o);
        bits = other > bits ? other : bits;
    }
    if (lane == 0 && bits) atomicMax(res, bits);
}

__device__ __forceinline__ unsigned long long splitmix64_dev(unsigned long long x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

// Counter-based field of stencil_inputs.counter (same bits), padding = 0.
template <typename T>
__global__ void fill_counter_kernel(T* __restrict__ buf, int nx, int ny, int r, long long pitch, int rows,
                                    int planes, int A, long long kz0, unsigned long long seed) {
    const long long total = (long long)planes * rows * pitch;
    const long long px = nx + 2 * r, py = ny + 2 * r;
    for (long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x; e < total;
         e += (long long)gridDim.x * blockDim.x) {
        const long long row = e / pitch;
        const int xe = (int)(e % pitch);
        const int i = xe - (A - r);  // outer x index in [0, nx + 2r)
        T v = T(0);
        if (i >= 0 && i < px) {
            const long long kk = row / rows + kz0, jj = row % rows;
            const unsigned long long lin = (unsigned long long)((kk * py + jj) * px + i);
            const unsigned long long h = splitmix64_dev(lin + (seed << 40));
            if constexpr (sizeof(T) == 4)
                v = (T)((double)(h >> 40) * 0x1.0p-24);
            else
                v = (T)((double)(h >> 11) * 0x1.0p-53);
        }
        buf[e] = v;
    }
}

// Load the plan's kernels now (cudaFuncGetAttributes forces a lazily loaded function in): with
// CUDA_MODULE_LOADING=LAZY a first launch can wait for the context to go idle, and slab plans whose
// streams wait on their neighbours' flags never let it (in-process p2p slabs, one host thread each).
void preload_kernels(stencil_plan_s* p) {
    cudaFuncAttributes a;
    if (p->dtype == STENCIL_F32) {
        cudaFuncGetAttributes(&a, residual_kernel<float>);
        cudaFuncGetAttributes(&a, shell_copy_kernel<float>);
        cudaFuncGetAttributes(&a, fill_counter_kernel<float>);
    } else {
        cudaFuncGetAttributes(&a, residual_kernel<double>);
        cudaFuncGetAttributes(&a, shell_copy_kernel<double>);
        cudaFuncGetAttributes(&a, fill_counter_kernel<double>);
    }
    Geometry g;
    const stencil_config_t& c = p->cfg;
    if (config_geometry(p->lay, c, &g, kernel_variant(p)) == STENCIL_SUCCESS) {
        const bool tma = tma_kernel(c.kernel);
        const KernelEntry* ke = find_kernel(c.kernel, p->dtype, p->r, tma ? c.tx : 0, tma ? c.rx / g.vec : 0, c.ry,
                                            kernel_variant(p), c.kernel == STENCIL_KERNEL_INPLANE_WS ? c.zbox : 0);
        if (ke) cudaFuncGetAttributes(&a, ke->func);
    }
    cudaGetLastError();
    set_error("");
}

// ============================================================================
// kernel registry (instantiations live in kern_<dtype>_r<R>.cu, compiled in parallel)
// ============================================================================
#define STENCIL_DECL_DG(d, r) void register_##d##_r##r##_dg(std::vector<KernelEntry>&);
#define STENCIL_DECL_REG(d, r)                          \
    void register_##d##_r##r(std::vector<KernelEntry>&); \
    void register_##d##_r##r##_g(std::vector<KernelEntry>&); \
    void register_##d##_r##r##_ax(std::vector<KernelEntry>&); \
    void register_##d##_r##r##_ps(std::vector<KernelEntry>&); \
    void register_##d##_r##r##_ws(std::vector<KernelEntry>&); \
    void register_##d##_r##r##_abl(std::vector<KernelEntry>&); \
    STENCIL_DECL_DG(d, r)
STENCIL_DECL_REG(f32, 1) STENCIL_DECL_REG(f32, 2) STENCIL_DECL_REG(f32, 3)
STENCIL_DECL_REG(f32, 4) STENCIL_DECL_REG(f32, 5) STENCIL_DECL_REG(f32, 6)
STENCIL_DECL_REG(f64, 1) STENCIL_DECL_REG(f64, 2) STENCIL_DECL_REG(f64, 3)
STENCIL_DECL_REG(f64, 4) STENCIL_DECL_REG(f64, 5) STENCIL_DECL_REG(f64, 6)
#undef STENCIL_DECL_REG

const std::vector<KernelEntry>& kernel_registry() {
    static const std::vector<KernelEntry> reg = [] {
        std::vector<KernelEntry> v;
        for (auto f : {register_f32_r1, register_f32_r2, register_f32_r3, register_f32_r4, register_f32_r5,
                       register_f32_r6, register_f64_r1, register_f64_r2, register_f64_r3, register_f64_r4,
                       register_f64_r5, register_f64_r6, register_f32_r1_g, register_f32_r2_g, register_f32_r3_g,
                       register_f32_r4_g, register_f32_r5_g, register_f32_r6_g, register_f64_r1_g, register_f64_r2_g,
                       register_f64_r3_g, register_f64_r4_g, register_f64_r5_g, register_f64_r6_g,
                       register_f32_r1_ax, register_f32_r2_ax, register_f32_r3_ax, register_f32_r4_ax,
                       register_f32_r5_ax, register_f32_r6_ax, register_f64_r1_ax, register_f64_r2_ax,
                       register_f64_r3_ax, register_f64_r4_ax, register_f64_r5_ax, register_f64_r6_ax,
                       register_f32_r1_ps, register_f32_r2_ps, register_f32_r3_ps, register_f32_r4_ps,
                       register_f32_r5_ps, register_f32_r6_ps, register_f64_r1_ps, register_f64_r2_ps,
                       register_f64_r3_ps, register_f64_r4_ps, register_f64_r5_ps, register_f64_r6_ps,
                       register_f32_r1_ws, register_f32_r2_ws, register_f32_r3_ws, register_f32_r4_ws,
                       register_f32_r5_ws, register_f32_r6_ws, register_f64_r1_ws, register_f64_r2_ws,
                       register_f64_r3_ws, register_f64_r4_ws, register_f64_r5_ws, register_f64_r6_ws,
                       register_f32_r1_abl, register_f32_r2_abl, register_f32_r3_abl, register_f32_r4_abl,
                       register_f32_r5_abl, register_f32_r6_abl, register_f64_r1_abl, register_f64_r2_abl,
                       register_f64_r3_abl, register_f64_r4_abl, register_f64_r5_abl, register_f64_r6_abl,
                       register_f32_r1_dg, register_f32_r2_dg, register_f32_r3_dg, register_f32_r4_dg,
                       register_f64_r1_dg, register_f64_r2_dg, register_f64_r3_dg, register_f64_r4_dg})
            f(v);
        return v;
    }();
    return reg;
}

const KernelEntry* find_kernel(int kernel, int dtype, int radius, int bx, int rxv, int ry, int source, int zb) {
    for (const auto& e : kernel_registry())
        if (e.kernel == kernel && e.dtype == dtype && e.radius == radius && e.source == source && e.ry == ry &&
            (!tma_kernel(kernel) || (e.bx == bx && e.rxv == rxv)) &&
            (kernel != STENCIL_KERNEL_INPLANE_WS || e.zb == zb))
            return &e;
    return nullptr;
}

// ============================================================================
// geometry / validation
// ============================================================================
static constexpr size_t kMaxSmem = 227 * 1024;

stencil_status_t config_geometry(const stencil_layout_t& lay, const stencil_config_t& c, Geometry* g, int source) {
    const int s = (int)lay.elem_size;
    const int r = lay.radius;
    Geometry o{};
    o.vec = 16 / s;
    o.hx = ((r + o.vec - 1) / o.vec) * o.vec;
    if (c.tx < 1 || c.ty < 1 || c.zsegs < 1)
        return fail(STENCIL_ERROR_INVALID_VALUE, "config: tx, ty, zsegs must be >= 1");
    if (c.zsegs > lay.nz) return fail(STENCIL_ERROR_INVALID_VALUE, "config: zsegs > nz");
    o.threads = c.tx * c.ty;
    if (tma_kernel(c.kernel)) {
        const bool ws = c.kernel == STENCIL_KERNEL_INPLANE_WS;
        // constraint (i) of P:L256: TX a multiple of a half-warp
        if (c.tx % 16 != 0) return fail(STENCIL_ERROR_INVALID_VALUE, "config: tx must be a multiple of 16");
        if (o.threads > 256) return fail(STENCIL_ERROR_INVALID_VALUE, "config: in-plane block limited to 256 threads");
        if (ws && o.threads % 32 != 0)
            return fail(STENCIL_ERROR_INVALID_VALUE, "config: warp-specialized in-plane needs tx*ty a multiple of 32");
        if (c.rx % o.vec != 0) return fail(STENCIL_ERROR_INVALID_VALUE, "config: rx must be a multiple of the 16-byte vector");
        const int rxv = c.rx / o.vec;
        if (!find_kernel(c.kernel, lay.dtype, r, c.tx, rxv, c.ry, source, ws ? c.zbox : 0))
            return fail(STENCIL_ERROR_NOT_SUPPORTED, "config: no in-plane instantiation for this (r, tx, rx, ry, zbox)");
        if (c.stages < 2 || c.stages > 16) return fail(STENCIL_ERROR_INVALID_VALUE, "config: stages must be in [2, 16]");
        // forward-plane + TMA (fp_tma.cuh): the ring holds planes z .. z+r plus the load in flight
        if (c.kernel == STENCIL_KERNEL_FP_TMA && c.zbox >= 1 && c.stages < (r + c.zbox - 1) / c.zbox + 2)
            return fail(STENCIL_ERROR_INVALID_VALUE, "config: forward-plane TMA needs stages >= ceil(r/zbox) + 2");
        o.W = c.tx * c.rx;
        o.H = c.ty * c.ry;
        // TMA box limits: <= 256 elements per dimension
        if (o.W + 2 * o.hx > 256 || o.H + 2 * r > 256)
            return fail(STENCIL_ERROR_INVALID_VALUE, "config: tile + halo exceeds the TMA box limit of 256");
        if (c.zbox < 1 || c.zbox > 8) return fail(STENCIL_ERROR_INVALID_VALUE, "config: zbox must be in [1, 8]");
        o.smem_pitch = o.W + 2 * o.hx;
        auto rnd = [](int bytes) { return ((bytes + 127) / 128) * 128; };
        if (source == 4) {
            // Div (divgrad.cuh): u x-halo box, v y-halo box, w centre box per stage
            const int ub = o.smem_pitch * o.H * s * c.zbox, vb = o.W * (o.H + 2 * r) * s * c.zbox,
                      wb = o.W * o.H * s * c.zbox;
            o.gstage_off = 0;
            o.stage_elems = (rnd(ub) + rnd(vb) + rnd(wb)) / s;
            o.box_bytes = (uint32_t)(ub + vb + wb);
        } else {
            const int stage_bytes = o.smem_pitch * (o.H + 2 * r) * s * c.zbox;
            // source plans: the g box (W x H x zbox, centre only) follows in the same stage
            const int g_bytes = source == 1 ? o.W * o.H * s * c.zbox : 0;  // (variant 1: second grid)
            o.gstage_off = rnd(stage_bytes) / s;
            o.stage_elems = o.gstage_off + rnd(g_bytes) / s;
            o.box_bytes = (uint32_t)(stage_bytes + g_bytes);
        }
        o.smem = 128 * (size_t)((2 * c.stages * 8 + 127) / 128) + (size_t)c.stages * o.stage_elems * s;
        // compute warps padded to whole warpgroups + the producer warpgroup (inplane_ws.cuh)
        if (ws) o.threads = (o.threads + 127) / 128 * 128 + 128;
    } else if (c.kernel == STENCIL_KERNEL_FORWARD ||
               (c.kernel >= STENCIL_KERNEL_IP_CLASSIC && c.kernel <= STENCIL_KERNEL_IP_FULLSLICE_V)) {
        const bool fwd = c.kernel == STENCIL_KERNEL_FORWARD;
        if (c.rx != 1 || c.zbox != 1)
            return fail(STENCIL_ERROR_INVALID_VALUE, "config: forward-plane / loading-variant kernels use rx = zbox = 1");
        if (c.tx % 16 != 0) return fail(STENCIL_ERROR_INVALID_VALUE, "config: tx must be a multiple of 16");
        if (o.threads > 512) return fail(STENCIL_ERROR_INVALID_VALUE, "config: block limited to 512 threads");
        if (c.tx < r || c.ty < r) return fail(STENCIL_ERROR_INVALID_VALUE, "config: halo loads need tx, ty >= r");
        if (!find_kernel(c.kernel, lay.dtype, r, 0, 0, c.ry, source))
            return fail(STENCIL_ERROR_NOT_SUPPORTED, "config: no instantiation for this (kernel, r, ry)");
        o.W = c.tx;
        o.H = c.ty * c.ry;
        if (fwd) {
            o.smem = (size_t)fp_tile_pitch(c.tx, r, s) * (o.H + 2 * r) * s;
        } else {
            const int v = 16 / s, hx = c.kernel == STENCIL_KERNEL_IP_FULLSLICE_V ? ((r + v - 1) / v) * v : r;
            int sp = c.tx + 2 * hx;
            if (c.kernel != STENCIL_KERNEL_IP_FULLSLICE_V && (sp * s / 4) % 32 == 0) sp += 1;  // AblGeom::pitch
            o.smem = 2 * (size_t)sp * (o.H + 2 * r) * s;
        }
    } else {
        return fail(STENCIL_ERROR_INVALID_VALUE, "config: unknown kernel");
    }
    if (o.smem > kMaxSmem) return fail(STENCIL_ERROR_INVALID_VALUE, "config: shared memory exceeds 227 KB");
    o.tiles_x = (int)((lay.nx + o.W - 1) / o.W);
    if (c.ytiles < 0) return fail(STENCIL_ERROR_INVALID_VALUE, "config: ytiles < 0");
    if (c.ytiles > 0 && !tma_kernel(c.kernel))
        return fail(STENCIL_ERROR_INVALID_VALUE, "config: ytiles is an in-plane option");
    o.tiles_y = c.ytiles > 0 ? c.ytiles : (int)((lay.ny + o.H - 1) / o.H);
    if (o.tiles_y > lay.ny || (lay.ny + o.tiles_y - 1) / o.tiles_y > o.H)
        return fail(STENCIL_ERROR_INVALID_VALUE, "config: ytiles leaves a tile taller than ty*ry");
    if (o.tiles_y > 65535) return fail(STENCIL_ERROR_INVALID_VALUE, "config: too many y tiles");
    *g = o;
    return STENCIL_SUCCESS;
}

// ============================================================================
// tensor maps
// ============================================================================
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &p, 12000, cudaEnableDefault, &q) ==
                cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    });
    return fn;
}

static stencil_status_t get_map(stencil_plan_s* plan, const void* ptr, int box0, int box1, int box2,
                                const CUtensorMap** out) {
    for (auto& m : plan->maps)
        if (m.ptr == ptr && m.box0 == box0 && m.box1 == box1 && m.box2 == box2) {
            *out = &m.map;
            return STENCIL_SUCCESS;
        }
    auto enc = get_encode();
    if (!enc) return fail(STENCIL_ERROR_CUDA, "cuTensorMapEncodeTiled unavailable from the driver");
    const stencil_layout_t& L = plan->lay;
    stencil_plan_s::MapEntry e{};
    e.ptr = ptr;
    e.box0 = box0;
    e.box1 = box1;
    e.box2 = box2;
    cuuint64_t dims[3] = {(cuuint64_t)L.pitch_x, (cuuint64_t)L.rows_y, (cuuint64_t)L.planes_z};
    cuuint64_t strides[2] = {(cuuint64_t)(L.pitch_x * L.elem_size), (cuuint64_t)(L.pitch_x * L.rows_y * L.elem_size)};
    cuuint32_t box[3] = {(cuuint32_t)box0, (cuuint32_t)box1, (cuuint32_t)box2};
    cuuint32_t estr[3] = {1, 1, 1};
    // L2 promotion: box rows are W+2HX elements starting 16 B before a 128-B
    // line, so the x halo of a row's first and last box (the shell columns at
    // the grid's x edges) sits in a line of its own; 128-B promotion fetches
    // that whole line (the row's pitch padding included) and 256-B fetched up
    // to 1.8x the bytes for 64-wide tiles.  Short rows (<= 24 lines, e.g.
    // 512^3 f32: 18) take 64-B promotion: 512^3 r=4 f32 reads 580-598 instead
    // of 629-648 MB per sweep and ran 716 vs 608 / 714 vs 711 Gpts/s in
    // same-box sustained A/Bs (profiles/r2e/promo, profiles/r2f); long rows
    // keep 128 B, where the edge lines are a few per cent of a row and 64-B
    // promotion measured 6-7 % slower (2048^2 x 1024 f32, 610 vs 654 Gpts/s,
    // profiles/r2f/c5promo*)
    CUtensorMapL2promotion promo = L.pitch_x * L.elem_size <= 24 * 128 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
                                                                        : CU_TENSOR_MAP_L2_PROMOTION_L2_128B;
    if (const char* e = getenv("STENCIL_L2_PROMO")) {
        const std::string v(e);
        if (v == "none") promo = CU_TENSOR_MAP_L2_PROMOTION_NONE;
        else if (v == "64") promo = CU_TENSOR_MAP_L2_PROMOTION_L2_64B;
        else if (v == "128") promo = CU_TENSOR_MAP_L2_PROMOTION_L2_128B;
        else if (v == "256") promo = CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
    }
    CUresult rc = enc(&e.map, plan->dtype == STENCIL_F32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64,
                      3, const_cast<void*>(ptr), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      CU_TENSOR_MAP_SWIZZLE_NONE, promo,
                      CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (rc != CUDA_SUCCESS) return fail(STENCIL_ERROR_CUDA, "cuTensorMapEncodeTiled failed: " + std::to_string((int)rc));
    if (plan->maps.size() >= 16) plan->maps.pop_front();
    plan->maps.push_back(e);
    *out = &plan->maps.back().map;
    return STENCIL_SUCCESS;
}

// ============================================================================
// launches
// ============================================================================
template <typename T>
static void fill_params(const stencil_plan_s* plan, const Geometry& g, const stencil_config_t& cfg,
                        const SweepSegments& segs, int dir, SweepParams<T>* p) {
    const stencil_layout_t& L = plan->lay;
    p->nx = (int)L.nx;
    p->ny = (int)L.ny;
    p->nz = (int)L.nz;
    p->rows = (int)L.rows_y;
    p->pitch = L.pitch_x;
    p->plane = L.pitch_x * L.rows_y;
    p->A = (int)L.interior_x0;
    p->tiles_x = g.tiles_x;
    p->tiles_y = g.tiles_y;
    p->zsegs = cfg.zsegs;
    p->seg_base = segs.seg_base;
    p->seg_stride = segs.seg_stride;
    p->stages = cfg.stages;
    p->smem_pitch = g.smem_pitch;
    p->stage_elems = g.stage_elems;
    p->zbox = cfg.zbox;
    static const int spol = getenv("STENCIL_STORE_POLICY") ? atoi(getenv("STENCIL_STORE_POLICY")) : 0;
    static const int lpol = getenv("STENCIL_LOAD_POLICY") ? atoi(getenv("STENCIL_LOAD_POLICY")) : 0;
    p->store_policy = spol;
    p->load_policy = lpol;
    p->dir = dir;
    static const int dbg = getenv("STENCIL_DEBUG") ? atoi(getenv("STENCIL_DEBUG")) : 0;
    p->debug = dbg;
    p->stage_tx_bytes = g.box_bytes;
    p->gstage_off = g.gstage_off;
    for (int m = 0; m <= STENCIL_MAX_RADIUS; ++m) {
        p->c[m] = (T)plan->coeffs[m];
        p->cy[m] = (T)plan->coeffs_y[m];
        p->cz[m] = (T)plan->coeffs_z[m];
    }
    p->peer_lo = static_cast<T*>(plan->sweep_peer_lo);
    p->peer_hi = static_cast<T*>(plan->sweep_peer_hi);
    p->lo_delta = plan->lo_delta;
    p->hi_delta = plan->hi_delta;
    p->d = (T)plan->d;
    p->ws_warps = cfg.tx * cfg.ty / 32;
}

stencil_status_t launch_sweep(stencil_plan_s* plan, const stencil_config_t& cfg, const void* src, const void* gsrc,
                              void* dst, const SweepSegments& segs, int dir, cudaStream_t st) {
    if (segs.count <= 0) return STENCIL_SUCCESS;
    const int source = kernel_variant(plan);
    if ((source == 1) != (gsrc != nullptr))
        return fail(STENCIL_ERROR_INVALID_VALUE, "sweep: second grid / plan kind mismatch");
    Geometry g;
    stencil_status_t rc = config_geometry(plan->lay, cfg, &g, source);
    if (rc != STENCIL_SUCCESS) return rc;
    const bool ws = cfg.kernel == STENCIL_KERNEL_INPLANE_WS;
    const bool tma = tma_kernel(cfg.kernel);
    const int rxv = tma ? cfg.rx / g.vec : 0;
    const KernelEntry* ke = find_kernel(cfg.kernel, plan->dtype, plan->r, cfg.tx, rxv, cfg.ry, source, ws ? cfg.zbox : 0);
    if (!ke) return fail(STENCIL_ERROR_NOT_SUPPORTED, "no kernel instantiation for this configuration");
    if (g.smem > 48 * 1024)
        STENCIL_CUDA_TRY(cudaFuncSetAttribute(ke->func, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g.smem));
    LaunchArgs a{};
    a.grid = dim3(g.tiles_x, g.tiles_y, segs.count);
    a.block = ws ? dim3(g.threads, 1, 1) : dim3(cfg.tx, cfg.ty, 1);
    a.smem = g.smem;
    a.stream = st;
    a.in = src;
    a.g = gsrc;
    a.out = dst;
    SweepParams<float> pf;
    SweepParams<double> pd;
    if (plan->dtype == STENCIL_F32) {
        fill_params(plan, g, cfg, segs, dir, &pf);
        a.params = &pf;
    } else {
        fill_params(plan, g, cfg, segs, dir, &pd);
        a.params = &pd;
    }
    // local copies: a later get_map may evict the cache entry an earlier one returned
    CUtensorMap map_in, map_g;
    if (tma) {
        const CUtensorMap* m = nullptr;
        rc = get_map(plan, src, g.W + 2 * g.hx, g.H + 2 * plan->r, cfg.zbox, &m);
        if (rc != STENCIL_SUCCESS) return rc;
        map_in = *m;
        a.tmap = &map_in;

        if (source == 1) {
            rc = get_map(plan, gsrc, g.W, g.H, cfg.zbox, &m);
            if (rc != STENCIL_SUCCESS) return rc;
            map_g = *m;
            a.tmap_g = &map_g;
        }
    }
    cudaError_t e = ke->launch(a);
    if (e != cudaSuccess) return cuda_fail(e, "sweep kernel launch");
    plan->launches++;
    return STENCIL_SUCCESS;
}

// One Div / Grad sweep (divgrad.cuh): in[0..2] = u, v, w (div) or f (grad), out[0..2] = out (div) or
// gx, gy, gz (grad); all segments, streamed upward.
stencil_status_t launch_divgrad(stencil_plan_s* plan, const stencil_config_t& cfg, const void* const* in,
                                void* const* out, cudaStream_t st) {
    const int source = kernel_variant(plan);
    Geometry g;
    stencil_status_t rc = config_geometry(plan->lay, cfg, &g, source);
    if (rc != STENCIL_SUCCESS) return rc;
    const KernelEntry* ke = find_kernel(cfg.kernel, plan->dtype, plan->r, cfg.tx, cfg.rx / g.vec, cfg.ry, source, cfg.zbox);
    if (!ke) return fail(STENCIL_ERROR_NOT_SUPPORTED, "no div/grad kernel for this configuration");
    if (g.smem > 48 * 1024)
        STENCIL_CUDA_TRY(cudaFuncSetAttribute(ke->func, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g.smem));
    LaunchArgs a{};
    a.grid = dim3(g.tiles_x, g.tiles_y, cfg.zsegs);
    a.block = dim3(g.threads, 1, 1);
    a.smem = g.smem;
    a.stream = st;
    a.out = out[0];
    a.out1 = out[1];
    a.out2 = out[2];
    SweepParams<float> pf;
    SweepParams<double> pd;
    const SweepSegments all{0, 1, cfg.zsegs};
    if (plan->dtype == STENCIL_F32) {
        fill_params(plan, g, cfg, all, 1, &pf);
        a.params = &pf;
    } else {
        fill_params(plan, g, cfg, all, 1, &pd);
        a.params = &pd;
    }
    CUtensorMap m0, m1, m2;
    const CUtensorMap* m = nullptr;
    const int r = plan->r;
    if (source == 4) {
        if ((rc = get_map(plan, in[0], g.W + 2 * g.hx, g.H, cfg.zbox, &m)) != STENCIL_SUCCESS) return rc;
        m0 = *m;
        if ((rc = get_map(plan, in[1], g.W, g.H + 2 * r, cfg.zbox, &m)) != STENCIL_SUCCESS) return rc;
        m1 = *m;
        if ((rc = get_map(plan, in[2], g.W, g.H, cfg.zbox, &m)) != STENCIL_SUCCESS) return rc;
        m2 = *m;
    } else {
        if ((rc = get_map(plan, in[0], g.W + 2 * g.hx, g.H + 2 * r, cfg.zbox, &m)) != STENCIL_SUCCESS) return rc;
        m0 = m1 = m2 = *m;
    }
    a.tmap = &m0;
    a.tmap_g = &m1;
    a.tmap_h = &m2;
    cudaError_t e = ke->launch(a);
    if (e != cudaSuccess) return cuda_fail(e, "div/grad kernel launch");
    plan->launches++;
    return STENCIL_SUCCESS;
}

stencil_status_t launch_shell_copy(stencil_plan_s* plan, const void* src, void* dst, cudaStream_t st) {
    const stencil_layout_t& L = plan->lay;
    const long long nrows = L.rows_y * L.planes_z;
    const int threads = 256;
    long long blocks = (nrows * 32 + threads - 1) / threads;
    blocks = std::min<long long>(blocks, (long long)plan->sm_count * 16);
    if (plan->dtype == STENCIL_F32)
        shell_copy_kernel<float><<<(unsigned)blocks, threads, 0, st>>>(
            (const float*)src, (float*)dst, (int)L.nx, (int)L.ny, (int)L.nz, plan->r, L.pitch_x, (int)L.rows_y,
            (int)L.x_origin);
    else
        shell_copy_kernel<double><<<(unsigned)blocks, threads, 0, st>>>(
            (const double*)src, (double*)dst, (int)L.nx, (int)L.ny, (int)L.nz, plan->r, L.pitch_x, (int)L.rows_y,
            (int)L.x_origin);
    STENCIL_CUDA_TRY(cudaGetLastError());
    plan->aux_launches++;
    return STENCIL_SUCCESS;
}

}  // namespace stencil

using namespace stencil;

// ============================================================================
// C ABI
// ============================================================================
extern "C" {

const char* stencil_status_string(stencil_status_t s) {
    switch (s) {
        case STENCIL_SUCCESS: return "STENCIL_SUCCESS";
        case STENCIL_ERROR_INVALID_VALUE: return "STENCIL_ERROR_INVALID_VALUE";
        case STENCIL_ERROR_NOT_SUPPORTED: return "STENCIL_ERROR_NOT_SUPPORTED";
        case STENCIL_ERROR_MISALIGNED: return "STENCIL_ERROR_MISALIGNED";
        case STENCIL_ERROR_OUT_OF_MEMORY: return "STENCIL_ERROR_OUT_OF_MEMORY";
        case STENCIL_ERROR_CUDA: return "STENCIL_ERROR_CUDA";
        case STENCIL_ERROR_NCCL: return "STENCIL_ERROR_NCCL";
    }
    return "STENCIL_ERROR_UNKNOWN";
}

const char* stencil_last_error_detail(void) { return g_err.c_str(); }

int stencil_abi_version(void) { return STENCIL_ABI_VERSION; }

stencil_status_t stencil_layout_compute(int64_t nx, int64_t ny, int64_t nz, int radius, stencil_dtype_t dtype,
                                        stencil_layout_t* out) {
    if (!out) return fail(STENCIL_ERROR_INVALID_VALUE, "layout: NULL output");
    if (nx < 1 || ny < 1 || nz < 1) return fail(STENCIL_ERROR_INVALID_VALUE, "layout: extents must be >= 1");
    if (radius < 1 || radius > STENCIL_MAX_RADIUS) return fail(STENCIL_ERROR_INVALID_VALUE, "layout: radius must be in [1, 6]");
    if (dtype != STENCIL_F32 && dtype != STENCIL_F64) return fail(STENCIL_ERROR_INVALID_VALUE, "layout: unknown dtype");
    if (nx > (1 << 28) || ny > (1 << 28) || nz > (1 << 28))
        return fail(STENCIL_ERROR_INVALID_VALUE, "layout: extent too large");
    stencil_layout_t L{};
    L.nx = nx;
    L.ny = ny;
    L.nz = nz;
    L.radius = radius;
    L.dtype = dtype;
    L.elem_size = dtype == STENCIL_F32 ? 4 : 8;
    const int64_t A = 128 / L.elem_size;
    L.interior_x0 = A;
    L.x_origin = A - radius;
    L.pitch_x = ((A + nx + radius + A - 1) / A) * A;
    L.rows_y = ny + 2 * radius;
    L.planes_z = nz + 2 * radius;
    L.bytes = L.planes_z * L.rows_y * L.pitch_x * L.elem_size;
    *out = L;
    return STENCIL_SUCCESS;
}

static stencil_status_t plan_init(stencil_plan_t p, int64_t nx, int64_t ny, int64_t nz, int radius,
                                  const double* coeffs, stencil_dtype_t dtype) {
    stencil_status_t rc = stencil_layout_compute(nx, ny, nz, radius, dtype, &p->lay);
    if (rc != STENCIL_SUCCESS) return rc;
    STENCIL_CUDA_TRY(cudaGetDevice(&p->device));
    cudaDeviceProp prop;
    STENCIL_CUDA_TRY(cudaGetDeviceProperties(&prop, p->device));
    if (prop.major != 10 || prop.minor != 0)
        return fail(STENCIL_ERROR_NOT_SUPPORTED, std::string("device is sm_") + std::to_string(prop.major) +
                                                     std::to_string(prop.minor) + ", this library is built for sm_100a");
    p->sm_count = prop.multiProcessorCount;
    p->r = radius;
    p->dtype = dtype;
    for (int m = 0; m <= STENCIL_MAX_RADIUS; ++m) p->coeffs[m] = m <= radius ? coeffs[m] : 0.0;
    // round to the plan's type once (what every kernel sees)
    if (dtype == STENCIL_F32)
        for (int m = 0; m <= radius; ++m) p->coeffs[m] = (double)(float)p->coeffs[m];
    for (int m = 0; m <= STENCIL_MAX_RADIUS; ++m) p->coeffs_y[m] = p->coeffs_z[m] = p->coeffs[m];
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_plan_create_app(stencil_plan_t* plan, int64_t nx, int64_t ny, int64_t nz, int radius,
                                         const double* coeffs, stencil_dtype_t dtype, stencil_app_t app, double d) {
    if (!plan || !coeffs) return fail(STENCIL_ERROR_INVALID_VALUE, "plan_create: NULL argument");
    *plan = nullptr;
    if (app != STENCIL_APP_JACOBI && app != STENCIL_APP_SOURCE && app != STENCIL_APP_WAVE)
        return fail(STENCIL_ERROR_INVALID_VALUE, "plan_create: unknown application kind");
    if (!std::isfinite(d)) return fail(STENCIL_ERROR_INVALID_VALUE, "plan_create: d must be finite");
    stencil_plan_t p = new (std::nothrow) stencil_plan_s();
    if (!p) return fail(STENCIL_ERROR_OUT_OF_MEMORY, "plan_create: host allocation");
    stencil_status_t rc = plan_init(p, nx, ny, nz, radius, coeffs, dtype);
    if (rc != STENCIL_SUCCESS) {
        stencil_destroy(p);
        return rc;
    }
    p->app = app;
    p->d = app == STENCIL_APP_JACOBI ? 0.0 : (dtype == STENCIL_F32 ? (double)(float)d : d);
    // plain sweeps default to the warp-specialized in-plane kernel (the faster one at the sustained
    // clock); application plans to the classic one
    p->cfg = default_config(p, app == STENCIL_APP_JACOBI ? STENCIL_KERNEL_INPLANE_WS : STENCIL_KERNEL_INPLANE);
    *plan = p;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_plan_create(stencil_plan_t* plan, int64_t nx, int64_t ny, int64_t nz, int radius,
                                     const double* coeffs, stencil_dtype_t dtype) {
    return stencil_plan_create_app(plan, nx, ny, nz, radius, coeffs, dtype, STENCIL_APP_JACOBI, 0.0);
}

stencil_status_t stencil_plan_create_axes(stencil_plan_t* plan, int64_t nx, int64_t ny, int64_t nz, int radius,
                                          const double* coeffs, stencil_dtype_t dtype) {
    if (!plan || !coeffs) return fail(STENCIL_ERROR_INVALID_VALUE, "plan_create_axes: NULL argument");
    *plan = nullptr;
    if (radius < 1 || radius > STENCIL_MAX_RADIUS)
        return fail(STENCIL_ERROR_INVALID_VALUE, "plan_create_axes: radius must be in [1, 6]");
    for (int i = 0; i <= 3 * radius; ++i)
        if (!std::isfinite(coeffs[i])) return fail(STENCIL_ERROR_INVALID_VALUE, "plan_create_axes: non-finite coefficient");
    // c0, cx_1..cx_r go through the common path; cy, cz follow
    double cx[STENCIL_MAX_RADIUS + 1] = {};
    for (int m = 0; m <= radius; ++m) cx[m] = m == 0 ? coeffs[0] : coeffs[m];
    stencil_plan_t p = new (std::nothrow) stencil_plan_s();
    if (!p) return fail(STENCIL_ERROR_OUT_OF_MEMORY, "plan_create_axes: host allocation");
    stencil_status_t rc = plan_init(p, nx, ny, nz, radius, cx, dtype);
    if (rc != STENCIL_SUCCESS) {
        stencil_destroy(p);
        return rc;
    }
    for (int m = 1; m <= radius; ++m) {
        const double cy = coeffs[radius + m], cz = coeffs[2 * radius + m];
        p->coeffs_y[m] = dtype == STENCIL_F32 ? (double)(float)cy : cy;
        p->coeffs_z[m] = dtype == STENCIL_F32 ? (double)(float)cz : cz;
    }
    p->axes = true;
    p->cfg = default_config(p, STENCIL_KERNEL_INPLANE);
    *plan = p;
    return STENCIL_SUCCESS;
}

// internal: used by dist.cu
stencil_status_t stencil_plan_init_internal(stencil_plan_t p, int64_t nx, int64_t ny, int64_t nz, int radius,
                                            const double* coeffs, stencil_dtype_t dtype) {
    return plan_init(p, nx, ny, nz, radius, coeffs, dtype);
}

void stencil_destroy(stencil_plan_t p) {
    if (!p) return;
    cudaSetDevice(p->device);
    cudaDeviceSynchronize();
    dist_destroy(p);
    if (p->scratch) cudaFree(p->scratch);
    if (p->d_res) cudaFree(p->d_res);
    p2p_destroy(p);
    for (auto& e : p->graphs) cudaGraphExecDestroy(e.exec);
    for (auto& h : p->hslot) {
        if (h.din) cudaFree(h.din);
        if (h.dout) cudaFree(h.dout);
        for (cudaEvent_t e : {h.h2d_done, h.comp_done, h.d2h_done})
            if (e) cudaEventDestroy(e);
    }
    for (cudaStream_t q : {p->hs_h2d, p->hs_comp, p->hs_d2h})
        if (q) cudaStreamDestroy(q);
    if (p->hs_fork) cudaEventDestroy(p->hs_fork);
    if (p->s_capture) cudaStreamDestroy(p->s_capture);
    if (p->h_res) cudaFreeHost(p->h_res);
    for (cudaEvent_t e : p->tev) cudaEventDestroy(e);
    delete p;
}

stencil_status_t stencil_plan_layout(stencil_plan_t p, stencil_layout_t* out) {
    if (!p || !out) return fail(STENCIL_ERROR_INVALID_VALUE, "plan_layout: NULL argument");
    *out = p->lay;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_plan_set_config(stencil_plan_t p, const stencil_config_t* cfg) {
    if (!p || !cfg) return fail(STENCIL_ERROR_INVALID_VALUE, "set_config: NULL argument");
    Geometry g;
    stencil_status_t rc = config_geometry(p->lay, *cfg, &g, kernel_variant(p));
    if (rc != STENCIL_SUCCESS) return rc;
    if (p->dist && cfg->zsegs < 1) return fail(STENCIL_ERROR_INVALID_VALUE, "set_config: zsegs");
    p->cfg = *cfg;
    if (p->p2p) preload_kernels(p);
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_plan_get_config(stencil_plan_t p, stencil_config_t* cfg) {
    if (!p || !cfg) return fail(STENCIL_ERROR_INVALID_VALUE, "get_config: NULL argument");
    *cfg = p->cfg;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_plan_reserve(stencil_plan_t p) {
    if (!p) return fail(STENCIL_ERROR_INVALID_VALUE, "reserve: NULL plan");
    if (p->scratch) return STENCIL_SUCCESS;
    cudaError_t e = cudaMalloc(&p->scratch, (size_t)p->lay.bytes);
    if (e == cudaErrorMemoryAllocation) {
        cudaGetLastError();
        p->scratch = nullptr;
        return fail(STENCIL_ERROR_OUT_OF_MEMORY, "reserve: scratch grid");
    }
    if (e != cudaSuccess) return cuda_fail(e, "cudaMalloc(scratch)");
    return STENCIL_SUCCESS;
}

static bool overlap(const void* a, const void* b, int64_t n) {
    const char* x = (const char*)a;
    const char* y = (const char*)b;
    return x < y + n && y < x + n;
}

// record the next pooled timing event on st
static stencil_status_t timing_mark(stencil_plan_s* p, cudaStream_t st) {
    if (p->tev_used == p->tev.size()) {
        cudaEvent_t e;
        STENCIL_CUDA_TRY(cudaEventCreate(&e));
        p->tev.push_back(e);
    }
    STENCIL_CUDA_TRY(cudaEventRecord(p->tev[p->tev_used++], st));
    return STENCIL_SUCCESS;
}

// One sweep src (+ d * g) -> dst of the whole (local) grid on st, with the
// per-sweep halo exchange of distributed plans: boundary segments first (they
// feed the exchange), the interior segments overlap the NCCL transfer.
static stencil_status_t sweep_step(stencil_plan_s* p, const void* src, const void* g, void* dst, int dir,
                                   cudaStream_t st) {
    stencil_status_t rc;
    const int zsegs = p->cfg.zsegs;
    if (!(p->dist && p->nranks > 1)) {
        SweepSegments all{0, 1, zsegs};
        return launch_sweep(p, p->cfg, src, g, dst, all, dir, st);
    }
    if (p->local_group)
        return fail(STENCIL_ERROR_NOT_SUPPORTED, "in-process rank groups run through stencil_run_dist_local");
    // the exchanged planes [0, r) and [nz - r, nz) must come from the two boundary segments alone
    // (else the interior launch, concurrent with the exchange, would still be writing some of them)
    if (zsegs >= 2 && p->lay.nz / zsegs >= p->r) {
        SweepSegments b{0, zsegs - 1, 2};
        if ((rc = launch_sweep(p, p->cfg, src, g, dst, b, dir, st)) != STENCIL_SUCCESS) return rc;
        STENCIL_CUDA_TRY(cudaEventRecord(p->ev_bnd, st));
        STENCIL_CUDA_TRY(cudaStreamWaitEvent(p->s_comm, p->ev_bnd, 0));
        if ((rc = dist_exchange(p, dst, p->s_comm)) != STENCIL_SUCCESS) return rc;
        SweepSegments in_segs{1, 1, zsegs - 2};
        if ((rc = launch_sweep(p, p->cfg, src, g, dst, in_segs, dir, st)) != STENCIL_SUCCESS) return rc;
    } else {
        SweepSegments all{0, 1, zsegs};
        if ((rc = launch_sweep(p, p->cfg, src, g, dst, all, dir, st)) != STENCIL_SUCCESS) return rc;
        STENCIL_CUDA_TRY(cudaEventRecord(p->ev_bnd, st));
        STENCIL_CUDA_TRY(cudaStreamWaitEvent(p->s_comm, p->ev_bnd, 0));
        if ((rc = dist_exchange(p, dst, p->s_comm)) != STENCIL_SUCCESS) return rc;
    }
    STENCIL_CUDA_TRY(cudaEventRecord(p->ev_xchg, p->s_comm));
    STENCIL_CUDA_TRY(cudaStreamWaitEvent(st, p->ev_xchg, 0));
    return STENCIL_SUCCESS;
}

static stencil_status_t check_buffers(stencil_plan_s* p, const char* what, std::initializer_list<const void*> bufs) {
    uintptr_t bits = 0;
    for (const void* b : bufs) {
        if (!b) return fail(STENCIL_ERROR_INVALID_VALUE, std::string(what) + ": NULL argument");
        bits |= (uintptr_t)b;
    }
    if (bits & 127) return fail(STENCIL_ERROR_MISALIGNED, std::string(what) + ": buffers must be 128-byte aligned");
    return STENCIL_SUCCESS;
}

// The Fig. 1 loop for plans without (g = NULL) and with a fixed
// second grid: dst <- S^iters(in) (+ d g each sweep); `in` is preserved.
// The launches of one Jacobi run (after validation): shell copies, then the
// ping-pong sweeps; the last sweep lands in out.
static stencil_status_t issue_jacobi(stencil_plan_s* p, const void* in, const void* g, void* out, int iters,
                                     cudaStream_t st) {
    // the frozen shell of every written buffer equals in's shell
    stencil_status_t rc = launch_shell_copy(p, in, out, st);
    if (rc != STENCIL_SUCCESS) return rc;
    if (iters >= 2) {
        rc = launch_shell_copy(p, in, p->scratch, st);
        if (rc != STENCIL_SUCCESS) return rc;
    }
    const size_t span0 = p->tev_used;
    if (p->timing && (rc = timing_mark(p, st)) != STENCIL_SUCCESS) return rc;
    const void* src = in;
    for (int t = 1; t <= iters; ++t) {
        // sweep t writes out when (iters - t) is even, else the scratch grid: the last lands in out
        void* dst = ((iters - t) % 2 == 0) ? out : p->scratch;
        // odd sweeps stream upward, even sweeps downward: each sweep starts on
        // the planes the previous one wrote last (still in L2)
        const int dir = (t % 2 == 1) ? 1 : -1;
        if ((rc = sweep_step(p, src, g, dst, dir, st)) != STENCIL_SUCCESS) return rc;
        src = dst;
        if ((p->timing == 2 || (p->timing && t == iters)) && (rc = timing_mark(p, st)) != STENCIL_SUCCESS) return rc;
    }
    if (p->timing) p->spans.push_back({span0, p->tev_used - 1, iters});
    p->last_sweeps = iters;
    return STENCIL_SUCCESS;
}

// CUDA graphs for repeated runs (launch-bound small grids, e.g. BASELINE
// config 1: 64^3 sweeps of ~1 us each): the first run of a (buffers, iters,
// configuration) key is captured on a private stream and instantiated; later
// runs launch the graph on the caller's stream.  STENCIL_GRAPHS=0 disables.
static bool graphs_enabled() {
    static const bool on = [] {
        const char* e = getenv("STENCIL_GRAPHS");
        return !(e && e[0] == '0');
    }();
    return on;
}

static stencil_status_t run_jacobi_graph(stencil_plan_s* p, const void* in, const void* g, void* out, int iters,
                                         cudaStream_t st) {
    for (auto& e : p->graphs)
        if (e.in == in && e.g == g && e.out == out && e.iters == iters && memcmp(&e.cfg, &p->cfg, sizeof e.cfg) == 0) {
            STENCIL_CUDA_TRY(cudaGraphLaunch(e.exec, st));
            p->launches += e.launches;
            p->aux_launches += e.aux_launches;
            p->last_sweeps = iters;
            return STENCIL_SUCCESS;
        }
    if (!p->s_capture) STENCIL_CUDA_TRY(cudaStreamCreateWithFlags(&p->s_capture, cudaStreamNonBlocking));
    const int64_t l0 = p->launches, a0 = p->aux_launches;
    STENCIL_CUDA_TRY(cudaStreamBeginCapture(p->s_capture, cudaStreamCaptureModeThreadLocal));
    stencil_status_t rc = issue_jacobi(p, in, g, out, iters, p->s_capture);
    cudaGraph_t graph = nullptr;
    cudaError_t ce = cudaStreamEndCapture(p->s_capture, &graph);
    if (rc != STENCIL_SUCCESS) {
        if (graph) cudaGraphDestroy(graph);
        return rc;
    }
    if (ce != cudaSuccess) return cuda_fail(ce, "run: graph capture");
    stencil_plan_s::GraphEntry e{};
    e.in = in;
    e.g = g;
    e.out = out;
    e.iters = iters;
    e.cfg = p->cfg;
    e.launches = p->launches - l0;
    e.aux_launches = p->aux_launches - a0;
    p->launches = l0;  // counted when the graph is launched
    p->aux_launches = a0;
    ce = cudaGraphInstantiate(&e.exec, graph, 0);
    cudaGraphDestroy(graph);
    if (ce != cudaSuccess) return cuda_fail(ce, "run: graph instantiate");
    if (p->graphs.size() >= 8) {
        cudaGraphExecDestroy(p->graphs.front().exec);
        p->graphs.erase(p->graphs.begin());
    }
    p->graphs.push_back(e);
    STENCIL_CUDA_TRY(cudaGraphLaunch(e.exec, st));
    p->launches += e.launches;
    p->aux_launches += e.aux_launches;
    p->last_sweeps = iters;
    return STENCIL_SUCCESS;
}

static stencil_status_t run_jacobi(stencil_plan_s* p, const void* in, const void* g, void* out, int iters,
                                   cudaStream_t st) {
    if (overlap(in, out, p->lay.bytes)) return fail(STENCIL_ERROR_INVALID_VALUE, "run: in and out overlap");
    if (g && overlap(g, out, p->lay.bytes)) return fail(STENCIL_ERROR_INVALID_VALUE, "run: f and out overlap");
    STENCIL_CUDA_TRY(cudaSetDevice(p->device));
    if (iters == 0) {
        STENCIL_CUDA_TRY(cudaMemcpyAsync(out, in, (size_t)p->lay.bytes, cudaMemcpyDeviceToDevice, st));
        p->last_sweeps = 0;
        return STENCIL_SUCCESS;
    }
    if (iters >= 2) {
        stencil_status_t rc = stencil_plan_reserve(p);
        if (rc != STENCIL_SUCCESS) return rc;
        if (overlap(p->scratch, in, p->lay.bytes) || overlap(p->scratch, out, p->lay.bytes) ||
            (g && overlap(p->scratch, g, p->lay.bytes)))
            return fail(STENCIL_ERROR_INVALID_VALUE, "run: buffer overlaps the plan scratch");
    }
    if (graphs_enabled() && !p->timing && !p->dist && !p->p2p) return run_jacobi_graph(p, in, g, out, iters, st);
    return issue_jacobi(p, in, g, out, iters, st);
}

stencil_status_t stencil_run(stencil_plan_t p, const void* in, void* out, int iters, stencil_stream_t stream) {
    if (!p) return fail(STENCIL_ERROR_INVALID_VALUE, "run: NULL argument");
    stencil_status_t rc = check_buffers(p, "run", {in, out});
    if (rc != STENCIL_SUCCESS) return rc;
    if (iters < 0) return fail(STENCIL_ERROR_INVALID_VALUE, "run: iters < 0");
    if (p->app != STENCIL_APP_JACOBI)
        return fail(STENCIL_ERROR_INVALID_VALUE, "run: plan was created for an application stencil (run_source / run_wave)");
    return run_jacobi(p, in, nullptr, out, iters, (cudaStream_t)stream);
}

// max over interior points |a - b| in the plan's dtype (residual_kernel) into the plan's
// device word d_res (as the bit pattern of a non-negative T), stream-ordered, no host sync
stencil_status_t stencil_residual_launch_internal(stencil_plan_t p, const void* a, const void* b, cudaStream_t st) {
    if (!p->d_res) STENCIL_CUDA_TRY(cudaMalloc(&p->d_res, sizeof(unsigned long long)));
    const stencil_layout_t& L = p->lay;
    const long long nrows = L.ny * L.nz;
    const int threads = 256;
    const unsigned blocks = (unsigned)std::min<long long>((nrows * 32 + threads - 1) / threads, (long long)p->sm_count * 8);
    STENCIL_CUDA_TRY(cudaMemsetAsync(p->d_res, 0, sizeof(unsigned long long), st));
    if (p->dtype == STENCIL_F32)
        residual_kernel<float><<<blocks, threads, 0, st>>>((const float*)a, (const float*)b, (int)L.nx, (int)L.ny,
                                                           (int)L.nz, p->r, L.pitch_x, (int)L.rows_y,
                                                           (int)L.interior_x0, p->d_res);
    else
        residual_kernel<double><<<blocks, threads, 0, st>>>((const double*)a, (const double*)b, (int)L.nx, (int)L.ny,
                                                            (int)L.nz, p->r, L.pitch_x, (int)L.rows_y,
                                                            (int)L.interior_x0, p->d_res);
    STENCIL_CUDA_TRY(cudaGetLastError());
    p->aux_launches++;
    return STENCIL_SUCCESS;
}

// read d_res back (host-synchronous on st) and decode it
stencil_status_t stencil_residual_read_internal(stencil_plan_t p, cudaStream_t st, double* res) {
    if (!p->h_res) STENCIL_CUDA_TRY(cudaMallocHost(&p->h_res, sizeof(unsigned long long)));
    STENCIL_CUDA_TRY(cudaMemcpyAsync(p->h_res, p->d_res, sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    STENCIL_CUDA_TRY(cudaStreamSynchronize(st));
    const unsigned long long bits = *p->h_res;
    if (p->dtype == STENCIL_F32) {
        float f;
        const unsigned u = (unsigned)bits;
        memcpy(&f, &u, sizeof f);
        *res = f;
    } else {
        memcpy(res, &bits, sizeof *res);
    }
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_residual_internal(stencil_plan_t p, const void* a, const void* b, cudaStream_t st,
                                           double* res) {
    stencil_status_t rc = stencil_residual_launch_internal(p, a, b, st);
    if (rc != STENCIL_SUCCESS) return rc;
    return stencil_residual_read_internal(p, st, res);
}

stencil_status_t stencil_residual(stencil_plan_t p, const void* a, const void* b, stencil_stream_t stream,
                                  double* residual) {
    if (!p || !residual) return fail(STENCIL_ERROR_INVALID_VALUE, "residual: NULL argument");
    stencil_status_t rc = check_buffers(p, "residual", {a, b});
    if (rc != STENCIL_SUCCESS) return rc;
    STENCIL_CUDA_TRY(cudaSetDevice(p->device));
    return stencil_residual_internal(p, a, b, (cudaStream_t)stream, residual);
}

// Fig. 1 with its stop criterion (reading R5b): sweep until the update
// residual max|u_t - u_{t-1}| at a check (every check_every sweeps) is <= tol,
// or max_iters sweeps.  u_t alternates between out (t odd) and the plan scratch
// (t even); the result is moved into out at the end.  Host-synchronous at
// every check (one 8-byte read back).
// internal: timing marks for p2p.cu
stencil_status_t stencil_timing_mark_internal(stencil_plan_t p, cudaStream_t st) { return timing_mark(p, st); }

stencil_status_t stencil_run_until(stencil_plan_t p, const void* in, void* out, int max_iters, double tol,
                                   int check_every, stencil_stream_t stream, int* iters_done, double* residual) {
    if (!p || !iters_done || !residual) return fail(STENCIL_ERROR_INVALID_VALUE, "run_until: NULL argument");
    stencil_status_t rc = check_buffers(p, "run_until", {in, out});
    if (rc != STENCIL_SUCCESS) return rc;
    if (max_iters < 1 || check_every < 1 || !(tol >= 0.0))
        return fail(STENCIL_ERROR_INVALID_VALUE, "run_until: max_iters, check_every >= 1 and tol >= 0 required");
    if (p->app != STENCIL_APP_JACOBI) return fail(STENCIL_ERROR_INVALID_VALUE, "run_until: Jacobi plans only");

    if (overlap(in, out, p->lay.bytes)) return fail(STENCIL_ERROR_INVALID_VALUE, "run_until: in and out overlap");
    cudaStream_t st = (cudaStream_t)stream;
    STENCIL_CUDA_TRY(cudaSetDevice(p->device));
    if ((rc = stencil_plan_reserve(p)) != STENCIL_SUCCESS) return rc;
    if (overlap(p->scratch, in, p->lay.bytes) || overlap(p->scratch, out, p->lay.bytes))
        return fail(STENCIL_ERROR_INVALID_VALUE, "run_until: buffer overlaps the plan scratch");
    if ((rc = launch_shell_copy(p, in, out, st)) != STENCIL_SUCCESS) return rc;
    if ((rc = launch_shell_copy(p, in, p->scratch, st)) != STENCIL_SUCCESS) return rc;
    const stencil_layout_t& L = p->lay;
    const void* src = in;
    int t = 0;
    double res = -1.0;
    while (t < max_iters) {
        ++t;
        void* dst = (t % 2 == 1) ? out : p->scratch;
        if ((rc = sweep_step(p, src, nullptr, dst, (t % 2 == 1) ? 1 : -1, st)) != STENCIL_SUCCESS) return rc;
        if (t % check_every == 0 || t == max_iters) {
            // distributed plans: the global residual is the max over ranks (one NCCL all-reduce of the
            // residual bits, which order like the values), so every rank stops at the same sweep
            if ((rc = stencil_residual_launch_internal(p, dst, src, st)) != STENCIL_SUCCESS) return rc;
            if (p->dist && p->nranks > 1 && (rc = dist_allreduce_max_u64(p, p->d_res, st)) != STENCIL_SUCCESS) return rc;
            if ((rc = stencil_residual_read_internal(p, st, &res)) != STENCIL_SUCCESS) return rc;
            if (res <= tol) {
                src = dst;
                break;
            }
        }
        src = dst;
    }
    if (src != out) STENCIL_CUDA_TRY(cudaMemcpyAsync(out, src, (size_t)L.bytes, cudaMemcpyDeviceToDevice, st));
    p->last_sweeps = t;
    *iters_done = t;
    *residual = res;
    return STENCIL_SUCCESS;
}

// Host-to-host runs, pipelined across calls: slot k = call % 2 owns a device
// input and output grid; the H2D copy of call n+1, the sweeps of call n and
// the D2H copy of call n-1 run on three plan streams at once, ordered by
// events (slot reuse waits for the previous user of the same slot).
stencil_status_t stencil_run_host(stencil_plan_t p, const void* host_in, void* host_out, int iters,
                                  stencil_stream_t stream) {
    if (!p || !host_in || !host_out) return fail(STENCIL_ERROR_INVALID_VALUE, "run_host: NULL argument");
    if (iters < 0) return fail(STENCIL_ERROR_INVALID_VALUE, "run_host: iters < 0");
    if (p->app != STENCIL_APP_JACOBI || p->dist || p->p2p)
        return fail(STENCIL_ERROR_INVALID_VALUE, "run_host: single-GPU Jacobi plans only");
    STENCIL_CUDA_TRY(cudaSetDevice(p->device));
    const size_t n = (size_t)p->lay.bytes;
    // lazily created; every object is created only if still missing, so a failed
    // first call (e.g. out of memory) leaks nothing and a later call can retry
    for (int k = 0; k < 2; ++k) {
        auto& h = p->hslot[k];
        if (!h.din) STENCIL_CUDA_TRY(cudaMalloc(&h.din, n));
        if (!h.dout) {
            STENCIL_CUDA_TRY(cudaMalloc(&h.dout, n));
            STENCIL_CUDA_TRY(cudaMemset(h.dout, 0, n));
        }
        for (cudaEvent_t* e : {&h.h2d_done, &h.comp_done, &h.d2h_done})
            if (!*e) STENCIL_CUDA_TRY(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
    }
    for (cudaStream_t* q : {&p->hs_h2d, &p->hs_comp, &p->hs_d2h})
        if (!*q) STENCIL_CUDA_TRY(cudaStreamCreateWithFlags(q, cudaStreamNonBlocking));
    if (!p->hs_fork) STENCIL_CUDA_TRY(cudaEventCreateWithFlags(&p->hs_fork, cudaEventDisableTiming));
    auto& sl = p->hslot[p->host_calls % 2];
    const bool reused = p->host_calls >= 2;
    // the caller's prior work on `stream` (e.g. filling host_in) comes first
    STENCIL_CUDA_TRY(cudaEventRecord(p->hs_fork, (cudaStream_t)stream));
    STENCIL_CUDA_TRY(cudaStreamWaitEvent(p->hs_h2d, p->hs_fork, 0));
    if (reused) STENCIL_CUDA_TRY(cudaStreamWaitEvent(p->hs_h2d, sl.comp_done, 0));  // din no longer read
    STENCIL_CUDA_TRY(cudaMemcpyAsync(sl.din, host_in, n, cudaMemcpyHostToDevice, p->hs_h2d));
    STENCIL_CUDA_TRY(cudaEventRecord(sl.h2d_done, p->hs_h2d));
    STENCIL_CUDA_TRY(cudaStreamWaitEvent(p->hs_comp, sl.h2d_done, 0));
    if (reused) STENCIL_CUDA_TRY(cudaStreamWaitEvent(p->hs_comp, sl.d2h_done, 0));  // dout no longer read
    stencil_status_t rc = run_jacobi(p, sl.din, nullptr, sl.dout, iters, p->hs_comp);
    if (rc != STENCIL_SUCCESS) return rc;
    STENCIL_CUDA_TRY(cudaEventRecord(sl.comp_done, p->hs_comp));
    STENCIL_CUDA_TRY(cudaStreamWaitEvent(p->hs_d2h, sl.comp_done, 0));
    STENCIL_CUDA_TRY(cudaMemcpyAsync(host_out, sl.dout, n, cudaMemcpyDeviceToHost, p->hs_d2h));
    STENCIL_CUDA_TRY(cudaEventRecord(sl.d2h_done, p->hs_d2h));
    p->host_calls++;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_run_host_wait(stencil_plan_t p, stencil_stream_t stream) {
    if (!p) return fail(STENCIL_ERROR_INVALID_VALUE, "run_host_wait: NULL plan");
    if (p->host_calls == 0) return STENCIL_SUCCESS;
    STENCIL_CUDA_TRY(cudaSetDevice(p->device));
    // downloads run in call order on one stream: the last call's event covers them all
    STENCIL_CUDA_TRY(cudaStreamWaitEvent((cudaStream_t)stream, p->hslot[(p->host_calls - 1) % 2].d2h_done, 0));
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_run_source(stencil_plan_t p, const void* in, const void* f, void* out, int iters,
                                    stencil_stream_t stream) {
    if (!p) return fail(STENCIL_ERROR_INVALID_VALUE, "run_source: NULL argument");
    stencil_status_t rc = check_buffers(p, "run_source", {in, f, out});
    if (rc != STENCIL_SUCCESS) return rc;
    if (iters < 0) return fail(STENCIL_ERROR_INVALID_VALUE, "run_source: iters < 0");
    if (p->app != STENCIL_APP_SOURCE) return fail(STENCIL_ERROR_INVALID_VALUE, "run_source: plan is not a SOURCE plan");
    return run_jacobi(p, in, f, out, iters, (cudaStream_t)stream);
}

// Leapfrog (config 3 "3D wave"): u_{n+1} = S(u_n) + d u_{n-1}, states rotate
// through u_prev (B0), u (B1) and the plan scratch (B2): state n+1 lands in
// B_{(n+1) mod 3}.  At the end the last two states are moved into (B0, B1) if
// iters is not a multiple of 3 (two grid copies).
stencil_status_t stencil_run_wave(stencil_plan_t p, void* u_prev, void* u, int iters, stencil_stream_t stream) {
    if (!p) return fail(STENCIL_ERROR_INVALID_VALUE, "run_wave: NULL argument");
    stencil_status_t rc = check_buffers(p, "run_wave", {u_prev, u});
    if (rc != STENCIL_SUCCESS) return rc;
    if (iters < 0) return fail(STENCIL_ERROR_INVALID_VALUE, "run_wave: iters < 0");
    if (p->app != STENCIL_APP_WAVE) return fail(STENCIL_ERROR_INVALID_VALUE, "run_wave: plan is not a WAVE plan");
    if (overlap(u_prev, u, p->lay.bytes)) return fail(STENCIL_ERROR_INVALID_VALUE, "run_wave: u_prev and u overlap");
    cudaStream_t st = (cudaStream_t)stream;
    STENCIL_CUDA_TRY(cudaSetDevice(p->device));
    p->last_sweeps = 0;
    if (iters == 0) return STENCIL_SUCCESS;
    if ((rc = stencil_plan_reserve(p)) != STENCIL_SUCCESS) return rc;
    if (overlap(p->scratch, u_prev, p->lay.bytes) || overlap(p->scratch, u, p->lay.bytes))
        return fail(STENCIL_ERROR_INVALID_VALUE, "run_wave: buffer overlaps the plan scratch");
    void* B[3] = {u_prev, u, p->scratch};
    // every state carries u's (frozen Dirichlet) shell
    if ((rc = launch_shell_copy(p, u, u_prev, st)) != STENCIL_SUCCESS) return rc;
    if ((rc = launch_shell_copy(p, u, p->scratch, st)) != STENCIL_SUCCESS) return rc;
    const size_t span0 = p->tev_used;
    if (p->timing && (rc = timing_mark(p, st)) != STENCIL_SUCCESS) return rc;
    for (int t = 1; t <= iters; ++t) {
        const int dir = (t % 2 == 1) ? 1 : -1;
        if ((rc = sweep_step(p, B[t % 3], B[(t - 1) % 3], B[(t + 1) % 3], dir, st)) != STENCIL_SUCCESS) return rc;
        if ((p->timing == 2 || (p->timing && t == iters)) && (rc = timing_mark(p, st)) != STENCIL_SUCCESS) return rc;
    }
    if (p->timing) p->spans.push_back({span0, p->tev_used - 1, iters});
    const size_t n = (size_t)p->lay.bytes;
    if (iters % 3 == 1) {  // newest in B2, previous in B1
        STENCIL_CUDA_TRY(cudaMemcpyAsync(B[0], B[1], n, cudaMemcpyDeviceToDevice, st));
        STENCIL_CUDA_TRY(cudaMemcpyAsync(B[1], B[2], n, cudaMemcpyDeviceToDevice, st));
    } else if (iters % 3 == 2) {  // newest in B0, previous in B2
        STENCIL_CUDA_TRY(cudaMemcpyAsync(B[1], B[0], n, cudaMemcpyDeviceToDevice, st));
        STENCIL_CUDA_TRY(cudaMemcpyAsync(B[0], B[2], n, cudaMemcpyDeviceToDevice, st));
    }
    p->last_sweeps = iters;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_plan_create_divgrad(stencil_plan_t* plan, int64_t nx, int64_t ny, int64_t nz, int radius,
                                             const double* a, stencil_dtype_t dtype, stencil_app_t app) {
    if (!plan || !a) return fail(STENCIL_ERROR_INVALID_VALUE, "plan_create_divgrad: NULL argument");
    *plan = nullptr;
    if (app != STENCIL_APP_DIV && app != STENCIL_APP_GRAD)
        return fail(STENCIL_ERROR_INVALID_VALUE, "plan_create_divgrad: app must be STENCIL_APP_DIV or STENCIL_APP_GRAD");
    if (radius > 4 && radius <= STENCIL_MAX_RADIUS)
        return fail(STENCIL_ERROR_NOT_SUPPORTED, "plan_create_divgrad: radius must be in [1, 4]");
    double c[STENCIL_MAX_RADIUS + 1] = {};
    for (int m = 1; m <= radius && m <= STENCIL_MAX_RADIUS; ++m) {
        if (!std::isfinite(a[m - 1])) return fail(STENCIL_ERROR_INVALID_VALUE, "plan_create_divgrad: non-finite weight");
        c[m] = a[m - 1];
    }
    stencil_plan_t p = new (std::nothrow) stencil_plan_s();
    if (!p) return fail(STENCIL_ERROR_OUT_OF_MEMORY, "plan_create_divgrad: host allocation");
    stencil_status_t rc = plan_init(p, nx, ny, nz, radius, c, dtype);
    if (rc != STENCIL_SUCCESS) {
        stencil_destroy(p);
        return rc;
    }
    p->app = app;
    // default: the registered tile (divgrad kernels: tx 16 / 32, ry 2 / 4, zbox 2) whose CTA count is closest
    // to a whole number of waves on this GPU, spill-free, eight compute warps first
    const int vec = 16 / (int)p->lay.elem_size;
    stencil_config_t best{};
    double best_score = -1e300;
    bool found = false;
    for (int tx : {32, 16})
        for (int ry : {2, 4})
            for (int warps : {8, 4}) {
                const int ty = warps * 32 / tx;
                for (int z = 1; z <= 32; ++z) {
                    stencil_config_t cf{STENCIL_KERNEL_INPLANE_WS, tx, ty, vec, ry, 4, z, 2, 0};
                    if (z > 1 && p->lay.nz / z < 4 * radius) break;
                    Geometry g;
                    if (config_geometry(p->lay, cf, &g, kernel_variant(p)) != STENCIL_SUCCESS) continue;
                    const KernelEntry* ke = find_kernel(cf.kernel, dtype, radius, tx, 1, ry, kernel_variant(p), 2);
                    cudaFuncAttributes at;
                    if (!ke || cudaFuncGetAttributes(&at, ke->func) != cudaSuccess || at.localSizeBytes > 0) {
                        cudaGetLastError();
                        continue;
                    }
                    const double ctas = (double)g.tiles_x * g.tiles_y * z;
                    const double waves = std::ceil(ctas / p->sm_count);
                    const double score = ctas / (waves * p->sm_count) - 0.01 * z - (warps == 4 ? 0.02 : 0.0);
                    if (score > best_score) {
                        best_score = score;
                        best = cf;
                        found = true;
                    }
                }
            }
    set_error("");
    if (!found) {
        stencil_destroy(p);
        return fail(STENCIL_ERROR_NOT_SUPPORTED, "plan_create_divgrad: no usable kernel configuration");
    }
    p->cfg = best;
    *plan = p;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_run_div(stencil_plan_t p, const void* u, const void* v, const void* w, void* out,
                                 stencil_stream_t stream) {
    if (!p) return fail(STENCIL_ERROR_INVALID_VALUE, "run_div: NULL plan");
    if (p->app != STENCIL_APP_DIV) return fail(STENCIL_ERROR_INVALID_VALUE, "run_div: plan is not a Div plan");
    stencil_status_t rc = check_buffers(p, "run_div", {u, v, w, out});
    if (rc != STENCIL_SUCCESS) return rc;
    for (const void* q : {u, v, w})
        if (overlap(q, out, p->lay.bytes)) return fail(STENCIL_ERROR_INVALID_VALUE, "run_div: out overlaps an input");
    STENCIL_CUDA_TRY(cudaSetDevice(p->device));
    const void* in[3] = {u, v, w};
    void* o[3] = {out, nullptr, nullptr};
    return launch_divgrad(p, p->cfg, in, o, (cudaStream_t)stream);
}

stencil_status_t stencil_run_grad(stencil_plan_t p, const void* f, void* gx, void* gy, void* gz,
                                  stencil_stream_t stream) {
    if (!p) return fail(STENCIL_ERROR_INVALID_VALUE, "run_grad: NULL plan");
    if (p->app != STENCIL_APP_GRAD) return fail(STENCIL_ERROR_INVALID_VALUE, "run_grad: plan is not a Grad plan");
    stencil_status_t rc = check_buffers(p, "run_grad", {f, gx, gy, gz});
    if (rc != STENCIL_SUCCESS) return rc;
    void* o[3] = {gx, gy, gz};
    for (int i = 0; i < 3; ++i) {
        if (overlap(f, o[i], p->lay.bytes)) return fail(STENCIL_ERROR_INVALID_VALUE, "run_grad: an output overlaps f");
        for (int j = i + 1; j < 3; ++j)
            if (overlap(o[i], o[j], p->lay.bytes)) return fail(STENCIL_ERROR_INVALID_VALUE, "run_grad: outputs overlap");
    }
    STENCIL_CUDA_TRY(cudaSetDevice(p->device));
    const void* in[3] = {f, nullptr, nullptr};
    return launch_divgrad(p, p->cfg, in, o, (cudaStream_t)stream);
}

stencil_status_t stencil_plan_set_timing(stencil_plan_t p, int enable) {
    if (!p) return fail(STENCIL_ERROR_INVALID_VALUE, "set_timing: NULL plan");
    if (enable < 0 || enable > 2) return fail(STENCIL_ERROR_INVALID_VALUE, "set_timing: mode must be 0, 1 or 2");
    p->timing = enable;
    p->spans.clear();
    p->tev_used = 0;
    p->acc_sweeps = 0;
    p->acc_ms = 0.0;
    p->acc_min = p->acc_max = p->last_ms = -1.0;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_plan_stats(stencil_plan_t p, stencil_stats_t* out) {
    if (!p || !out) return fail(STENCIL_ERROR_INVALID_VALUE, "stats: NULL argument");
    stencil_stats_t s{};
    s.launches = p->launches;
    s.aux_launches = p->aux_launches;
    s.timing_enabled = p->timing;
    s.last_run_sweeps = p->last_sweeps;
    // fold the runs recorded since the last call into the totals, then reuse their events
    if (!p->spans.empty()) STENCIL_CUDA_TRY(cudaEventSynchronize(p->tev[p->spans.back().last]));
    for (const auto& sp : p->spans) {
        double run_ms = 0.0;
        for (size_t e = sp.first; e < sp.last; ++e) {
            float ms = 0.f;
            STENCIL_CUDA_TRY(cudaEventElapsedTime(&ms, p->tev[e], p->tev[e + 1]));
            run_ms += ms;
            if (p->timing == 2) {
                if (p->acc_min < 0 || ms < p->acc_min) p->acc_min = ms;
                if (ms > p->acc_max) p->acc_max = ms;
            }
        }
        p->acc_ms += run_ms;
        p->acc_sweeps += sp.sweeps;
        p->last_ms = run_ms;
    }
    p->spans.clear();
    p->tev_used = 0;
    s.last_run_sweep_ms = p->last_ms;
    s.timed_sweeps = p->acc_sweeps;
    s.timed_sweep_ms = p->acc_sweeps ? p->acc_ms : -1.0;
    s.sweep_ms_min = p->acc_min;
    s.sweep_ms_max = p->acc_max;
    *out = s;
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_fill_counter(stencil_plan_t p, void* buf, uint64_t seed, stencil_stream_t stream) {
    if (!p || !buf) return fail(STENCIL_ERROR_INVALID_VALUE, "fill_counter: NULL argument");
    if ((uintptr_t)buf & 127) return fail(STENCIL_ERROR_MISALIGNED, "fill_counter: buffer must be 128-byte aligned");
    const stencil_layout_t& L = p->lay;
    const int threads = 256;
    const unsigned blocks = (unsigned)p->sm_count * 8;
    const long long kz0 = p->z0_global;  // global outer plane of local outer plane 0 (0 for single plans)
    if (p->dtype == STENCIL_F32)
        fill_counter_kernel<float><<<blocks, threads, 0, (cudaStream_t)stream>>>(
            (float*)buf, (int)L.nx, (int)L.ny, p->r, L.pitch_x, (int)L.rows_y, (int)L.planes_z, (int)L.interior_x0, kz0,
            seed);
    else
        fill_counter_kernel<double><<<blocks, threads, 0, (cudaStream_t)stream>>>(
            (double*)buf, (int)L.nx, (int)L.ny, p->r, L.pitch_x, (int)L.rows_y, (int)L.planes_z, (int)L.interior_x0,
            kz0, seed);
    STENCIL_CUDA_TRY(cudaGetLastError());
    p->aux_launches++;
    return STENCIL_SUCCESS;
}

}  // extern "C"
