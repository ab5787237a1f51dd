// tune.cu -- performance models (Sec. VI) and the auto-tuner
// (Sec. IV-C exhaustive search P:L254-258; model-based beta pruning P:L372).
#include <algorithm>
#include <cstdio>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <numeric>
#include <vector>

#include "internal.h"

namespace stencil {

static double env_double(const char* name, double dflt) {
    const char* v = getenv(name);
    if (!v || !*v) return dflt;
    char* end = nullptr;
    double x = strtod(v, &end);
    return (end && end != v) ? x : dflt;
}

// GPU parameter set of P:L331-333 for the current device.  BW is the pin
// bandwidth x 0.8 (the B200 copy kernel reaches ~80% of pin, MEASURED_PEAKS)
// unless STENCIL_BW_GBS overrides it; Lat (cycles) from STENCIL_LAT_CYCLES.
void gpu_params(int device, stencil_gpu_params_t* g) {
    cudaDeviceProp prop;
    cudaGetDeviceProperties(&prop, device);
    int mem_khz = 0, bus_bits = 0, clk_khz = 0;
    cudaDeviceGetAttribute(&mem_khz, cudaDevAttrMemoryClockRate, device);
    cudaDeviceGetAttribute(&bus_bits, cudaDevAttrGlobalMemoryBusWidth, device);
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, device);
    const double pin = 2.0 * mem_khz * 1e3 * bus_bits / 8.0;
    g->sm = prop.multiProcessorCount;
    g->bw = env_double("STENCIL_BW_GBS", pin > 0 ? 0.8 * pin / 1e9 : 6552.0) * 1e9;
    g->smem = (int32_t)prop.sharedMemPerMultiprocessor;
    g->reg = prop.regsPerMultiprocessor;
    g->blk_sm = prop.maxBlocksPerMultiProcessor;
    g->warp_sm = prop.maxThreadsPerMultiProcessor / 32;
    g->lat_cycles = env_double("STENCIL_LAT_CYCLES", 600.0);
    g->clock_hz = clk_khz > 0 ? clk_khz * 1e3 : 1.965e9;
}

// ----------------------------------------------------------------------------
// model-P: Eqs. (6)-(14) with readings R12-R15 (mirrors oracle/model_p.py)
// ----------------------------------------------------------------------------
static int warp_blk(const stencil_model_kernel_t& k) { return (k.tx * k.ty + 31) / 32; }

static double f_hide(const stencil_gpu_params_t& g, const stencil_model_kernel_t& k, int n) {
    if (n <= 1) return 1.0;
    if (g.warp_sm <= 1) return (double)n;
    const double w = (double)n * warp_blk(k);
    double v = 1.0 + (n - 1) * (1.0 - (w - 1.0) / (g.warp_sm - 1.0));
    return std::min(std::max(v, 1.0), (double)n);
}

double model_paper(const stencil_gpu_params_t& g, const stencil_model_kernel_t& k, bool literal_tc, double* blks_o,
                   int* act_o, int* stages_o, int* rem_o) {
    const double W = (double)k.tx * k.rx, H = (double)k.ty * k.ry;
    const double blks = (double)k.lx * k.ly / (W * H);                           // Eq. (6)
    const long long KR = (long long)k.regs_per_thread * k.tx * k.ty;            // R12
    const long long KS = std::max(1, k.smem_per_block);
    const int wb = warp_blk(k);
    long long act = std::min<long long>(KR > 0 ? g.reg / KR : g.blk_sm, g.smem / KS);  // Eq. (7)
    act = std::min<long long>(act, g.warp_sm / wb);
    act = std::min<long long>(act, g.blk_sm);
    if (blks_o) *blks_o = blks;
    if (act_o) *act_o = (int)act;
    if (act < 1) {
        if (stages_o) *stages_o = 0;
        if (rem_o) *rem_o = 0;
        return 0.0;
    }
    const int stages = (int)std::ceil(blks / ((double)g.sm * act));               // Eq. (8)
    const int rem = (int)std::ceil((blks - (double)(stages - 1) * act * g.sm) / g.sm);  // Eq. (9)
    const double bytes_blk = (double)k.elem_size * ((W + 2 * k.radius) * (H + 2 * k.radius) + W * H);
    const double tm = g.lat_cycles / g.clock_hz + bytes_blk / (g.bw / g.sm);      // Eq. (10)
    double tc = (double)k.ops_per_point * k.rx * k.ry * wb / g.clock_hz;          // Eq. (11), R13
    if (literal_tc) tc *= (double)act;
    const double ts = f_hide(g, k, (int)act) * tm + act * tc;                     // Eq. (12)
    const double tl = f_hide(g, k, rem) * tm + rem * tc;                          // Eq. (13)
    if (stages_o) *stages_o = stages;
    if (rem_o) *rem_o = rem;
    return (double)k.lx * k.ly / (ts * (stages - 1) + tl);                        // Eq. (14)
}

// ----------------------------------------------------------------------------
// model-B: the B200 model.  Time of one sweep =
//   max(T_sm, T_dram) + T_launch
// T_sm: the busiest SM runs ceil(CTAs / SMs) CTAs, each streaming nz/zsegs + 2r
//   planes of a W x H tile (ragged / balanced tiles included); per plane every
//   thread issues its FP lane-ops (FP32 pipe 128 lanes/clk/SM, DFMA at half
//   rate; FFMA2 packs two lanes per issue slot), its 16-byte LDS (128 B/clk/SM)
//   and a fixed overhead; the bound is the largest of the three, divided by a
//   latency-hiding efficiency min(1, resident warps / 8).
// T_dram: compulsory read + write (+ the second grid of application plans) and
//   the warm-up re-reads of every extra z segment, at the copy bandwidth scaled
//   by min(1, bytes in flight / (BW x 1 us)); a CTA keeps at most ~4 TMA
//   tensor loads in flight on B200 (tools/membench3.cu).
// Fitted on exhaustive B200 measurements of 12 search spaces
// (profiles/tune_space, tools/model_fit.py): beta = 5 % picks 99.8 % of the
// exhaustive best on average, 98.7 % worst.
// ----------------------------------------------------------------------------
double model_b200(const stencil_gpu_params_t& g, const stencil_model_kernel_t& k) {
    const int r = k.radius;
    const double s = k.elem_size;
    const double vec = 16.0 / s;
    const double hx = std::ceil(r / vec) * vec;
    const double W = (double)k.tx * k.rx, H = (double)k.ty * k.ry;
    const double tiles = std::ceil((double)k.lx / W) * (k.ytiles > 0 ? k.ytiles : std::ceil((double)k.ly / H));
    const double zsegs = std::max(1, k.zsegs);
    const double P = (double)k.lx * k.ly * k.lz;
    const bool inplane = k.stages > 0;
    const int inputs = k.inputs >= 2 ? 2 : 1;
    const double ctas = tiles * (inplane ? zsegs : 1.0);
    const double act = k.active_blocks > 0 ? k.active_blocks : 1;
    const double threads = (double)k.tx * k.ty;
    const double warps = std::ceil(threads / 32.0);
    const double planes = (double)k.lz / (inplane ? zsegs : 1.0) + (inplane ? 2.0 * r : 0.0);  // per CTA
    // per thread per streamed plane
    double fp, lds_bytes, slots;
    const double pts = (double)k.rx * k.ry;
    if (inplane) {
        const double rxv = k.rx / vec;
        fp = (6.0 * r + 1 + (inputs - 1)) * pts * (s == 8 ? 2.0 : 1.0);          // in FP32-lane units
        lds_bytes = 16.0 * ((k.ry + 2.0 * r) * rxv + 2.0 * k.ry * (hx / vec) + (inputs - 1) * k.ry * rxv);
        slots = (s == 4 ? fp / 2.0 : fp / 2.0) + lds_bytes / 16.0 + 2.0;           // FFMA2: 2 lanes / slot
    } else {
        fp = (6.0 * r + 1 + (inputs - 1)) * (s == 8 ? 2.0 : 1.0);
        lds_bytes = (4.0 * r + 1) * s;
        slots = fp + (4.0 * r + 1) + 12.0;
    }
    const double cyc = std::max({threads * fp / 128.0, threads * lds_bytes / 128.0, threads * slots / 128.0});
    const double per_sm = std::ceil(ctas / g.sm);
    const double resident_warps = std::min(act, per_sm) * warps;
    const double eff = std::min(1.0, resident_warps / 8.0);
    const double t_sm = per_sm * planes * cyc / eff / g.clock_hz;
    const double dram = s * P * (1.0 + inputs) + (inplane ? s * (double)k.lx * k.ly * 2.0 * r * (zsegs - 1) : 0.0);
    const double box = inplane ? ((W + 2 * hx) * (H + 2 * r) + (inputs - 1) * W * H) * s : 0.0;
    const double inflight = inplane ? std::min(ctas, act * g.sm) * std::min(4, std::max(1, k.stages - 1)) * box *
                                          std::max(1, k.zbox)
                                    : std::min(ctas, act * g.sm) * threads * s * (1.0 + r);
    const double eta = std::min(1.0, inflight / (g.bw * 1.0e-6));
    const double t_dram = dram / (g.bw * eta);
    return P / (std::max(t_sm, t_dram) + 3e-6);
}

// ----------------------------------------------------------------------------
// search space
// ----------------------------------------------------------------------------
static void zseg_candidates(int64_t nz, int r, std::vector<int>* out) {
    static const int cands[] = {1, 2, 3, 4, 5, 6, 8, 10, 12, 16, 24, 32};
    for (int z : cands)
        if (z == 1 || nz / z >= 4 * r) out->push_back(z);
}

static std::vector<stencil_config_t> enumerate_space(const stencil_layout_t& lay, int kernel, int sm_count) {
    std::vector<stencil_config_t> v;
    const int vec = 16 / (int)lay.elem_size;
    std::vector<int> zs;
    zseg_candidates(lay.nz, lay.radius, &zs);
    if (tma_kernel(kernel)) {
        // ty runs over every integer so that tile counts can match the 148 SMs
        // (e.g. 512 = 36 x 14 + 8: 4 x 37 = 148 tiles); wave balance is filtered in describe().
        // Warp-specialized kernels: only the registered tiles (kern_inst.cuh register_ws) are valid
        for (int tx : {16, 32, 64})
            for (int ty = 1; ty <= 16; ++ty)
                for (int rxv : {1, 2})
                    for (int ry : {1, 2, 4, 8})
                        for (int si = 0; si < 3; ++si)
                            for (int zb : {1, 2, 4})
                            for (int z : zs) {
                                // forward-plane + TMA holds r planes more in the ring (fp_tma.cuh)
                                const int st = kernel == STENCIL_KERNEL_FP_TMA
                                                   ? (lay.radius + zb - 1) / zb + 2 + si
                                                   : (si == 0 ? 3 : (si == 1 ? 4 : 6));
                                stencil_config_t c{kernel, tx, ty, rxv * vec, ry, st, z, zb, 0};
                                if (tx * ty < 64) continue;
                                Geometry g;
                                if (config_geometry(lay, c, &g) != STENCIL_SUCCESS) continue;
                                v.push_back(c);
                                // balanced y partitions whose CTA count fills the SMs (1 or 2 CTAs per SM)
                                for (int per_sm : {1, 2}) {
                                    const int yt = (sm_count * per_sm) / (g.tiles_x * z);
                                    if (yt < 1 || yt == g.tiles_y) continue;
                                    stencil_config_t b = c;
                                    b.ytiles = yt;
                                    Geometry gb;
                                    if (config_geometry(lay, b, &gb) == STENCIL_SUCCESS) v.push_back(b);
                                }
                            }
    } else if (kernel == STENCIL_KERNEL_FORWARD) {
        // ry: register rows per thread (1 = the SDK shape; 2, 4 = Fig. 10 case (i))
        for (int tx : {16, 32, 64})
            for (int ty : {2, 4, 8, 16, 32})
                for (int ry : {1, 2, 4}) {
                    stencil_config_t c{STENCIL_KERNEL_FORWARD, tx, ty, 1, ry, 1, 1, 1, 0};
                    Geometry g;
                    if (config_geometry(lay, c, &g) != STENCIL_SUCCESS) continue;
                    v.push_back(c);
                }
    } else {
        // the in-plane loading variants with per-thread loads (Fig. 6): thread block and register rows
        for (int tx : {16, 32, 64, 128})
            for (int ty : {2, 4, 8, 16})
                for (int ry : {1, 2, 4})
                    for (int z : zs) {
                        stencil_config_t c{kernel, tx, ty, 1, ry, 1, z, 1, 0};
                        Geometry g;
                        if (config_geometry(lay, c, &g) != STENCIL_SUCCESS) continue;
                        v.push_back(c);
                    }
    }
    set_error("");
    return v;
}

struct Candidate {
    stencil_config_t cfg;
    stencil_tune_entry_t entry;
    double score;
};

static bool describe(stencil_plan_s* plan, const stencil_config_t& c, const stencil_gpu_params_t& gp,
                     stencil_tune_entry_t* e) {
    Geometry g;
    const int source = kernel_variant(plan);
    if (config_geometry(plan->lay, c, &g, source) != STENCIL_SUCCESS) return false;
    const bool tma = tma_kernel(c.kernel);
    const int rxv = tma ? c.rx / g.vec : 0;
    const KernelEntry* ke = find_kernel(c.kernel, plan->dtype, plan->r, tma ? c.tx : 0, rxv, c.ry, source,
                                        c.kernel == STENCIL_KERNEL_INPLANE_WS ? c.zbox : 0);
    if (!ke) return false;
    cudaFuncAttributes attr;
    if (cudaFuncGetAttributes(&attr, ke->func) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    if (attr.localSizeBytes > 0) return false;  // register spills: excluded (constraint on registers)
    if (g.smem > 48 * 1024 &&
        cudaFuncSetAttribute(ke->func, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)g.smem) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    int act = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&act, ke->func, g.threads, g.smem) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    if (act < 1) return false;
    if (tma) {
        // wave balance: CTAs / (SMs x max CTAs on one SM) -- skip badly quantised grids
        const double ctas = (double)g.tiles_x * g.tiles_y * c.zsegs;
        const double per_sm = std::ceil(ctas / plan->sm_count);
        if (ctas / (plan->sm_count * per_sm) < 0.8 && ctas > plan->sm_count) return false;
    }
    stencil_model_kernel_t mk{};
    mk.lx = plan->lay.nx;
    mk.ly = plan->lay.ny;
    mk.lz = plan->lay.nz;
    mk.tx = c.tx;
    mk.ty = c.ty;
    mk.rx = c.rx;
    mk.ry = c.ry;
    mk.radius = plan->r;
    mk.elem_size = (int)plan->lay.elem_size;
    mk.regs_per_thread = attr.numRegs;
    mk.smem_per_block = (int)g.smem;
    mk.ops_per_point = 8 * plan->r + 1;  // Table II (in-plane)
    mk.stages = tma ? c.stages : 0;
    mk.zbox = c.zbox;
    mk.ytiles = g.tiles_y;
    mk.zsegs = c.zsegs;
    mk.active_blocks = act;
    mk.inputs = source == 1 ? 2 : 1;
    e->cfg = c;
    e->pred_paper_gpts = model_paper(gp, mk, false, nullptr, nullptr, nullptr, nullptr) / 1e9;  // Eq. (14): points/s
    e->pred_b200_gpts = model_b200(gp, mk) / 1e9;
    e->measured_gpts = -1.0;
    e->regs_per_thread = attr.numRegs;
    e->smem_bytes = (int)g.smem;
    e->active_blocks = act;
    return true;
}

// ----------------------------------------------------------------------------
// tuning cache (STENCIL_TUNE_CACHE): one line per tuning run,
//   stencil-tune-v1 dtype r nx ny nz variant sm kernel tx ty rx ry stages zsegs zbox ytiles gpts
// ----------------------------------------------------------------------------
static void cache_append(const stencil_plan_s* plan, const stencil_config_t& c, double gpts) {
    const char* path = getenv("STENCIL_TUNE_CACHE");
    if (!path || !*path) return;
    FILE* f = fopen(path, "a");
    if (!f) return;
    const stencil_layout_t& L = plan->lay;
    fprintf(f, "stencil-tune-v1 %d %d %lld %lld %lld %d %d %d %d %d %d %d %d %d %d %d %.3f\n", (int)plan->dtype,
            plan->r, (long long)L.nx, (long long)L.ny, (long long)L.nz, kernel_variant(plan), plan->sm_count,
            c.kernel, c.tx, c.ty, c.rx, c.ry, c.stages, c.zsegs, c.zbox, c.ytiles, gpts);
    fclose(f);
}

// best cached configuration for this plan's (dtype, r, extents, kind, SM count), if any
static bool cache_lookup(const stencil_plan_s* plan, stencil_config_t* out) {
    const char* path = getenv("STENCIL_TUNE_CACHE");
    if (!path || !*path) return false;
    FILE* f = fopen(path, "r");
    if (!f) return false;
    const stencil_layout_t& L = plan->lay;
    char tag[32];
    int dt, r, var, sm;
    long long nx, ny, nz;
    stencil_config_t c{};
    double gpts, best = -1.0;
    char line[512];
    while (fgets(line, sizeof line, f)) {  // line by line: a malformed line is skipped, not the rest
        if (sscanf(line, "%31s %d %d %lld %lld %lld %d %d %d %d %d %d %d %d %d %d %d %lf", tag, &dt, &r, &nx, &ny, &nz,
                   &var, &sm, &c.kernel, &c.tx, &c.ty, &c.rx, &c.ry, &c.stages, &c.zsegs, &c.zbox, &c.ytiles,
                   &gpts) != 18)
            continue;
        if (strcmp(tag, "stencil-tune-v1") != 0 || dt != (int)plan->dtype || r != plan->r || nx != L.nx ||
            ny != L.ny || nz != L.nz || var != kernel_variant(plan) || sm != plan->sm_count || gpts <= best)
            continue;
        Geometry g;
        if (config_geometry(L, c, &g, kernel_variant(plan)) != STENCIL_SUCCESS) continue;
        best = gpts;
        *out = c;
    }
    fclose(f);
    set_error("");
    return best > 0;
}

stencil_config_t default_config(stencil_plan_s* plan, int kernel) {
    {
        stencil_config_t c;
        if (cache_lookup(plan, &c)) return c;
    }
    stencil_gpu_params_t gp;
    gpu_params(plan->device, &gp);
    stencil_config_t best{};
    double best_score = -1.0;
    for (const auto& c : enumerate_space(plan->lay, kernel, plan->sm_count)) {
        stencil_tune_entry_t e;
        if (!describe(plan, c, gp, &e)) continue;
        if (e.pred_b200_gpts > best_score) {
            best_score = e.pred_b200_gpts;
            best = c;
        }
    }
    if (best_score < 0 && kernel == STENCIL_KERNEL_INPLANE_WS) return default_config(plan, STENCIL_KERNEL_INPLANE);
    if (best_score < 0) {  // fall back to the smallest valid configuration
        const int vec = 16 / (int)plan->lay.elem_size;
        best = kernel == STENCIL_KERNEL_INPLANE ? stencil_config_t{STENCIL_KERNEL_INPLANE, 32, 4, vec, 1, 2, 1, 1, 0}
                                                : stencil_config_t{STENCIL_KERNEL_FORWARD, 32, 8, 1, 1, 1, 1, 1, 0};
    }
    set_error("");
    return best;
}

static stencil_status_t time_config(stencil_plan_s* plan, const stencil_config_t& c, void* a, void* b, const void* g,
                                    cudaStream_t st, int iters, int reps, double* ms_per_iter) {
    cudaEvent_t e0, e1;
    STENCIL_CUDA_TRY(cudaEventCreate(&e0));
    STENCIL_CUDA_TRY(cudaEventCreate(&e1));
    std::vector<float> t;
    stencil_status_t rc = STENCIL_SUCCESS;
    SweepSegments all{0, 1, c.zsegs};
    for (int rep = 0; rep <= reps && rc == STENCIL_SUCCESS; ++rep) {  // rep 0 = warm-up
        cudaEventRecord(e0, st);
        for (int i = 0; i < iters && rc == STENCIL_SUCCESS; ++i)
            rc = launch_sweep(plan, c, (i % 2) ? b : a, g, (i % 2) ? a : b, all, (i % 2) ? -1 : 1, st);
        cudaEventRecord(e1, st);
        if (cudaEventSynchronize(e1) != cudaSuccess) rc = cuda_fail(cudaGetLastError(), "tune timing");
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep > 0) t.push_back(ms / iters);
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    if (rc != STENCIL_SUCCESS) return rc;
    std::sort(t.begin(), t.end());
    *ms_per_iter = t[t.size() / 2];
    return STENCIL_SUCCESS;
}

}  // namespace stencil

using namespace stencil;

extern "C" {

double stencil_model_paper(const stencil_gpu_params_t* g, const stencil_model_kernel_t* k, int literal_tc, double* blks,
                           int* act_blks, int* stages, int* rem_blks) {
    if (!g || !k) return -1.0;
    return model_paper(*g, *k, literal_tc != 0, blks, act_blks, stages, rem_blks);
}

double stencil_model_b200(const stencil_gpu_params_t* g, const stencil_model_kernel_t* k) {
    if (!g || !k) return -1.0;
    return model_b200(*g, *k);
}

stencil_status_t stencil_tune(stencil_plan_t plan, stencil_kernel_t kernel, stencil_model_t model, double beta_percent,
                              int iters_per_rep, int reps, void* scratch_in, void* scratch_out, stencil_stream_t stream,
                              stencil_tune_report_t* report) {
    if (!plan || !scratch_in || !scratch_out) return fail(STENCIL_ERROR_INVALID_VALUE, "tune: NULL argument");
    if (((uintptr_t)scratch_in | (uintptr_t)scratch_out) & 127)
        return fail(STENCIL_ERROR_MISALIGNED, "tune: buffers must be 128-byte aligned");
    if (kernel < STENCIL_KERNEL_INPLANE || kernel > STENCIL_KERNEL_FP_TMA)
        return fail(STENCIL_ERROR_INVALID_VALUE, "tune: unknown kernel");
    if (iters_per_rep < 1 || reps < 1) return fail(STENCIL_ERROR_INVALID_VALUE, "tune: iters_per_rep, reps >= 1");
    STENCIL_CUDA_TRY(cudaSetDevice(plan->device));
    cudaStream_t st = (cudaStream_t)stream;
    stencil_gpu_params_t gp;
    gpu_params(plan->device, &gp);
    // both scratch grids carry the input's shell already (caller's contents); sweeps only write interiors
    std::vector<stencil_tune_entry_t> cands;
    for (const auto& c : enumerate_space(plan->lay, kernel, plan->sm_count)) {
        stencil_tune_entry_t e;
        if (describe(plan, c, gp, &e)) cands.push_back(e);
    }
    if (cands.empty()) return fail(STENCIL_ERROR_NOT_SUPPORTED, "tune: empty search space");
    // rank by the chosen model ("ranked in decreasing order")
    std::stable_sort(cands.begin(), cands.end(), [&](const stencil_tune_entry_t& a, const stencil_tune_entry_t& b) {
        const double pa = model == STENCIL_MODEL_PAPER ? a.pred_paper_gpts : a.pred_b200_gpts;
        const double pb = model == STENCIL_MODEL_PAPER ? b.pred_paper_gpts : b.pred_b200_gpts;
        return pa > pb;
    });
    const int M = (int)cands.size();
    int N = M;
    if (beta_percent > 0 && beta_percent < 100) N = std::max(1, (int)std::ceil(beta_percent * M / 100.0));
    int best = -1;
    double best_ms = 1e300;
    // application plans read a second grid every sweep: time with a zero-filled one of the plan's layout
    void* g = nullptr;
    if (plan->app != STENCIL_APP_JACOBI) {
        STENCIL_CUDA_TRY(cudaMalloc(&g, (size_t)plan->lay.bytes));
        STENCIL_CUDA_TRY(cudaMemsetAsync(g, 0, (size_t)plan->lay.bytes, st));
    }
    for (int i = 0; i < N; ++i) {
        double ms = 0.0;
        stencil_status_t rc = time_config(plan, cands[i].cfg, scratch_in, scratch_out, g, st, iters_per_rep, reps, &ms);
        if (rc != STENCIL_SUCCESS) {
            if (g) cudaFree(g);
            return rc;
        }
        const double pts = (double)plan->lay.nx * plan->lay.ny * plan->lay.nz;
        cands[i].measured_gpts = pts / (ms * 1e-3) / 1e9;
        if (ms < best_ms) {
            best_ms = ms;
            best = i;
        }
    }
    // refinement at the sustained clock: the per-candidate timings are short (iters_per_rep sweeps,
    // boost clocks), so near-equal candidates swap places run to run and the winner of a burst is
    // not the winner of a long run under the power cap.  The twelve fastest, plus the four fastest of
    // the largest register tiles (RX*RY) if not among them -- bursts favour small tiles that draw more
    // energy per point, which the power cap then takes back -- are re-timed with runs
    // of ~STENCIL_TUNE_SUSTAIN_MS (default 300) ms each, after ~0.5 s of sweeps that bring the GPU
    // to its steady clock, in two interleaved rounds (forward, backward); the mean decides and is
    // what the report calls the measured rate.
    double burst_gpts = -1.0;
    {
        std::vector<int> order;
        for (int i = 0; i < N; ++i)
            if (cands[i].measured_gpts > 0) order.push_back(i);
        std::sort(order.begin(), order.end(),
                  [&](int x, int y) { return cands[x].measured_gpts > cands[y].measured_gpts; });
        int max_tile = 0;
        for (int i : order) max_tile = std::max(max_tile, cands[i].cfg.rx * cands[i].cfg.ry);
        std::vector<int> big;
        for (int i : order)
            if (cands[i].cfg.rx * cands[i].cfg.ry == max_tile) big.push_back(i);
        if (order.size() > 12) order.resize(12);
        for (size_t k = 0, added = 0; k < big.size() && added < 4; ++k)
            if (std::find(order.begin(), order.end(), big[k]) == order.end()) {
                order.push_back(big[k]);
                ++added;
            }
        burst_gpts = cands[best].measured_gpts;
        const double sustain_ms = env_double("STENCIL_TUNE_SUSTAIN_MS", 300.0);
        if (order.size() > 1 && sustain_ms > 0) {
            const double pts = (double)plan->lay.nx * plan->lay.ny * plan->lay.nz;
            auto sweeps_for = [&](int i, double ms) {
                const double ms_sweep = pts / (cands[i].measured_gpts * 1e9) * 1e3;
                return std::max(2 * iters_per_rep, (int)std::ceil(ms / ms_sweep / 2.0) * 2);
            };
            double tmp = 0.0;
            stencil_status_t rc = time_config(plan, cands[order[0]].cfg, scratch_in, scratch_out, g, st,
                                              sweeps_for(order[0], 500.0), 1, &tmp);  // reach the steady clock
            std::vector<double> sum(order.size(), 0.0);
            for (int round = 0; round < 2 && rc == STENCIL_SUCCESS; ++round)
                for (size_t k = 0; k < order.size() && rc == STENCIL_SUCCESS; ++k) {
                    const size_t j = round == 0 ? k : order.size() - 1 - k;
                    double ms = 0.0;
                    rc = time_config(plan, cands[order[j]].cfg, scratch_in, scratch_out, g, st,
                                     sweeps_for(order[j], sustain_ms), 1, &ms);
                    sum[j] += ms;
                }
            if (rc != STENCIL_SUCCESS) {
                if (g) cudaFree(g);
                return rc;
            }
            double best_long = 1e300;
            for (size_t j = 0; j < order.size(); ++j) {
                const double ms = sum[j] / 2.0;
                if (ms < best_long) {
                    best_long = ms;
                    best = order[j];
                }
            }
            best_ms = best_long;
            burst_gpts = cands[best].measured_gpts;
        }
    }
    if (g) cudaFree(g);
    plan->cfg = cands[best].cfg;
    cache_append(plan, cands[best].cfg, (double)plan->lay.nx * plan->lay.ny * plan->lay.nz / (best_ms * 1e-3) / 1e9);
    plan->tune_results = cands;
    if (report) {
        stencil_tune_report_t r{};
        r.model = model;
        r.beta_percent = beta_percent;
        r.space_size = M;
        r.timed = N;
        r.best = cands[best].cfg;
        r.best_ms_per_iter = best_ms;
        r.best_predicted_gpts = model == STENCIL_MODEL_PAPER ? cands[best].pred_paper_gpts : cands[best].pred_b200_gpts;
        r.best_measured_gpts = (double)plan->lay.nx * plan->lay.ny * plan->lay.nz / (best_ms * 1e-3) / 1e9;
        r.best_rank_by_model = best;
        r.best_burst_gpts = burst_gpts;
        *report = r;
    }
    return STENCIL_SUCCESS;
}

stencil_status_t stencil_tune_results(stencil_plan_t plan, stencil_tune_entry_t* out, int cap, int* count) {
    if (!plan || !count) return fail(STENCIL_ERROR_INVALID_VALUE, "tune_results: NULL argument");
    *count = (int)plan->tune_results.size();
    if (out)
        for (int i = 0; i < cap && i < *count; ++i) out[i] = plan->tune_results[i];
    return STENCIL_SUCCESS;
}

}  // extern "C"
