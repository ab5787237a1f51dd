// common.cuh -- device helpers shared by the sweep kernels (sm_100a).
//
// PTX wrappers for mbarriers and TMA tensor loads, 16-byte vector moves and
// the fixed per-point arithmetic order used by EVERY sweep kernel (DESIGN.md
// reading R7: one order for all kernels / tiles / segments / GPU counts, so
// they are bit-identical to each other).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace stencil {

// ---------------------------------------------------------------------------
// Kernel parameters
// ---------------------------------------------------------------------------
template <typename T>
struct SweepParams {
    int nx, ny, nz;          // interior extents of the (local) grid
    int rows;                // ny + 2r
    long long pitch;         // elements per row
    long long plane;         // elements per plane = rows * pitch
    int A;                   // element offset of interior x = 0 within a row
    int tiles_x, tiles_y;    // xy tiles
    int zsegs;               // z segments of [0, nz) (segment s = [s*nz/zsegs, (s+1)*nz/zsegs))
    int seg_base, seg_stride;  // this launch sweeps segments seg_base + blockIdx.z * seg_stride
    int stages;              // TMA ring depth (in-plane)
    int smem_pitch;          // elements per smem tile row (in-plane)
    int stage_elems;         // elements per ring stage (in-plane; 128 B multiple)
    int zbox;                // planes per TMA load (in-plane)
    int store_policy;        // L2 policy of output stores: 0 evict_normal, 1 evict_first, 2 evict_last
    int load_policy;         // L2 policy of TMA plane loads (same coding)
    int dir;                 // sweep direction along z: +1 upward, -1 downward
    int debug;               // experiments only (STENCIL_DEBUG): bit0 skip TMA waits/refills, bit1 skip stores
    unsigned stage_tx_bytes; // bytes one ring stage receives (in-plane box + g box)
    int gstage_off;          // element offset of the g box inside a stage (G kernels)
    T c[7];                  // c0..cr of Eq. (1), rounded to T (r <= STENCIL_MAX_RADIUS = 6); per-axis
                             // kernels (AX): c0 and cx_1..cx_r
    T cy[7], cz[7];          // per-axis kernels only: cy_m, cz_m (index m = 1..r)
    T* peer_lo;              // PS kernels: lower / upper neighbour's output grid (mapped peer memory) or null
    T* peer_hi;
    long long lo_delta;      // element offset of our plane z in the lower neighbour's grid: + nz_lo * plane
    long long hi_delta;      // ... in the upper neighbour's grid: - nz * plane
    T d;                     // coefficient of the second, centre-only grid g (G kernels)
    int ws_warps;            // warp-specialized in-plane: compute warps (tx*ty/32)
};

// Element index of interior point (x, y, z) (each in [-r, n + r)) in the pitched layout.
template <typename T, int R>
__device__ __forceinline__ long long gidx(const SweepParams<T>& p, int x, int y, int z) {
    return (long long)(z + R) * p.plane + (long long)(y + R) * p.pitch + p.A + x;
}

// ---------------------------------------------------------------------------
// Fixed arithmetic order (reading R7), used by every kernel, tile, segment and
// GPU count so all of them are bit-identical.  With z[-m], z[+m] the values of
// planes k-m, k+m IN SWEEP ORDER (for a downward sweep, dir = -1, z[-m] is
// plane k+m) and x[.], y[.] the in-plane neighbours:
//   acc = c_r * z[-r]
//   acc = fma(c_m, z[-m], acc)                          m = r-1 .. 1
//   acc = fma(c_0, centre, acc)
//   acc = fma(c_m, (x[i-m] + x[i+m]), acc); acc = fma(c_m, (y[j-m] + y[j+m]), acc)   m = 1 .. r
//   acc = fma(c_m, z[+m], acc)                          m = 1 .. r
//   acc = fma(d, g, acc)       (application stencils with a second grid only)
// i.e. the order in which the planes stream past an in-plane sweep.  6r+1
// FP instructions per point (r FMA for the behind terms, 1 + 4r for the plane
// itself, r for the forward terms).  Explicit round-to-nearest intrinsics:
// no contraction ambiguity, no fast-math.
// Per-axis kernels (AX, reading R3b) use the same order with cx_m, cy_m and
// cz_m in place of c_m on the x, y and z terms.
// ---------------------------------------------------------------------------
__device__ __forceinline__ float f_add(float a, float b) { return __fadd_rn(a, b); }
__device__ __forceinline__ double f_add(double a, double b) { return __dadd_rn(a, b); }
__device__ __forceinline__ float f_mul(float a, float b) { return __fmul_rn(a, b); }
__device__ __forceinline__ double f_mul(double a, double b) { return __dmul_rn(a, b); }
__device__ __forceinline__ float f_fma(float a, float b, float c) { return __fmaf_rn(a, b, c); }
__device__ __forceinline__ double f_fma(double a, double b, double c) { return __fma_rn(a, b, c); }

// ---------------------------------------------------------------------------
// 16-byte vectors
// ---------------------------------------------------------------------------
template <typename T> struct Vec;
template <> struct Vec<float> { static constexpr int N = 4; };
template <> struct Vec<double> { static constexpr int N = 2; };

template <typename T>
__device__ __forceinline__ void lds16(T* dst, const T* src) {
    if constexpr (sizeof(T) == 4) {
        float4 v = *reinterpret_cast<const float4*>(src);
        dst[0] = v.x; dst[1] = v.y; dst[2] = v.z; dst[3] = v.w;
    } else {
        double2 v = *reinterpret_cast<const double2*>(src);
        dst[0] = v.x; dst[1] = v.y;
    }
}

// Streaming 128-bit global store (the output plane is not re-read by this launch).
template <typename T>
__device__ __forceinline__ void stg16(T* dst, const T* src) {
    if constexpr (sizeof(T) == 4) {
        float4 v = make_float4(src[0], src[1], src[2], src[3]);
        *reinterpret_cast<float4*>(dst) = v;
    } else {
        double2 v = make_double2(src[0], src[1]);
        *reinterpret_cast<double2*>(dst) = v;
    }
}

// ---------------------------------------------------------------------------
// mbarrier + TMA (PTX ISA: mbarrier.*, cp.async.bulk.tensor)
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    while (!mbar_try_wait(bar, parity)) {
    }
}

// try_wait with a suspend-time hint: the thread sleeps until the phase completes (or the hint,
// in ns, elapses) instead of re-issuing the test -- for warps that only wait (the producer)
__device__ __forceinline__ bool mbar_try_wait_sleep(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity), "r"(1000000u)
        : "memory");
    return ok != 0;
}

__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity) {
    while (!mbar_try_wait_sleep(bar, parity)) {
    }
}

// 3-D tiled TMA load of one box into shared memory, completing on `bar`.
__device__ __forceinline__ void tma_load_3d(void* smem_dst, const CUtensorMap* map, int c0, int c1, int c2,
                                            uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(smem_u32(smem_dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(bar))
        : "memory");
}

// TMA load with an L2 eviction-priority hint (createpolicy descriptor).
__device__ __forceinline__ void tma_load_3d_hint(void* smem_dst, const CUtensorMap* map, int c0, int c1, int c2,
                                                 uint64_t* bar, uint64_t policy) {
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
        " [%0], [%1, {%2, %3, %4}], [%5], %6;" ::"r"(smem_u32(smem_dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(bar)), "l"(policy)
        : "memory");
}

// L2 eviction-priority descriptor: 0 evict_normal, 1 evict_first, 2 evict_last.
__device__ __forceinline__ uint64_t l2_policy(int kind) {
    uint64_t pol;
    if (kind == 1)
        asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    else if (kind == 2)
        asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    else
        asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

__device__ __forceinline__ void prefetch_tensormap(const CUtensorMap* map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

// 3-D tiled TMA store of one box from shared memory (bulk async-group of the
// issuing thread).  Elements outside the tensor map's extents are not written.
__device__ __forceinline__ void tma_store_3d(const CUtensorMap* map, const void* smem_src, int c0, int c1, int c2) {
    asm volatile(
        "cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
            reinterpret_cast<uint64_t>(map)),
        "r"(smem_u32(smem_src)), "r"(c0), "r"(c1), "r"(c2)
        : "memory");
}

__device__ __forceinline__ void bulk_commit_group() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }

// wait until at most N of this thread's bulk groups still READ shared memory
template <int N>
__device__ __forceinline__ void bulk_wait_group_read() {
    asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}

// wait until at most N of this thread's bulk groups are incomplete (writes done)
template <int N>
__device__ __forceinline__ void bulk_wait_group() {
    asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory");
}

// make this thread's generic-proxy shared-memory writes visible to the async proxy (TMA)
__device__ __forceinline__ void fence_proxy_async_smem() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

}  // namespace stencil
