// kern_inst.cuh -- template instantiations of the sweep kernels for one
// (dtype, radius), registered into the plan's kernel table.  Included by the
// kern_<dtype>_r<R>.cu files so the instantiations compile in parallel.
#pragma once

#include "ablation.cuh"
#include "forward.cuh"
#include "inplane.cuh"
#include "inplane_ws.cuh"
#include "divgrad.cuh"
#include "fp_tma.cuh"
#include "internal.h"

namespace stencil {

template <typename T, int R, int BX, int RXV, int RY, bool G, bool AX, bool PS>
static cudaError_t launch_ip(const LaunchArgs& a) {
    inplane_sweep_kernel<T, R, BX, RXV, RY, G, AX, PS><<<a.grid, a.block, a.smem, a.stream>>>(
        *a.tmap, G ? *a.tmap_g : *a.tmap, static_cast<T*>(a.out), *static_cast<const SweepParams<T>*>(a.params));
    return cudaGetLastError();
}

template <typename T, int R, int BX, int RXV, int RY, int ZB, bool G, bool AX, bool PS = false>
static cudaError_t launch_ws(const LaunchArgs& a) {
    inplane_ws_kernel<T, R, BX, RXV, RY, ZB, G, AX, PS><<<a.grid, a.block, a.smem, a.stream>>>(
        *a.tmap, G ? *a.tmap_g : *a.tmap, static_cast<T*>(a.out), *static_cast<const SweepParams<T>*>(a.params));
    return cudaGetLastError();
}

template <typename T, int R, int BX, int RXV, int RY, int ZB, int KIND>
static cudaError_t launch_dg(const LaunchArgs& a) {
    divgrad_kernel<T, R, BX, RXV, RY, ZB, KIND><<<a.grid, a.block, a.smem, a.stream>>>(
        *a.tmap, KIND == DG_DIV ? *a.tmap_g : *a.tmap, KIND == DG_DIV ? *a.tmap_h : *a.tmap, static_cast<T*>(a.out),
        static_cast<T*>(a.out1), static_cast<T*>(a.out2), *static_cast<const SweepParams<T>*>(a.params));
    return cudaGetLastError();
}

template <typename T, int R, bool G, bool AX, int RY = 1>
static cudaError_t launch_fp(const LaunchArgs& a) {
    forward_sweep_kernel<T, R, G, AX, RY><<<a.grid, a.block, a.smem, a.stream>>>(
        static_cast<const T*>(a.in), static_cast<const T*>(a.g), static_cast<T*>(a.out),
        *static_cast<const SweepParams<T>*>(a.params));
    return cudaGetLastError();
}

template <typename T, int R, int BX, int RXV, int RY>
static cudaError_t launch_fpt(const LaunchArgs& a) {
    fp_tma_kernel<T, R, BX, RXV, RY><<<a.grid, a.block, a.smem, a.stream>>>(
        *a.tmap, static_cast<T*>(a.out), *static_cast<const SweepParams<T>*>(a.params));
    return cudaGetLastError();
}

template <typename T, int R, int LOAD, int RY>
static cudaError_t launch_ldg(const LaunchArgs& a) {
    inplane_ldg_kernel<T, R, LOAD, RY><<<a.grid, a.block, a.smem, a.stream>>>(
        static_cast<const T*>(a.in), static_cast<T*>(a.out), *static_cast<const SweepParams<T>*>(a.params));
    return cudaGetLastError();
}

template <typename T>
constexpr int dtype_of() {
    return sizeof(T) == 4 ? STENCIL_F32 : STENCIL_F64;
}

// kernel variant recorded in KernelEntry::source: 0 plain Eq. (1), 1 second
// centre-only grid (G), 2 per-axis coefficients (AX), 3 fused peer-store
// halo exchange (PS)
template <bool G, bool AX, bool PS = false>
constexpr int variant_of() {
    return G ? 1 : (AX ? 2 : (PS ? 3 : 0));
}

template <typename T, int R, int BX, int RXV, int RY, bool G, bool AX, bool PS>
static void add_ip(std::vector<KernelEntry>& v) {
    constexpr int W = BX * RXV * Vec<T>::N;
    if constexpr (inplane_fits<T, R, RXV, RY, AX>() && W + 2 * InplaceGeom<T, R>::HX <= 256) {
        v.push_back({STENCIL_KERNEL_INPLANE, dtype_of<T>(), R, BX, RXV, RY, variant_of<G, AX, PS>(), 0,
                     reinterpret_cast<const void*>(&inplane_sweep_kernel<T, R, BX, RXV, RY, G, AX, PS>),
                     &launch_ip<T, R, BX, RXV, RY, G, AX, PS>});
    }
}

template <typename T, int R, int BX, bool G, bool AX, bool PS>
static void add_bx(std::vector<KernelEntry>& v) {
    add_ip<T, R, BX, 1, 1, G, AX, PS>(v);
    add_ip<T, R, BX, 1, 2, G, AX, PS>(v);
    add_ip<T, R, BX, 1, 4, G, AX, PS>(v);
    add_ip<T, R, BX, 1, 8, G, AX, PS>(v);
    add_ip<T, R, BX, 2, 1, G, AX, PS>(v);
    add_ip<T, R, BX, 2, 2, G, AX, PS>(v);
    add_ip<T, R, BX, 2, 4, G, AX, PS>(v);
}

template <typename T, int R, int BX, int RXV, int RY, int ZB, bool G, bool AX, bool PS = false>
static void add_ws(std::vector<KernelEntry>& v) {
    constexpr int W = BX * RXV * Vec<T>::N;
    if constexpr (inplane_fits<T, R, RXV, RY, AX>() && W + 2 * InplaceGeom<T, R>::HX <= 256) {
        v.push_back({STENCIL_KERNEL_INPLANE_WS, dtype_of<T>(), R, BX, RXV, RY, variant_of<G, AX, PS>(), ZB,
                     reinterpret_cast<const void*>(&inplane_ws_kernel<T, R, BX, RXV, RY, ZB, G, AX, PS>),
                     &launch_ws<T, R, BX, RXV, RY, ZB, G, AX, PS>});
    }
}

template <typename T, int R, int BX, int RXV, int RY, bool G, bool AX, bool PS = false>
static void add_ws_zb(std::vector<KernelEntry>& v) {
    add_ws<T, R, BX, RXV, RY, 1, G, AX, PS>(v);
    add_ws<T, R, BX, RXV, RY, 2, G, AX, PS>(v);
    add_ws<T, R, BX, RXV, RY, 4, G, AX, PS>(v);
}

// warp-specialized in-plane kernels (inplane_ws.cuh): the register tiles that
// win on B200 (16-byte x vectors, 2 or 4 rows) for block widths 16 and 32;
// PS = the fused peer-store slab variant (kern_<dtype>_r<R>_ps.cu)
template <typename T, int R, bool G, bool AX = false, bool PS = false>
static void register_ws(std::vector<KernelEntry>& v) {
    add_ws_zb<T, R, 16, 1, 2, G, AX, PS>(v);
    add_ws_zb<T, R, 16, 1, 4, G, AX, PS>(v);
    add_ws_zb<T, R, 32, 1, 2, G, AX, PS>(v);
    add_ws_zb<T, R, 32, 1, 4, G, AX, PS>(v);
}

// G = false: the plain sweep (Eq. 1); G = true: the application-stencil variant
// with a second, centre-only input grid (kern_<dtype>_r<R>_g.cu); AX = true:
// per-axis coefficients (kern_<dtype>_r<R>_ax.cu); PS = true: fused peer-store
// halo exchange (kern_<dtype>_r<R>_ps.cu, in-plane only).  AX / PS register
// block widths 16 and 32 only, to bound build time -- the tuner sees only what
// is registered.
template <typename T, int R, bool G, bool AX = false, bool PS = false>
static void register_radius(std::vector<KernelEntry>& v) {
    add_bx<T, R, 16, G, AX, PS>(v);
    add_bx<T, R, 32, G, AX, PS>(v);
    if constexpr (!AX && !PS) add_bx<T, R, 64, G, AX, PS>(v);
    if constexpr (!PS)
        v.push_back({STENCIL_KERNEL_FORWARD, dtype_of<T>(), R, 0, 0, 1, variant_of<G, AX>(), 0,
                     reinterpret_cast<const void*>(&forward_sweep_kernel<T, R, G, AX>), &launch_fp<T, R, G, AX>});
}

}  // namespace stencil

#define STENCIL_REGISTER(NAME, T, R, G) \
    namespace stencil {                 \
    void NAME(std::vector<KernelEntry>& v) { register_radius<T, R, G>(v); } \
    }
namespace stencil {

// the ablation kernels (ablation.cuh): forward-plane with register rows, and the paper's in-plane
// loading variants with per-thread loads, each with 1, 2 and 4 register rows
template <typename T, int R, int LOAD>
static void add_ldg(std::vector<KernelEntry>& v) {
    constexpr int kind = STENCIL_KERNEL_IP_CLASSIC + LOAD;
    v.push_back({kind, dtype_of<T>(), R, 0, 0, 1, 0, 0, reinterpret_cast<const void*>(&inplane_ldg_kernel<T, R, LOAD, 1>),
                 &launch_ldg<T, R, LOAD, 1>});
    v.push_back({kind, dtype_of<T>(), R, 0, 0, 2, 0, 0, reinterpret_cast<const void*>(&inplane_ldg_kernel<T, R, LOAD, 2>),
                 &launch_ldg<T, R, LOAD, 2>});
    v.push_back({kind, dtype_of<T>(), R, 0, 0, 4, 0, 0, reinterpret_cast<const void*>(&inplane_ldg_kernel<T, R, LOAD, 4>),
                 &launch_ldg<T, R, LOAD, 4>});
}

// forward-plane with K-IP's TMA loads and register tiles (fp_tma.cuh)
template <typename T, int R, int BX, int RY>
static void add_fpt(std::vector<KernelEntry>& v) {
    constexpr int W = BX * Vec<T>::N;
    if constexpr (fp_tma_fits<T, R, 1, RY>() && W + 2 * InplaceGeom<T, R>::HX <= 256)
        v.push_back({STENCIL_KERNEL_FP_TMA, dtype_of<T>(), R, BX, 1, RY, 0, 0,
                     reinterpret_cast<const void*>(&fp_tma_kernel<T, R, BX, 1, RY>), &launch_fpt<T, R, BX, 1, RY>});
}

template <typename T, int R>
static void register_ablation(std::vector<KernelEntry>& v) {
    add_fpt<T, R, 16, 1>(v);
    add_fpt<T, R, 16, 2>(v);
    add_fpt<T, R, 16, 4>(v);
    add_fpt<T, R, 32, 1>(v);
    add_fpt<T, R, 32, 2>(v);
    add_fpt<T, R, 32, 4>(v);
    add_ldg<T, R, LOAD_CLASSIC>(v);
    add_ldg<T, R, LOAD_VERTICAL>(v);
    add_ldg<T, R, LOAD_HORIZONTAL>(v);
    add_ldg<T, R, LOAD_FULLSLICE>(v);
    add_ldg<T, R, LOAD_FULLSLICE_V>(v);
    v.push_back({STENCIL_KERNEL_FORWARD, dtype_of<T>(), R, 0, 0, 2, 0, 0,
                 reinterpret_cast<const void*>(&forward_sweep_kernel<T, R, false, false, 2>), &launch_fp<T, R, false, false, 2>});
    v.push_back({STENCIL_KERNEL_FORWARD, dtype_of<T>(), R, 0, 0, 4, 0, 0,
                 reinterpret_cast<const void*>(&forward_sweep_kernel<T, R, false, false, 4>), &launch_fp<T, R, false, false, 4>});
}

}  // namespace stencil

namespace stencil {

// Div / Grad (divgrad.cuh): kernel kind INPLANE_WS, plan variants 4 (div) and 5 (grad)
template <typename T, int R, int BX, int RY, int KIND>
static void add_dg(std::vector<KernelEntry>& v) {
    v.push_back({STENCIL_KERNEL_INPLANE_WS, dtype_of<T>(), R, BX, 1, RY, 4 + KIND, 2,
                 reinterpret_cast<const void*>(&divgrad_kernel<T, R, BX, 1, RY, 2, KIND>),
                 &launch_dg<T, R, BX, 1, RY, 2, KIND>});
}

template <typename T, int R>
static void register_divgrad(std::vector<KernelEntry>& v) {
    add_dg<T, R, 16, 2, DG_DIV>(v);
    add_dg<T, R, 16, 4, DG_DIV>(v);
    add_dg<T, R, 32, 2, DG_DIV>(v);
    add_dg<T, R, 32, 4, DG_DIV>(v);
    add_dg<T, R, 16, 2, DG_GRAD>(v);
    add_dg<T, R, 16, 4, DG_GRAD>(v);
    add_dg<T, R, 32, 2, DG_GRAD>(v);
    add_dg<T, R, 32, 4, DG_GRAD>(v);
}

}  // namespace stencil

#define STENCIL_REGISTER_DG(NAME, T, R) \
    namespace stencil {                 \
    void NAME(std::vector<KernelEntry>& v) { register_divgrad<T, R>(v); } \
    }
#define STENCIL_REGISTER_ABL(NAME, T, R) \
    namespace stencil {                 \
    void NAME(std::vector<KernelEntry>& v) { register_ablation<T, R>(v); } \
    }
#define STENCIL_REGISTER_WS(NAME, T, R, G) \
    namespace stencil {                 \
    void NAME(std::vector<KernelEntry>& v) { register_ws<T, R, G>(v); } \
    }
#define STENCIL_REGISTER_AX(NAME, T, R) \
    namespace stencil {                 \
    void NAME(std::vector<KernelEntry>& v) { register_radius<T, R, false, true>(v); } \
    }
#define STENCIL_REGISTER_PS(NAME, T, R) \
    namespace stencil {                 \
    void NAME(std::vector<KernelEntry>& v) {                \
        register_radius<T, R, false, false, true>(v);       \
        register_ws<T, R, false, false, true>(v);           \
    }                                                       \
    }
