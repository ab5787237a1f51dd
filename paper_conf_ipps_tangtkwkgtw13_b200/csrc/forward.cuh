// forward.cuh -- K-FP: the forward-plane baseline ("nvstencil", the CUDA SDK
// FDTD3d shape), compiled for sm_100a.
//
// Paper: forward-plane method P:L113-134 (Eq. 2), halo loading
// pattern of Fig. 4, SDK sample ref. [25].
//
// Thread block TX x TY (TX = 32 as in the SDK), one output point per thread
// per plane, full z sweep (no segments), 2r+1 register queue over
// [z-r, z+r].  At each z step:
//   - the queue shifts; the thread loads the INTERIOR point of the forward
//     plane z+r (one scalar load, "input elements are loaded ... a
//     distance r away");
//   - the current plane is written to a (TY+2r) x (TX+2r) shared tile; threads
//     with ty < r load the top/bottom halos and threads with tx < r the
//     left/right halos of the CURRENT plane (2-4 separate loads for
//     perimeter threads, Fig. 4);
//   - __syncthreads, Eq. (2) in the fixed order of common.cuh (so K-FP and
//     K-IP are bit-identical), store.
#pragma once

#include "common.cuh"

namespace stencil {

// G: application stencils with a second, centre-only input grid g (see
// inplane.cuh): out = Eq. (2) + p.d * g, the g term last.  AX: per-axis
// coefficients (reading R3b), common.cuh order.
template <typename T, int R, bool G, bool AX = false>
__global__ void __launch_bounds__(512, 1)
    forward_sweep_kernel(const T* __restrict__ in, const T* __restrict__ g, T* __restrict__ out,
                         const SweepParams<T> p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    T* tile = reinterpret_cast<T*>(smem_raw);
    const int tx = threadIdx.x, ty = threadIdx.y;
    const int TX = blockDim.x, TY = blockDim.y;
    const int tp = TX + 2 * R;  // tile pitch
    const int x = blockIdx.x * TX + tx;
    const int y = blockIdx.y * TY + ty;
    const int seg = p.seg_base + blockIdx.z * p.seg_stride;
    const int z0 = (int)(((long long)seg * p.nz) / p.zsegs);
    const int z1 = (int)(((long long)(seg + 1) * p.nz) / p.zsegs);
    // a point exists in the outer grid iff x, y in [-R, n + R)
    const bool c_ok = (x < p.nx + R) && (y < p.ny + R);
    const bool inside = (x < p.nx) && (y < p.ny);

#define FP_LD(xx, yy, zz) __ldg(&in[gidx<T, R>(p, (xx), (yy), (zz))])

    // sweep direction (same convention as K-IP): "behind" = planes already passed
    const int dir = p.dir;
    const int zs = dir > 0 ? z0 : z1 - 1;  // first plane of the sweep
    T behind[R], infront[R], cur = T(0);
#pragma unroll
    for (int m = 0; m < R; ++m) { behind[m] = T(0); infront[m] = T(0); }
    if (c_ok) {
#pragma unroll
        for (int m = 1; m <= R; ++m) behind[m - 1] = FP_LD(x, y, zs - dir * m);  // plane zs - dir*m
        cur = FP_LD(x, y, zs);
#pragma unroll
        for (int m = 1; m <= R; ++m) infront[m - 1] = FP_LD(x, y, zs + dir * m);  // plane zs + dir*m
    }

#pragma unroll 4  // (unroll 2 spilled for double r = 2; __launch_bounds__(512) alone let ptxas pick 32 registers + spills for float r = 4)
    for (int i = 0; i < z1 - z0; ++i) {
        const int z = zs + dir * i;
        __syncthreads();  // previous plane's compute is done with the tile
        tile[(ty + R) * tp + tx + R] = cur;
        if (ty < R) {  // top / bottom halo rows of the current plane
            if (x < p.nx + R && y - R >= -R) tile[ty * tp + tx + R] = FP_LD(x, y - R, z);
            if (x < p.nx + R && y + TY < p.ny + R) tile[(ty + TY + R) * tp + tx + R] = FP_LD(x, y + TY, z);
        }
        if (tx < R) {  // left / right halo columns of the current plane
            if (y < p.ny + R) tile[(ty + R) * tp + tx] = FP_LD(x - R, y, z);
            if (y < p.ny + R && x + TX < p.nx + R) tile[(ty + R) * tp + tx + TX + R] = FP_LD(x + TX, y, z);
        }
        __syncthreads();
        if (inside) {  // Eq. (2) in the fixed order of common.cuh
            const T* cz = AX ? p.cz : p.c;  // z-axis coefficients
            T acc = f_mul(cz[R], behind[R - 1]);
#pragma unroll
            for (int m = R - 1; m >= 1; --m) acc = f_fma(cz[m], behind[m - 1], acc);
            acc = f_fma(p.c[0], cur, acc);
#pragma unroll
            for (int m = 1; m <= R; ++m) {
                const T xs = f_add(tile[(ty + R) * tp + tx + R - m], tile[(ty + R) * tp + tx + R + m]);
                const T ys = f_add(tile[(ty + R - m) * tp + tx + R], tile[(ty + R + m) * tp + tx + R]);
                acc = f_fma(p.c[m], xs, acc);
                acc = f_fma(AX ? p.cy[m] : p.c[m], ys, acc);
            }
#pragma unroll
            for (int m = 1; m <= R; ++m) acc = f_fma(cz[m], infront[m - 1], acc);
            if constexpr (G) acc = f_fma(p.d, __ldg(&g[gidx<T, R>(p, x, y, z)]), acc);
            out[gidx<T, R>(p, x, y, z)] = acc;
        }
        // shift the 2r+1 queue and fetch the forward plane z + dir*(1+R)
#pragma unroll
        for (int m = R - 1; m > 0; --m) behind[m] = behind[m - 1];
        behind[0] = cur;
        cur = infront[0];
#pragma unroll
        for (int m = 0; m < R - 1; ++m) infront[m] = infront[m + 1];
        if (c_ok && i + 1 < z1 - z0) infront[R - 1] = FP_LD(x, y, z + dir * (1 + R));
    }
#undef FP_LD
}

}  // namespace stencil
