// forward.cuh -- K-FP: the forward-plane baseline ("nvstencil", the CUDA SDK
// FDTD3d shape), compiled for sm_100a.
//
// Paper: forward-plane method P:L113-134 (Eq. 2), halo loading
// pattern of Fig. 4, SDK sample ref. [25]; with
// register blocking (RY > 1) it is case (i) of Fig. 10.
//
// Thread block TX x TY (TX = 32 as in the SDK), one output point per thread
// per plane per register row (RY rows strided by TY), 2r+1 register
// queue over [z-r, z+r] per point.  At each z step:
//   - the queue shifts; the thread loads the INTERIOR point of the forward
//     plane z+r (one scalar load per point, "input elements are loaded
//     ... a distance r away");
//   - the current plane is written to a (H+2r) x (TX+2r) shared tile; threads
//     with ty < r load the top/bottom halos and threads with tx < r the
//     left/right halos of the CURRENT plane (2-4 separate loads for
//     perimeter threads, Fig. 4);
//   - __syncthreads, Eq. (2) in the fixed order of common.cuh (so K-FP and
//     K-IP are bit-identical), store.
// A fair baseline: every address is a pointer advanced by one plane per step
// (no per-load index arithmetic), and the tile pitch is padded off a multiple
// of 32 banks.
#pragma once

#include "common.cuh"

namespace stencil {

__host__ __device__ inline int fp_tile_pitch(int TX, int R, int s) {
    const int p = TX + 2 * R;
    return ((p * s / 4) % 32 == 0) ? p + 1 : p;
}

// G: application stencils with a second, centre-only input grid g (see
// inplane.cuh): out = Eq. (2) + p.d * g, the g term last.  AX: per-axis
// coefficients (reading R3b), common.cuh order.  RY: register rows per thread.
template <typename T, int R, bool G, bool AX = false, int RY = 1>
__global__ void __launch_bounds__(512, 1)
    forward_sweep_kernel(const T* __restrict__ in, const T* __restrict__ g, T* __restrict__ out,
                         const SweepParams<T> p) {
    extern __shared__ __align__(128) unsigned char smem_raw[];
    T* tile = reinterpret_cast<T*>(smem_raw);
    const int tx = threadIdx.x, ty = threadIdx.y;
    const int TX = blockDim.x, TY = blockDim.y, H = TY * RY;
    const int tp = fp_tile_pitch(TX, R, (int)sizeof(T));  // tile pitch
    const int x = blockIdx.x * TX + tx;
    const int yb = blockIdx.y * H;  // first interior row of the tile
    const int seg = p.seg_base + blockIdx.z * p.seg_stride;
    const int z0 = (int)(((long long)seg * p.nz) / p.zsegs);
    const int z1 = (int)(((long long)(seg + 1) * p.nz) / p.zsegs);
    const long long pitch = p.pitch;
    // sweep direction (same convention as K-IP): "behind" = planes already passed
    const int dir = p.dir;
    const int zs = dir > 0 ? z0 : z1 - 1;  // first plane of the sweep
    const long long dpl = dir > 0 ? p.plane : -p.plane;
    // a point exists in the outer grid iff x, y in [-R, n + R)
    const bool x_ok = x < p.nx + R;
    // pointer to (x, row yb - R, plane zs) in the input; every other address is a fixed offset of it
    const T* pc = in + gidx<T, R>(p, x, yb - R, zs);
    T* po = out + gidx<T, R>(p, x, yb, zs);
    const T* pg = G ? g + gidx<T, R>(p, x, yb, zs) : nullptr;

    T behind[RY][R], infront[RY][R], cur[RY];
#pragma unroll
    for (int j = 0; j < RY; ++j) {
        const int y = yb + ty + j * TY;
        const bool ok = x_ok && y < p.ny + R;
        const T* q = pc + (long long)(R + ty + j * TY) * pitch;
#pragma unroll
        for (int m = 1; m <= R; ++m) behind[j][m - 1] = ok ? __ldg(q - m * dpl) : T(0);
        cur[j] = ok ? __ldg(q) : T(0);
#pragma unroll
        for (int m = 1; m <= R; ++m) infront[j][m - 1] = ok ? __ldg(q + m * dpl) : T(0);
    }

#pragma unroll 2
    for (int i = 0; i < z1 - z0; ++i) {
        __syncthreads();  // previous plane's compute is done with the tile
#pragma unroll
        for (int j = 0; j < RY; ++j) tile[(ty + j * TY + R) * tp + tx + R] = cur[j];
        if (ty < R && x_ok) {  // top / bottom halo rows of the current plane
            if (yb - R + ty >= -R) tile[ty * tp + tx + R] = __ldg(pc + (long long)ty * pitch);
            if (yb + H + ty < p.ny + R) tile[(ty + H + R) * tp + tx + R] = __ldg(pc + (long long)(ty + H + R) * pitch);
        }
        if (tx < R) {  // left / right halo columns of the current plane
#pragma unroll
            for (int j = 0; j < RY; ++j) {
                const int rr = ty + j * TY + R;
                if (yb + rr - R < p.ny + R) {
                    tile[rr * tp + tx] = __ldg(pc + (long long)rr * pitch - R);
                    if (x + TX < p.nx + R) tile[rr * tp + tx + TX + R] = __ldg(pc + (long long)rr * pitch + TX);
                }
            }
        }
        __syncthreads();
#pragma unroll
        for (int j = 0; j < RY; ++j) {
            const int y = yb + ty + j * TY;
            if (x < p.nx && y < p.ny) {  // Eq. (2) in the fixed order of common.cuh
                const T* cz = AX ? p.cz : p.c;  // z-axis coefficients
                const int rr = ty + j * TY + R;
                T acc = f_mul(cz[R], behind[j][R - 1]);
#pragma unroll
                for (int m = R - 1; m >= 1; --m) acc = f_fma(cz[m], behind[j][m - 1], acc);
                acc = f_fma(p.c[0], cur[j], acc);
#pragma unroll
                for (int m = 1; m <= R; ++m) {
                    const T xs = f_add(tile[rr * tp + tx + R - m], tile[rr * tp + tx + R + m]);
                    const T ys = f_add(tile[(rr - m) * tp + tx + R], tile[(rr + m) * tp + tx + R]);
                    acc = f_fma(p.c[m], xs, acc);
                    acc = f_fma(AX ? p.cy[m] : p.c[m], ys, acc);
                }
#pragma unroll
                for (int m = 1; m <= R; ++m) acc = f_fma(cz[m], infront[j][m - 1], acc);
                if constexpr (G) acc = f_fma(p.d, __ldg(pg + (long long)(ty + j * TY) * pitch), acc);
                po[(long long)(ty + j * TY) * pitch] = acc;
            }
        }
        // shift the 2r+1 queues and fetch the forward plane z + dir*(1+R)
        const bool more = i + 1 < z1 - z0;
#pragma unroll
        for (int j = 0; j < RY; ++j) {
#pragma unroll
            for (int m = R - 1; m > 0; --m) behind[j][m] = behind[j][m - 1];
            behind[j][0] = cur[j];
            cur[j] = infront[j][0];
#pragma unroll
            for (int m = 0; m < R - 1; ++m) infront[j][m] = infront[j][m + 1];
            const bool ok = x_ok && yb + ty + j * TY < p.ny + R;
            if (ok && more) infront[j][R - 1] = __ldg(pc + (long long)(R + ty + j * TY) * pitch + (1 + R) * dpl);
        }
        pc += dpl;
        po += dpl;
        if constexpr (G) pg += dpl;
    }
}

}  // namespace stencil
