// ablation.cuh -- the paper's loading variants with per-thread global loads
// (Sec. III-C 1-3, Fig. 6; evaluated in Fig. 7 and Fig. 10,
// P:L216-226), for the NEXT-2 ablation.
//
// K-IP (inplane.cuh / inplane_ws.cuh) moves a plane tile with ONE TMA box; the
// paper's kernels move it with per-thread loads, and how those loads are
// grouped is what Fig. 6 varies.  These kernels keep everything else fixed --
// the in-plane schedule of Eqs. (3)-(5) with the register queue, the fixed
// per-point order of common.cuh (so every variant is bit-identical to K-IP and
// K-FP), one point per thread in x and RY rows per thread in y (register
// blocking, outputs strided by TY as the paper does) -- and vary only
// how plane k reaches shared memory:
//   LOAD_CLASSIC     interior by each thread, top/bottom halos by threads
//                    ty < r, left/right halos by threads tx < r (Fig. 6a: the
//                    nvstencil pattern applied to the in-plane schedule);
//   LOAD_VERTICAL    interior columns together with their top/bottom halos
//                    (one coalesced strip per row), left/right halos apart
//                    (Fig. 6b);
//   LOAD_HORIZONTAL  interior rows together with their left/right halos, the
//                    top/bottom halo rows apart (Fig. 6c);
//   LOAD_FULLSLICE   the whole (W+2r) x (H+2r) slice, corners included, by a
//                    warp-aligned flat assignment (Fig. 6d);
//   LOAD_FULLSLICE_V the full slice in 16-byte vectors (the "memory-level
//                    parallelism" of P:L189-191): rows start HX = r rounded up
//                    to a vector before the tile, as the TMA box of K-IP.
// The plane tile is double-buffered in shared memory: one __syncthreads per
// plane.  Sweep direction, z segments and warm-up / drain planes as K-IP.
#pragma once

#include "common.cuh"

namespace stencil {

enum { LOAD_CLASSIC = 0, LOAD_VERTICAL = 1, LOAD_HORIZONTAL = 2, LOAD_FULLSLICE = 3, LOAD_FULLSLICE_V = 4 };

// shared-memory row pitch of the ablation tile: W + 2*HXA (+1 element when that is a multiple of
// 32 words, so the column accesses of neighbouring rows do not share banks)
template <typename T, int R, int LOAD>
struct AblGeom {
    static constexpr int VEC = Vec<T>::N;
    static constexpr int HXA = LOAD == LOAD_FULLSLICE_V ? ((R + VEC - 1) / VEC) * VEC : R;  // x halo in smem
    static __host__ __device__ int pitch(int W) {
        const int p = W + 2 * HXA;
        return (LOAD != LOAD_FULLSLICE_V && (p * (int)sizeof(T) / 4) % 32 == 0) ? p + 1 : p;
    }
};

template <typename T, int R, int LOAD, int RY>
__global__ void __launch_bounds__(512, 1)
    inplane_ldg_kernel(const T* __restrict__ in, T* __restrict__ out, const SweepParams<T> p) {
    using G = AblGeom<T, R, LOAD>;
    constexpr int HXA = G::HXA;
    constexpr int VEC = G::VEC;
    constexpr int Q = 2 * R;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    const int TX = blockDim.x, TY = blockDim.y;
    const int W = TX, H = TY * RY;
    const int SP = G::pitch(W);
    const int plane_elems = SP * (H + 2 * R);
    T* buf0 = reinterpret_cast<T*>(smem_raw);
    const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * TX + tx, nth = TX * TY;
    const int x0 = blockIdx.x * W;          // interior x of the tile's first column
    const int y0 = blockIdx.y * H;
    const int seg = p.seg_base + blockIdx.z * p.seg_stride;
    const int z0 = (int)(((long long)seg * p.nz) / p.zsegs);
    const int z1 = (int)(((long long)(seg + 1) * p.nz) / p.zsegs);
    const int Lp = (z1 - z0) + 2 * R;
    const int dir = p.dir;
    const long long pitch = p.pitch;

    // value of outer-grid point (interior coordinates xx, yy in [-R, n + R)), 0 outside the grid
    auto ld = [&](const T* pl, int xx, int yy) -> T {
        return (xx >= -R && xx < p.nx + R && yy >= -R && yy < p.ny + R) ? __ldg(pl + (long long)(yy + R) * pitch + p.A + xx)
                                                                       : T(0);
    };
    // load streamed plane q (outer plane index zo) into tile buffer b: element (row, col) of the tile is
    // outer point (x0 - HXA + col, y0 - R + row)
    auto load_plane = [&](T* b, int zo) {
        const T* pl = in + (long long)zo * p.plane;
        if constexpr (LOAD == LOAD_FULLSLICE) {
            const int rw = W + 2 * R, n = rw * (H + 2 * R);
            for (int i = tid; i < n; i += nth) {
                const int row = i / rw, col = i - row * rw;
                b[row * SP + col] = ld(pl, x0 - R + col, y0 - R + row);
            }
        } else if constexpr (LOAD == LOAD_FULLSLICE_V) {
            // 16-byte vectors; the row of W + 2 HXA elements starts at a vector boundary (A is 128 B aligned)
            const int nv = (W + 2 * HXA) / VEC, n = nv * (H + 2 * R);
            for (int i = tid; i < n; i += nth) {
                const int row = i / nv, v = i - row * nv;
                const int xx = x0 - HXA + v * VEC, yy = y0 - R + row;
                T* d = b + row * SP + v * VEC;
                if (yy >= -R && yy < p.ny + R && xx + VEC <= p.pitch - p.A) {  // inside the pitched row
                    const T* s = pl + (long long)(yy + R) * pitch + p.A + xx;
                    if constexpr (sizeof(T) == 4) {
                        const float4 w = __ldg(reinterpret_cast<const float4*>(s));
                        d[0] = w.x; d[1] = w.y; d[2] = w.z; d[3] = w.w;
                    } else {
                        const double2 w = __ldg(reinterpret_cast<const double2*>(s));
                        d[0] = w.x; d[1] = w.y;
                    }
                } else {
#pragma unroll
                    for (int e = 0; e < VEC; ++e) d[e] = T(0);
                }
            }
        } else if constexpr (LOAD == LOAD_VERTICAL) {
            for (int row = ty; row < H + 2 * R; row += TY) b[row * SP + HXA + tx] = ld(pl, x0 + tx, y0 - R + row);
            if (tx < R)
                for (int row = ty; row < H + 2 * R; row += TY) {
                    b[row * SP + HXA - R + tx] = ld(pl, x0 - R + tx, y0 - R + row);
                    b[row * SP + HXA + W + tx] = ld(pl, x0 + W + tx, y0 - R + row);
                }
        } else if constexpr (LOAD == LOAD_HORIZONTAL) {
            const int rw = W + 2 * R, n = rw * H;
            for (int i = tid; i < n; i += nth) {
                const int row = i / rw, col = i - row * rw;
                b[(row + R) * SP + col] = ld(pl, x0 - R + col, y0 + row);
            }
            if (ty < R) {
                b[ty * SP + HXA + tx] = ld(pl, x0 + tx, y0 - R + ty);
                b[(H + R + ty) * SP + HXA + tx] = ld(pl, x0 + tx, y0 + H + ty);
            }
        } else {  // LOAD_CLASSIC
#pragma unroll
            for (int j = 0; j < RY; ++j) b[(R + ty + j * TY) * SP + HXA + tx] = ld(pl, x0 + tx, y0 + ty + j * TY);
            if (ty < R) {
                b[ty * SP + HXA + tx] = ld(pl, x0 + tx, y0 - R + ty);
                b[(H + R + ty) * SP + HXA + tx] = ld(pl, x0 + tx, y0 + H + ty);
            }
            if (tx < R)
#pragma unroll
                for (int j = 0; j < RY; ++j) {
                    const int row = R + ty + j * TY;
                    b[row * SP + HXA - R + tx] = ld(pl, x0 - R + tx, y0 + ty + j * TY);
                    b[row * SP + HXA + W + tx] = ld(pl, x0 + W + tx, y0 + ty + j * TY);
                }
        }
    };

    T acc[Q][RY];
#pragma unroll
    for (int a = 0; a < Q; ++a)
#pragma unroll
        for (int j = 0; j < RY; ++j) acc[a][j] = T(0);
    const T* cz = p.c;
    const int gx = x0 + tx;
    // output rows strided by TY
    long long obase = (long long)R * pitch + p.A + gx;  // + (y + 0) * pitch per row, + plane offset
    auto zo_of = [&](int q) { return dir > 0 ? z0 - R + q + R : z1 + R - 1 - q + R; };  // outer plane of step q

    for (int q0 = 0; q0 < Lp; q0 += Q) {
#pragma unroll
        for (int u = 0; u < Q; ++u) {
            const int q = q0 + u;
            if (q < Lp) {
                T* b = buf0 + (q & 1) * plane_elems;
                load_plane(b, zo_of(q));
                __syncthreads();
                const bool write = q >= 2 * R;
                const int zout = (dir > 0 ? z0 - R + q : z1 + R - 1 - q) - dir * R;  // interior plane k - R
#pragma unroll
                for (int j = 0; j < RY; ++j) {
                    const int row = R + ty + j * TY;
                    const T* c0p = b + row * SP + HXA + tx;
                    const T x = c0p[0];
                    // step 3 (Eq. 5): forward terms into planes k-1 .. k-R; plane k-R completes
#pragma unroll
                    for (int m = 1; m <= R; ++m) acc[(u - m + Q) % Q][j] = f_fma(cz[m], x, acc[(u - m + Q) % Q][j]);
                    const int gy = y0 + ty + j * TY;
                    if (write && gx < p.nx && gy < p.ny)
                        out[obase + (long long)gy * pitch + (long long)(zout + R) * p.plane] = acc[(u + R) % Q][j];
                    // step 4: behind terms for planes k+R .. k+1
                    acc[(u + R) % Q][j] = f_mul(cz[R], x);
#pragma unroll
                    for (int m = R - 1; m >= 1; --m) acc[(u + m) % Q][j] = f_fma(cz[m], x, acc[(u + m) % Q][j]);
                    // step 5: Eq. (3) in-plane terms of plane k
                    T a = f_fma(p.c[0], x, acc[u % Q][j]);
#pragma unroll
                    for (int m = 1; m <= R; ++m) {
                        const T xs = f_add(c0p[-m], c0p[m]);
                        const T ys = f_add(c0p[-m * SP], c0p[m * SP]);
                        a = f_fma(p.c[m], xs, a);
                        a = f_fma(p.c[m], ys, a);
                    }
                    acc[u % Q][j] = a;
                }
            }
        }
    }
}

}  // namespace stencil
