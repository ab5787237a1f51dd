// divgrad.cuh -- Table V application stencils with several grids:
// Div (3 inputs -> 1 output) and Grad (1 input -> 3 outputs), computed with
// the in-plane method (Sec. III-C), SURVEY.md NEXT-1.
//
// Definitions (reading R19; the paper takes them from [17]):
// order-2r central first derivatives with one coefficient set a_1..a_r,
//   Div : out = sum_m a_m ((u[i+m]-u[i-m]) + (v[j+m]-v[j-m]) + (w[k+m]-w[k-m]))
//   Grad: gx = sum_m a_m (f[i+m]-f[i-m]),  gy (j),  gz (k)
// One sweep (no Fig. 1 loop).  The in-plane form: every input value is read
// in the plane it lives in; the z differences are built incrementally in a
// register queue of 2r partial outputs per point exactly as Eqs. (3)-(5) build
// Eq. (1) -- plane k adds -a_m w[k] to the outputs of planes k+m ("behind"
// terms) and +a_m w[k] to those of planes k-m ("forward" terms); the output
// of plane k-r is complete when plane k has streamed.  The x / y differences
// of plane k come from shared memory:
//   Div : a stage holds, per plane, an x-halo box of u ((W+2HX) x H), a
//         y-halo box of v (W x (H+2r)) and the centre box of w (W x H) -- the
//         three grids are in-plane'd separately, so only the halos each one
//         needs are moved (the paper's point that speedup falls as grids are
//         added, is about exactly these extra streams);
//   Grad: one full-slice box of f per plane; gx, gy of plane k are complete at
//         once and stored, gz goes through the queue.
// Per-point order (fixed, one for every configuration): behind terms m = r..1,
// then the in-plane differences m = 1..r (x then y), then forward terms
// m = 1..r.  Same warp-specialized structure as inplane_ws.cuh (producer
// warpgroup, compile-time planes per box, branch-free step body).
#pragma once

#include "inplane_ws.cuh"

namespace stencil {

enum { DG_DIV = 0, DG_GRAD = 1 };

template <typename T, int R, int BX, int RXV, int RY, int ZB, int KIND>
__global__ void __launch_bounds__(384, 1)
    divgrad_kernel(const __grid_constant__ CUtensorMap tm0, const __grid_constant__ CUtensorMap tm1,
                   const __grid_constant__ CUtensorMap tm2, T* __restrict__ out0, T* __restrict__ out1,
                   T* __restrict__ out2, const SweepParams<T> p) {
    using G = InplaceGeom<T, R>;
    using A = Lanes<T>;
    using L = typename A::L;
    constexpr int VEC = G::VEC;
    constexpr int HX = G::HX;
    constexpr int NVH = G::NVH;
    constexpr int NX = RXV * VEC;
    constexpr int NL = NX / A::PER;
    constexpr int LV = VEC / A::PER;
    constexpr int HL = HX / A::PER;
    constexpr int W = BX * NX;
    constexpr int SPU = W + 2 * HX;  // row pitch of an x-halo box
    constexpr int NCOL = RY + 2 * R;
    constexpr int Q = 2 * R;
    constexpr int U = Q / ws_gcd(Q, ZB) * ZB;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    const int S = p.stages;
    uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw);
    uint64_t* empty = full + S;
    T* ring = reinterpret_cast<T*>(smem_raw + 128 * ((2 * S * 8 + 127) / 128));
    const int ncw = p.ws_warps;
    const int pw = (ncw + 3) & ~3;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int H = (ncw * 32 / BX) * RY;
    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int seg = p.seg_base + blockIdx.z * p.seg_stride;
    const int z0 = (int)(((long long)seg * p.nz) / p.zsegs);
    const int z1 = (int)(((long long)(seg + 1) * p.nz) / p.zsegs);
    const int Lp = (z1 - z0) + 2 * R;
    const int y0 = (int)(((long long)tile_y * p.ny) / p.tiles_y);
    const int nloads = (Lp + ZB - 1) / ZB;
    // box offsets inside a stage (elements; each box a multiple of 128 bytes)
    auto rnd = [](int e) { return ((e * (int)sizeof(T) + 127) / 128) * 128 / (int)sizeof(T); };
    const int u_pl = (KIND == DG_DIV ? H : H + 2 * R) * SPU;  // per plane: u (div) or f (grad) box
    const int v_off = rnd(ZB * u_pl);
    const int v_pl = (H + 2 * R) * W;
    const int w_off = v_off + rnd(ZB * v_pl);
    const int w_pl = H * W;

    if (threadIdx.x == 0) {
        prefetch_tensormap(&tm0);
        if constexpr (KIND == DG_DIV) {
            prefetch_tensormap(&tm1);
            prefetch_tensormap(&tm2);
        }
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], ncw);
        }
        fence_mbar_init();
    }
    __syncthreads();

    if (warp >= pw) {  // producer warpgroup (inplane_ws.cuh)
        asm volatile("setmaxnreg.dec.sync.aligned.u32 24;\n" ::: "memory");
        if (warp == pw && lane == 0) {
            const uint64_t lpol = l2_policy(p.load_policy);
            const int xh = p.A - HX + tile_x * W, xc = p.A + tile_x * W;
            for (int l = 0, slot = 0, ph = 0; l < nloads; ++l) {
                if (l >= S) mbar_wait_sleep(&empty[slot], ph ^ 1u);
                const int bz = z0 + l * ZB;  // outer plane of the box's first plane (streamed upward)
                T* st = ring + (size_t)slot * p.stage_elems;
                mbar_arrive_expect_tx(&full[slot], p.stage_tx_bytes);
                if constexpr (KIND == DG_DIV) {
                    tma_load_3d_hint(st, &tm0, xh, y0 + R, bz, &full[slot], lpol);         // u: x halos
                    tma_load_3d_hint(st + v_off, &tm1, xc, y0, bz, &full[slot], lpol);     // v: y halos
                    tma_load_3d_hint(st + w_off, &tm2, xc, y0 + R, bz, &full[slot], lpol); // w: centre
                } else {
                    tma_load_3d_hint(st, &tm0, xh, y0, bz, &full[slot], lpol);             // f: full slice
                }
                if (++slot == S) {
                    slot = 0;
                    ph ^= 1u;
                }
            }
        }
        return;
    }
    asm volatile("setmaxnreg.inc.sync.aligned.u32 240;\n" ::: "memory");
    if (warp >= ncw) return;

    const int tx = threadIdx.x % BX, ty = threadIdx.x / BX;
    L acc[Q][RY][NL];
#pragma unroll
    for (int a = 0; a < Q; ++a)
#pragma unroll
        for (int b = 0; b < RY; ++b)
#pragma unroll
            for (int e = 0; e < NL; ++e) acc[a][b][e] = A::bcast(T(0));
    L ap[R + 1], an[R + 1];  // +a_m (forward / in-plane) and -a_m (behind), index m
#pragma unroll
    for (int m = 1; m <= R; ++m) {
        ap[m] = A::bcast(p.c[m]);
        an[m] = A::bcast(-p.c[m]);
    }
    const int gx0 = tile_x * W + tx * NX;
    const int gy0 = y0 + ty * RY;
    const bool fast = (tile_x + 1) * W <= p.nx && y0 + H <= p.ny;
    // plane-k output pointers (z = z0 - R at step 0; the z output of plane k-R lags by R planes)
    T* dz = (KIND == DG_DIV ? out0 : out2) + gidx<T, R>(p, gx0, gy0, z0 - 2 * R);
    T* dx = out0 + gidx<T, R>(p, gx0, gy0, z0 - R);  // grad only
    T* dy = out1 + gidx<T, R>(p, gx0, gy0, z0 - R);
    const long long dplane = p.plane;
#ifdef STENCIL_STG16
    const uint64_t spol = l2_policy(p.store_policy);
#endif
    auto store_rows = [&](T* base, L (&v)[RY][NL], bool pred, auto fast_tag) {
        constexpr bool FAST = decltype(fast_tag)::value;
#pragma unroll
        for (int jj = 0; jj < RY; ++jj) {
            if constexpr (FAST) {
#ifdef STENCIL_STG16  // experiment hook: 16-byte vector stores (measured 4-8 % slower for Grad, profiles/r2c/stg16_*)
#pragma unroll
                for (int q = 0; q < RXV; ++q)
                    stg16_if(base + jj * p.pitch + q * VEC, v[jj][q * LV], v[jj][q * LV + 1], pred, spol);
#else
#pragma unroll
                for (int e = 0; e < NL; ++e) stg8_if(base + jj * p.pitch + e * A::PER, v[jj][e], pred);
#endif
            } else {
#pragma unroll
                for (int e = 0; e < NX; ++e)
                    stg_if(base + jj * p.pitch + e, A::elem(&v[jj][0], e), pred && gy0 + jj < p.ny && gx0 + e < p.nx);
            }
        }
    };
    // thread offsets inside a stage plane
    const int off_x = (ty * RY) * SPU + HX + tx * NX;  // u / f box: my first row, first point
    const int off_v = (ty * RY) * W + tx * NX;         // v box: my column block (rows -R .. RY+R-1)
    const int off_w = (ty * RY) * W + tx * NX;         // w box: my rows

    int slot = 0;
    uint32_t phase = 0;
    const T* stage = ring;
    int q0 = 0;
    auto sweep = [&](auto fast_tag, auto checked_tag) {
        constexpr bool CHECKED = decltype(checked_tag)::value;
        for (; CHECKED ? q0 < Lp : q0 + U <= Lp; q0 += U) {
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int q = q0 + u;
                if (!CHECKED || q < Lp) {
                    const int zs = u % ZB;
                    if (zs == 0) mbar_wait(&full[slot], phase);
                    const bool write_z = q >= 2 * R;                // plane k-R is an output
                    const bool write_c = q >= R && q < Lp - R;      // plane k is an output (grad gx, gy)
                    // centre values of plane k (z terms): w (div) or f (grad)
                    L zc[RY][NL];
                    L colf[NCOL][NL];  // grad: f column block incl. y halos
                    if constexpr (KIND == DG_DIV) {
                        const T* sw = stage + w_off + zs * w_pl + off_w;
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                            for (int v = 0; v < RXV; ++v) A::lds16(&zc[jj][v * LV], sw + jj * W + v * VEC);
                    } else {
                        const T* sf = stage + zs * u_pl + off_x;
#pragma unroll
                        for (int rr = 0; rr < NCOL; ++rr)
#pragma unroll
                            for (int v = 0; v < RXV; ++v) A::lds16(&colf[rr][v * LV], sf + rr * SPU + v * VEC);
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                            for (int e = 0; e < NL; ++e) zc[jj][e] = colf[R + jj][e];
                    }
                    // ---- forward terms (+a_m z[k]) into planes k-1 .. k-R; plane k-R completes
#pragma unroll
                    for (int m = 1; m < R; ++m)
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                            for (int e = 0; e < NL; ++e)
                                acc[(u - m + Q) % Q][jj][e] = A::fma(ap[m], zc[jj][e], acc[(u - m + Q) % Q][jj][e]);
                    L fin[RY][NL];
#pragma unroll
                    for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                        for (int e = 0; e < NL; ++e) fin[jj][e] = A::fma(ap[R], zc[jj][e], acc[(u + R) % Q][jj][e]);
                    store_rows(dz, fin, write_z, fast_tag);
                    dz += dplane;
                    // ---- in-plane differences of plane k
                    if constexpr (KIND == DG_DIV) {
                        // x differences of u (its x-halo box) then y differences of v (its y-halo box)
                        const T* su = stage + zs * u_pl + off_x;
                        const T* sv = stage + v_off + zs * v_pl + off_v;
                        L colv[NCOL][NL];
#pragma unroll
                        for (int rr = 0; rr < NCOL; ++rr)
#pragma unroll
                            for (int v = 0; v < RXV; ++v) A::lds16(&colv[rr][v * LV], sv + rr * W + v * VEC);
                        L ext[RY][NL + 2 * HL];
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj) {
#pragma unroll
                            for (int h = 0; h < NVH; ++h) {
                                A::lds16(&ext[jj][h * LV], su + jj * SPU - HX + h * VEC);
                                A::lds16(&ext[jj][HL + NL + h * LV], su + jj * SPU + NX + h * VEC);
                            }
#pragma unroll
                            for (int v = 0; v < RXV; ++v) A::lds16(&ext[jj][HL + v * LV], su + jj * SPU + v * VEC);
                        }
#pragma unroll
                        for (int m = 1; m <= R; ++m)
#pragma unroll
                            for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                                for (int e = 0; e < NL; ++e) {
                                    const L xd = A::xdiff(ext[jj], HX + e * A::PER, m);
                                    const L yd = A::sub(colv[R + jj + m][e], colv[R + jj - m][e]);
                                    acc[u % Q][jj][e] = A::fma(ap[m], xd, acc[u % Q][jj][e]);
                                    acc[u % Q][jj][e] = A::fma(ap[m], yd, acc[u % Q][jj][e]);
                                }
                    } else {
                        // gx, gy of plane k, complete now
                        const T* sf = stage + zs * u_pl + off_x;
                        L ext[RY][NL + 2 * HL];
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj) {
#pragma unroll
                            for (int h = 0; h < NVH; ++h) {
                                A::lds16(&ext[jj][h * LV], sf + (R + jj) * SPU - HX + h * VEC);
                                A::lds16(&ext[jj][HL + NL + h * LV], sf + (R + jj) * SPU + NX + h * VEC);
                            }
#pragma unroll
                            for (int e = 0; e < NL; ++e) ext[jj][HL + e] = colf[R + jj][e];
                        }
                        L gxv[RY][NL], gyv[RY][NL];
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                            for (int e = 0; e < NL; ++e) {
                                gxv[jj][e] = A::mul(ap[1], A::xdiff(ext[jj], HX + e * A::PER, 1));
                                gyv[jj][e] = A::mul(ap[1], A::sub(colf[R + jj + 1][e], colf[R + jj - 1][e]));
                            }
#pragma unroll
                        for (int m = 2; m <= R; ++m)
#pragma unroll
                            for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                                for (int e = 0; e < NL; ++e) {
                                    gxv[jj][e] = A::fma(ap[m], A::xdiff(ext[jj], HX + e * A::PER, m), gxv[jj][e]);
                                    gyv[jj][e] = A::fma(ap[m], A::sub(colf[R + jj + m][e], colf[R + jj - m][e]), gyv[jj][e]);
                                }
                        store_rows(dx, gxv, write_c, fast_tag);
                        store_rows(dy, gyv, write_c, fast_tag);
                        dx += dplane;
                        dy += dplane;
                    }
                    // ---- behind terms (-a_m z[k]) for planes k+R .. k+1 (-a_R first)
#pragma unroll
                    for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                        for (int e = 0; e < NL; ++e) acc[(u + R) % Q][jj][e] = A::mul(an[R], zc[jj][e]);
#pragma unroll
                    for (int m = R - 1; m >= 1; --m)
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                            for (int e = 0; e < NL; ++e)
                                acc[(u + m) % Q][jj][e] = A::fma(an[m], zc[jj][e], acc[(u + m) % Q][jj][e]);
                    if (zs == ZB - 1) {
                        __syncwarp();
                        if (lane == 0) mbar_arrive(&empty[slot]);
                        if (++slot == S) {
                            slot = 0;
                            phase ^= 1u;
                        }
                        stage = ring + (size_t)slot * p.stage_elems;
                    }
                }
            }
        }
    };
    if (fast) {
        sweep(std::integral_constant<bool, true>{}, std::integral_constant<bool, false>{});
        sweep(std::integral_constant<bool, true>{}, std::integral_constant<bool, true>{});
    } else {
        sweep(std::integral_constant<bool, false>{}, std::integral_constant<bool, true>{});
    }
}

}  // namespace stencil
