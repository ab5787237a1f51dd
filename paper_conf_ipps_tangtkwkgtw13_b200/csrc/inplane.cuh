// inplane.cuh -- K-IP: the in-plane full-slice sweep with register tiling,
// written for sm_100a.
//
// Paper: in-plane method Sec. III-C, Eqs. (3)-(5),
// steps 1-6, full-slice loading (Fig. 6d), vector loads
// (P:L189-191), register tiling.
//
// One thread block owns a W x H xy tile (W = TX*RX, H = TY*RY) and sweeps one
// z segment [z0, z1) of it.  Per plane k (interior index, k from z0-r to
// z1+r-1):
//   step 1  TMA loads the full slice (W+2HX) x (H+2r) of plane k -- interior and
//           halo as ONE box (HX = r rounded up to a 16-byte vector) -- into
//           stage k mod S of a shared-memory ring, S-1 planes ahead of use,
//           completing on an mbarrier (one elected thread issues it);
//   step 2  Eq. (3): each thread forms the partial output of its RX x RY points
//           from the in-plane neighbours (shared memory, 128-bit loads) and the
//           r "behind" centre values cached in registers;
//   step 3  Eq. (5): adds c_p * in[k] into the r queued partial outputs of
//           planes k-1..k-r (registers);
//   step 4  plane k-r is now complete: 128-bit coalesced stores to HBM;
//   step 5  the new partial and the centre values enter the register queues.
// The z loop is unrolled by r so that queue rotation is register renaming.
// Planes z0-r..z0-1 (warm-up) and z1..z1+r-1 (drain) are loaded so segments
// are independent; their outputs are never stored.
//
// Differences from the paper's Fermi/Kepler design:
// TMA + mbarrier ring instead of per-thread loads; contiguous RX vectors
// instead of strided outputs (reading R17); z segments to fill 148 SMs.
#pragma once

#include "common.cuh"

namespace stencil {

template <typename T, int R>
struct InplaceGeom {
    static constexpr int VEC = Vec<T>::N;                  // elements per 16-byte vector
    static constexpr int HX = ((R + VEC - 1) / VEC) * VEC;  // x halo, padded to a vector
    static constexpr int NVH = HX / VEC;                    // halo vectors per side
};

// Registers the queues need: 2r values per point (r partials + r behind).
template <typename T, int R, int RXV, int RY>
constexpr bool inplane_fits() {
    constexpr int pts = RXV * Vec<T>::N * RY;
    constexpr int words = 2 * R * pts * (int)(sizeof(T) / 4);
    return words <= 128;
}

template <typename T, int R, int RXV, int RY>
__global__ void __launch_bounds__(256, 1)
    inplane_sweep_kernel(const __grid_constant__ CUtensorMap tmap_in, T* __restrict__ out,
                         const SweepParams<T> p) {
    using G = InplaceGeom<T, R>;
    constexpr int VEC = G::VEC;
    constexpr int HX = G::HX;
    constexpr int NVH = G::NVH;
    constexpr int NX = RXV * VEC;  // points per thread along x

    extern __shared__ __align__(128) unsigned char smem_raw[];
    uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw);            // S mbarriers
    T* ring = reinterpret_cast<T*>(smem_raw + 128 * ((p.stages * 8 + 127) / 128));

    const int tx = threadIdx.x, ty = threadIdx.y;
    const int TX = blockDim.x;
    const int W = TX * NX, H = blockDim.y * RY;
    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int seg = p.seg_base + blockIdx.z * p.seg_stride;
    const int z0 = (int)(((long long)seg * p.nz) / p.zsegs);
    const int z1 = (int)(((long long)(seg + 1) * p.nz) / p.zsegs);
    const int L = (z1 - z0) + 2 * R;  // planes streamed: z0-R .. z1+R-1
    const bool leader = (tx == 0 && ty == 0);
    const uint32_t box_bytes = (uint32_t)((W + 2 * HX) * (H + 2 * R) * sizeof(T));
    // TMA box origin: outer x = tile_x*W - HX (element A - HX + ...), outer row tile_y*H
    const int bx0 = p.A - HX + tile_x * W;
    const int by0 = tile_y * H;

    if (leader) {
        prefetch_tensormap(&tmap_in);
        for (int s = 0; s < p.stages; ++s) mbar_init(&full[s], 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (leader) {
        const int npre = L < p.stages ? L : p.stages;
        for (int q = 0; q < npre; ++q) {
            mbar_arrive_expect_tx(&full[q], box_bytes);
            tma_load_3d(ring + (size_t)q * p.stage_elems, &tmap_in, bx0, by0, z0 - R + q + R, &full[q]);
        }
    }

    // Register queues.  Slot u holds plane (k mod R) == u.
    T qpart[R][RY][NX];  // partial outputs of the r previous planes (Eq. 5 targets)
    T behind[R][RY][NX]; // centre values of the r previous planes (Eq. 3 behind terms)
#pragma unroll
    for (int a = 0; a < R; ++a)
#pragma unroll
        for (int b = 0; b < RY; ++b)
#pragma unroll
            for (int e = 0; e < NX; ++e) { qpart[a][b][e] = T(0); behind[a][b][e] = T(0); }

    const int sp = p.smem_pitch;
    const int col0 = HX + tx * NX;   // my first centre column in the tile
    const int row0 = R + ty * RY;    // my first output row in the tile
    const int gx0 = tile_x * W + tx * NX;
    const int gy0 = tile_y * H + ty * RY;

    int stage = 0;
    uint32_t phase = 0;
    for (int q0 = 0; q0 < L; q0 += R) {
#pragma unroll
        for (int u = 0; u < R; ++u) {
            const int q = q0 + u;
            if (q < L) {
                mbar_wait(&full[stage], phase);
                const T* sb = ring + (size_t)stage * p.stage_elems;
                const int k = z0 - R + q;            // plane being consumed
                const bool write = (q >= 2 * R);     // plane k-R is an output of this segment
#pragma unroll
                for (int jj = 0; jj < RY; ++jj) {
                    // --- step 2 loads: row jj extended by the x halo, and the y column
                    T ext[NX + 2 * HX];
#pragma unroll
                    for (int h = 0; h < NVH; ++h)
                        lds16(&ext[h * VEC], sb + (row0 + jj) * sp + col0 - HX + h * VEC);
#pragma unroll
                    for (int v = 0; v < RXV; ++v)
                        lds16(&ext[HX + v * VEC], sb + (row0 + jj) * sp + col0 + v * VEC);
#pragma unroll
                    for (int h = 0; h < NVH; ++h)
                        lds16(&ext[HX + NX + h * VEC], sb + (row0 + jj) * sp + col0 + NX + h * VEC);
                    T ydn[R][NX], yup[R][NX];
#pragma unroll
                    for (int m = 1; m <= R; ++m)
#pragma unroll
                        for (int v = 0; v < RXV; ++v) {
                            lds16(&ydn[m - 1][v * VEC], sb + (row0 + jj - m) * sp + col0 + v * VEC);
                            lds16(&yup[m - 1][v * VEC], sb + (row0 + jj + m) * sp + col0 + v * VEC);
                        }
                    T part[NX];
#pragma unroll
                    for (int e = 0; e < NX; ++e) {
                        const T x = ext[HX + e];
                        // Eq. (3): in-plane + behind terms, fixed order (common.cuh)
                        T acc = f_mul(p.c[0], x);
#pragma unroll
                        for (int m = 1; m <= R; ++m)
                            acc = term(p.c[m], ext[HX + e - m], ext[HX + e + m], ydn[m - 1][e], yup[m - 1][e],
                                       behind[(u - m + R) % R][jj][e], acc);
                        part[e] = acc;
                        // Eq. (5): forward contributions to planes k-1..k-R, in arrival order
#pragma unroll
                        for (int pp = 1; pp <= R; ++pp)
                            qpart[(u - pp + R) % R][jj][e] = f_fma(p.c[pp], x, qpart[(u - pp + R) % R][jj][e]);
                    }
                    // --- step 4: plane k-R (slot u) is complete
                    if (write) {
                        const int gy = gy0 + jj;
                        if (gy < p.ny) {
                            T* dst = out + gidx<T, R>(p, gx0, gy, k - R);
#pragma unroll
                            for (int v = 0; v < RXV; ++v) {
                                const int xv = gx0 + v * VEC;
                                if (xv + VEC <= p.nx) {
                                    stg16(dst + v * VEC, &qpart[u][jj][v * VEC]);
                                } else {
#pragma unroll
                                    for (int e = 0; e < VEC; ++e)
                                        if (xv + e < p.nx) dst[v * VEC + e] = qpart[u][jj][v * VEC + e];
                                }
                            }
                        }
                    }
                    // --- step 5: shift in the new partial and the centre values
#pragma unroll
                    for (int e = 0; e < NX; ++e) {
                        qpart[u][jj][e] = part[e];
                        behind[u][jj][e] = ext[HX + e];
                    }
                }
                __syncthreads();  // every thread is done with this stage
                if (leader && q + p.stages < L) {
                    mbar_arrive_expect_tx(&full[stage], box_bytes);
                    tma_load_3d(ring + (size_t)stage * p.stage_elems, &tmap_in, bx0, by0,
                                z0 - R + q + p.stages + R, &full[stage]);
                }
                if (++stage == p.stages) { stage = 0; phase ^= 1u; }
            }
        }
    }
}

}  // namespace stencil
