// fp_tma.cuh -- the forward-plane method with K-IP's loads: TMA full-slice
// boxes into an mbarrier ring, 16-byte column loads, register tiling and the
// FP32x2 lane arithmetic of inplane.cuh.  The NEXT-2 ablation row "forward
// plane + the same vector/TMA loads" (paper Fig. 10 case
// (i)): with the loading held fixed, what remains between this
// kernel and K-IP is the method itself.
//
// Forward-plane schedule (Eq. 2): output plane z is computed in
// ONE step, when plane z+r arrives, from a register queue of the 2r+1 input
// values in[z-r .. z+r] of each point plus the x / y neighbours of
// plane z, read from shared memory.  So plane z's slice must still be in the
// ring r planes after it arrived: the ring holds the slices of planes
// z .. z+r (and the loads in flight), against K-IP's one plane per step --
// the shared-memory cost of the forward-plane method that the in-plane
// method removes.  Two cursors walk the ring in stream order:
// the FRONT (plane q: its centre rows enter the queue) and the BACK (plane
// q-r: its neighbours are read, then its stage is released).  The ring needs
// at least ceil(r/ZB) + 2 stages (config_geometry enforces it): load
// floor(q/ZB) is waited for while load floor((q-r)/ZB) is still held and the
// refill runs one load behind.
//
// Per point the arithmetic is the fixed order of common.cuh (reading R7):
// c_r in[z-r], c_{r-1} in[z-r+1] .. c_1 in[z-1], c_0 in[z], (x pair, y pair)
// for m = 1..r, then c_1 in[z+1] .. c_r in[z+r] -- so the outputs are
// bit-identical to K-IP and K-FP.  The queue is indexed by plane mod 2r+1 and
// the z loop unrolled by 2r+1: no value moves between registers.
#pragma once

#include "inplane.cuh"

namespace stencil {

// registers: the (2r+1)-deep queue plus the column block of the back plane
template <typename T, int R, int RXV, int RY>
constexpr bool fp_tma_fits() {
    constexpr int w = (int)(sizeof(T) / 4);
    constexpr int pts = RXV * Vec<T>::N * RY;
    constexpr int words = ((2 * R + 1) * pts + 2 * R * RXV * Vec<T>::N) * w;
    return words <= 176;
}

template <typename T, int R, int BX, int RXV, int RY>
__global__ void __launch_bounds__(256, 1)
    fp_tma_kernel(const __grid_constant__ CUtensorMap tmap_in, T* __restrict__ out, const SweepParams<T> p) {
    using G = InplaceGeom<T, R>;
    using A = Lanes<T>;
    using L = typename A::L;
    constexpr int VEC = G::VEC;
    constexpr int HX = G::HX;
    constexpr int NVH = G::NVH;
    constexpr int NX = RXV * VEC;     // points per thread along x
    constexpr int NL = NX / A::PER;   // lanes per thread-row
    constexpr int LV = VEC / A::PER;  // lanes per 16-byte vector
    constexpr int HL = HX / A::PER;   // lanes of x halo
    constexpr int W = BX * NX;
    constexpr int SP = W + 2 * HX;
    constexpr int P = 2 * R + 1;      // queue depth (planes z-r .. z+r)

    extern __shared__ __align__(128) unsigned char smem_raw[];
    uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw);
    uint64_t* empty = full + p.stages;
    T* ring = reinterpret_cast<T*>(smem_raw + 128 * ((2 * p.stages * 8 + 127) / 128));

    const int tx = threadIdx.x, ty = threadIdx.y;
    const int lane = (ty * BX + tx) & 31;
    const int nwarps = (BX * blockDim.y + 31) / 32;
    const int H = blockDim.y * RY;
    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int seg = p.seg_base + blockIdx.z * p.seg_stride;
    const int z0 = (int)(((long long)seg * p.nz) / p.zsegs);
    const int z1 = (int)(((long long)(seg + 1) * p.nz) / p.zsegs);
    const int Lp = (z1 - z0) + 2 * R;  // planes streamed: z0-R .. z1+R-1
    const bool leader = (tx == 0 && ty == 0);
    const int pstride = SP * (H + 2 * R);
    const int bx0 = p.A - HX + tile_x * W;
    const int y0 = (int)(((long long)tile_y * p.ny) / p.tiles_y);
    const int y1 = (int)(((long long)(tile_y + 1) * p.ny) / p.tiles_y);

    if (leader) {
        prefetch_tensormap(&tmap_in);
        for (int s = 0; s < p.stages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], nwarps);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const uint64_t spol = l2_policy(p.store_policy), lpol = l2_policy(p.load_policy);
    const int ZB = p.zbox;
    const int dir = p.dir;
    const int nloads = (Lp + ZB - 1) / ZB;
    auto box_z = [&](int l) { return dir > 0 ? z0 + l * ZB : z1 + 2 * R - (l + 1) * ZB; };
    auto issue = [&](int slot, int l) {
        mbar_arrive_expect_tx(&full[slot], p.stage_tx_bytes);
        tma_load_3d_hint(ring + (size_t)slot * p.stage_elems, &tmap_in, bx0, y0, box_z(l), &full[slot], lpol);
    };
    if (leader) {
        const int npre = nloads < p.stages ? nloads : p.stages;
        for (int l = 0; l < npre; ++l) issue(l, l);
    }

    L c[R + 1];
#pragma unroll
    for (int m = 0; m <= R; ++m) c[m] = A::bcast(p.c[m]);
    L qv[P][RY][NL];  // centre rows of planes (slot = streamed plane index mod 2r+1)

    const int my_off = (ty * RY) * SP + HX + tx * NX;  // column block origin (first row - R)
    const int gx0 = tile_x * W + tx * NX;
    const int gy0 = y0 + ty * RY;
    const bool x_full = (tile_x + 1) * W <= p.nx;
    const int store_mode = !x_full ? 2 : (y1 - y0 == H ? 0 : 1);
    T* dst = out + gidx<T, R>(p, gx0, gy0, dir > 0 ? z0 : z1 - 1);
    const long long dplane = dir > 0 ? p.plane : -p.plane;

    int fstage = 0, fzin = 0;  // front cursor (plane q)
    uint32_t fphase = 0;
    int bstage = 0, bzin = 0;  // back cursor (plane q - R)
    uint32_t bphase = 0;
    int lrel = 0;              // loads released so far
    auto sweep = [&](auto mode_tag) {
    constexpr int MODE = decltype(mode_tag)::value;
    for (int q0 = 0; q0 < Lp; q0 += P) {
#pragma unroll
        for (int u = 0; u < P; ++u) {
            const int q = q0 + u;
            if (q < Lp) {
                // ---- front: the centre rows of plane q enter the queue
                if (fzin == 0) mbar_wait(&full[fstage], fphase);
                {
                    const int zi = dir > 0 ? fzin : ZB - 1 - fzin;
                    const T* sf = ring + (size_t)fstage * p.stage_elems + zi * pstride + my_off + R * SP;
#pragma unroll
                    for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                        for (int v = 0; v < RXV; ++v) A::lds16(&qv[u][jj][v * LV], sf + jj * SP + v * VEC);
                }
                if (++fzin == ZB) {
                    fzin = 0;
                    if (++fstage == p.stages) {
                        fstage = 0;
                        fphase ^= 1u;
                    }
                }
                if (q >= R) {
                    // ---- back: plane q - R is the current plane z
                    const int zi = dir > 0 ? bzin : ZB - 1 - bzin;
                    const T* sb = ring + (size_t)bstage * p.stage_elems + zi * pstride + my_off;
                    if (q >= 2 * R) {
                        // y neighbours: rows -R..-1 and RY..RY+R-1 from shared memory, the RY centre
                        // rows from the queue
                        L col[RY + 2 * R][NL];
#pragma unroll
                        for (int rr = 0; rr < R; ++rr)
#pragma unroll
                            for (int v = 0; v < RXV; ++v) {
                                A::lds16(&col[rr][v * LV], sb + rr * SP + v * VEC);
                                A::lds16(&col[R + RY + rr][v * LV], sb + (R + RY + rr) * SP + v * VEC);
                            }
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                            for (int e = 0; e < NL; ++e) col[R + jj][e] = qv[(u - R + P) % P][jj][e];
                        L ext[RY][NL + 2 * HL];  // rows with their x halo
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj) {
#pragma unroll
                            for (int h = 0; h < NVH; ++h) {
                                A::lds16(&ext[jj][h * LV], sb + (R + jj) * SP - HX + h * VEC);
                                A::lds16(&ext[jj][HL + NL + h * LV], sb + (R + jj) * SP + NX + h * VEC);
                            }
#pragma unroll
                            for (int e = 0; e < NL; ++e) ext[jj][HL + e] = col[R + jj][e];
                        }
                        // Eq. (2) in the fixed order: behind, centre, in-plane pairs, forward
                        L acc[RY][NL];
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                            for (int e = 0; e < NL; ++e) acc[jj][e] = A::mul(c[R], qv[(u - 2 * R + P) % P][jj][e]);
#pragma unroll
                        for (int m = R - 1; m >= 1; --m)
#pragma unroll
                            for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                                for (int e = 0; e < NL; ++e)
                                    acc[jj][e] = A::fma(c[m], qv[(u - R - m + 2 * P) % P][jj][e], acc[jj][e]);
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                            for (int e = 0; e < NL; ++e) acc[jj][e] = A::fma(c[0], col[R + jj][e], acc[jj][e]);
#pragma unroll
                        for (int m = 1; m <= R; ++m)
#pragma unroll
                            for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                                for (int e = 0; e < NL; ++e) {
                                    acc[jj][e] = A::fma(c[m], A::xsum(ext[jj], HX + e * A::PER, m), acc[jj][e]);
                                    acc[jj][e] = A::fma(c[m], A::add(col[R + jj - m][e], col[R + jj + m][e]), acc[jj][e]);
                                }
#pragma unroll
                        for (int m = 1; m <= R; ++m)
#pragma unroll
                            for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                                for (int e = 0; e < NL; ++e)
                                    acc[jj][e] = A::fma(c[m], qv[(u - R + m + P) % P][jj][e], acc[jj][e]);
                        if constexpr (MODE <= 1) {
#pragma unroll
                            for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                                for (int v = 0; v < RXV; ++v)
                                    A::stg16(dst + (long long)jj * p.pitch + v * VEC, &acc[jj][v * LV],
                                             MODE == 0 ? true : gy0 + jj < y1, spol);
                        } else {
#pragma unroll
                            for (int jj = 0; jj < RY; ++jj)
                                if (gy0 + jj < y1) {
#pragma unroll
                                    for (int e = 0; e < NX; ++e)
                                        if (gx0 + e < p.nx) dst[(long long)jj * p.pitch + e] = A::elem(&acc[jj][0], e);
                                }
                        }
                        dst += dplane;
                    }
                    // release the back stage after its last plane; the leader refills the stage of the
                    // load before it (one load behind, as K-IP)
                    if (++bzin == ZB) {
                        bzin = 0;
                        __syncwarp();
                        if (lane == 0) mbar_arrive(&empty[bstage]);
                        const int l = lrel++;
                        if (leader && l >= 1 && l - 1 + p.stages < nloads) {
                            const int ps = bstage == 0 ? p.stages - 1 : bstage - 1;
                            mbar_wait(&empty[ps], bstage == 0 ? bphase ^ 1u : bphase);
                            issue(ps, l - 1 + p.stages);
                        }
                        if (++bstage == p.stages) {
                            bstage = 0;
                            bphase ^= 1u;
                        }
                    }
                }
            }
        }
    }
    };
    if (store_mode == 0)
        sweep(std::integral_constant<int, 0>{});
    else if (store_mode == 1)
        sweep(std::integral_constant<int, 1>{});
    else
        sweep(std::integral_constant<int, 2>{});
}

}  // namespace stencil
