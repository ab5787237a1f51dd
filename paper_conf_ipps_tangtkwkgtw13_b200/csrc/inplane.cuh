// inplane.cuh -- K-IP: the in-plane full-slice sweep with register tiling,
// written for sm_100a.
//
// Paper: in-plane method Sec. III-C, Eqs. (3)-(5),
// steps 1-6, full-slice loading (Fig. 6d), vector loads
// (P:L189-191), register tiling.
//
// One thread block owns a W x H xy tile (W = BX*RX, H = TY*RY) and sweeps one
// z segment [z0, z1) of it.  Every input value is read from the plane it
// lives in (the in-plane property, Fig. 5b), and every output is built by
// incremental updates as the planes stream past:
//   step 1  TMA loads the full slice (W+2HX) x (H+2r) of ZB consecutive planes
//           -- interior and halo as ONE 3-D box (HX = r rounded up to a
//           16-byte vector) -- into a stage of a shared-memory ring, S-1
//           loads ahead of use, completing on a "full" mbarrier; one elected
//           thread issues it after every warp has released the stage on its
//           "empty" mbarrier.  (On B200 a CTA keeps only ~4 TMA tensor loads
//           in flight, so the box depth ZB sets the bytes in flight, see
//           tools/membench3.cu and DESIGN.md section 5);
//   step 2  each thread loads its column block (RY+2r rows of its RX x-points,
//           128-bit loads at compile-time offsets) and x halos once per plane;
//   step 3  Eq. (5): c_m * in[k] is added to the queued outputs of planes
//           k-1..k-r; plane k-r is now complete and is stored (128-bit,
//           coalesced);
//   step 4  symmetric to Eq. (5) for the planes AHEAD: c_m * in[k] starts /
//           updates the outputs of planes k+r..k+1 (the "behind" terms of
//           Eq. (3) for those planes);
//   step 5  Eq. (3) in-plane terms of plane k: c0*in[k] and the x/y
//           neighbours from shared memory are added to the output of plane k.
// So the register queue holds 2r partial outputs per point (planes k-r+1 ..
// k+r), the same register budget as the paper's r partials + r cached behind
// values, but no value is ever copied between registers: the
// z loop is unrolled by 2r, and the slot of plane k-r, completed and stored
// in step 3, is re-initialised in place for plane k+r in step 4.  The per-point summation
// order is the fixed one of common.cuh (reading R7), shared with K-FP.
// fp32 arithmetic runs on the packed FP32x2 pipe instructions of sm_100
// (FADD2 / FFMA2 / FMUL2: two IEEE round-to-nearest operations each, so the
// order -- and the bits -- are unchanged).  Planes z0-r..z0-1 (warm-up) and
// z1..z1+r-1 (drain) are streamed so segments are independent; their outputs
// are never stored.
#pragma once

#include <type_traits>

#include "common.cuh"

// Experiment hooks (tools/ab.sh): compiled in only with -DSTENCIL_DEBUG_HOOKS.
#ifdef STENCIL_DEBUG_HOOKS
#define STENCIL_DBG(p) ((p).debug)
#else
#define STENCIL_DBG(p) 0
#endif

namespace stencil {

template <typename T, int R>
struct InplaceGeom {
    static constexpr int VEC = Vec<T>::N;                  // elements per 16-byte vector
    static constexpr int HX = ((R + VEC - 1) / VEC) * VEC;  // x halo, padded to a vector
    static constexpr int NVH = HX / VEC;                    // halo vectors per side
};

// Registers: 2r accumulators per point plus the column block (RY+2r rows),
// kept under the 255-register limit.
template <typename T, int R, int RXV, int RY, bool AX = false>
constexpr bool inplane_fits() {
    constexpr int w = (int)(sizeof(T) / 4);
    constexpr int pts = RXV * Vec<T>::N * RY;
    constexpr int words = (2 * R * pts + (RY + 2 * R) * RXV * Vec<T>::N + (AX ? 4 * R : 0)) * w;
    return words <= 176;
}

// ---------------------------------------------------------------------------
// Lane arithmetic: fp32 works on packed pairs of x-adjacent points held in
// 64-bit registers (FP32x2 instructions); fp64 on scalars.
// ---------------------------------------------------------------------------
template <typename T>
struct Lanes;

template <>
struct Lanes<float> {
    using L = unsigned long long;  // two floats: lo = even x, hi = odd x
    static constexpr int PER = 2;
    static __device__ __forceinline__ L add(L a, L b) {
        L r;
        asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
        return r;
    }
    static __device__ __forceinline__ L sub(L a, L b) {
        L r;
        asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
        return r;
    }
    static __device__ __forceinline__ L mul(L a, L b) {
        L r;
        asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
        return r;
    }
    static __device__ __forceinline__ L fma(L a, L b, L c) {
        L r;
        asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
        return r;
    }
    static __device__ __forceinline__ L make(float lo, float hi) {
        L r;
        asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
        return r;
    }
    static __device__ __forceinline__ float lo(L a) { return __uint_as_float((unsigned)(a & 0xffffffffull)); }
    static __device__ __forceinline__ float hi(L a) { return __uint_as_float((unsigned)(a >> 32)); }
    static __device__ __forceinline__ L bcast(float c) { return make(c, c); }
    // 16 bytes of shared memory -> two lanes
    static __device__ __forceinline__ void lds16(L* d, const float* s) {
#ifdef STENCIL_LDS_PLAIN
        const ulonglong2 v = *reinterpret_cast<const ulonglong2*>(s);
        d[0] = v.x;
        d[1] = v.y;
#else
        asm volatile("ld.shared.v2.u64 {%0, %1}, [%2];" : "=l"(d[0]), "=l"(d[1]) : "r"(smem_u32(s)));
#endif
    }
    // predicated 16-byte store (no branch).  STENCIL_STG64: as two 8-byte stores of the two lanes
    static __device__ __forceinline__ void stg16(float* g, const L* v, bool pred, uint64_t pol) {
#ifdef STENCIL_STG64
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\t@p st.global.L2::cache_hint.u64 [%0], %1, %4;\n\t"
            "@p st.global.L2::cache_hint.u64 [%0+8], %2, %4;\n\t}" ::"l"(g),
            "l"(v[0]), "l"(v[1]), "r"((int)pred), "l"(pol)
            : "memory");
#else
        asm volatile(
#ifdef STENCIL_STG_U64  // experiment hook: the round-2 form (two u64 operands)
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\t@p st.global.L2::cache_hint.v2.u64 [%0], {%1, %2}, %4;\n\t}" ::"l"(g),
            "l"(v[0]), "l"(v[1]), "r"((int)pred), "l"(pol)
            : "memory");
#else
            // four f32 operands, not two u64: ptxas then stores the FFMA2 result registers in place
            // (with u64 operands it copied most of them into fresh register pairs first)
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %5, 0;\n\t@p st.global.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %6;\n\t}" ::"l"(g),
            "f"(lo(v[0])), "f"(hi(v[0])), "f"(lo(v[1])), "f"(hi(v[1])), "r"((int)pred), "l"(pol)
            : "memory");
#endif
#endif
    }
    // one lane (two x-adjacent floats) -> 8 bytes of global memory
    static __device__ __forceinline__ void stg8(float* g, L v) {
        asm volatile("st.global.u64 [%0], %1;" ::"l"(g), "l"(v) : "memory");
    }
    static __device__ __forceinline__ float elem(const L* row, int i) { return (i & 1) ? hi(row[i >> 1]) : lo(row[i >> 1]); }
    // x-neighbour sum (x[a-m] + x[a+m]) for the lane starting at element a (even)
    static __device__ __forceinline__ L xsum(const L* row, int a, int m) {
        if ((m & 1) == 0) return add(row[(a - m) >> 1], row[(a + m) >> 1]);
        // odd offsets straddle lanes: two scalar round-to-nearest adds form one lane
        return make(__fadd_rn(elem(row, a - m), elem(row, a + m)), __fadd_rn(elem(row, a + 1 - m), elem(row, a + 1 + m)));
    }
    // x-neighbour difference (x[a+m] - x[a-m]) (first-derivative stencils, divgrad.cuh)
    static __device__ __forceinline__ L xdiff(const L* row, int a, int m) {
        if ((m & 1) == 0) return sub(row[(a + m) >> 1], row[(a - m) >> 1]);
        return make(__fsub_rn(elem(row, a + m), elem(row, a - m)), __fsub_rn(elem(row, a + 1 + m), elem(row, a + 1 - m)));
    }
};

template <>
struct Lanes<double> {
    using L = double;
    static constexpr int PER = 1;
    static __device__ __forceinline__ L add(L a, L b) { return __dadd_rn(a, b); }
    static __device__ __forceinline__ L sub(L a, L b) { return __dsub_rn(a, b); }
    static __device__ __forceinline__ L mul(L a, L b) { return __dmul_rn(a, b); }
    static __device__ __forceinline__ L fma(L a, L b, L c) { return __fma_rn(a, b, c); }
    static __device__ __forceinline__ L bcast(double c) { return c; }
    static __device__ __forceinline__ void lds16(L* d, const double* s) {
        double2 v = *reinterpret_cast<const double2*>(s);
        d[0] = v.x;
        d[1] = v.y;
    }
    static __device__ __forceinline__ void stg16(double* g, const L* v, bool pred, uint64_t pol) {
        asm volatile(
            "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\t@p st.global.L2::cache_hint.v2.f64 [%0], {%1, %2}, %4;\n\t}" ::"l"(g),
            "d"(v[0]), "d"(v[1]), "r"((int)pred), "l"(pol)
            : "memory");
    }
    static __device__ __forceinline__ void stg8(double* g, L v) {
        asm volatile("st.global.f64 [%0], %1;" ::"l"(g), "d"(v) : "memory");
    }
    static __device__ __forceinline__ double elem(const L* row, int i) { return row[i]; }
    static __device__ __forceinline__ L xsum(const L* row, int a, int m) { return add(row[a - m], row[a + m]); }
    static __device__ __forceinline__ L xdiff(const L* row, int a, int m) { return sub(row[a + m], row[a - m]); }
};

// SRC (application stencils with a second, centre-only input grid g, Table V
// "Poisson"-type 2 in -> 1 out, and the leapfrog wave step): the
// output is Eq. (1) on `in` plus p.d * g at the output point, added last
// (common.cuh order).  g arrives by TMA in the same ring stage as the in-plane
// box whose output plane it belongs to: box (W, H, ZB) at the output planes,
// completing on the same "full" barrier.
// AX (per-axis symmetric coefficients, reading R3b): c0 and c_{x,m},
// c_{y,m}, c_{z,m}: the in-plane terms fma(cx_m, x-pair) then fma(cy_m, y-pair),
// the z terms with cz_m (common.cuh order; the isotropic kernel is the same
// code with one c_m).
// PS (fused z-slab halo exchange): a multi-GPU slab plan
// whose neighbours' grids are mapped into this process (CUDA IPC over NVLink /
// NVSwitch).  Every completed output plane z < r is ALSO stored into the lower
// neighbour's grid (its halo plane nz_lo + z) and every plane z >= nz - r into
// the upper neighbour's (its halo plane z - nz), straight from the same
// registers, so the exchange rides on the sweep's own stores with no separate
// copy, kernel or NCCL call; stream-ordered flags (p2p.cu) order the sweeps.
template <typename T, int R, int BX, int RXV, int RY, bool SRC, bool AX = false, bool PS = false>
__global__ void __launch_bounds__(256, 1)
    inplane_sweep_kernel(const __grid_constant__ CUtensorMap tmap_in, const __grid_constant__ CUtensorMap tmap_g,
                         T* __restrict__ out, const SweepParams<T> p) {
    using G = InplaceGeom<T, R>;
    using A = Lanes<T>;
    using L = typename A::L;
    constexpr int VEC = G::VEC;
    constexpr int HX = G::HX;
    constexpr int NVH = G::NVH;
    constexpr int NX = RXV * VEC;        // points per thread along x
    constexpr int NL = NX / A::PER;      // lanes per thread-row
    constexpr int LV = VEC / A::PER;     // lanes per 16-byte vector
    constexpr int HL = HX / A::PER;      // lanes of x halo
    constexpr int W = BX * NX;           // tile width
    constexpr int SP = W + 2 * HX;       // smem row pitch (elements), compile time
    constexpr int NCOL = RY + 2 * R;     // rows of the column block
    constexpr int Q = 2 * R;             // accumulator slots (planes k-r+1 .. k+r)

    extern __shared__ __align__(128) unsigned char smem_raw[];
    uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw);   // S "full" mbarriers
    uint64_t* empty = full + p.stages;                          // S "empty" mbarriers
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
    const int pstride = SP * (H + 2 * R);  // elements per plane inside a stage
    const uint32_t box_bytes = p.stage_tx_bytes;  // in-plane box (+ g box when G) per stage
    const int bx0 = p.A - HX + tile_x * W;  // TMA box origin (element x, outer row, outer plane)
    // balanced y partition: tile t owns interior rows [t*ny/tiles_y, (t+1)*ny/tiles_y), at most H of them
    const int y0 = (int)(((long long)tile_y * p.ny) / p.tiles_y);
    const int y1 = (int)(((long long)(tile_y + 1) * p.ny) / p.tiles_y);
    const int by0 = y0;  // outer row of interior row y0 - R

    if (leader) {
        prefetch_tensormap(&tmap_in);
        if constexpr (SRC) prefetch_tensormap(&tmap_g);
        for (int s = 0; s < p.stages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], nwarps);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const uint64_t spol = l2_policy(p.store_policy), lpol = l2_policy(p.load_policy);
    // Stream order: dir = +1 streams planes z0-R .. z1+R-1 upward, dir = -1
    // streams z1+R-1 .. z0-R downward (stencil_run alternates so a sweep starts
    // where the previous one ended and finds its first inputs in L2).  Load l
    // brings ZB consecutive streamed planes as one TMA box; the box origin is
    // its lowest plane (outer index).
    const int ZB = p.zbox;
    const int dir = p.dir;
    const int nloads = (Lp + ZB - 1) / ZB;
    auto box_z = [&](int l) { return dir > 0 ? z0 + l * ZB : z1 + 2 * R - (l + 1) * ZB; };
    // g box of load l: the output planes of its streamed planes (R behind in stream order), x and y
    // at the tile's interior origin
    const int gbx0 = p.A + tile_x * W, gby0 = y0 + R;
    auto issue = [&](int slot, int l) {
        mbar_arrive_expect_tx(&full[slot], box_bytes);
        tma_load_3d_hint(ring + (size_t)slot * p.stage_elems, &tmap_in, bx0, by0, box_z(l), &full[slot], lpol);
        if constexpr (SRC)
            tma_load_3d_hint(ring + (size_t)slot * p.stage_elems + p.gstage_off, &tmap_g, gbx0, gby0,
                             box_z(l) - R * dir, &full[slot], lpol);
    };
    if (leader) {
        const int npre = nloads < p.stages ? nloads : p.stages;
        for (int l = 0; l < npre; ++l) issue(l, l);
    }

    // acc[s]: partial output of the plane whose index is congruent to s mod 2r
    L acc[Q][RY][NL];
#pragma unroll
    for (int a = 0; a < Q; ++a)
#pragma unroll
        for (int b = 0; b < RY; ++b)
#pragma unroll
            for (int e = 0; e < NL; ++e) acc[a][b][e] = A::bcast(T(0));
    L c[R + 1];  // c0, and c_m (isotropic) or cx_m (AX)
#pragma unroll
    for (int m = 0; m <= R; ++m) c[m] = A::bcast(p.c[m]);
    L cyv[AX ? R + 1 : 1], czv[AX ? R + 1 : 1];  // AX only: cy_m, cz_m
#pragma unroll
    for (int m = 0; m <= (AX ? R : 0); ++m) {
        cyv[m] = A::bcast(p.cy[m]);
        czv[m] = A::bcast(p.cz[m]);
    }
    // z-axis coefficient (steps 3 and 4)
    auto cz = [&](int m) -> L { if constexpr (AX) return czv[m]; else return c[m]; };
    const L dg = A::bcast(p.d);  // coefficient of the second grid (SRC only)

    // my column block starts at tile row ty*RY (= my first row - R), column HX + tx*NX
    const int my_off = (ty * RY) * SP + HX + tx * NX;
    const int gx0 = tile_x * W + tx * NX;
    const int gy0 = y0 + ty * RY;
    // whole-tile flags are uniform: interior tiles take the unpredicated store path
    // uniform per CTA: store mode 0 = every x-point and row valid (no checks), 1 = every x-point valid
    // (rows predicated), 2 = partial in x (element-wise checks)
    const bool x_full = (tile_x + 1) * W <= p.nx;
    const int store_mode = !x_full ? 2 : (y1 - y0 == H ? 0 : 1);
    // the first output (step q = 2R) is plane z0 (dir +1) or z1-1 (dir -1)
    T* dst = out + gidx<T, R>(p, gx0, gy0, dir > 0 ? z0 : z1 - 1);
    const long long dplane = dir > 0 ? p.plane : -p.plane;
    int zout = dir > 0 ? z0 : z1 - 1;  // interior plane of the next output (PS only)

    int stage = 0, zin = 0;  // ring stage and plane index inside it
    uint32_t phase = 0;      // parity of the current stage's full barrier
    int lcons = 0;           // loads consumed so far
    // three copies of the sweep loop, one per store mode: interior tiles store without any branch
    auto sweep = [&](auto mode_tag) {
    constexpr int MODE = decltype(mode_tag)::value;
    for (int q0 = 0; q0 < Lp; q0 += Q) {
#pragma unroll
        for (int u = 0; u < Q; ++u) {
            const int q = q0 + u;
            if (q < Lp) {
                if (zin == 0 && !(STENCIL_DBG(p) & 1)) mbar_wait(&full[stage], phase);
                const int zi = dir > 0 ? zin : ZB - 1 - zin;  // plane inside the stage
                const T* sb = ring + (size_t)stage * p.stage_elems + zi * pstride + my_off;
                // ---- step 2: column block (rows -R .. RY+R-1) and x halos
                L col[NCOL][NL];
#pragma unroll
                for (int rr = 0; rr < NCOL; ++rr)
#pragma unroll
                    for (int v = 0; v < RXV; ++v) A::lds16(&col[rr][v * LV], sb + rr * SP + v * VEC);
                const bool write = (q >= 2 * R);  // plane k-R is an output of this segment
                // ---- step 3: forward terms (Eq. 5) into planes k-1 .. k-R, arrival order; the last
                // term of plane k-R lands in fresh registers `fin` (stored below; step 4 re-initialises
                // the slot), which lets ptxas place them as the 128-bit store operands without moves
#pragma unroll
                for (int m = 1; m < R; ++m)
#pragma unroll
                    for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                        for (int e = 0; e < NL; ++e)
                            acc[(u - m + Q) % Q][jj][e] = A::fma(cz(m), col[R + jj][e], acc[(u - m + Q) % Q][jj][e]);
                L fin[RY][NL];
#pragma unroll
                for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                    for (int e = 0; e < NL; ++e) fin[jj][e] = A::fma(cz(R), col[R + jj][e], acc[(u + R) % Q][jj][e]);
                if constexpr (SRC) {
                    // + d * g at the output point, last in the fixed order (common.cuh)
                    const T* gb = ring + (size_t)stage * p.stage_elems + p.gstage_off + (zi * H + ty * RY) * W + tx * NX;
#pragma unroll
                    for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                        for (int v = 0; v < RXV; ++v) {
                            L gv[LV];
                            A::lds16(gv, gb + jj * W + v * VEC);
#pragma unroll
                            for (int e = 0; e < LV; ++e) fin[jj][v * LV + e] = A::fma(dg, gv[e], fin[jj][v * LV + e]);
                        }
                }
                // plane k-R (slot (u+R) mod 2R) is complete: one uniform store region per step
                if constexpr (MODE <= 1) {
                    // stores predicated on `write` (and the row, mode 1): no branch in the step
                    const bool wp = write && !(STENCIL_DBG(p) & 2);
#pragma unroll
                    for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                        for (int v = 0; v < RXV; ++v)
                            A::stg16(dst + (long long)jj * p.pitch + v * VEC, &fin[jj][v * LV],
                                     MODE == 0 ? wp : (wp && gy0 + jj < y1), spol);
                } else if (write) {
                    {
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
                            if (gy0 + jj < y1) {
#pragma unroll
                                for (int e = 0; e < NX; ++e)
                                    if (gx0 + e < p.nx) dst[(long long)jj * p.pitch + e] = A::elem(&fin[jj][0], e);
                            }
                    }
                }
                if constexpr (PS) {
                    // fused halo exchange: planes [0, r) -> lower neighbour, [nz - r, nz) -> upper; a
                    // slab of r <= nz < 2r planes sends some planes to both
#pragma unroll
                    for (int side = 0; side < 2; ++side) {
                    T* peer = nullptr;
                    if (side == 0 && write && zout < R && p.peer_lo) peer = p.peer_lo + ((dst - out) + p.lo_delta);
                    if (side == 1 && write && zout >= p.nz - R && p.peer_hi) peer = p.peer_hi + ((dst - out) + p.hi_delta);
                    if (peer) {
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
                            if (gy0 + jj < y1) {
                                if (MODE <= 1) {
#pragma unroll
                                    for (int v = 0; v < RXV; ++v)
                                        A::stg16(peer + (long long)jj * p.pitch + v * VEC, &fin[jj][v * LV], true, spol);
                                } else {
#pragma unroll
                                    for (int e = 0; e < NX; ++e)
                                        if (gx0 + e < p.nx) peer[(long long)jj * p.pitch + e] = A::elem(&fin[jj][0], e);
                                }
                            }
                    }
                    }
                    zout += write ? dir : 0;
                }
                // ---- step 4: behind terms for planes k+R .. k+1 (c_R first: fixed order)
#pragma unroll
                for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                    for (int e = 0; e < NL; ++e) acc[(u + R) % Q][jj][e] = A::mul(cz(R), col[R + jj][e]);
#pragma unroll
                for (int m = R - 1; m >= 1; --m)
#pragma unroll
                    for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                        for (int e = 0; e < NL; ++e)
                            acc[(u + m) % Q][jj][e] = A::fma(cz(m), col[R + jj][e], acc[(u + m) % Q][jj][e]);
                // ---- step 5: Eq. (3) in-plane terms of plane k, all rows interleaved
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
#pragma unroll
                for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                    for (int e = 0; e < NL; ++e) acc[u][jj][e] = A::fma(c[0], col[R + jj][e], acc[u][jj][e]);
#pragma unroll
                for (int m = 1; m <= R; ++m)
#pragma unroll
                    for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                        for (int e = 0; e < NL; ++e) {
                            const L xs = A::xsum(ext[jj], HX + e * A::PER, m);
                            const L ys = A::add(col[R + jj - m][e], col[R + jj + m][e]);
                            // x pair then y pair, each with its own FMA (common.cuh order): the
                            // same 4 FP instructions per m as fma(c_m, xs + ys), measured 0-3 %
                            // faster on B200 (tools/ab1.sh), and the per-axis variant is the
                            // same code with cy_m
                            acc[u][jj][e] = A::fma(c[m], xs, acc[u][jj][e]);
                            if constexpr (AX)
                                acc[u][jj][e] = A::fma(cyv[m], ys, acc[u][jj][e]);
                            else
                                acc[u][jj][e] = A::fma(c[m], ys, acc[u][jj][e]);
                        }
                dst += write ? dplane : 0;
                // after the last plane of a stage: release it (one arrival per warp) and refill the previous one
                if (++zin == ZB || q == Lp - 1) {
                    zin = 0;
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&empty[stage]);
                    const int l = lcons++;  // load just consumed
                    if (leader && l >= 1 && l - 1 + p.stages < nloads && !(STENCIL_DBG(p) & 1)) {
                        // the previous stage held load l-1: same ring round unless we just wrapped
                        const int ps = stage == 0 ? p.stages - 1 : stage - 1;
                        mbar_wait(&empty[ps], stage == 0 ? phase ^ 1u : phase);
                        issue(ps, l - 1 + p.stages);
                    }
                    if (++stage == p.stages) {
                        stage = 0;
                        phase ^= 1u;
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
