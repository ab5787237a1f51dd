// inplane_ws.cuh -- K-IP/WS: the in-plane sweep (Sec. III-C, Eqs. 3-5,
// P:L136-173) in a warp-specialized B200 form.
//
// Same method, same per-point arithmetic order (common.cuh, reading R7) and
// the same register queue as inplane.cuh -- so both kernels are bit-identical --
// but the data movement is taken off the compute warps:
//   * a producer warp (first warp of the CTA's last warpgroup) is the only
//     issuer of the full-slice TMA loads (step 1): it waits on the ring's
//     "empty" mbarriers and re-arms the "full" ones; compute warps never block
//     on a refill.  The producer warpgroup gives its registers to the compute
//     warps (setmaxnreg: 24 vs 240 per thread);
//   * the completed plane k-r leaves as 8- or 16-byte global stores taken straight
//     from the FFMA2 result register pairs (no operand moves), addressed from
//     one plane pointer advanced once per plane; tiles inside the interior store with
//     no checks, only ragged edge tiles take a predicated element path (one
//     uniform branch per plane);
//   * the planes per TMA box (ZB) are a template parameter, so every
//     shared-memory address in the unrolled loop is a compile-time offset;
// Rows of a balanced y tile beyond its partition (y >= y1) are computed and
// stored with the same values the next tile stores (identical per-point
// order).  (A TMA tensor store of each warp's rows was tried first: the
// generic-to-async proxy fence it needs before every store costs a
// MEMBAR.ALL.CTA per plane per warp.)
#pragma once

#include "inplane.cuh"

// Experiment hook (tools/variants): -DSTENCIL_STG_NOCLOBBER drops the "memory" clobber of the
// output stores, which lets the compiler hoist shared-memory loads above them.
#ifdef STENCIL_STG_NOCLOBBER
#define STENCIL_STG_CLOBBER
#else
#define STENCIL_STG_CLOBBER : "memory"
#endif

namespace stencil {

#ifdef STENCIL_TIMESTAMPS
// Experiment hook (tools/ts_gaps.py): every CTA of every launch records its start / end %globaltimer into a
// device ring (slot = arrival order), read by stencil_dbg_timestamps.  Built into A/B variants only, and
// only in ONE translation unit (the reader below is an extern "C" definition; tools/variant_lib.py).
static __device__ unsigned long long g_ts[4 * 32768];
static __device__ unsigned g_ts_n;
__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#endif

__host__ __device__ constexpr int ws_gcd(int a, int b) { return b == 0 ? a : ws_gcd(b, a % b); }

// predicated scalar store (ragged edge tiles of the warp-specialized kernel)
__device__ __forceinline__ void stg_if(float* g, float v, bool pred) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %2, 0;\n\t@p st.global.f32 [%0], %1;\n\t}" ::"l"(g), "f"(v),
                 "r"((int)pred)
                 STENCIL_STG_CLOBBER);
}
__device__ __forceinline__ void stg_if(double* g, double v, bool pred) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %2, 0;\n\t@p st.global.f64 [%0], %1;\n\t}" ::"l"(g), "d"(v),
                 "r"((int)pred)
                 STENCIL_STG_CLOBBER);
}

// The two lanes go out as a v2.f32 pair: ptxas then stores the FFMA2 result registers in place
// (as one u64 operand it copied most of them into fresh register pairs first: 1.4 MOV per point)
__device__ __forceinline__ void stg8_if(float* g, unsigned long long v, bool pred) {
#ifdef STENCIL_STG_U64  // experiment hook: the round-2 form (one u64 operand)
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %2, 0;\n\t@p st.global.u64 [%0], %1;\n\t}" ::"l"(g), "l"(v),
                 "r"((int)pred)
                 STENCIL_STG_CLOBBER);
    return;
#endif
    const float lo = __uint_as_float((unsigned)(v & 0xffffffffull)), hi = __uint_as_float((unsigned)(v >> 32));
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\t@p st.global.v2.f32 [%0], {%1, %2};\n\t}" ::"l"(g),
                 "f"(lo), "f"(hi), "r"((int)pred)
                 STENCIL_STG_CLOBBER);
}
__device__ __forceinline__ void stg8_if(double* g, double v, bool pred) { stg_if(g, v, pred); }
// the same with an L2 eviction-priority hint (createpolicy descriptor, SweepParams::store_policy)
__device__ __forceinline__ void stg8_if(float* g, unsigned long long v, bool pred, uint64_t pol) {
#ifdef STENCIL_STG_U64
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %2, 0;\n\t@p st.global.L2::cache_hint.u64 [%0], %1, %3;\n\t}" ::"l"(g),
        "l"(v), "r"((int)pred), "l"(pol)
        STENCIL_STG_CLOBBER);
    return;
#endif
    const float lo = __uint_as_float((unsigned)(v & 0xffffffffull)), hi = __uint_as_float((unsigned)(v >> 32));
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\t@p st.global.L2::cache_hint.v2.f32 [%0], {%1, %2}, %4;\n\t}" ::"l"(g),
        "f"(lo), "f"(hi), "r"((int)pred), "l"(pol)
        STENCIL_STG_CLOBBER);
}
__device__ __forceinline__ void stg8_if(double* g, double v, bool pred, uint64_t pol) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %2, 0;\n\t@p st.global.L2::cache_hint.f64 [%0], %1, %3;\n\t}" ::"l"(g),
        "d"(v), "r"((int)pred), "l"(pol)
        STENCIL_STG_CLOBBER);
}

// 16-byte predicated store of two lanes (f32: two FFMA2 result pairs as v4.f32; f64: two doubles as v2.f64):
// one store instruction per 16-byte vector, and a warp's row of vectors is one contiguous span, which halves
// the L1 data-pipe wavefronts the output stores take against two 8-byte stores 16 bytes apart per lane
__device__ __forceinline__ void stg16_if(float* g, unsigned long long a, unsigned long long b, bool pred, uint64_t pol) {
    const float a0 = __uint_as_float((unsigned)(a & 0xffffffffull)), a1 = __uint_as_float((unsigned)(a >> 32));
    const float b0 = __uint_as_float((unsigned)(b & 0xffffffffull)), b1 = __uint_as_float((unsigned)(b >> 32));
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %5, 0;\n\t@p st.global.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %6;\n\t}" ::"l"(g),
        "f"(a0), "f"(a1), "f"(b0), "f"(b1), "r"((int)pred), "l"(pol)
        STENCIL_STG_CLOBBER);
}
__device__ __forceinline__ void stg16_if(double* g, double a, double b, bool pred, uint64_t pol) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\t@p st.global.L2::cache_hint.v2.f64 [%0], {%1, %2}, %4;\n\t}" ::"l"(g),
        "d"(a), "d"(b), "r"((int)pred), "l"(pol)
        STENCIL_STG_CLOBBER);
}

// PS (fused z-slab halo exchange, as inplane.cuh): completed output planes z < r are also stored into the
// lower neighbour's grid and planes z >= nz - r into the upper one's, from the same registers.  Only the
// blocks of U steps whose outputs can be such planes (q < 3r, q >= Lp - r) carry the peer stores: the
// middle of the sweep runs the plain body.
template <typename T, int R, int BX, int RXV, int RY, int ZB, bool SRC, bool AX, bool PS = false>
__global__ void __launch_bounds__(384, 1)
    inplane_ws_kernel(const __grid_constant__ CUtensorMap tmap_in, const __grid_constant__ CUtensorMap tmap_g,
                      T* __restrict__ out, const SweepParams<T> p) {
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
    constexpr int SP = W + 2 * HX;
    constexpr int NCOL = RY + 2 * R;
    constexpr int Q = 2 * R;
    constexpr int U = Q / ws_gcd(Q, ZB) * ZB;
    // Output store width (measured, profiles/r2c/stg16_*): one 16-byte store per vector is faster for fp64 and
    // for r >= 5 (3-4 %), two 8-byte lane stores for fp32 r <= 4 (8 %: with 16-byte stores the sweep read more
    // from DRAM and ran slower at a higher clock)
#if defined(STENCIL_STG8)
    constexpr bool STG16 = false;
#elif defined(STENCIL_STG16)
    constexpr bool STG16 = true;
#else
    constexpr bool STG16 = sizeof(T) == 8 || R >= 5;
#endif  // lcm(2r, ZB): slots, stage planes and (2r even) out buffers fixed

    extern __shared__ __align__(128) unsigned char smem_raw[];
    const int S = p.stages;
    uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw);
    uint64_t* empty = full + S;
    T* ring = reinterpret_cast<T*>(smem_raw + 128 * ((2 * S * 8 + 127) / 128));
    const int ncw = p.ws_warps;             // compute warps (tx*ty/32)
    const int pw = (ncw + 3) & ~3;          // first warp of the producer warpgroup

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int H = (ncw * 32 / BX) * RY;
    const int tile_x = blockIdx.x, tile_y = blockIdx.y;
    const int seg = p.seg_base + blockIdx.z * p.seg_stride;
    const int z0 = (int)(((long long)seg * p.nz) / p.zsegs);
    const int z1 = (int)(((long long)(seg + 1) * p.nz) / p.zsegs);
    const int Lp = (z1 - z0) + 2 * R;
    const int pstride = SP * (H + 2 * R);
    const int y0 = (int)(((long long)tile_y * p.ny) / p.tiles_y);
    const int dir = p.dir;
    const int nloads = (Lp + ZB - 1) / ZB;

#ifdef STENCIL_TIMESTAMPS
    unsigned long long ts0 = 0;
    unsigned ts_slot = 0;
    if (threadIdx.x == 0) {
        ts0 = gtimer();
        ts_slot = atomicAdd(&g_ts_n, 1u) & 32767u;
    }
#endif
    if (threadIdx.x == 0) {
        prefetch_tensormap(&tmap_in);
        if constexpr (SRC) prefetch_tensormap(&tmap_g);
        for (int s = 0; s < S; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], ncw);
        }
        fence_mbar_init();
    }
    __syncthreads();

    // ------------------------------------------------------------ producer warp
    // Registers go where the arithmetic is.  The block is the compute warpgroups plus one producer
    // warpgroup (setmaxnreg works per warpgroup), launched at 168 registers per thread; the producer
    // warpgroup drops to 24 and the compute warps grow to 240 (8 x 240 + 4 x 24 = 12 x 168).
    if (warp >= pw) {
        asm volatile("setmaxnreg.dec.sync.aligned.u32 24;\n" ::: "memory");
        if (warp == pw && lane == 0) {
            const uint64_t lpol = l2_policy(p.load_policy);
            const int bx0 = p.A - HX + tile_x * W;
            const int gbx0 = p.A + tile_x * W, gby0 = y0 + R;
            for (int l = 0, slot = 0, ph = 0; l < nloads; ++l) {
                if (l >= S) mbar_wait_sleep(&empty[slot], ph ^ 1u);
                const int bz = dir > 0 ? z0 + l * ZB : z1 + 2 * R - (l + 1) * ZB;
                mbar_arrive_expect_tx(&full[slot], p.stage_tx_bytes);
                tma_load_3d_hint(ring + (size_t)slot * p.stage_elems, &tmap_in, bx0, y0, bz, &full[slot], lpol);
                if constexpr (SRC)
                    tma_load_3d_hint(ring + (size_t)slot * p.stage_elems + p.gstage_off, &tmap_g, gbx0, gby0,
                                     bz - R * dir, &full[slot], lpol);
                if (++slot == S) {
                    slot = 0;
                    ph ^= 1u;
                }
            }
        }
        return;
    }

    // ------------------------------------------------------------ compute warps
    asm volatile("setmaxnreg.inc.sync.aligned.u32 240;\n" ::: "memory");
    if (warp >= ncw) return;  // padding warps of the last compute warpgroup
    const int tx = threadIdx.x % BX, ty = threadIdx.x / BX;
    L acc[Q][RY][NL];
#pragma unroll
    for (int a = 0; a < Q; ++a)
#pragma unroll
        for (int b = 0; b < RY; ++b)
#pragma unroll
            for (int e = 0; e < NL; ++e) acc[a][b][e] = A::bcast(T(0));
    L c[R + 1];
#pragma unroll
    for (int m = 0; m <= R; ++m) c[m] = A::bcast(p.c[m]);
    L cyv[AX ? R + 1 : 1], czv[AX ? R + 1 : 1];
#pragma unroll
    for (int m = 0; m <= (AX ? R : 0); ++m) {
        cyv[m] = A::bcast(p.cy[m]);
        czv[m] = A::bcast(p.cz[m]);
    }
    auto cz = [&](int m) -> L { if constexpr (AX) return czv[m]; else return c[m]; };
    const L dg = A::bcast(p.d);

    const int my_off = (ty * RY) * SP + HX + tx * NX;
    const int gx0 = tile_x * W + tx * NX;   // my first interior point
    const int gy0 = y0 + ty * RY;
    // whole tile inside the interior (uniform per CTA): unchecked stores.  Rows of a balanced
    // y tile past its partition (y >= y1) hold the values the next tile writes too (same order)
    const bool fast = (tile_x + 1) * W <= p.nx && y0 + H <= p.ny;
    T* dst = out + gidx<T, R>(p, gx0, gy0, dir > 0 ? z0 : z1 - 1);
    const long long dplane = dir > 0 ? p.plane : -p.plane;
    const uint64_t spol = l2_policy(p.store_policy);
    const int poff0 = dir > 0 ? 0 : (ZB - 1) * pstride;
    const int pdel = dir > 0 ? pstride : -pstride;

    int slot = 0;
    uint32_t phase = 0;
    const T* stage = ring;
    // two copies of the loop: interior tiles (FAST) store without checks, edge tiles element-wise.
    // The step body has no branch besides the ring waits: a branch inside the unrolled loop splits
    // it into blocks the scheduler cannot interleave, which costs more than the work it would skip
    // (measured: skipping the warm-up / drain steps this way made the sweep 3-30 % slower)
    // CHECKED: steps past the segment's last plane are skipped (the tail block); the main blocks of
    // U steps run without that test, so the unrolled steps form one block the scheduler interleaves
    int q0 = 0;
    // PEER: this copy of the body also issues the fused halo-exchange stores (PS only); q0 runs up to
    // `qend` (unchecked copies: whole blocks of U steps ending at or before it)
    auto sweep = [&](auto fast_tag, auto checked_tag, auto peer_tag, int qend) {
        constexpr bool FAST = decltype(fast_tag)::value;
        constexpr bool CHECKED = decltype(checked_tag)::value;
        constexpr bool PEER = decltype(peer_tag)::value;
        for (; CHECKED ? q0 < qend : q0 + U <= qend; q0 += U) {
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int q = q0 + u;
                if (!CHECKED || q < Lp) {
                    const int zs = u % ZB;  // plane of the current load (compile time)
                    if (zs == 0) mbar_wait(&full[slot], phase);
                    const T* sb = stage + poff0 + zs * pdel + my_off;
                    const bool write = q >= 2 * R;  // plane k-R is an output of this segment
                    L col[NCOL][NL];
#pragma unroll
                    for (int rr = 0; rr < NCOL; ++rr)
#pragma unroll
                        for (int v = 0; v < RXV; ++v) A::lds16(&col[rr][v * LV], sb + rr * SP + v * VEC);
                    // ---- step 3 (Eq. 5): forward terms into planes k-1 .. k-R; plane k-R completes
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
                        const int zi = dir > 0 ? zs : ZB - 1 - zs;
                        const T* gb = stage + p.gstage_off + (zi * H + ty * RY) * W + tx * NX;
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
                    // plane k-R: 8- / 16-byte stores straight from the FFMA2 result pairs (no operand moves),
                    // predicated on `write`; row addresses are formed from the plane base every step
                    // (a store reads its address register late, so its pointer is not bumped in place)
#pragma unroll
                    for (int jj = 0; jj < RY; ++jj) {
                        if constexpr (FAST) {
                            if constexpr (STG16) {
#pragma unroll
                                for (int v = 0; v < RXV; ++v)
                                    stg16_if(dst + jj * p.pitch + v * VEC, fin[jj][v * LV], fin[jj][v * LV + 1], write, spol);
                            } else {
#pragma unroll
                                for (int e = 0; e < NL; ++e) stg8_if(dst + jj * p.pitch + e * A::PER, fin[jj][e], write, spol);
                            }
                        } else {
#pragma unroll
                            for (int e = 0; e < NX; ++e)
                                stg_if(dst + jj * p.pitch + e, A::elem(&fin[jj][0], e),
                                       write && gy0 + jj < p.ny && gx0 + e < p.nx);
                        }
                    }
                    if constexpr (PEER) {
                        // interior plane of this output; planes [0, r) -> lower neighbour, [nz - r, nz) ->
                        // upper (a slab of r <= nz < 2r sends some planes to both)
                        const int zout = dir > 0 ? z0 + (q - 2 * R) : z1 - 1 - (q - 2 * R);
#pragma unroll
                        for (int side = 0; side < 2; ++side) {
                            T* peer = nullptr;
                            if (side == 0 && write && zout < R && p.peer_lo) peer = p.peer_lo + ((dst - out) + p.lo_delta);
                            if (side == 1 && write && zout >= p.nz - R && p.peer_hi)
                                peer = p.peer_hi + ((dst - out) + p.hi_delta);
                            if (peer) {
#pragma unroll
                                for (int jj = 0; jj < RY; ++jj) {
                                    if constexpr (FAST && STG16) {
#pragma unroll
                                        for (int v = 0; v < RXV; ++v)
                                            stg16_if(peer + jj * p.pitch + v * VEC, fin[jj][v * LV], fin[jj][v * LV + 1], true, spol);
                                    } else if constexpr (FAST) {
#pragma unroll
                                        for (int e = 0; e < NL; ++e) stg8_if(peer + jj * p.pitch + e * A::PER, fin[jj][e], true);
                                    } else {
#pragma unroll
                                        for (int e = 0; e < NX; ++e)
                                            stg_if(peer + jj * p.pitch + e, A::elem(&fin[jj][0], e),
                                                   gy0 + jj < p.ny && gx0 + e < p.nx);
                                    }
                                }
                            }
                        }
                    }
                    dst += write ? dplane : 0;
                    // ---- step 5: Eq. (3) in-plane terms of plane k
                    L ext[RY][NL + 2 * HL];
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
                        for (int e = 0; e < NL; ++e) acc[u % Q][jj][e] = A::fma(c[0], col[R + jj][e], acc[u % Q][jj][e]);
#pragma unroll
                    for (int m = 1; m <= R; ++m)
#pragma unroll
                        for (int jj = 0; jj < RY; ++jj)
#pragma unroll
                            for (int e = 0; e < NL; ++e) {
                                const L xs = A::xsum(ext[jj], HX + e * A::PER, m);
                                const L ys = A::add(col[R + jj - m][e], col[R + jj + m][e]);
                                acc[u % Q][jj][e] = A::fma(c[m], xs, acc[u % Q][jj][e]);
                                if constexpr (AX)
                                    acc[u % Q][jj][e] = A::fma(cyv[m], ys, acc[u % Q][jj][e]);
                                else
                                    acc[u % Q][jj][e] = A::fma(c[m], ys, acc[u % Q][jj][e]);
                            }
                    // ---- step 4: behind terms for planes k+R .. k+1 (c_R first).  Issued after
                    // step 5 (other accumulators, so the per-point order is unchanged): the slot it
                    // re-initialises held plane k-R, whose stores must first read their registers
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
                    // last plane of the load: release the stage (one arrival per warp).  A load the
                    // segment ends inside is never refilled, so it needs no release
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
    using yes = std::integral_constant<bool, true>;
    using no = std::integral_constant<bool, false>;
#ifdef STENCIL_TIMESTAMPS
    struct TsGuard {
        unsigned long long t0;
        unsigned slot;
        bool on;
        __device__ ~TsGuard() {
            if (on) {
                unsigned smid;
                asm volatile("mov.u32 %0, %smid;" : "=r"(smid));
                g_ts[4 * slot] = t0;
                g_ts[4 * slot + 1] = gtimer();
                g_ts[4 * slot + 2] = blockIdx.x + 1000ull * blockIdx.y + 1000000ull * blockIdx.z;
                g_ts[4 * slot + 3] = smid;
            }
        }
    } ts_guard{ts0, ts_slot, threadIdx.x == 0};
#endif
    if constexpr (PS) {
        // head blocks (outputs q - 2r < r) and tail blocks (q >= Lp - r) with the peer stores, the middle
        // without; every block runs exactly once, in order
        if (fast) {
            sweep(yes{}, no{}, yes{}, 3 * R + U - 1 < Lp ? 3 * R + U - 1 : Lp);
            sweep(yes{}, no{}, no{}, Lp - R);
            sweep(yes{}, yes{}, yes{}, Lp);
        } else {
            sweep(no{}, yes{}, yes{}, Lp);
        }
    } else {
        if (fast) {
            sweep(yes{}, no{}, no{}, Lp);
            sweep(yes{}, yes{}, no{}, Lp);
        } else {
            sweep(no{}, yes{}, no{}, Lp);
        }
    }
}

}  // namespace stencil

#ifdef STENCIL_TIMESTAMPS
// copies the ring and its arrival count to the host and resets the count (experiments only)
extern "C" int stencil_dbg_timestamps(unsigned long long* host, unsigned* count) {
    if (cudaMemcpyFromSymbol(count, stencil::g_ts_n, sizeof(unsigned)) != cudaSuccess) return -1;
    if (cudaMemcpyFromSymbol(host, stencil::g_ts, sizeof(stencil::g_ts)) != cudaSuccess) return -1;
    const unsigned z = 0;
    return cudaMemcpyToSymbol(stencil::g_ts_n, &z, sizeof(unsigned)) == cudaSuccess ? 0 : -1;
}
#endif
