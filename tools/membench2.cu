// membench2.cu -- which way of staging plane tiles into shared memory streams
// HBM fastest on B200?  TMA 3-D boxes (L2 promotion / alignment variants) vs
// cp.async 16-byte copies vs LDG+STS, each with and without the 128-bit row
// stores of the sweep.  Geometry of the in-plane kernel at 512^3, r = 4.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <stdio.h>
#include <stdlib.h>

#include <vector>

#define CK(x)                                                                                  \
    do {                                                                                       \
        cudaError_t e = (x);                                                                   \
        if (e != cudaSuccess) {                                                                \
            fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e));          \
            exit(1);                                                                           \
        }                                                                                      \
    } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

struct P {
    long long pitch, plane;
    int A, R, nz, zsegs, stages, RY, H, W, HXL, HXR, mode;  // mode bit0: store, bit1: load
};

// staging method: 0 = TMA box, 1 = cp.async 16 B, 2 = LDG.128 -> STS.128
template <int METHOD>
__global__ void __launch_bounds__(256, 1) stream(const __grid_constant__ CUtensorMap tm, const float* __restrict__ in,
                                                  float* __restrict__ out, P p) {
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t* full = (uint64_t*)sm;
    uint64_t* empty = full + p.stages;
    const int SP = p.W + p.HXL + p.HXR;
    const int rowsb = p.H + 2 * p.R;
    const int stage_elems = ((SP * rowsb * 4 + 127) / 128) * 32;
    float* ring = (float*)(sm + 128 * ((2 * p.stages * 8 + 127) / 128));
    const int tx = threadIdx.x, ty = threadIdx.y, nthr = blockDim.x * blockDim.y, tid = ty * blockDim.x + tx;
    const int nwarps = nthr / 32, lane = tid & 31;
    const int seg = blockIdx.z;
    const int z0 = (int)((long long)seg * p.nz / p.zsegs), z1 = (int)((long long)(seg + 1) * p.nz / p.zsegs);
    const int L = z1 - z0 + 2 * p.R;
    const bool leader = tid == 0;
    const uint32_t box = SP * rowsb * 4;
    const int bx0 = p.A - p.HXL + blockIdx.x * p.W, by0 = blockIdx.y * p.H;
    const bool do_load = p.mode & 2, do_store = p.mode & 1;
    if (leader) {
        for (int s = 0; s < p.stages; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&empty[s])), "r"(nwarps));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    const int vec_per_row = SP / 4, nvec = vec_per_row * rowsb;
    auto issue = [&](int q, int s) {  // METHOD 0 only (leader)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(box));
        asm volatile(
            "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
            "%4}], [%5];" ::"r"(su32(ring + (size_t)s * stage_elems)),
            "l"((uint64_t)&tm), "r"(bx0), "r"(by0), "r"(z0 + q), "r"(su32(&full[s]))
            : "memory");
    };
    auto issue_thr = [&](int q, int s) {  // METHOD 1: all threads, cp.async 16 B
        const float* g = in + (long long)(z0 + q) * p.plane + (long long)by0 * p.pitch + bx0;
        float* d = ring + (size_t)s * stage_elems;
        for (int v = tid; v < nvec; v += nthr) {
            const int r = v / vec_per_row, c = (v % vec_per_row) * 4;
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(d + r * SP + c)), "l"(g + r * p.pitch + c)
                         : "memory");
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    auto wait = [&](uint64_t* b, uint32_t ph) {
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                         : "=r"(ok)
                         : "r"(su32(b)), "r"(ph)
                         : "memory");
    };
    if (do_load) {
        if (METHOD == 0 && leader)
            for (int q = 0; q < p.stages && q < L; ++q) issue(q, q);
        if (METHOD == 1)
            for (int q = 0; q < p.stages - 1; ++q) {
                if (q < L) issue_thr(q, q);
                else asm volatile("cp.async.commit_group;" ::: "memory");
            }
    }
    float accum = 0.f;
    const int gx0 = blockIdx.x * p.W + tx * 4;
    int stage = 0;
    uint32_t phase = 0;
    float4 v[8];
    for (int q = 0; q < L; ++q) {
        if (do_load) {
            if (METHOD == 0) {
                wait(&full[stage], phase);
            } else if (METHOD == 1) {
                asm volatile("cp.async.wait_group %0;" ::"n"(1) : "memory");
                __syncthreads();
            } else {
                // LDG.128 -> STS.128 of this plane, synchronous
                const float* g = in + (long long)(z0 + q) * p.plane + (long long)by0 * p.pitch + bx0;
                float* d = ring + (size_t)stage * stage_elems;
                float4 t[8];
                int n = 0;
                for (int vv = tid; vv < nvec; vv += nthr, ++n) {
                    const int r = vv / vec_per_row, c = (vv % vec_per_row) * 4;
                    t[n & 7] = __ldg((const float4*)(g + r * p.pitch + c));
                    if ((n & 7) == 7 || vv + nthr >= nvec)
                        for (int k = 0, vk = vv - (n & 7) * nthr; k <= (n & 7); ++k, vk += nthr) {
                            const int rk = vk / vec_per_row, ck = (vk % vec_per_row) * 4;
                            *(float4*)(d + rk * SP + ck) = t[k];
                        }
                }
                __syncthreads();
            }
            const float* sb = ring + (size_t)stage * stage_elems + (p.R + ty * p.RY) * SP + p.HXL + tx * 4;
            for (int jj = 0; jj < p.RY; ++jj) v[jj] = *(const float4*)(sb + jj * SP);
        } else {
            for (int jj = 0; jj < p.RY; ++jj) v[jj] = make_float4(q, 0, 0, 0);
        }
        if (q >= 2 * p.R && do_store) {
            float* d = out + (long long)(z0 + q - p.R) * p.plane + (long long)(by0 + ty * p.RY + p.R) * p.pitch + p.A + gx0;
            for (int jj = 0; jj < p.RY; ++jj) *(float4*)(d + jj * p.pitch) = v[jj];
        } else {
            for (int jj = 0; jj < p.RY; ++jj) accum += v[jj].x + v[jj].w;
        }
        if (do_load) {
            if (METHOD == 0) {
                __syncwarp();
                if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[stage])));
                if (leader && q >= 1 && q - 1 + p.stages < L) {
                    int ps = stage == 0 ? p.stages - 1 : stage - 1;
                    wait(&empty[ps], ((q - 1) / p.stages) & 1);
                    issue(q - 1 + p.stages, ps);
                }
            } else if (METHOD == 1) {
                __syncthreads();
                const int nq = q + p.stages - 1;
                if (nq < L) issue_thr(nq, nq % p.stages);
                else asm volatile("cp.async.commit_group;" ::: "memory");
            } else {
                __syncthreads();
            }
        }
        if (++stage == p.stages) {
            stage = 0;
            phase ^= 1;
        }
    }
    if (accum == 1234.5f) out[0] = accum;
}

int main() {
    const int n = 512, R = 4, A = 32;
    const long long pitch = 576, rows = n + 2 * R, planes = n + 2 * R;
    const long long plane = pitch * rows, elems = plane * planes;
    float *a, *b;
    CK(cudaMalloc(&a, elems * 4));
    CK(cudaMalloc(&b, elems * 4));
    CK(cudaMemset(a, 0, elems * 4));
    CK(cudaMemset(b, 0, elems * 4));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const double alg = 2.0 * 4.0 * n * n * (double)n;
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult qr;
    CK(cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &fn, 12000, cudaEnableDefault, &qr));
    auto enc = (PFN_cuTensorMapEncodeTiled_v12000)fn;
    struct V {
        const char* name;
        int method, hxl, hxr, promo;
    };
    std::vector<V> vs = {{"TMA halo4 promo128", 0, 4, 4, 1}, {"TMA halo0 promo128", 0, 0, 0, 1}};
    struct C { int ty, ry, stages, zsegs; };
    std::vector<C> cs = {{8, 4, 3, 2}, {8, 4, 6, 2}, {8, 4, 9, 2}, {8, 4, 6, 4}, {8, 2, 3, 4}, {8, 2, 6, 4}, {8, 2, 12, 4}, {4, 4, 6, 4}, {4, 4, 10, 4}};
    for (int mode : {2})
        for (auto vv : vs)
            for (auto c : cs) {
                const int W = 128, H = c.ty * c.ry;
                if (vv.hxl + vv.hxr + W > 256 && vv.method == 0) continue;
                CUtensorMap tm;
                cuuint64_t dims[3] = {(cuuint64_t)pitch, (cuuint64_t)rows, (cuuint64_t)planes};
                cuuint64_t str[2] = {(cuuint64_t)pitch * 4, (cuuint64_t)plane * 4};
                cuuint32_t box[3] = {(cuuint32_t)(W + vv.hxl + vv.hxr), (cuuint32_t)(H + 2 * R), 1};
                cuuint32_t es[3] = {1, 1, 1};
                CUtensorMapL2promotion pr = vv.promo == 2 ? CU_TENSOR_MAP_L2_PROMOTION_L2_256B
                                            : vv.promo == 1 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B
                                                            : CU_TENSOR_MAP_L2_PROMOTION_NONE;
                if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, a, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        CU_TENSOR_MAP_SWIZZLE_NONE, pr, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
                    printf("encode failed %s\n", vv.name);
                    continue;
                }
                P p{pitch, plane, A, R, n, c.zsegs, c.stages, c.ry, H, W, vv.hxl, vv.hxr, mode};
                const int SP = W + vv.hxl + vv.hxr;
                const int stage_elems = ((SP * (H + 2 * R) * 4 + 127) / 128) * 32;
                size_t smem = 128 * ((2 * c.stages * 8 + 127) / 128) + (size_t)c.stages * stage_elems * 4;
                dim3 grid(n / W, n / H, c.zsegs), block(32, c.ty);
                auto k = vv.method == 0 ? stream<0> : vv.method == 1 ? stream<1> : stream<2>;
                CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                for (int it = 0; it < 3; ++it) k<<<grid, block, smem>>>(tm, a, b, p);
                CK(cudaGetLastError());
                cudaEventRecord(e0);
                for (int it = 0; it < 20; ++it) k<<<grid, block, smem>>>(tm, a, b, p);
                cudaEventRecord(e1);
                CK(cudaEventSynchronize(e1));
                float ms;
                cudaEventElapsedTime(&ms, e0, e1);
                const double bytes = mode == 3 ? alg : alg / 2;
                printf("%-42s %-10s ty=%d ry=%d st=%d zs=%d: %7.1f us %7.1f GB/s\n", vv.name,
                       mode == 3 ? "load+store" : "load", c.ty, c.ry, c.stages, c.zsegs, ms / 20 * 1e3,
                       bytes / (ms / 20 * 1e-3) / 1e9);
            }
    return 0;
}
