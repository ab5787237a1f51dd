// membench.cu -- memory-pattern microbenchmarks for the sweep kernels (B200).
// Not part of the library: isolates the HBM ceiling of the in-plane kernel's
// access pattern (TMA full-slice box loads + 128-bit row stores) from its
// arithmetic.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17
//                     tools/membench.cu -o tools/membench -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <stdio.h>
#include <stdlib.h>

#include <vector>

#define CK(x)                                                                    \
    do {                                                                         \
        cudaError_t e = (x);                                                     \
        if (e != cudaSuccess) {                                                  \
            fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); \
            exit(1);                                                             \
        }                                                                        \
    } while (0)

__global__ void copy_kernel(const float4* __restrict__ a, float4* __restrict__ b, long long n) {
    long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    long long st = (long long)gridDim.x * blockDim.x;
    for (; i + 3 * st < n; i += 4 * st) {
        float4 v0 = a[i], v1 = a[i + st], v2 = a[i + 2 * st], v3 = a[i + 3 * st];
        b[i] = v0;
        b[i + st] = v1;
        b[i + 2 * st] = v2;
        b[i + 3 * st] = v3;
    }
    for (; i < n; i += st) b[i] = a[i];
}

// z-streaming copy with plain 128-bit loads: each CTA owns a W x H tile column
// and walks planes z0..z1 (the sweep's order), copying the tile centre.
__global__ void zstream_ldg(const float* __restrict__ in, float* __restrict__ out, int W, int H, int nz, long long pitch,
                            long long plane, int A, int R, int zsegs, int RY, int unroll) {
    const int tx = threadIdx.x, ty = threadIdx.y;
    const int seg = blockIdx.z;
    const int z0 = (int)((long long)seg * nz / zsegs), z1 = (int)((long long)(seg + 1) * nz / zsegs);
    const long long off = (long long)(blockIdx.y * H + ty * RY + R) * pitch + A + blockIdx.x * W + tx * 4;
    for (int z = z0; z < z1; z += 4) {
        float4 v[4][4];
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int jj = 0; jj < 4; ++jj)
                if (jj < RY && z + u < z1) v[u][jj] = *(const float4*)(in + (long long)(z + u + R) * plane + off + jj * pitch);
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int jj = 0; jj < 4; ++jj)
                if (jj < RY && z + u < z1) *(float4*)(out + (long long)(z + u + R) * plane + off + jj * pitch) = v[u][jj];
    }
}

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// TMA box stream: same geometry as the in-plane kernel.  mode 0: load + store
// centre; mode 1: load only (sum into a register); mode 2: store only.
template <int W, int HX>
__global__ void __launch_bounds__(256, 1) box_stream(const __grid_constant__ CUtensorMap tm, float* out, int nx, int ny,
                                                      int nz, long long pitch, long long plane, int A, int R, int zsegs,
                                                      int stages, int mode, int RY) {
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t* full = (uint64_t*)sm;
    uint64_t* empty = full + stages;
    const int SP = W + 2 * HX;
    const int H = blockDim.y * RY;
    const int stage_elems = ((SP * (H + 2 * R) * 4 + 127) / 128) * 32;
    float* ring = (float*)(sm + 128 * ((2 * stages * 8 + 127) / 128));
    const int tx = threadIdx.x, ty = threadIdx.y;
    const int nwarps = (blockDim.x * blockDim.y) / 32;
    const int lane = (ty * blockDim.x + tx) & 31;
    const int seg = blockIdx.z;
    const int z0 = (int)((long long)seg * nz / zsegs), z1 = (int)((long long)(seg + 1) * nz / zsegs);
    const int L = z1 - z0 + 2 * R;
    const bool leader = tx == 0 && ty == 0;
    const uint32_t box = SP * (H + 2 * R) * 4;
    const int bx0 = A - HX + blockIdx.x * W, by0 = blockIdx.y * H;
    if (leader) {
        for (int s = 0; s < stages; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&empty[s])), "r"(nwarps));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    auto issue = [&](int q, int s) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(box));
        asm volatile(
            "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(
                su32(ring + (size_t)s * stage_elems)),
            "l"((uint64_t)&tm), "r"(bx0), "r"(by0), "r"(z0 + q), "r"(su32(&full[s]))
            : "memory");
    };
    auto wait = [&](uint64_t* b, uint32_t ph) {
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                         : "=r"(ok)
                         : "r"(su32(b)), "r"(ph)
                         : "memory");
    };
    if (leader && mode != 2)
        for (int q = 0; q < stages && q < L; ++q) issue(q, q);
    float accum = 0.f;
    const int gx0 = blockIdx.x * W + tx * 4;
    int stage = 0;
    uint32_t phase = 0;
    for (int q = 0; q < L; ++q) {
        float4 v[8];
        if (mode != 2) {
            wait(&full[stage], phase);
            const float* sb = ring + (size_t)stage * stage_elems + (R + ty * RY) * SP + HX + tx * 4;
            for (int jj = 0; jj < RY; ++jj) v[jj] = *(const float4*)(sb + jj * SP);
        } else {
            for (int jj = 0; jj < RY; ++jj) v[jj] = make_float4(q, 0, 0, 0);
        }
        if (q >= 2 * R && mode != 1) {
            float* d = out + (long long)(z0 + q - 2 * R + R) * plane + (long long)(blockIdx.y * H + ty * RY + R) * pitch + A + gx0;
            for (int jj = 0; jj < RY; ++jj) *(float4*)(d + jj * pitch) = v[jj];
        } else {
            for (int jj = 0; jj < RY; ++jj) accum += v[jj].x + v[jj].w;
        }
        if (mode != 2) {
            __syncwarp();
            if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[stage])));
            if (leader && q >= 1 && q - 1 + stages < L) {
                int ps = stage == 0 ? stages - 1 : stage - 1;
                wait(&empty[ps], ((q - 1) / stages) & 1);
                issue(q - 1 + stages, ps);
            }
        }
        if (++stage == stages) { stage = 0; phase ^= 1; }
    }
    if (accum == 1234.5f) out[0] = accum;
}

int main(int argc, char** argv) {
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
    const double alg = 2.0 * 4.0 * n * n * (double)n;  // compulsory bytes of one sweep
    // 1. plain copy of the whole buffer
    {
        long long nv = elems / 4;
        for (int it = 0; it < 3; ++it) copy_kernel<<<148 * 8, 256>>>((float4*)a, (float4*)b, nv);
        cudaEventRecord(e0);
        for (int it = 0; it < 20; ++it) copy_kernel<<<148 * 8, 256>>>((float4*)a, (float4*)b, nv);
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        printf("copy (LDG/STG.128, %lld MB): %.1f GB/s\n", elems * 4 >> 20, 2.0 * elems * 4 / (ms / 20 * 1e-3) / 1e9);
    }
    // 2. TMA box streams
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult qr;
    CK(cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &fn, 12000, cudaEnableDefault, &qr));
    auto enc = (PFN_cuTensorMapEncodeTiled_v12000)fn;
    struct Cfg { int bx, ty, ry, stages, zsegs; };
    std::vector<Cfg> cfgs = {{32, 8, 4, 6, 2}, {32, 4, 4, 6, 3}, {32, 8, 2, 6, 4}, {32, 4, 2, 6, 5}, {32, 8, 4, 4, 1},
                             {32, 16, 1, 6, 4}, {32, 4, 1, 8, 4}};
    for (int mode = 0; mode < 3; ++mode)
        for (auto c : cfgs) {
            const int W = 128, HX = 4;
            const int H = c.ty * c.ry;
            CUtensorMap tm;
            cuuint64_t dims[3] = {(cuuint64_t)pitch, (cuuint64_t)rows, (cuuint64_t)planes};
            cuuint64_t str[2] = {(cuuint64_t)pitch * 4, (cuuint64_t)plane * 4};
            cuuint32_t box[3] = {(cuuint32_t)(W + 2 * HX), (cuuint32_t)(H + 2 * R), 1};
            cuuint32_t es[3] = {1, 1, 1};
            if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, a, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                    CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) !=
                CUDA_SUCCESS) {
                printf("encode failed\n");
                continue;
            }
            const int stage_elems = (((W + 2 * HX) * (H + 2 * R) * 4 + 127) / 128) * 32;
            size_t smem = 128 * ((2 * c.stages * 8 + 127) / 128) + (size_t)c.stages * stage_elems * 4;
            if (c.bx * c.ty > 256) continue;
            CK(cudaFuncSetAttribute(box_stream<128, 4>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            dim3 grid(n / W, n / H, c.zsegs), block(c.bx, c.ty);
            for (int it = 0; it < 3; ++it)
                box_stream<128, 4><<<grid, block, smem>>>(tm, b, n, n, n, pitch, plane, A, R, c.zsegs, c.stages, mode, c.ry);
            CK(cudaGetLastError());
            cudaEventRecord(e0);
            for (int it = 0; it < 20; ++it)
                box_stream<128, 4><<<grid, block, smem>>>(tm, b, n, n, n, pitch, plane, A, R, c.zsegs, c.stages, mode, c.ry);
            cudaEventRecord(e1);
            CK(cudaEventSynchronize(e1));
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            const double bytes = mode == 0 ? alg : alg / 2;
            printf("box stream mode=%d (%s) bx=%d ty=%d ry=%d stages=%d zsegs=%d ctas=%d: %.1f us, %.1f GB/s (compulsory)\n",
                   mode, mode == 0 ? "load+store" : mode == 1 ? "load only" : "store only", c.bx, c.ty, c.ry, c.stages,
                   c.zsegs, grid.x * grid.y * grid.z, ms / 20 * 1e3, bytes / (ms / 20 * 1e-3) / 1e9);
        }
    // 3. z-streaming with plain loads
    struct Z { int ty, ry, zsegs; };
    for (Z c : std::vector<Z>{{8, 4, 2}, {4, 4, 4}, {8, 2, 4}, {8, 4, 8}, {4, 2, 8}, {8, 1, 8}}) {
        const int W = 128, H = c.ty * c.ry;
        dim3 grid(n / W, n / H, c.zsegs), block(32, c.ty);
        for (int it = 0; it < 3; ++it)
            zstream_ldg<<<grid, block>>>(a, b, W, H, n, pitch, plane, A, R, c.zsegs, c.ry, 4);
        CK(cudaGetLastError());
        cudaEventRecord(e0);
        for (int it = 0; it < 20; ++it) zstream_ldg<<<grid, block>>>(a, b, W, H, n, pitch, plane, A, R, c.zsegs, c.ry, 4);
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        printf("zstream LDG ty=%d ry=%d zsegs=%d ctas=%d: %.1f us, %.1f GB/s\n", c.ty, c.ry, c.zsegs,
               grid.x * grid.y * grid.z, ms / 20 * 1e3, alg / (ms / 20 * 1e-3) / 1e9);
    }
    return 0;
}
