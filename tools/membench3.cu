// membench3.cu -- TMA streaming ceilings on B200: 1-D bulk copies of
// contiguous chunks vs 3-D boxes with short rows, load-only, persistent CTAs.
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

__device__ __forceinline__ void wait(uint64_t* b, uint32_t ph) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }"
                     : "=r"(ok)
                     : "r"(su32(b)), "r"(ph)
                     : "memory");
}

// Each CTA streams chunks [blockIdx.x + i*gridDim.x] of `chunk` bytes with a
// `stages`-deep ring of 1-D bulk copies; one thread issues, all consume 1 word.
__global__ void bulk1d(const char* __restrict__ src, long long nbytes, int chunk, int stages, float* sink) {
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t* full = (uint64_t*)sm;
    char* ring = (char*)(sm + 1024);
    const long long nchunks = nbytes / chunk;
    if (threadIdx.x == 0) {
        for (int s = 0; s < stages; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    auto issue = [&](long long c, int s) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(chunk));
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         su32(ring + (size_t)s * chunk)),
                     "l"(src + c * chunk), "r"(chunk), "r"(su32(&full[s]))
                     : "memory");
    };
    long long my = (nchunks - blockIdx.x + gridDim.x - 1) / gridDim.x;
    if (threadIdx.x == 0)
        for (int s = 0; s < stages && s < my; ++s) issue(blockIdx.x + (long long)s * gridDim.x, s);
    float acc = 0;
    int stage = 0;
    uint32_t ph = 0;
    for (long long i = 0; i < my; ++i) {
        wait(&full[stage], ph);
        acc += ((const float*)(ring + (size_t)stage * chunk))[threadIdx.x];
        __syncthreads();
        if (threadIdx.x == 0 && i + stages < my) issue(blockIdx.x + (i + stages) * gridDim.x, stage);
        if (++stage == stages) { stage = 0; ph ^= 1; }
    }
    if (acc == 12345.f) sink[0] = acc;
}

// 3-D boxes of (bw x bh x 1) tiling the whole (pitch x rows x planes) array,
// CTAs persistent over boxes in z-major order.
__global__ void box3d(const __grid_constant__ CUtensorMap tm, int bw, int bh, int nbx, int nby, int nplanes, int stages,
                      float* sink, int bd) {
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t* full = (uint64_t*)sm;
    float* ring = (float*)(sm + 1024);
    const int bytes = bw * bh * 4 * bd;
    const int stage_elems = ((bytes + 127) / 128) * 32;
    const long long nboxes = (long long)nbx * nby * (nplanes / bd);
    if (threadIdx.x == 0) {
        for (int s = 0; s < stages; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    auto issue = [&](long long b, int s) {
        const int x = (int)(b % nbx) * bw, y = (int)((b / nbx) % nby) * bh, z = (int)(b / ((long long)nbx * nby)) * bd;
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(bytes));
        asm volatile(
            "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
            "%4}], [%5];" ::"r"(su32(ring + (size_t)s * stage_elems)),
            "l"((uint64_t)&tm), "r"(x), "r"(y), "r"(z), "r"(su32(&full[s]))
            : "memory");
    };
    long long my = (nboxes - blockIdx.x + gridDim.x - 1) / gridDim.x;
    if (threadIdx.x == 0)
        for (int s = 0; s < stages && s < my; ++s) issue(blockIdx.x + (long long)s * gridDim.x, s);
    float acc = 0;
    int stage = 0;
    uint32_t ph = 0;
    for (long long i = 0; i < my; ++i) {
        wait(&full[stage], ph);
        acc += ring[(size_t)stage * stage_elems + threadIdx.x];
        __syncthreads();
        if (threadIdx.x == 0 && i + stages < my) issue(blockIdx.x + (i + stages) * gridDim.x, stage);
        if (++stage == stages) { stage = 0; ph ^= 1; }
    }
    if (acc == 12345.f) sink[0] = acc;
}

int main() {
    const long long nbytes = 1LL << 30;  // 1 GiB
    char* a;
    float* sink;
    CK(cudaMalloc(&a, nbytes));
    CK(cudaMalloc(&sink, 64));
    CK(cudaMemset(a, 0, nbytes));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    auto timeit = [&](auto launch, double bytes, const char* name) {
        for (int i = 0; i < 2; ++i) launch();
        CK(cudaGetLastError());
        cudaEventRecord(e0);
        for (int i = 0; i < 5; ++i) launch();
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        printf("%-60s %8.1f GB/s\n", name, bytes / (ms / 5 * 1e-3) / 1e9);
    };
    char name[256];
    for (int chunk : {8192})
        for (int stages : {2, 4, 6})
            for (int cps : {1, 2, 4}) {
                size_t smem = 1024 + (size_t)stages * chunk;
                if (smem * cps > 220 * 1024) continue;
                CK(cudaFuncSetAttribute(bulk1d, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                snprintf(name, sizeof name, "bulk1d chunk=%d stages=%d ctas/SM=%d (in flight/SM %d KB)", chunk, stages, cps,
                         (int)(chunk * stages * cps / 1024));
                timeit([&] { bulk1d<<<148 * cps, 256, smem>>>(a, nbytes, chunk, stages, sink); }, (double)nbytes, name);
            }
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult qr;
    CK(cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &fn, 12000, cudaEnableDefault, &qr));
    auto enc = (PFN_cuTensorMapEncodeTiled_v12000)fn;
    struct B { int bw, bh, bd, stages, cps; };
    const int pitch = 576, rows = 520;
    const int planes = (int)(nbytes / 4 / pitch / rows);
    for (B b : std::vector<B>{{128, 32, 1, 4, 1}, {128, 32, 1, 8, 1}, {128, 32, 2, 4, 1}, {128, 32, 3, 3, 1},
                              {128, 16, 1, 8, 1}, {128, 16, 2, 4, 1}, {128, 16, 4, 3, 1}, {128, 16, 2, 4, 2},
                              {128, 8, 1, 12, 1}, {128, 8, 4, 4, 1}, {136, 40, 1, 6, 1}, {136, 40, 2, 3, 1},
                              {136, 24, 2, 4, 1}, {136, 24, 3, 3, 1}, {136, 24, 2, 3, 2}}) {
        CUtensorMap tm;
        cuuint64_t dims[3] = {(cuuint64_t)pitch, (cuuint64_t)rows, (cuuint64_t)planes};
        cuuint64_t str[2] = {(cuuint64_t)pitch * 4, (cuuint64_t)pitch * rows * 4};
        cuuint32_t box[3] = {(cuuint32_t)b.bw, (cuuint32_t)b.bh, (cuuint32_t)b.bd};
        cuuint32_t es[3] = {1, 1, 1};
        if (enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, a, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) !=
            CUDA_SUCCESS) {
            printf("encode failed\n");
            continue;
        }
        const int bytes = b.bw * b.bh * 4 * b.bd;
        size_t smem = 1024 + (size_t)b.stages * (((bytes + 127) / 128) * 128);
        if (smem * b.cps > 227 * 1024) { printf("skip %dx%dx%d\n", b.bw, b.bh, b.bd); continue; }
        CK(cudaFuncSetAttribute(box3d, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        const int nbx = 512 / b.bw, nby = 512 / b.bh;
        snprintf(name, sizeof name, "box3d %dx%dx%d stages=%d ctas/SM=%d (in flight/SM %d KB)", b.bw, b.bh, b.bd, b.stages,
                 b.cps, bytes * b.stages * b.cps / 1024);
        timeit([&] { box3d<<<148 * b.cps, 256, smem>>>(tm, b.bw, b.bh, nbx, nby, planes, b.stages, sink, b.bd); },
               (double)nbx * b.bw * nby * b.bh * 4.0 * (planes / b.bd) * b.bd, name);
    }
    return 0;
}
