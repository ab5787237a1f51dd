// mbar_repro_c.cu -- mbar_repro_b.cu with the refilling thread chosen at compile time (-DWAITER=n):
// does synccheck still flag the empty-barrier wait when the waiter is not one of its arrivers?
// Minimal full/empty mbarrier ring fed by 1-D bulk copies (the in-plane kernel's
// pattern) to check whether compute-sanitizer synccheck flags it.
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void wait(uint64_t* b, uint32_t par) {
    uint32_t ok = 0;
    while (!ok) asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }" : "=r"(ok) : "r"(su32(b)), "r"(par) : "memory");
}
__global__ void k(const float* src, int* out, int S, int N) {
    extern __shared__ __align__(128) unsigned char sm[];
    uint64_t* full = (uint64_t*)sm;
    uint64_t* empty = full + S;
    float* ring = (float*)(sm + 128 * ((2 * S * 8 + 127) / 128));
    const int chunk = 4096;
    const int nw = blockDim.x / 32;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])) : "memory");
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&empty[s])), "r"(nw) : "memory");
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto issue = [&](int l) {
        const int s = l % S;
        asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&full[s])) : "memory");
    };
    if (threadIdx.x == WAITER) for (int l = 0; l < S; ++l) issue(l);
    __syncthreads();
    float acc = 0;
    int stage = 0; uint32_t phase = 0;
    for (int l = 0; l < N; ++l) {
        wait(&full[stage], phase);
        acc += ring[stage * chunk / 4 + threadIdx.x];
        __syncwarp();
        if ((threadIdx.x & 31) == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[stage])) : "memory");
        if (threadIdx.x == WAITER && l >= 1 && l - 1 + S < N) {
            const int ps = stage == 0 ? S - 1 : stage - 1;
            wait(&empty[ps], stage == 0 ? phase ^ 1u : phase);
            issue(l - 1 + S);
        }
        if (++stage == S) { stage = 0; phase ^= 1; }
    }
    if (acc == 1.2345f) out[0] = 1;
}
int main() {
    float* s; int* o;
    cudaMalloc(&s, 64 << 20); cudaMemset(s, 0, 64 << 20); cudaMalloc(&o, 64);
    const int S = 3;
    k<<<4, 128, 128 + S * 4096>>>(s, o, S, 20);
    printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
