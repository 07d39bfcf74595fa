// Bandwidth probe (measurement aid, not part of libmsp): read-only streaming
// of a large buffer with (a) LDG.128 grid-stride loads and (b) a TMA bulk
// copy ring per CTA, to find what the SpMV producer design can reach.
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void ldg_sum(const int4 *__restrict__ a, int64_t n16, int unroll_dummy, unsigned long long *out)
{
    int acc = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (; i + 3 * stride < n16; i += 4 * stride) {
        int4 v0 = __ldcs(a + i), v1 = __ldcs(a + i + stride), v2 = __ldcs(a + i + 2 * stride), v3 = __ldcs(a + i + 3 * stride);
        acc ^= v0.x ^ v1.y ^ v2.z ^ v3.w;
    }
    for (; i < n16; i += stride) { int4 v = __ldcs(a + i); acc ^= v.x; }
    if (acc == 0x7fffffff) atomicAdd(out, 1ull);
}

// One producer thread, (blockDim-32) consumer threads that touch one word of
// each landed stage (so the wait is real), ST stages of `chunk` bytes.
__global__ void tma_stream(const char *__restrict__ a, int64_t bytes, int chunk, int ST, unsigned long long *out)
{
    extern __shared__ __align__(128) char sm[];
    uint64_t *full = (uint64_t *)(sm + (size_t)ST * chunk);
    uint64_t *empty = full + ST;
    const int64_t per = (bytes / gridDim.x) & ~int64_t(15);
    const char *base = a + per * blockIdx.x;
    const int nt = (int)(per / chunk);
    if (threadIdx.x == 0) {
        for (int s = 0; s < ST; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&empty[s])), "r"((int)(blockDim.x / 32 - 1)));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    const int warp = threadIdx.x / 32, lane = threadIdx.x & 31;
    int acc = 0;
    if (warp == 0) {
        if (lane == 0) {
            for (int t = 0; t < nt; ++t) {
                const int s = t % ST;
                if (t >= ST) {
                    uint32_t ok = 0, par = ((t / ST) - 1) & 1;
                    while (!ok) asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}" : "=r"(ok) : "r"(su32(&empty[s])), "r"(par) : "memory");
                }
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(chunk) : "memory");
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(su32(sm + (size_t)s * chunk)), "l"(base + (int64_t)t * chunk), "r"(chunk), "r"(su32(&full[s])) : "memory");
            }
        }
    } else {
        for (int t = 0; t < nt; ++t) {
            const int s = t % ST;
            uint32_t ok = 0, par = (t / ST) & 1;
            while (!ok) asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}" : "=r"(ok) : "r"(su32(&full[s])), "r"(par) : "memory");
            acc ^= ((const int *)(sm + (size_t)s * chunk))[(threadIdx.x * 97) % (chunk / 4)];
            __syncwarp();
            if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[s])) : "memory");
        }
    }
    if (acc == 0x7fffffff) atomicAdd(out, 1ull);
}

extern "C" int probe_ldg(const void *a, long long bytes, int blocks, int threads, void *out, void *stream)
{
    ldg_sum<<<blocks, threads, 0, (cudaStream_t)stream>>>((const int4 *)a, bytes / 16, 0, (unsigned long long *)out);
    return (int)cudaGetLastError();
}

extern "C" int probe_tma(const void *a, long long bytes, int blocks, int threads, int chunk, int ST, void *out, void *stream)
{
    const int smem = ST * chunk + 2 * ST * 8;
    cudaFuncSetAttribute(tma_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    tma_stream<<<blocks, threads, smem, (cudaStream_t)stream>>>((const char *)a, bytes, chunk, ST, (unsigned long long *)out);
    return (int)cudaGetLastError();
}
