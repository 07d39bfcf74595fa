// Measurement aid (not part of libmsp): TMA bulk-copy ring whose consumers
// hold every landed stage for `hold` SM cycles before releasing it -- the
// bandwidth a streaming kernel gets as a function of the time its consumers
// keep a stage (bytes in flight per SM = (STAGES - held) * chunk).
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void tma_hold(const char *__restrict__ a, int64_t bytes, int chunk, int ST, int hold, unsigned long long *out)
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
            const long long t0 = clock64();
            while (clock64() - t0 < hold) {}
            __syncwarp();
            if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[s])) : "memory");
        }
    }
    if (acc == 0x7fffffff) atomicAdd(out, 1ull);
}

extern "C" int probe_hold(const void *a, long long bytes, int blocks, int threads, int chunk, int ST, int hold, void *out,
                          void *stream)
{
    const int smem = ST * chunk + 2 * ST * 8;
    cudaFuncSetAttribute(tma_hold, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    tma_hold<<<blocks, threads, smem, (cudaStream_t)stream>>>((const char *)a, bytes, chunk, ST, hold,
                                                             (unsigned long long *)out);
    return (int)cudaGetLastError();
}
