// Measurement aid (not part of libmsp): random 8-byte gathers from an x of
// `n` doubles, 4 per output (the C5 SpMV access pattern without the CSR
// stream) -- how many DRAM bytes one random gather costs on this GPU and how
// the load's cache operator changes it.
#include <cstdint>
#include <cuda_runtime.h>

__global__ void fill_idx(int *idx, int64_t m, uint32_t n, uint32_t seed)
{
    for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < m; i += int64_t(gridDim.x) * blockDim.x) {
        uint64_t z = uint64_t(i) * 0x9E3779B97F4A7C15ull + seed;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z ^= z >> 31;
        idx[i] = int(uint32_t(z % n));
    }
}

template <int MODE>
__device__ __forceinline__ double gld(const double *p)
{
    double v;
    if (MODE == 0) v = __ldg(p);
    else if (MODE == 1) v = __ldcg(p);
    else if (MODE == 2) asm volatile("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(v) : "l"(p));
    else if (MODE == 3) asm volatile("ld.global.nc.L2::64B.f64 %0, [%1];" : "=d"(v) : "l"(p));
    else asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(0ull));
    return v;
}

template <int MODE>
__global__ void __launch_bounds__(256) gather4(const int *__restrict__ idx, const double *__restrict__ x, double *y, int64_t m)
{
    for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < m; i += int64_t(gridDim.x) * blockDim.x) {
        const int4 c = __ldcs(reinterpret_cast<const int4 *>(idx) + i);
        y[i] = gld<MODE>(x + c.x) + gld<MODE>(x + c.y) + gld<MODE>(x + c.z) + gld<MODE>(x + c.w);
    }
}

extern "C" int probe_fill(int *idx, long long m, unsigned n, unsigned seed, void *s)
{
    fill_idx<<<148 * 8, 256, 0, (cudaStream_t)s>>>(idx, m, n, seed);
    return int(cudaGetLastError());
}

extern "C" int probe_gather(int mode, const int *idx, const double *x, double *y, long long m, int blocks, void *s)
{
    cudaStream_t st = (cudaStream_t)s;
    switch (mode) {
    case 0: gather4<0><<<blocks, 256, 0, st>>>(idx, x, y, m); break;
    case 1: gather4<1><<<blocks, 256, 0, st>>>(idx, x, y, m); break;
    case 2: gather4<2><<<blocks, 256, 0, st>>>(idx, x, y, m); break;
    case 3: gather4<3><<<blocks, 256, 0, st>>>(idx, x, y, m); break;
    default: gather4<4><<<blocks, 256, 0, st>>>(idx, x, y, m); break;
    }
    return int(cudaGetLastError());
}
