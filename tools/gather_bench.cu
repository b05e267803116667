// Microbenchmark: the random-gather ceiling of the hook phase on a given graph.
// For every CSR entry (v, u) with u < v, load parent[u] (one random 4-byte gather per
// hooked edge, exactly the first hop of find_repres) and accumulate; no hooking.
// Variants: hint 0 = plain loads, 1 = nlist/src streamed with L2::evict_first and
// parent with L2::evict_last cache policies.
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ int ld_first(const int *p, unsigned long long pol)
{
    int v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;"
                 : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int ld_last(const int *p, unsigned long long pol)
{
    int v;
    asm volatile("ld.global.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}

template <int HINT, int U>
__global__ void __launch_bounds__(256) gather_kernel(long long m, const int *__restrict__ src,
                                                     const int *__restrict__ nlist,
                                                     const int *parent,
                                                     unsigned long long *out)
{
    unsigned long long pf = 0, pl = 0;
    if (HINT) {
        asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pf));
        asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pl));
    }
    unsigned long long acc = 0;
    const long long stride = (long long)gridDim.x * blockDim.x * U;
    for (long long e0 = (long long)blockIdx.x * blockDim.x * U + threadIdx.x; e0 < m; e0 += stride) {
        int u[U], v[U], p[U];
#pragma unroll
        for (int j = 0; j < U; j++) {
            const long long e = e0 + (long long)j * blockDim.x;
            u[j] = 0;
            v[j] = 0;
            if (e < m) {
                u[j] = HINT ? ld_first(nlist + e, pf) : __ldg(nlist + e);
                v[j] = HINT ? ld_first(src + e, pf) : __ldg(src + e);
            }
        }
#pragma unroll
        for (int j = 0; j < U; j++) {
            p[j] = 0;
            if (u[j] < v[j]) p[j] = HINT ? ld_last(parent + u[j], pl) : parent[u[j]];
        }
#pragma unroll
        for (int j = 0; j < U; j++) acc += (unsigned)p[j];
    }
    if (acc == 0x123456789ull) out[0] = acc;  // keep the loads alive
}

extern "C" int gather_run(int hint, long long m, const int *src, const int *nlist,
                          const int *parent, unsigned long long *out, void *stream)
{
    const int grid = 148 * 8;
    if (hint) gather_kernel<1, 8><<<grid, 256, 0, (cudaStream_t)stream>>>(m, src, nlist, parent, out);
    else gather_kernel<0, 8><<<grid, 256, 0, (cudaStream_t)stream>>>(m, src, nlist, parent, out);
    return (int)cudaGetLastError();
}
