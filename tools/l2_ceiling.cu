// Microbenchmark: the L2 random-sector ceiling that bounds the hook kernels.
//   mode 0: P random 4-byte loads from a table of T bytes (indices from a counter hash)
//   mode 1: the R21 probe pattern: stream E int32 entries u (coalesced, L1::no_allocate)
//           and, for the half with (u & 1) == 0, load the table word u >> 5
// Reported by tools/l2_ceiling.py as loads (sectors) per second.
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long mix(unsigned long long z)
{
    z += 0x9e3779b97f4a7c15ull;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
    return z ^ (z >> 31);
}

template <int U>
__global__ void __launch_bounds__(256) random_kernel(long long P, const unsigned *table,
                                                     unsigned long long words, unsigned *out)
{
    unsigned acc = 0;
    const long long stride = (long long)gridDim.x * blockDim.x * U;
    for (long long i = ((long long)blockIdx.x * blockDim.x + threadIdx.x) * U; i < P; i += stride) {
        unsigned v[U];
#pragma unroll
        for (int j = 0; j < U; j++) {
            const unsigned long long k = mix(i + j) % words;
            asm volatile("ld.global.b32 %0, [%1];" : "=r"(v[j]) : "l"(table + k));
        }
#pragma unroll
        for (int j = 0; j < U; j++) acc += v[j];
    }
    if (acc == 0x9e3779b9u) out[0] = acc;
}

template <int F>
__device__ __forceinline__ unsigned ld_probe(const unsigned *p)
{
    unsigned v;
    if (F == 0) asm volatile("ld.global.b32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (F == 1) asm volatile("ld.global.cg.b32 %0, [%1];" : "=r"(v) : "l"(p));
    else if (F == 2) asm volatile("ld.global.L1::no_allocate.b32 %0, [%1];" : "=r"(v) : "l"(p));
    else asm volatile("ld.relaxed.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}

template <int U, int F = 0>
__global__ void __launch_bounds__(256) probe_kernel(long long E, const int *list,
                                                    const unsigned *table, unsigned *out)
{
    unsigned acc = 0;
    const long long stride = (long long)gridDim.x * blockDim.x * U;
    for (long long i = (long long)blockIdx.x * blockDim.x * U + threadIdx.x; i < E; i += stride) {
        int u[U];
#pragma unroll
        for (int j = 0; j < U; j++) {
            const long long e = i + (long long)j * blockDim.x;
            u[j] = 1;
            if (e < E) asm volatile("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(u[j]) : "l"(list + e));
        }
        unsigned w[U];
#pragma unroll
        for (int j = 0; j < U; j++) {
            w[j] = 0;
            if ((u[j] & 1) == 0) w[j] = ld_probe<F>(table + (u[j] >> 5));
        }
#pragma unroll
        for (int j = 0; j < U; j++) acc += w[j];
    }
    if (acc == 0x9e3779b9u) out[0] = acc;
}

extern "C" int l2c_random(long long P, const unsigned *table, unsigned long long words,
                          unsigned *out, int grid)
{
    random_kernel<8><<<grid, 256>>>(P, table, words, out);
    return (int)cudaGetLastError();
}

extern "C" int l2c_probe(long long E, const int *list, const unsigned *table, unsigned *out,
                         int grid)
{
    probe_kernel<8><<<grid, 256>>>(E, list, table, out);
    return (int)cudaGetLastError();
}

// probe-load flavour / loads-per-thread sweep: flavour 0 ld.global, 1 .cg, 2 L1::no_allocate,
// 3 ld.relaxed.gpu; U = 4, 8 or 16 entries per thread per iteration
extern "C" int l2c_probe_v(long long E, const int *list, const unsigned *table, unsigned *out,
                           int grid, int flavour, int U)
{
#define L2C_CASE(UU, FF) if (U == UU && flavour == FF) probe_kernel<UU, FF><<<grid, 256>>>(E, list, table, out);
    L2C_CASE(4, 0) L2C_CASE(4, 1) L2C_CASE(4, 2) L2C_CASE(4, 3)
    L2C_CASE(8, 0) L2C_CASE(8, 1) L2C_CASE(8, 2) L2C_CASE(8, 3)
    L2C_CASE(16, 0) L2C_CASE(16, 1) L2C_CASE(16, 2) L2C_CASE(16, 3)
#undef L2C_CASE
    return (int)cudaGetLastError();
}
