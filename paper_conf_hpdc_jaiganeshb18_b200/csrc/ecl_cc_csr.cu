// ecl_cc_csr.cu — input preparation beside the hot path: build the
// symmetric CSR that ECL-CC consumes from an undirected edge list, exactly as the paper
// prepared its inputs (§4: "we modified the graphs to eliminate loops and multiple
// edges between the same two vertices.  We added any missing back edges to make the
// graphs undirected.  ... each undirected edge is represented by two directed edges").
//
//   expand_kernel   each pair (a,b), a != b, becomes the keys a*n+b and b*n+a; self-loops
//                   become the sentinel n*n (sorted last); out-of-range IDs raise a flag
//   CUB radix sort  ascending keys = rows in vertex order, each row ascending
//   CUB unique      drops duplicate entries (multiple edges)
//   emit kernels    nlist[i] = key % n; nindex[v] = lower bound of v*n among the keys
//                   (isolated vertices get empty rows)
//
// The sort and unique are CUB library primitives (header-only, CUDA toolkit); the
// expansion, the sentinel handling and the CSR emission are this file's kernels.
#include "ecl_cc_ctx.h"

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_select.cuh>

using namespace eclcc_host;

namespace {

constexpr int kThreads = 256;

__global__ void __launch_bounds__(kThreads) expand_kernel(long long E, int n, const int *src,
                                                          const int *dst,
                                                          unsigned long long *keys, int *flags)
{
    const unsigned long long N = (unsigned long long)n, S = N * N;
    const long long stride = (long long)gridDim.x * kThreads;
    for (long long i = (long long)blockIdx.x * kThreads + threadIdx.x; i < E; i += stride) {
        const int a = src[i], b = dst[i];
        unsigned long long k0 = S, k1 = S;
        if (a < 0 || a >= n || b < 0 || b >= n) {
            atomicOr(flags, 1);
        } else if (a != b) {                                   // loops are eliminated
            k0 = (unsigned long long)a * N + (unsigned)b;
            k1 = (unsigned long long)b * N + (unsigned)a;      // the back edge
        }
        keys[2 * i] = k0;
        keys[2 * i + 1] = k1;
    }
}

// uniq[0..m) ascending and duplicate-free (sentinel excluded): entry i of row r = key / n
// is the neighbour key % n
__global__ void __launch_bounds__(kThreads) emit_list_kernel(long long m, int n,
                                                             const unsigned long long *uniq,
                                                             int *nlist)
{
    const unsigned long long N = (unsigned long long)n;
    const long long stride = (long long)gridDim.x * kThreads;
    for (long long i = (long long)blockIdx.x * kThreads + threadIdx.x; i < m; i += stride)
        nlist[i] = (int)(uniq[i] % N);
}

// nindex[v] = number of keys < v*n (lower bound by binary search), v = 0..n
__global__ void __launch_bounds__(kThreads) emit_offsets_kernel(long long m, int n,
                                                                const unsigned long long *uniq,
                                                                long long *nindex)
{
    const unsigned long long N = (unsigned long long)n;
    const int stride = gridDim.x * kThreads;
    for (int v = blockIdx.x * kThreads + threadIdx.x; v <= n; v += stride) {
        const unsigned long long t = (unsigned long long)v * N;
        long long lo = 0, hi = m;
        while (lo < hi) {
            const long long mid = lo + (hi - lo) / 2;
            if (uniq[mid] < t) lo = mid + 1;
            else hi = mid;
        }
        nindex[v] = lo;
    }
}

__global__ void empty_offsets_kernel(int n, long long *nindex)
{
    const int stride = gridDim.x * kThreads;
    for (int v = blockIdx.x * kThreads + threadIdx.x; v <= n; v += stride) nindex[v] = 0;
}

int end_bit_for(unsigned long long S)
{
    int b = 1;
    while (b < 64 && (S >> b) != 0) b++;
    return b;   // every key <= S has no bits at or above b
}

}  // namespace

extern "C" {

ecl_cc_status ecl_cc_build_csr(ecl_cc_handle h, int32_t n, int64_t num_edges, const int32_t *src,
                               const int32_t *dst, int64_t *nindex_out, int32_t *nlist_out,
                               int64_t nlist_capacity, int64_t *m_out, void *stream)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    if (n < 0 || num_edges < 0) return fail_arg(h, "negative size");
    if (!m_out) return fail_arg(h, "null m_out");
    if (!nindex_out) return fail_arg(h, "null nindex_out");
    if (num_edges > 0 && (!src || !dst)) return fail_arg(h, "null edge list");
    if ((unsigned long long)n * (unsigned long long)n >= (1ull << 62))
        return fail_arg(h, "n too large");
    DeviceGuard g(h->device);
    if (!g.ok) return fail_arg(h, "cannot select the handle's device");
    cudaStream_t s = (cudaStream_t)stream;
    *m_out = 0;
    {
        ecl_cc_status st = begin_call(h, s);
        if (st != ECL_CC_OK) return st;
        h->last_stream = s;   // every return below follows a synchronisation of `s`
    }
    const int grid = h->sms * 8;
    if (num_edges == 0 || n == 0) {
        if (num_edges > 0) return fail_arg(h, "edges given for an empty vertex set");
        empty_offsets_kernel<<<grid, kThreads, 0, s>>>(n, (long long *)nindex_out);
        CK(cudaGetLastError(), "empty_offsets launch");
        CK(cudaStreamSynchronize(s), "sync");
        return ECL_CC_OK;
    }
    const long long K = 2 * (long long)num_edges;
    const unsigned long long S = (unsigned long long)n * (unsigned long long)n;
    const int end_bit = end_bit_for(S);

    // scratch: keys, sorted keys (reused as the unique output), count, flags, CUB temp
    size_t sort_tmp = 0, uniq_tmp = 0;
    unsigned long long *kp = nullptr;
    CK(cub::DeviceRadixSort::SortKeys(nullptr, sort_tmp, kp, kp, K, 0, end_bit, s), "cub sort size");
    CK(cub::DeviceSelect::Unique(nullptr, uniq_tmp, kp, kp, (long long *)nullptr, (int64_t)K, s),
       "cub unique size");
    const size_t keys_b = sizeof(unsigned long long) * (size_t)K;
    const size_t tmp_b = (sort_tmp > uniq_tmp ? sort_tmp : uniq_tmp) + 256;
    const size_t need = 2 * keys_b + tmp_b + 64;
    if (need > h->csr_tmp_bytes) {
        if (h->csr_tmp) CK(cudaFreeAsync(h->csr_tmp, s), "cudaFreeAsync(csr)");
        h->csr_tmp = nullptr;
        h->csr_tmp_bytes = 0;
        CK(cudaMallocAsync(&h->csr_tmp, need, s), "cudaMallocAsync(csr)");
        h->csr_tmp_bytes = need;
    }
    char *base = (char *)h->csr_tmp;
    unsigned long long *keys = (unsigned long long *)base;
    unsigned long long *sorted = (unsigned long long *)(base + keys_b);
    long long *cnt = (long long *)(base + 2 * keys_b);
    int *flags = (int *)(base + 2 * keys_b + 16);
    void *tmp = base + 2 * keys_b + 64;

    CK(cudaMemsetAsync(flags, 0, sizeof(int), s), "memset flags");
    expand_kernel<<<grid, kThreads, 0, s>>>(num_edges, n, src, dst, keys, flags);
    CK(cudaGetLastError(), "expand launch");
    size_t tb = tmp_b;
    CK(cub::DeviceRadixSort::SortKeys(tmp, tb, keys, sorted, K, 0, end_bit, s), "cub sort");
    tb = tmp_b;
    CK(cub::DeviceSelect::Unique(tmp, tb, sorted, keys, cnt, (int64_t)K, s), "cub unique");
    long long host[2] = {0, 0};
    CK(cudaMemcpyAsync(&host[0], cnt, sizeof(long long), cudaMemcpyDeviceToHost, s), "D2H count");
    int hflags = 0;
    CK(cudaMemcpyAsync(&hflags, flags, sizeof(int), cudaMemcpyDeviceToHost, s), "D2H flags");
    CK(cudaStreamSynchronize(s), "sync");
    if (hflags) {
        snprintf(h->err, sizeof(h->err), "invalid graph: vertex ID out of [0, n)");
        return ECL_CC_ERR_INVALID_GRAPH;
    }
    long long m = host[0];
    if (m > 0) {   // the sentinel, if present, is the last unique key
        unsigned long long last = 0;
        CK(cudaMemcpy(&last, keys + (m - 1), sizeof(last), cudaMemcpyDeviceToHost), "D2H last");
        if (last == S) m--;
    }
    if (m > nlist_capacity) {
        snprintf(h->err, sizeof(h->err), "nlist capacity %lld < %lld entries",
                 (long long)nlist_capacity, m);
        *m_out = m;
        return ECL_CC_ERR_INVALID_ARG;
    }
    if (m > 0 && !nlist_out) return fail_arg(h, "null nlist_out");
    if (m == 0) {
        empty_offsets_kernel<<<grid, kThreads, 0, s>>>(n, (long long *)nindex_out);
    } else {
        emit_list_kernel<<<grid, kThreads, 0, s>>>(m, n, keys, nlist_out);
        emit_offsets_kernel<<<grid, kThreads, 0, s>>>(m, n, keys, (long long *)nindex_out);
    }
    CK(cudaGetLastError(), "emit launch");
    CK(cudaStreamSynchronize(s), "sync");
    *m_out = m;
    return ECL_CC_OK;
}

}  // extern "C"
