// ecl_cc.cu — host side of libecl_cc.so: the C ABI declared in include/ecl_cc.h.
//
// Launch sequence of one run (init, three compute kernels, finalize):
//   memset(counters) -> init_bin -> depth_probe -> prejump (R23, no-op unless deep)
//   -> hook_thread -> hook_range<front> -> hook_range<back>
//   -> finalize, all enqueued on the caller's stream with no host synchronisation.
#include "ecl_cc.h"
#include "ecl_cc_kernels.cuh"
#include "ecl_cc_ctx.h"

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <unordered_map>

using namespace eclcc;
using namespace eclcc_host;

namespace {

constexpr int kCnt = 32;        // 64-bit counter words owned by the handle
constexpr int kStatsOff = 16;   // ECL_CC_STATS counters live at cnt[16..31]
constexpr int kNumStats = 16;
#ifndef ECL_FAST_FINI
#define ECL_FAST_FINI 1
#endif
constexpr bool kFastFini = ECL_FAST_FINI != 0;   // Fini3 via finalize3_kernel
// R33 auto mode: the single-launch path for graphs up to this size (measured crossover,
// profiles/r2/ab_fused_size_r2z: faster up to ~4 M entries on every family; at ~8 M
// entries slower on R-MAT, whose hub chunks want more blocks than one per SM)
constexpr int kFusedMaxRows = 1 << 20;
constexpr long long kFusedMaxEntries = 1LL << 22;

const char *kVersion = "ecl_cc-b200 0.1 (sm_100a)";

int blocks_per_sm(ecl_cc_handle h, const void *kernel, size_t dsmem)
{
    auto it = h->occ.find(kernel);
    if (it != h->occ.end()) return it->second;
    if (dsmem > 0)
        cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsmem);
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kernel, kBlock, dsmem) != cudaSuccess ||
        b < 1)
        b = 1;
    h->occ[kernel] = b;
    return b;
}

// grid for a grid-stride kernel over `work` threads (or a persistent kernel if work < 0)
int grid_for(ecl_cc_handle h, const void *kernel, long long work_threads, size_t dsmem = 0,
             int occ_cap = 0)
{
    int b = blocks_per_sm(h, kernel, dsmem);
    if (occ_cap > 0 && occ_cap < b) b = occ_cap;
    const long long full = (long long)h->sms * b;
    if (h->grid_blocks > 0) return h->grid_blocks;
    if (work_threads < 0) return (int)full;
    long long need = (work_threads + kBlock - 1) / kBlock;
    if (need < 1) need = 1;
    return (int)(need < full ? need : full);
}

ecl_cc_status ensure_scratch(ecl_cc_handle h, int need, cudaStream_t s)
{
    if (need <= h->cap) return ECL_CC_OK;
    if (h->wl) CK(cudaFreeAsync(h->wl, s), "cudaFreeAsync(wl)");
    if (h->ub) CK(cudaFreeAsync(h->ub, s), "cudaFreeAsync(ub)");
    if (h->tbits) CK(cudaFreeAsync(h->tbits, s), "cudaFreeAsync(tbits)");
    h->wl = nullptr;
    h->ub = nullptr;
    h->tbits = nullptr;
    h->cap = 0;
    CK(cudaMallocAsync((void **)&h->wl, sizeof(int) * (size_t)need, s), "cudaMallocAsync(wl)");
    CK(cudaMallocAsync((void **)&h->ub, sizeof(unsigned) * (size_t)need, s), "cudaMallocAsync(ub)");
    CK(cudaMallocAsync((void **)&h->tbits, sizeof(unsigned) * (((size_t)need + 31) / 32), s),
       "cudaMallocAsync(tbits)");
    h->cap = need;
    return ECL_CC_OK;
}

template <int MODE, typename idx_t>
ecl_cc_status launch_path(ecl_cc_handle h, int n, long long m, int row_lo, int nrows,
                          const idx_t *nindex, const int *nlist, int *parent, cudaStream_t s,
                          bool rows_mode)
{
    ecl_cc_status st = ensure_scratch(h, nrows > 0 ? nrows : 1, s);
    if (st != ECL_CC_OK) return st;
    CK(cudaMemsetAsync(h->cnt, 0, kCnt * sizeof(unsigned long long), s), "cudaMemsetAsync");

    Params p;
    p.n = n;
    p.row_lo = row_lo;
    p.nrows = nrows;
    p.m = m;
    p.nindex = nindex;
    p.nlist = nlist;
    p.parent = parent;
    p.wl = h->wl;
    p.ub = h->ub;
    p.tbits = h->tbits;
    p.cap = h->cap;
    p.cnt = h->cnt;
    p.stats = h->cnt + kStatsOff;
    p.sched = (int *)(h->cnt + 8);
    p.t1 = h->t1;
    p.t2 = h->t2;
    p.ttas = h->ttas;
    // R28: Init3 folded into the hook kernels (the separate pass over every row start is
    // then a degree-only binning pass).  Auto: off for long rows (m >= 16 n: the R21
    // filter needs Init3's forest), else decided on the device by the locality probe
    // (random vertex IDs: on; meshes, whose Init3 chains R23 shortens: off)
    const bool can = h->init_mode == 3 && h->stop_after != 1 && nrows > 0;
    p.lazy = !can ? 0 : h->fuse_init == 1 ? 1
           : (h->fuse_init == 2 && m < 16LL * nrows) ? 2 : 0;
    p.lazy_flag = (const int *)(h->cnt + 7);
    h->last_lazy = p.lazy;
    p.init_mode = h->init_mode;
    p.jump = h->jump;
    p.batch = h->batch;
    p.anchor = h->cnt + 10;
    p.nthr = h->cnt + 3;
    p.gbits = nullptr;
    p.fa = h->fa;
    p.fb = h->fb;
    // R31: quads need a 16-byte aligned adjacency base (quad q = entries 4q..4q+3) and
    // 32-bit quad indices (m < 2^33).  p.vec: bit 0 hook_warp, bit 1 hook_block.  Default
    // (2): hook_warp only, and only with int32 offsets — quads cut the multi-piece
    // rounds' per-entry owner work (C4: 2.23 vs 2.33 ms) but cost the hubs' uniform rounds
    // (hook_block) and, with int64 offsets, hook_warp too (C5 hook_warp 3.75 vs 3.56 ms)
    const bool quads_ok = ((reinterpret_cast<uintptr_t>(nlist) & 15) == 0) && m < (1LL << 33);
    p.vec = !quads_ok ? 0 : h->vec == 1 ? 3 : (h->vec == 2 && sizeof(idx_t) == 4) ? 1 : 0;
    {
        // auto: on when parent[] (4n bytes) cannot stay in the 126 MB L2
        const bool on = h->filter == 1 || (h->filter == 2 && (long long)n * 4 > (128ll << 20));
        h->gbits_live = on;
        if (on) {
            const size_t words = ((size_t)n + 31) / 32;
            if (words > h->gbits_words) {
                if (h->gbits) CK(cudaFreeAsync(h->gbits, s), "cudaFreeAsync(gbits)");
                h->gbits = nullptr;
                h->gbits_words = 0;
                CK(cudaMallocAsync((void **)&h->gbits, words * 4, s), "cudaMallocAsync(gbits)");
                h->gbits_words = words;
            }
            CK(cudaMemsetAsync(h->gbits, 0, words * 4, s), "cudaMemsetAsync(gbits)");
            p.gbits = h->gbits;
        }
    }

    // R33: the whole path as one cooperative launch for small graphs (no per-phase
    // timing events inside it, so ECL_CC_OPT_TIMING keeps the multi-kernel path)
    const bool fuse = !rows_mode && h->timing == 0 && h->stop_after != 1 && nrows > 0 &&
                      (h->fused == 1 ||
                       (h->fused == 2 && nrows <= kFusedMaxRows && m <= kFusedMaxEntries));
    h->last_fused = fuse;
    if (fuse) {
        auto k = fused_small_kernel<MODE, idx_t>;
        const size_t sm = fused_smem_bytes<idx_t>();
        const int cap = h->sms * blocks_per_sm(h, (const void *)k, sm);
        // one block per SM: on C1 148 blocks ran 0.082 ms, 256 / 296 / 592 blocks
        // 0.09 / 0.09-0.10 / 0.115 ms (fewer CAS collisions, cheaper grid barriers)
        long long want = h->sms;
        if (h->grid_blocks > 0) want = h->grid_blocks;
        const int blocks = (int)std::min<long long>(cap, want);
        FusedArgs fa;
        fa.prejump = h->prejump;
        fa.fini = h->stop_after == 2 ? 0 : h->fini;
        fa.ctl = (int *)(h->cnt + 4);
        fa.bar = (unsigned *)(h->cnt + 12);
        void *args[] = {&p, &fa};
        CK(cudaLaunchCooperativeKernel((const void *)k, dim3(blocks), dim3(kBlock), args, sm, s),
           "fused launch");
        return ECL_CC_OK;
    }

    const bool tm = h->timing != 0;
    if (tm) {
        for (int i = 0; i < 8; i++)
            if (!h->ev[i]) CK(cudaEventCreate(&h->ev[i]), "cudaEventCreate");
        CK(cudaEventRecord(h->ev[0], s), "cudaEventRecord");
    }
    h->ev_valid = 0;
    auto mark = [&](int i) {
        if (tm) cudaEventRecord(h->ev[i], s);
    };
    if (rows_mode) {
        auto k = identity_outside_kernel;
        k<<<grid_for(h, (const void *)k, n), kBlock, 0, s>>>(n, row_lo, row_lo + nrows, parent);
    }
    if (p.lazy == 2)
        locality_probe_kernel<idx_t><<<1, kBlock, 0, s>>>(row_lo, nrows, nindex, nlist,
                                                           (int *)(h->cnt + 7));
    {
        auto k = init_bin_kernel<idx_t>;
        k<<<grid_for(h, (const void *)k, ((long long)nrows + kInitPerThread - 1) / kInitPerThread), kBlock, 0, s>>>(p);
    }
    if (h->prejump != 0 && h->stop_after != 1 && nrows > 0 && p.lazy != 1) {
        // R23: depth probe, then the passes (cooperative launch guarantees the
        // co-residency their grid barrier needs); both are no-ops on shallow forests
        int *ctl = (int *)(h->cnt + 4);
        depth_probe_kernel<<<1, kBlock, 0, s>>>(row_lo, nrows, parent, ctl, h->prejump,
                                                p.lazy ? p.lazy_flag : nullptr);
        auto k = prejump_kernel;
        const int blocks = std::min(h->sms * blocks_per_sm(h, (const void *)k, 0),
                                    (int)std::max(1LL, ((long long)nrows + kBlock - 1) / kBlock));
        int a0 = row_lo, a1 = nrows;
        int *a2 = parent, *a3 = ctl;
        void *args[] = {&a0, &a1, &a2, &a3};
        CK(cudaLaunchCooperativeKernel((const void *)k, dim3(blocks), dim3(kBlock), args, 0, s),
           "prejump launch");
    }
    mark(1);
    if (h->stop_after != 1) {
        // the three compute kernels depend only on init_bin; events record each
        // kernel's span whatever the launch order (ev[2+i] ends phase i)
        auto thread_k = [&] {
            auto k = hook_thread_kernel<MODE, idx_t>;
            const long long tiles = (nrows + kWarp - 1) / kWarp;
            const size_t sm = hook_smem_bytes<idx_t>();
            k<<<grid_for(h, (const void *)k, tiles * kWarp, sm, h->occ_thread), kBlock, sm, s>>>(p);
        };
        // R31 quad engine as its own instantiation (the scalar kernels keep their
        // register allocation)
        void (*const front_k)(Params) = (p.vec & 1) ? hook_range_kernel<MODE, idx_t, kUnitFront, true, true>
                                              : hook_range_kernel<MODE, idx_t, kUnitFront, true, false>;
        void (*const back_k)(Params) = (p.vec & 2) ? hook_range_kernel<MODE, idx_t, kUnitBack, false, true>
                                             : hook_range_kernel<MODE, idx_t, kUnitBack, false, false>;
        auto warp_k = [&] {
            auto k = front_k;
            const size_t sm = hook_smem_bytes<idx_t>();
            k<<<grid_for(h, (const void *)k, -1, sm, h->occ_range), kBlock, sm, s>>>(p);
        };
        auto block_k = [&] {
            auto k = back_k;
            const size_t sm = hook_smem_bytes<idx_t>();
            k<<<grid_for(h, (const void *)k, -1, sm, h->occ_range), kBlock, sm, s>>>(p);
        };
        if (h->order == 2) {
            // concurrent: hub chunks (L2-request bound) on a side stream next to the
            // warp and thread bins (issue / latency bound), occupancy split per SM
            const size_t sm = hook_smem_bytes<idx_t>();
            const int full = blocks_per_sm(h, (const void *)front_k, sm);
            // hook_block is launched first with a capped grid; hook_warp / hook_thread get
            // full persistent grids whose surplus blocks start as hook_block's retire (a
            // graph without hubs gives the whole GPU to the other two at once)
            // (3/4 of the SM's blocks measured best at C5: 12.99 vs 13.48 ms sequential)
            const int cb = h->occ_range > 0 ? h->occ_range : std::max(1, (3 * full) / 4);
            const int cw = h->occ_thread;
            // the side stream and both events exist for the handle's lifetime (created
            // together in ecl_cc_create); once the fork is recorded the join is always
            // recorded and waited on, so no error return leaves work of this call running
            // on the side stream unordered with `stream`
            CK(cudaEventRecord(h->fork, s), "fork");
            CK(cudaStreamWaitEvent(h->side, h->fork, 0), "fork wait");
            if (tm) cudaEventRecord(h->ev[6], h->side);
            {
                auto k = back_k;
                k<<<grid_for(h, (const void *)k, -1, sm, cb), kBlock, sm, h->side>>>(p);
            }
            if (tm) cudaEventRecord(h->ev[7], h->side);
            {
                auto k = hook_thread_kernel<MODE, idx_t>;
                const long long tiles = (nrows + kWarp - 1) / kWarp;
                const size_t smt = hook_smem_bytes<idx_t>();
                k<<<grid_for(h, (const void *)k, tiles * kWarp, smt, cw), kBlock, smt, s>>>(p);
            }
            mark(2);
            {
                auto k = front_k;
                k<<<grid_for(h, (const void *)k, -1, sm, cw), kBlock, sm, s>>>(p);
            }
            mark(3);
            cudaError_t ej = cudaEventRecord(h->join, h->side);
            if (ej == cudaSuccess) ej = cudaStreamWaitEvent(s, h->join, 0);
            if (ej != cudaSuccess) {
                cudaStreamSynchronize(h->side);   // cannot order it on `stream`: drain it
                return fail_cuda(h, ej, "join");
            }
            mark(4);
        } else if (h->order == 1) {
            block_k();
            mark(4);
            warp_k();
            mark(3);
            thread_k();
            mark(2);
        } else {
            thread_k();
            mark(2);
            warp_k();
            mark(3);
            block_k();
            mark(4);
        }
        if (h->stop_after != 2) {
            if (h->fini == 3 && kFastFini) {
                auto k = finalize3_kernel<MODE>;
                k<<<grid_for(h, (const void *)k, ((long long)n + kFinPer - 1) / kFinPer), kBlock, 0, s>>>(n, parent);
            } else {
                auto k = finalize_kernel<MODE>;
                k<<<grid_for(h, (const void *)k, n), kBlock, 0, s>>>(n, parent, h->fini);
            }
        }
        mark(5);
        if (tm && h->stop_after == 0) h->ev_valid = 1 + h->order;   // 3: hooks overlap
    }
    CK(cudaGetLastError(), "kernel launch");
    return ECL_CC_OK;
}

template <typename idx_t>
ecl_cc_status run_impl(ecl_cc_handle h, int32_t n, int64_t m, const idx_t *nindex,
                       const int32_t *nlist, int32_t *out, void *stream, int row_lo,
                       int nrows, bool rows_mode)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    if (n < 0) return fail_arg(h, "n < 0");
    if (m < 0) return fail_arg(h, "m < 0");
    if (n == 0) return ECL_CC_OK;
    if (!out) return fail_arg(h, "null output/parent pointer");
    if (nrows > 0 && !nindex) return fail_arg(h, "null nindex");
    if (m > 0 && !nlist) return fail_arg(h, "null nlist");
    if (m / kUnitFront + (long long)nrows >= (1LL << 32))
        return fail_arg(h, "graph too large for 32-bit worklist unit counters");
    DeviceGuard g(h->device);
    if (!g.ok) return fail_arg(h, "cannot select the handle's device");
    cudaStream_t s = (cudaStream_t)stream;
    ecl_cc_status st = begin_call(h, s);
    if (st != ECL_CC_OK) return st;
    switch (h->load_mode) {
    case 0: st = launch_path<0, idx_t>(h, n, m, row_lo, nrows, nindex, nlist, out, s, rows_mode); break;
    case 2: st = launch_path<2, idx_t>(h, n, m, row_lo, nrows, nindex, nlist, out, s, rows_mode); break;
    case 3: st = launch_path<3, idx_t>(h, n, m, row_lo, nrows, nindex, nlist, out, s, rows_mode); break;
    default: st = launch_path<1, idx_t>(h, n, m, row_lo, nrows, nindex, nlist, out, s, rows_mode); break;
    }
    ecl_cc_status se = end_call(h, s);
    return st != ECL_CC_OK ? st : se;
}

// pointers handed out by ecl_cc_ipc_open -> the mapping's base (for ecl_cc_ipc_close)
std::mutex &ipc_lock()
{
    static std::mutex m;
    return m;
}
std::unordered_map<void *, void *> &ipc_bases()
{
    static std::unordered_map<void *, void *> b;
    return b;
}

typedef int CUresult_compat;   // CUresult (driver API enum; 0 = CUDA_SUCCESS)

}  // namespace

extern "C" {

ecl_cc_status ecl_cc_create(ecl_cc_handle *out, int device)
{
    if (!out) return ECL_CC_ERR_INVALID_ARG;
    *out = nullptr;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev)
        return ECL_CC_ERR_INVALID_ARG;
    ecl_cc_handle h = new (std::nothrow) ecl_cc_ctx();
    if (!h) return ECL_CC_ERR_OOM;
    h->device = device;
    DeviceGuard g(device);
    // everything the handle owns for its lifetime is created here, all or nothing: the
    // side stream (hook_block under order 2; the stream destroy frees on), the fork/join
    // events of the concurrent order, the end-of-call event, the counters
    cudaError_t e = cudaDeviceGetAttribute(&h->sms, cudaDevAttrMultiProcessorCount, device);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->side, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->fork, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->join, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->done, cudaEventDisableTiming);
    if (e == cudaSuccess)
        e = cudaMallocAsync((void **)&h->cnt, kCnt * sizeof(unsigned long long), h->side);
    if (e == cudaSuccess) e = cudaMallocAsync((void **)&h->flags, 4 * sizeof(int), h->side);
    if (e == cudaSuccess) e = cudaStreamSynchronize(h->side);
    if (e != cudaSuccess) {
        if (h->side) {
            if (h->cnt) cudaFreeAsync(h->cnt, h->side);
            if (h->flags) cudaFreeAsync(h->flags, h->side);
            cudaStreamSynchronize(h->side);
            cudaStreamDestroy(h->side);
        }
        if (h->fork) cudaEventDestroy(h->fork);
        if (h->join) cudaEventDestroy(h->join);
        if (h->done) cudaEventDestroy(h->done);
        delete h;
        return e == cudaErrorMemoryAllocation ? ECL_CC_ERR_OOM : ECL_CC_ERR_CUDA;
    }
    *out = h;
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_destroy(ecl_cc_handle h)
{
    if (!h) return ECL_CC_OK;
    {
        // no device-wide synchronisation: the frees are stream-ordered on the handle's own
        // stream after the handle's last call (its `done` event), and only that stream is
        // waited for
        DeviceGuard g(h->device);
        cudaStream_t s = h->side;
        if (h->done_valid) cudaStreamWaitEvent(s, h->done, 0);
        void *bufs[] = {h->wl, h->ub, h->tbits, h->cnt, h->flags, h->e2e_index, h->e2e_list,
                        h->e2e_labels, h->gbits, h->csr_tmp};
        for (void *b : bufs)
            if (b) cudaFreeAsync(b, s);
        cudaStreamSynchronize(s);
        for (int i = 0; i < 8; i++)
            if (h->ev[i]) cudaEventDestroy(h->ev[i]);
        cudaEventDestroy(h->fork);
        cudaEventDestroy(h->join);
        cudaEventDestroy(h->done);
        cudaStreamDestroy(s);
    }
    delete h;
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_run(ecl_cc_handle h, int32_t n, int64_t m, const int32_t *nindex,
                         const int32_t *nlist, int32_t *nstat_out, void *stream)
{
    if (m > INT32_MAX) return fail_arg(h, "m > INT32_MAX: use ecl_cc_run_i64");
    return run_impl<int>(h, n, m, nindex, nlist, nstat_out, stream, 0, n, false);
}

ecl_cc_status ecl_cc_run_i64(ecl_cc_handle h, int32_t n, int64_t m, const int64_t *nindex,
                             const int32_t *nlist, int32_t *nstat_out, void *stream)
{
    return run_impl<long long>(h, n, m, (const long long *)nindex, nlist, nstat_out, stream, 0,
                               n, false);
}

ecl_cc_status ecl_cc_spanning_forest(ecl_cc_handle h, int32_t n, int64_t m, const void *nindex,
                                     int index_bytes, const int32_t *nlist,
                                     int32_t *labels_out, int32_t *tree_a, int32_t *tree_b,
                                     void *stream)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    if (index_bytes != 4 && index_bytes != 8) return fail_arg(h, "index_bytes must be 4 or 8");
    if (n > 0 && (!tree_a || !tree_b)) return fail_arg(h, "null tree-edge output");
    if (h->stop_after != 0) return fail_arg(h, "spanning forest needs a full run (stop_after 0)");
    h->fa = tree_a;
    h->fb = tree_b;
    ecl_cc_status st = index_bytes == 4
        ? ecl_cc_run(h, n, m, (const int32_t *)nindex, nlist, labels_out, stream)
        : ecl_cc_run_i64(h, n, m, (const int64_t *)nindex, nlist, labels_out, stream);
    h->fa = nullptr;
    h->fb = nullptr;
    return st;
}

ecl_cc_status ecl_cc_run_rows(ecl_cc_handle h, int32_t n, int32_t row_lo, int32_t row_hi,
                              int64_t m_rows, const int64_t *nindex_rows,
                              const int32_t *nlist_rows, int32_t *parent, void *stream)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    if (row_lo < 0 || row_hi < row_lo || row_hi > n) return fail_arg(h, "bad row range");
    return run_impl<long long>(h, n, m_rows, (const long long *)nindex_rows, nlist_rows, parent,
                               stream, row_lo, row_hi - row_lo, true);
}

ecl_cc_status ecl_cc_merge(ecl_cc_handle h, int32_t n, int32_t v_lo, int32_t v_hi,
                           const int32_t *peer_labels, int32_t *parent, void *stream)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    if (n < 0 || v_lo < 0 || v_hi < v_lo || v_hi > n) return fail_arg(h, "bad merge range");
    if (v_hi == v_lo) return ECL_CC_OK;
    if (!peer_labels || !parent) return fail_arg(h, "null pointer");
    DeviceGuard g(h->device);
    cudaStream_t s = (cudaStream_t)stream;
    ecl_cc_status st = begin_call(h, s);
    if (st != ECL_CC_OK) return st;
    const int cnt = v_hi - v_lo;
    if (h->load_mode == 1) {
        auto k = merge_hook_kernel<1>;
        k<<<grid_for(h, (const void *)k, ((long long)cnt + 3) / 4), kBlock, 0, s>>>(v_lo, cnt, peer_labels, parent, h->ttas
#ifdef ECL_CC_STATS
                                                                 , h->cnt + kStatsOff
#endif
        );
    } else {
        auto k = merge_hook_kernel<0>;
        k<<<grid_for(h, (const void *)k, ((long long)cnt + 3) / 4), kBlock, 0, s>>>(v_lo, cnt, peer_labels, parent, h->ttas
#ifdef ECL_CC_STATS
                                                                 , h->cnt + kStatsOff
#endif
        );
    }
    CK(cudaGetLastError(), "merge_hook launch");
    return end_call(h, s);
}

ecl_cc_status ecl_cc_forest_encode(ecl_cc_handle h, int32_t n, const int32_t *labels,
                                   int32_t anchor, uint32_t *bits, int32_t *pairs,
                                   int64_t cap, uint64_t *meta, void *stream)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    if (n <= 0) return fail_arg(h, "n must be > 0");
    if (anchor < -1 || anchor >= n) return fail_arg(h, "anchor out of range");
    if (cap < 0) return fail_arg(h, "cap < 0");
    if (!labels || !bits || !meta || (cap > 0 && !pairs)) return fail_arg(h, "null pointer");
    DeviceGuard g(h->device);
    cudaStream_t s = (cudaStream_t)stream;
    ecl_cc_status st = begin_call(h, s);
    if (st != ECL_CC_OK) return st;
    CK(cudaMemsetAsync(meta, 0, sizeof(uint64_t), s), "memset meta");
    auto k = encode_kernel;
    const long long words = ((long long)n + kWarp - 1) / kWarp;
    // ECL_CC_OPT_MERGE_FILTER: `labels` is the forest this handle's last run built; that
    // run's R21 bitmap and anchor (which then replaces `anchor`) prove most vertices'
    // class without a walk
    const bool filt = h->merge_filter && h->gbits_live;
    k<<<grid_for(h, (const void *)k, words * kWarp), kBlock, 0, s>>>(
        n, labels, anchor, bits, pairs, cap, (unsigned long long *)meta,
        filt ? h->gbits : nullptr, h->cnt + 10);
    CK(cudaGetLastError(), "encode launch");
    return end_call(h, s);
}

ecl_cc_status ecl_cc_merge_encoded(ecl_cc_handle h, int32_t n, int npeers,
                                   const uint32_t *const *bits, const int32_t *const *pairs,
                                   const uint64_t *const *meta, const int64_t *caps,
                                   int32_t *parent, void *stream)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    if (n <= 0) return fail_arg(h, "n must be > 0");
    if (npeers < 0 || npeers > kMaxPeers) return fail_arg(h, "npeers must be 0..8");
    if (!parent || (npeers > 0 && (!bits || !pairs || !meta || !caps)))
        return fail_arg(h, "null pointer");
    PeerSet ps{};
    ps.np = npeers;
    for (int i = 0; i < npeers; i++) {
        if (!bits[i] || !meta[i] || caps[i] < 0 || (caps[i] > 0 && !pairs[i]))
            return fail_arg(h, "null peer buffer");
        ps.bits[i] = bits[i];
        ps.pairs[i] = pairs[i];
        ps.meta[i] = (const unsigned long long *)meta[i];
        ps.cap[i] = caps[i];
    }
    if (npeers == 0) return ECL_CC_OK;
    DeviceGuard g(h->device);
    cudaStream_t s = (cudaStream_t)stream;
    ecl_cc_status st = begin_call(h, s);
    if (st != ECL_CC_OK) return st;
    const long long words = ((long long)n + kWarp - 1) / kWarp;
#ifdef ECL_CC_STATS
#define ECL_SA , h->cnt + kStatsOff
#else
#define ECL_SA
#endif
    unsigned *filt = (h->merge_filter && h->gbits_live) ? h->gbits : nullptr;
    if (h->load_mode == 1) {
        auto kb = merge_bits_kernel<1>;
        kb<<<grid_for(h, (const void *)kb, words * kWarp), kBlock, 0, s>>>(n, ps, parent, h->ttas,
                                                                            filt, h->cnt + 10 ECL_SA);
        auto kp = merge_pairs_kernel<1>;
        kp<<<grid_for(h, (const void *)kp, -1), kBlock, 0, s>>>(ps, parent, h->ttas ECL_SA);
    } else {
        auto kb = merge_bits_kernel<0>;
        kb<<<grid_for(h, (const void *)kb, words * kWarp), kBlock, 0, s>>>(n, ps, parent, h->ttas,
                                                                            filt, h->cnt + 10 ECL_SA);
        auto kp = merge_pairs_kernel<0>;
        kp<<<grid_for(h, (const void *)kp, -1), kBlock, 0, s>>>(ps, parent, h->ttas ECL_SA);
    }
#undef ECL_SA
    CK(cudaGetLastError(), "merge_encoded launch");
    return end_call(h, s);
}

// CUDA IPC (the peer mappings of the P2P merge): the handle of the allocation holding
// dev_ptr (cudaIpcGetMemHandle) followed by dev_ptr's byte offset inside it.
typedef CUresult_compat (*mem_range_fn)(unsigned long long *, size_t *, unsigned long long);

ecl_cc_status ecl_cc_ipc_export(const void *dev_ptr, void *handle_out)
{
    if (!dev_ptr || !handle_out) return ECL_CC_ERR_INVALID_ARG;
    static mem_range_fn range = nullptr;
    if (!range) {
        void *fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q) !=
                cudaSuccess || !fn)
            return ECL_CC_ERR_CUDA;
        range = (mem_range_fn)fn;
    }
    unsigned long long base = 0;
    size_t size = 0;
    if (range(&base, &size, (unsigned long long)(uintptr_t)dev_ptr) != 0) return ECL_CC_ERR_CUDA;
    cudaIpcMemHandle_t mh;
    if (cudaIpcGetMemHandle(&mh, (void *)(uintptr_t)base) != cudaSuccess) return ECL_CC_ERR_CUDA;
    const uint64_t off = (uint64_t)((uintptr_t)dev_ptr - base);
    memcpy(handle_out, &mh, sizeof(mh));
    memcpy((char *)handle_out + sizeof(mh), &off, sizeof(off));
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_ipc_open(int device, const void *handle, void **dev_ptr_out)
{
    if (!handle || !dev_ptr_out) return ECL_CC_ERR_INVALID_ARG;
    *dev_ptr_out = nullptr;
    DeviceGuard g(device);
    if (!g.ok) return ECL_CC_ERR_INVALID_ARG;
    cudaIpcMemHandle_t mh;
    uint64_t off = 0;
    memcpy(&mh, handle, sizeof(mh));
    memcpy(&off, (const char *)handle + sizeof(mh), sizeof(off));
    void *base = nullptr;
    if (cudaIpcOpenMemHandle(&base, mh, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess)
        return ECL_CC_ERR_CUDA;
    std::lock_guard<std::mutex> lk(ipc_lock());
    ipc_bases()[(char *)base + off] = base;
    *dev_ptr_out = (char *)base + off;
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_ipc_close(void *dev_ptr)
{
    if (!dev_ptr) return ECL_CC_ERR_INVALID_ARG;
    void *base = nullptr;
    {
        std::lock_guard<std::mutex> lk(ipc_lock());
        auto it = ipc_bases().find(dev_ptr);
        if (it == ipc_bases().end()) return ECL_CC_ERR_INVALID_ARG;
        base = it->second;
        ipc_bases().erase(it);
    }
    return cudaIpcCloseMemHandle(base) == cudaSuccess ? ECL_CC_OK : ECL_CC_ERR_CUDA;
}

ecl_cc_status ecl_cc_finalize(ecl_cc_handle h, int32_t n, int32_t *parent, void *stream)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    if (n < 0) return fail_arg(h, "n < 0");
    if (n == 0) return ECL_CC_OK;
    if (!parent) return fail_arg(h, "null parent");
    DeviceGuard g(h->device);
    cudaStream_t s = (cudaStream_t)stream;
    ecl_cc_status st = begin_call(h, s);
    if (st != ECL_CC_OK) return st;
    if (h->flatten_passes) {
        // R23's synchronous pointer-jumping passes first (forests merged from several
        // ranks can hold long chains of former roots, which Fini3 would walk per vertex)
        int *ctl = (int *)(h->cnt + 4);
        CK(cudaMemsetAsync(ctl, 0, 4 * sizeof(unsigned long long), s), "memset ctl");
        depth_probe_kernel<<<1, kBlock, 0, s>>>(0, n, parent, ctl, h->flatten_passes, nullptr);
        auto k = prejump_kernel;
        const int blocks = std::min(h->sms * blocks_per_sm(h, (const void *)k, 0),
                                    (int)std::max(1LL, ((long long)n + kBlock - 1) / kBlock));
        int a0 = 0, a1 = n;
        int *a2 = parent, *a3 = ctl;
        void *args[] = {&a0, &a1, &a2, &a3};
        CK(cudaLaunchCooperativeKernel((const void *)k, dim3(blocks), dim3(kBlock), args, 0, s),
           "flatten passes launch");
    }
    if (h->merge_filter && h->gbits_live && h->fini == 3) {
        // the R21 bitmap of the run that built `parent` (extended by merge_bits) proves
        // most vertices' root without a walk
        auto k = finalize_filter_kernel;
        k<<<grid_for(h, (const void *)k, ((long long)n + kWarp - 1) / kWarp * kWarp), kBlock, 0, s>>>(
            n, parent, h->gbits, h->cnt + 10);
    } else if (h->fini == 3 && kFastFini) {
        auto k = finalize3_kernel<0>;
        k<<<grid_for(h, (const void *)k, ((long long)n + kFinPer - 1) / kFinPer), kBlock, 0, s>>>(n, parent);
    } else {
        auto k = finalize_kernel<0>;
        k<<<grid_for(h, (const void *)k, n), kBlock, 0, s>>>(n, parent, h->fini);
    }
    CK(cudaGetLastError(), "finalize launch");
    return end_call(h, s);
}

ecl_cc_status ecl_cc_run_host(ecl_cc_handle h, int32_t n, int64_t m, const void *nindex_host,
                              int index_bytes, const int32_t *nlist_host,
                              int32_t *labels_host, void *stream)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    if (index_bytes != 4 && index_bytes != 8) return fail_arg(h, "index_bytes must be 4 or 8");
    if (n < 0 || m < 0) return fail_arg(h, "negative size");
    if (n == 0) return ECL_CC_OK;
    if (!nindex_host || !labels_host || (m > 0 && !nlist_host)) return fail_arg(h, "null pointer");
    if (index_bytes == 4 && m > INT32_MAX) return fail_arg(h, "m > INT32_MAX with int32 offsets");
    DeviceGuard g(h->device);
    cudaStream_t s = (cudaStream_t)stream;
    {
        ecl_cc_status st = begin_call(h, s);
        if (st != ECL_CC_OK) return st;
    }
    const size_t ib = (size_t)index_bytes * ((size_t)n + 1);
    if (ib > h->e2e_index_bytes) {
        if (h->e2e_index) CK(cudaFreeAsync(h->e2e_index, s), "cudaFreeAsync");
        h->e2e_index = nullptr;
        h->e2e_index_bytes = 0;
        CK(cudaMallocAsync(&h->e2e_index, ib, s), "cudaMallocAsync(index)");
        h->e2e_index_bytes = ib;
    }
    if ((size_t)m > h->e2e_list_n) {
        if (h->e2e_list) CK(cudaFreeAsync(h->e2e_list, s), "cudaFreeAsync");
        h->e2e_list = nullptr;
        h->e2e_list_n = 0;
        CK(cudaMallocAsync((void **)&h->e2e_list, sizeof(int) * (size_t)m, s), "cudaMallocAsync(list)");
        h->e2e_list_n = (size_t)m;
    }
    if ((size_t)n > h->e2e_labels_n) {
        if (h->e2e_labels) CK(cudaFreeAsync(h->e2e_labels, s), "cudaFreeAsync");
        h->e2e_labels = nullptr;
        h->e2e_labels_n = 0;
        CK(cudaMallocAsync((void **)&h->e2e_labels, sizeof(int) * (size_t)n, s), "cudaMallocAsync(labels)");
        h->e2e_labels_n = (size_t)n;
    }
    CK(cudaMemcpyAsync(h->e2e_index, nindex_host, ib, cudaMemcpyHostToDevice, s), "H2D nindex");
    if (m > 0)
        CK(cudaMemcpyAsync(h->e2e_list, nlist_host, sizeof(int) * (size_t)m, cudaMemcpyHostToDevice, s),
           "H2D nlist");
    ecl_cc_status st = index_bytes == 4
        ? ecl_cc_run(h, n, m, (const int32_t *)h->e2e_index, h->e2e_list, h->e2e_labels, stream)
        : ecl_cc_run_i64(h, n, m, (const int64_t *)h->e2e_index, h->e2e_list, h->e2e_labels, stream);
    if (st != ECL_CC_OK) return st;
    CK(cudaMemcpyAsync(labels_host, h->e2e_labels, sizeof(int) * (size_t)n, cudaMemcpyDeviceToHost, s),
       "D2H labels");
    CK(cudaStreamSynchronize(s), "cudaStreamSynchronize");
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_validate(ecl_cc_handle h, int32_t n, int64_t m, const void *nindex,
                              int index_bytes, const int32_t *nlist, void *stream)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    if (index_bytes != 4 && index_bytes != 8) return fail_arg(h, "index_bytes must be 4 or 8");
    if (n < 0 || m < 0) return fail_arg(h, "negative size");
    if (!nindex || (m > 0 && !nlist)) return fail_arg(h, "null pointer");
    DeviceGuard g(h->device);
    cudaStream_t s = (cudaStream_t)stream;
    {
        ecl_cc_status st = begin_call(h, s);
        if (st != ECL_CC_OK) return st;
        h->last_stream = s;   // every return below follows a synchronisation of `s`
    }
    int flags = 0;
    CK(cudaMemsetAsync(h->flags, 0, sizeof(int), s), "memset");
    const int grid = (int)std::min<long long>(((long long)n + kBlock) / kBlock, 148LL * 8);
    if (index_bytes == 4) {
        validate_offsets_kernel<int><<<grid, kBlock, 0, s>>>(n, m, (const int *)nindex, h->flags);
    } else {
        validate_offsets_kernel<long long><<<grid, kBlock, 0, s>>>(n, m, (const long long *)nindex, h->flags);
    }
    CK(cudaMemcpyAsync(&flags, h->flags, sizeof(int), cudaMemcpyDeviceToHost, s), "D2H");
    CK(cudaStreamSynchronize(s), "sync");
    if (flags) {
        snprintf(h->err, sizeof(h->err), "invalid graph: bad offsets");
        return ECL_CC_ERR_INVALID_GRAPH;
    }
    if (n > 0) {
        if (index_bytes == 4)
            validate_rows_kernel<int><<<grid, kBlock, 0, s>>>(n, (const int *)nindex, nlist, h->flags);
        else
            validate_rows_kernel<long long><<<grid, kBlock, 0, s>>>(n, (const long long *)nindex, nlist, h->flags);
        CK(cudaMemcpyAsync(&flags, h->flags, sizeof(int), cudaMemcpyDeviceToHost, s), "D2H");
        CK(cudaStreamSynchronize(s), "sync");
        if (flags & 2) {
            snprintf(h->err, sizeof(h->err), "invalid graph: neighbour ID out of range");
            return ECL_CC_ERR_INVALID_GRAPH;
        }
        const int sorted = (flags & 8) ? 0 : 1;
        if (index_bytes == 4)
            validate_symmetry_kernel<int><<<grid, kBlock, 0, s>>>(n, (const int *)nindex, nlist, sorted, h->flags);
        else
            validate_symmetry_kernel<long long><<<grid, kBlock, 0, s>>>(n, (const long long *)nindex, nlist, sorted, h->flags);
        CK(cudaMemcpyAsync(&flags, h->flags, sizeof(int), cudaMemcpyDeviceToHost, s), "D2H");
        CK(cudaStreamSynchronize(s), "sync");
        if (flags & 4) {
            snprintf(h->err, sizeof(h->err), "invalid graph: not symmetric");
            return ECL_CC_ERR_INVALID_GRAPH;
        }
    }
    CK(cudaGetLastError(), "validate launch");
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_set_option(ecl_cc_handle h, int option, int64_t value)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    switch (option) {
    case ECL_CC_OPT_THRESH_THREAD:
        if (value < 0 || value > (1 << 30)) return fail_arg(h, "thread threshold");
        h->t1 = (int)value;
        break;
    case ECL_CC_OPT_THRESH_WARP:
        if (value < 0 || value > (1 << 30)) return fail_arg(h, "warp threshold");
        h->t2 = (int)value;
        break;
    case ECL_CC_OPT_GRID_BLOCKS:
        if (value < 0 || value > (1 << 24)) return fail_arg(h, "grid blocks");
        h->grid_blocks = (int)value;
        break;
    case ECL_CC_OPT_STOP_AFTER:
        if (value < 0 || value > 2) return fail_arg(h, "stop_after");
        h->stop_after = (int)value;
        break;
    case ECL_CC_OPT_L2_FETCH: {
        if (value != 0 && value != 32 && value != 64 && value != 128)
            return fail_arg(h, "L2 fetch granularity must be 0, 32, 64 or 128");
        DeviceGuard g(h->device);
        if (value) CK(cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, (size_t)value), "cudaDeviceSetLimit");
        break;
    }
    case ECL_CC_OPT_OCC_THREAD:
        if (value < 0 || value > 64) return fail_arg(h, "occupancy cap");
        h->occ_thread = (int)value;
        break;
    case ECL_CC_OPT_OCC_RANGE:
        if (value < 0 || value > 64) return fail_arg(h, "occupancy cap");
        h->occ_range = (int)value;
        break;
    case ECL_CC_OPT_INIT:
        if (value < 1 || value > 3) return fail_arg(h, "init variant must be 1, 2 or 3");
        h->init_mode = (int)value;
        break;
    case ECL_CC_OPT_JUMP:
        if (value < 1 || value > 4) return fail_arg(h, "jump variant must be 1..4");
        h->jump = (int)value;
        break;
    case ECL_CC_OPT_FINI:
        if (value < 1 || value > 3) return fail_arg(h, "fini variant must be 1, 2 or 3");
        h->fini = (int)value;
        break;
    case ECL_CC_OPT_FILTER:
        if (value < 0 || value > 2) return fail_arg(h, "filter must be 0, 1 or 2");
        h->filter = (int)value;
        break;
    case ECL_CC_OPT_ORDER:
        if (value < 0 || value > 2) return fail_arg(h, "order must be 0, 1 or 2");
        h->order = (int)value;
        break;
    case ECL_CC_OPT_PREJUMP:
        if (value < 0 || value > 2) return fail_arg(h, "prejump must be 0, 1 or 2");
        h->prejump = (int)value;
        break;
    case ECL_CC_OPT_MERGE_FILTER:
        h->merge_filter = value != 0;
        break;
    case ECL_CC_OPT_FUSED:
        if (value < 0 || value > 2) return fail_arg(h, "fused must be 0, 1 or 2");
        h->fused = (int)value;
        break;
    case ECL_CC_OPT_VEC:
        if (value < 0 || value > 2) return fail_arg(h, "vec must be 0, 1 or 2");
        h->vec = (int)value;
        break;
    case ECL_CC_OPT_FUSE_INIT:
        if (value < 0 || value > 2) return fail_arg(h, "fuse_init must be 0, 1 or 2");
        h->fuse_init = (int)value;
        break;
    case ECL_CC_OPT_FLATTEN_PASSES:
        if (value < 0 || value > 2) return fail_arg(h, "flatten_passes must be 0, 1 or 2");
        h->flatten_passes = (int)value;
        break;
    case ECL_CC_OPT_BATCH:
        h->batch = value != 0;
        break;
    case ECL_CC_OPT_TTAS:
        h->ttas = value != 0;
        break;
    case ECL_CC_OPT_TIMING:
        h->timing = value != 0;
        break;
    case ECL_CC_OPT_LOAD_MODE:
        if (value < 0 || value > 3) return fail_arg(h, "load mode");
        h->load_mode = (int)value;
        break;
    default:
        return fail_arg(h, "unknown option");
    }
    if (h->t2 < h->t1) h->t2 = h->t1;
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_get_worklist(ecl_cc_handle h, int32_t *front, int64_t *nfront,
                                  int32_t *back, int64_t *nback)
{
    if (!h) return ECL_CC_ERR_INVALID_ARG;
    DeviceGuard g(h->device);
    cudaStream_t s = h->last_stream;
    unsigned long long c[2] = {0, 0};
    CK(cudaMemcpyAsync(c, h->cnt, sizeof(c), cudaMemcpyDeviceToHost, s), "D2H counters");
    CK(cudaStreamSynchronize(s), "sync");
    const long long nf = (long long)(unsigned)c[0], nb = (long long)(unsigned)c[1];
    if (nfront) *nfront = nf;
    if (nback) *nback = nb;
    if (front && nf > 0)
        CK(cudaMemcpyAsync(front, h->wl, sizeof(int) * nf, cudaMemcpyDeviceToDevice, s), "D2D front");
    if (back && nb > 0)
        CK(cudaMemcpyAsync(back, h->wl + h->cap - nb, sizeof(int) * nb, cudaMemcpyDeviceToDevice, s),
           "D2D back");
    CK(cudaStreamSynchronize(s), "sync");
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_get_run_info(ecl_cc_handle h, int64_t *out, int count)
{
    if (!h || !out || count < 0 || count > 5) return ECL_CC_ERR_INVALID_ARG;
    DeviceGuard g(h->device);
    unsigned long long c[11] = {};
    CK(cudaStreamSynchronize(h->last_stream), "sync");
    CK(cudaMemcpy(c, h->cnt, sizeof(c), cudaMemcpyDeviceToHost), "D2H counters");
    const int *ctl = (const int *)(c + 4);
    const int lazy_flag = (int)(unsigned)c[7];
    const int64_t v[5] = {h->last_lazy == 1 || (h->last_lazy == 2 && lazy_flag) ? 1 : 0,
                          ctl[0] ? 1 : 0, h->gbits_live ? 1 : 0,
                          c[10] ? (int64_t)(unsigned)c[10] : -1, h->last_fused ? 1 : 0};
    for (int i = 0; i < count; i++) out[i] = v[i];
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_get_filter(ecl_cc_handle h, const uint32_t **bits, int64_t *words,
                                int32_t *anchor)
{
    if (!h || !bits || !words || !anchor) return ECL_CC_ERR_INVALID_ARG;
    DeviceGuard g(h->device);
    *bits = h->gbits_live ? h->gbits : nullptr;
    *words = h->gbits_live ? (int64_t)h->gbits_words : 0;
    *anchor = -1;
    if (!h->gbits_live) return ECL_CC_OK;
    unsigned long long a = 0;
    CK(cudaStreamSynchronize(h->last_stream), "sync");
    CK(cudaMemcpy(&a, h->cnt + 10, sizeof(a), cudaMemcpyDeviceToHost), "D2H anchor");
    *anchor = a ? (int32_t)(unsigned)a : -1;
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_get_stats_ex(ecl_cc_handle h, int64_t *out, int count)
{
    if (!h || !out || count < 0 || count > kNumStats) return ECL_CC_ERR_INVALID_ARG;
    DeviceGuard g(h->device);
    unsigned long long c[kNumStats] = {};
    CK(cudaStreamSynchronize(h->last_stream), "sync");
    CK(cudaMemcpy(c, h->cnt + kStatsOff, sizeof(c), cudaMemcpyDeviceToHost), "D2H stats");
    for (int i = 0; i < count; i++) out[i] = (int64_t)c[i];
    return ECL_CC_OK;
}

ecl_cc_status ecl_cc_get_stats(ecl_cc_handle h, int64_t out[4])
{
    return ecl_cc_get_stats_ex(h, out, 4);
}

ecl_cc_status ecl_cc_get_timing(ecl_cc_handle h, float ms[5])
{
    if (!h || !ms) return ECL_CC_ERR_INVALID_ARG;
    if (!h->ev_valid) return fail_arg(h, "no timed full run recorded (set ECL_CC_OPT_TIMING)");
    DeviceGuard g(h->device);
    CK(cudaEventSynchronize(h->ev[5]), "cudaEventSynchronize");
    // phase i spans ev[from[i]] -> ev[to[i]] (the hook kernels may run in reverse order)
    static const int from0[5] = {0, 1, 2, 3, 4}, to0[5] = {1, 2, 3, 4, 5};
    static const int from1[5] = {0, 3, 4, 1, 2}, to1[5] = {1, 2, 3, 4, 5};
    // order 2 (concurrent hook kernels): each kernel's own span (hook_block's on the side
    // stream), so the phases overlap and their sum exceeds the run
    static const int from2[5] = {0, 1, 2, 6, 4}, to2[5] = {1, 2, 3, 7, 5};
    const int *from = h->ev_valid == 2 ? from1 : h->ev_valid == 3 ? from2 : from0;
    const int *to = h->ev_valid == 2 ? to1 : h->ev_valid == 3 ? to2 : to0;
    for (int i = 0; i < 5; i++) CK(cudaEventElapsedTime(&ms[i], h->ev[from[i]], h->ev[to[i]]), "elapsed");
    return ECL_CC_OK;
}

int ecl_cc_stats_enabled(void)
{
#ifdef ECL_CC_STATS
    return 1;
#else
    return 0;
#endif
}

const char *ecl_cc_status_string(ecl_cc_status s)
{
    switch (s) {
    case ECL_CC_OK: return "ok";
    case ECL_CC_ERR_INVALID_ARG: return "invalid argument";
    case ECL_CC_ERR_CUDA: return "CUDA error";
    case ECL_CC_ERR_OOM: return "out of device memory";
    case ECL_CC_ERR_INVALID_GRAPH: return "invalid graph";
    }
    return "unknown status";
}

const char *ecl_cc_last_error(ecl_cc_handle h) { return h ? h->err : "null handle"; }

const char *ecl_cc_version(void) { return kVersion; }

}  // extern "C"
