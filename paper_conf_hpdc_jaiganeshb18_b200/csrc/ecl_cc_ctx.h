// ecl_cc_ctx.h — internal: the handle struct and host helpers shared by the library's
// translation units (ecl_cc.cu: the ECL-CC path; ecl_cc_csr.cu: CSR preparation).
// Not part of the public ABI (include/ecl_cc.h).
#pragma once

#include "ecl_cc.h"

#include <cstdio>
#include <cuda_runtime.h>
#include <unordered_map>

struct ecl_cc_ctx {
    int device = 0;
    int sms = 0;
    // scratch (device, grow-only)
    int *wl = nullptr;
    unsigned *ub = nullptr;
    unsigned *tbits = nullptr;            // R24 thread-bin work bitmap (one bit per row)
    int cap = 0;
    unsigned long long *cnt = nullptr;    // [0..1] worklist counters, [8..9] int
                                          // scheduling counters, [10] R21 anchor,
                                          // [16..31] ECL_CC_STATS counters
    int *flags = nullptr;                 // validate flags
    // end-to-end buffers (device, grow-only)
    void *e2e_index = nullptr;
    size_t e2e_index_bytes = 0;
    int *e2e_list = nullptr;
    size_t e2e_list_n = 0;
    int *e2e_labels = nullptr;
    size_t e2e_labels_n = 0;
    // options
    int t1 = 16, t2 = 352;
    int grid_blocks = 0;
    int occ_thread = 0, occ_range = 0;    // blocks per SM caps (0 = max occupancy)
    int init_mode = 3, jump = 4, fini = 3; // paper ablation variants (defaults = ECL-CC)
    int batch = 1;                        // batched two-hop gathers (R16, R19)
    int filter = 2;                       // R21 membership filter: 0 off, 1 on, 2 auto
    int order = 2;                        // 0 thread, warp, block; 1 block, warp, thread;
                                          // 2 (default) block on a side stream || thread, warp
    cudaStream_t side = nullptr;          // handle-owned stream: hook_block under order 2,
                                          //   and the stream destroy() frees on
    cudaEvent_t fork = nullptr, join = nullptr;
    cudaEvent_t done = nullptr;           // recorded at the end of every enqueueing call
    bool done_valid = false;
    int prejump = 2;                      // R23 pointer-doubling passes: 0 off, 1 on, 2 auto
    int fuse_init = 2;                    // R28 lazy Init3: 0 off, 1 on, 2 auto (m >= 16n)
    int flatten_passes = 0;               // ecl_cc_finalize: R23 passes first (0 off,
                                          //   1 always, 2 if the depth probe finds it deep)
    int *fa = nullptr, *fb = nullptr;     // spanning-forest outputs of the current call
    // CSR builder scratch (ecl_cc_build_csr; device, grow-only)
    void *csr_tmp = nullptr;
    size_t csr_tmp_bytes = 0;
    unsigned *gbits = nullptr;            // R21 bitmap (grow-only)
    size_t gbits_words = 0;
    bool gbits_live = false;              // the last run used the R21 bitmap
    int last_lazy = 0;                    // the last run's R28 mode (0 off, 1 on, 2 probe)
    int merge_filter = 0;                 // merge_encoded / finalize use the last run's R21
                                          //   bitmap as membership proofs (multi-GPU)
    int vec = 2;                          // R31 quad engine: 0 off, 1 both range kernels,
                                          //   2 hook_warp with int32 offsets
    int fused = 2;                        // R33 single launch: 0 off, 1 on, 2 small graphs
    bool last_fused = false;              // the last run took the single-launch path
    int stop_after = 0;
    int load_mode = 1;
    int ttas = 1;                         // test-and-test-and-set hooks
    int timing = 0;                       // record per-kernel CUDA events
    cudaEvent_t ev[8] = {};               // phase ends on the run's stream; [6..7] side stream
    int ev_valid = 0;
    // last run (for ecl_cc_get_worklist)
    cudaStream_t last_stream = nullptr;
    std::unordered_map<const void *, int> occ;
    char err[512] = {0};
};

namespace eclcc_host {

inline ecl_cc_status fail_cuda(ecl_cc_handle h, cudaError_t e, const char *where)
{
    if (h) snprintf(h->err, sizeof(h->err), "%s: %s (%s)", where, cudaGetErrorString(e),
                    cudaGetErrorName(e));
    return e == cudaErrorMemoryAllocation ? ECL_CC_ERR_OOM : ECL_CC_ERR_CUDA;
}

inline ecl_cc_status fail_arg(ecl_cc_handle h, const char *msg)
{
    if (h) snprintf(h->err, sizeof(h->err), "invalid argument: %s", msg);
    return ECL_CC_ERR_INVALID_ARG;
}

#define CK(call, where)                                      \
    do {                                                     \
        cudaError_t e_ = (call);                             \
        if (e_ != cudaSuccess) return fail_cuda(h, e_, where); \
    } while (0)

// Stream ordering of the handle's scratch across calls.  begin_call: a call on a stream
// other than the previous call's waits for that call (the scratch is shared), end_call:
// record where this call ends.  Skipped while `s` is being captured into a CUDA graph
// (the graph replays in the capturing stream's order).
inline bool capturing(cudaStream_t s)
{
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    return cudaStreamIsCapturing(s, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone;
}

inline ecl_cc_status begin_call(ecl_cc_handle h, cudaStream_t s)
{
    if (h->done_valid && h->last_stream != s && !capturing(s))
        CK(cudaStreamWaitEvent(s, h->done, 0), "wait for the handle's previous call");
    return ECL_CC_OK;
}

inline ecl_cc_status end_call(ecl_cc_handle h, cudaStream_t s)
{
    h->last_stream = s;
    if (capturing(s)) return ECL_CC_OK;
    CK(cudaEventRecord(h->done, s), "record call end");
    h->done_valid = true;
    return ECL_CC_OK;
}

// Make `dev` current for the duration of a call, restoring the caller's device.
struct DeviceGuard {
    int prev = -1;
    bool ok = true;
    explicit DeviceGuard(int dev)
    {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != dev) ok = cudaSetDevice(dev) == cudaSuccess;
    }
    ~DeviceGuard()
    {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};

}  // namespace eclcc_host
