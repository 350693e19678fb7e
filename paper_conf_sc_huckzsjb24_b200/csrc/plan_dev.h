// Device-side planning (step a2 on the GPU, plan_dev.cu).  Not part of the C ABI.
#pragma once

#include <cuda_runtime.h>

#include <functional>
#include <vector>

#include "kernel.cuh"

namespace cusan {

// Range sizing rules of build_span_tables (check_api.cpp), passed to the device planner.
struct DevPlanArgs {
    uint64_t R_MIN, R_MAX, R_PER_ACC, R_BAL_MIN, R_PER_WARP, TAIL_PCT, TAIL_DIV;
    int max_blocks;
};

// Device memory of one device plan: scratch and the tables the check reads (inc, span tables),
// plus the stream the planning kernels run on (a plan is built while another check may run on its
// own stream).  Pooled per device (plan_dev_acquire / plan_dev_release): no allocation per plan
// once warm.
struct DevScratch {
    int device = 0;
    cudaStream_t stream = nullptr;
    char* a = nullptr;          // per-access buffers (pooled: held only while planning)
    uint64_t a_cap = 0;
    char* b = nullptr;          // per-incidence / per-span buffers (pooled: held only while planning)
    uint64_t b_cap = 0;
    char* o = nullptr;          // the output tables the check reads (kept with the plan)
    uint64_t o_cap = 0;
    unsigned long long* hdr_host = nullptr;   // pinned
    std::vector<WinDesc> wins_host;
    ~DevScratch();
};

struct DevPlanOut {
    const AccRec* inc = nullptr;      // incidence table (device)
    const DSpan* ds = nullptr;        // span tables of every window, each with its sentinel (device)
    std::vector<WinDesc> wins;        // non-empty windows
    uint64_t n_intervals = 0, n_inc = 0, n_ds = 0, n_spans = 0, shadow_cells = 0, shard_granules = 0, d_lo = 0;
    uint64_t tracked_bytes_shard = 0, rec_units = 0, spill_spans = 0, cell_bytes = 0;
    bool need_shadow = false;
    uint64_t h2d_bytes = 0, launches = 0;
};

// a2 on S.stream (waits for it) from the accesses' granule ranges (hp.acc_g0 / acc_g1) and a1's
// records.  host_a1 (if given) runs a1 on the host while the device's first phase — which needs
// only the ranges — builds the intervals; otherwise a1 must be done already.
int device_plan_a2(HostPlan& hp, const DevPlanArgs& args, DevScratch& S, DevPlanOut& out,
                   const std::function<int()>& host_a1 = nullptr);

DevScratch* plan_dev_acquire(int device);      // nullptr: no memory / stream
void plan_dev_release(DevScratch* s);          // the caller's work on it is complete
void plan_dev_release_all();                   // frees every pooled scratch and planning buffer

}  // namespace cusan
