// ts_timeline.cu -- canonical order of a recorded R23 timeline (R23): tasks by (gpu, prog),
// flows by (release_s, code).  The K3 LOG instantiation appends records in the order lanes reach them;
// this device sort makes the output independent of that order.
#include <cuda_runtime.h>
#include <thrust/execution_policy.h>
#include <thrust/sort.h>
#include "ts_internal.h"

namespace ts {

struct TaskLess {
    __host__ __device__ bool operator()(const triosim_task_rec &x, const triosim_task_rec &y) const {
        return x.gpu != y.gpu ? x.gpu < y.gpu : x.prog < y.prog;
    }
};
struct FlowLess {
    __host__ __device__ bool operator()(const triosim_flow_rec &x, const triosim_flow_rec &y) const {
        return x.release_s != y.release_s ? x.release_s < y.release_s : x.code < y.code;
    }
};

cudaError_t sort_timeline(triosim_task_rec *tasks, uint64_t nt, triosim_flow_rec *flows, uint64_t nf, cudaStream_t s) {
    if (nt > 1) thrust::sort(thrust::cuda::par.on(s), tasks, tasks + nt, TaskLess());
    if (nf > 1) thrust::sort(thrust::cuda::par.on(s), flows, flows + nf, FlowLess());
    return cudaGetLastError();
}

}  // namespace ts
