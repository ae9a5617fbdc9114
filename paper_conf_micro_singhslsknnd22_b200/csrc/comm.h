// comm.h - K5: batch-sharded data parallelism.
// A library-owned NCCL communicator, resolved with dlopen so the library loads (and its CPU
// tests run) without NCCL; over NVLink 5 / NVSwitch on the B200 box.  Two collectives per step:
// allreduce(s_t, int64) before SST so every rank computes the same keep mask, and
// allreduce(dW, fp32) before Adam.
#pragma once
#include <cstddef>
#include <string>
#include <cuda_runtime.h>

namespace sk {

// Host allreduce callback (skipper_comm_init_callback): sums `count` elements of dtype (0 f32, 1 f64,
// 2 i64) at buf over all ranks in place, ordered after the work already issued to `stream` and complete
// before it returns; 0 = success.  Exercises the multi-rank schedule where NCCL cannot run (one GPU, CPU
// process groups in tests).
typedef int (*AllreduceFn)(void *buf, size_t count, int dtype, void *stream, void *user);

struct Comm {
    void *comm = nullptr;  // ncclComm_t (or this Comm itself in callback mode: non-null = active)
    int rank = 0, world = 1;
    AllreduceFn cb = nullptr;
    void *cb_user = nullptr;
    bool init_callback(AllreduceFn fn, void *user, int rank, int world, std::string *err);
    static bool unique_id(unsigned char id[128], std::string *err);
    bool init(const unsigned char id[128], int rank, int world, std::string *err);
    bool allreduce_i64(long long *buf, size_t n, cudaStream_t s, std::string *err);
    bool allreduce_f32(float *buf, size_t n, cudaStream_t s, std::string *err);
    bool allreduce_f64(double *buf, size_t n, cudaStream_t s, std::string *err);
    void destroy();
};

}  // namespace sk
