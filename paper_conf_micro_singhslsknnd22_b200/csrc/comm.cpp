// comm.cpp - NCCL entry points resolved at run time (see comm.h).
#include "comm.h"

#include <dlfcn.h>
#include <cstring>
#include <mutex>

#include <nccl.h>

namespace sk {
namespace {

struct Nccl {
    void *h = nullptr;
    decltype(&ncclGetUniqueId) getUniqueId = nullptr;
    decltype(&ncclCommInitRank) commInitRank = nullptr;
    decltype(&ncclAllReduce) allReduce = nullptr;
    decltype(&ncclCommDestroy) commDestroy = nullptr;
    decltype(&ncclGetErrorString) errStr = nullptr;
    bool ok = false;
};

Nccl &nccl() {
    static Nccl n;
    static std::once_flag once;
    std::call_once(once, [] {
        const char *names[] = {"libnccl.so.2", "libnccl.so"};
        for (const char *nm : names) {
            n.h = dlopen(nm, RTLD_NOW | RTLD_GLOBAL);
            if (n.h) break;
        }
        if (!n.h) return;
        n.getUniqueId = reinterpret_cast<decltype(n.getUniqueId)>(dlsym(n.h, "ncclGetUniqueId"));
        n.commInitRank = reinterpret_cast<decltype(n.commInitRank)>(dlsym(n.h, "ncclCommInitRank"));
        n.allReduce = reinterpret_cast<decltype(n.allReduce)>(dlsym(n.h, "ncclAllReduce"));
        n.commDestroy = reinterpret_cast<decltype(n.commDestroy)>(dlsym(n.h, "ncclCommDestroy"));
        n.errStr = reinterpret_cast<decltype(n.errStr)>(dlsym(n.h, "ncclGetErrorString"));
        n.ok = n.getUniqueId && n.commInitRank && n.allReduce && n.commDestroy && n.errStr;
    });
    return n;
}

bool check(ncclResult_t r, const char *what, std::string *err) {
    if (r == ncclSuccess) return true;
    if (err) *err = std::string(what) + ": " + (nccl().errStr ? nccl().errStr(r) : "nccl error");
    return false;
}

}  // namespace

bool Comm::unique_id(unsigned char id[128], std::string *err) {
    Nccl &n = nccl();
    if (!n.ok) {
        if (err) *err = "libnccl.so.2 not found (dlopen)";
        return false;
    }
    ncclUniqueId u;
    if (!check(n.getUniqueId(&u), "ncclGetUniqueId", err)) return false;
    static_assert(sizeof(u) == 128, "ncclUniqueId is 128 bytes");
    std::memcpy(id, &u, 128);
    return true;
}

bool Comm::init(const unsigned char id[128], int r, int w, std::string *err) {
    Nccl &n = nccl();
    if (!n.ok) {
        if (err) *err = "libnccl.so.2 not found (dlopen)";
        return false;
    }
    ncclUniqueId u;
    std::memcpy(&u, id, 128);
    ncclComm_t c = nullptr;
    if (!check(n.commInitRank(&c, w, u, r), "ncclCommInitRank", err)) return false;
    comm = c;
    rank = r;
    world = w;
    return true;
}

bool Comm::init_callback(AllreduceFn fn, void *user, int r, int w, std::string *err) {
    if (!fn) {
        if (err) *err = "null allreduce callback";
        return false;
    }
    cb = fn;
    cb_user = user;
    comm = this;
    rank = r;
    world = w;
    return true;
}

static bool run_cb(const Comm &c, void *buf, size_t cnt, int dtype, cudaStream_t s, const char *what,
                   std::string *err) {
    if (c.cb(buf, cnt, dtype, s, c.cb_user) == 0) return true;
    if (err) *err = std::string(what) + ": allreduce callback failed";
    return false;
}

bool Comm::allreduce_i64(long long *buf, size_t cnt, cudaStream_t s, std::string *err) {
    if (cb) return run_cb(*this, buf, cnt, 2, s, "allreduce(s)", err);
    return check(nccl().allReduce(buf, buf, cnt, ncclInt64, ncclSum, static_cast<ncclComm_t>(comm), s),
                 "ncclAllReduce(s)", err);
}

bool Comm::allreduce_f64(double *buf, size_t cnt, cudaStream_t s, std::string *err) {
    if (cb) return run_cb(*this, buf, cnt, 1, s, "allreduce(u2)", err);
    return check(nccl().allReduce(buf, buf, cnt, ncclFloat64, ncclSum, static_cast<ncclComm_t>(comm), s),
                 "ncclAllReduce(u2)", err);
}

bool Comm::allreduce_f32(float *buf, size_t cnt, cudaStream_t s, std::string *err) {
    if (cb) return run_cb(*this, buf, cnt, 0, s, "allreduce(dW)", err);
    return check(nccl().allReduce(buf, buf, cnt, ncclFloat32, ncclSum, static_cast<ncclComm_t>(comm), s),
                 "ncclAllReduce(dW)", err);
}

void Comm::destroy() {
    if (comm && !cb && nccl().ok) nccl().commDestroy(static_cast<ncclComm_t>(comm));
    comm = nullptr;
    cb = nullptr;
    cb_user = nullptr;
    world = 1;
    rank = 0;
}

}  // namespace sk
