// cc_comm.cu -- multi-GPU exchange steps of the hot path (S§8(e)) behind the C
// ABI: NCCL over NVLink / NVSwitch, one communicator per process (one process
// per GPU).  libnccl is resolved at run time (dlopen of the copy the process
// already maps -- PyTorch's -- or CC_NCCL_LIBRARY), so the library itself has
// no link-time NCCL dependency and loads on machines without it.
#include "../../include/ctaclust.h"

#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>

extern "C" __attribute__((visibility("hidden"))) cc_status cc_internal_fail(cc_status s, const char* msg);  // ctaclust.cu

namespace {

struct Nccl {
    bool ok = false;
    std::string why;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

Nccl& nccl() {
    static Nccl n;
    static std::once_flag once;
    std::call_once(once, [] {
        const char* env = getenv("CC_NCCL_LIBRARY");
        void* h = dlopen(env ? env : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
        if (!h) h = dlopen(env ? env : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) { n.why = std::string("cannot load libnccl.so.2: ") + dlerror(); return; }
#define SYM(field, name)                                                     \
        *(void**)&n.field = dlsym(h, name);                                  \
        if (!n.field) { n.why = std::string("missing symbol ") + name; return; }
        SYM(GetUniqueId, "ncclGetUniqueId");
        SYM(CommInitRank, "ncclCommInitRank");
        SYM(CommDestroy, "ncclCommDestroy");
        SYM(AllReduce, "ncclAllReduce");
        SYM(AllGather, "ncclAllGather");
        SYM(Send, "ncclSend");
        SYM(Recv, "ncclRecv");
        SYM(GroupStart, "ncclGroupStart");
        SYM(GroupEnd, "ncclGroupEnd");
        SYM(GetErrorString, "ncclGetErrorString");
#undef SYM
        n.ok = true;
    });
    return n;
}

cc_status nfail(ncclResult_t r, const char* what) {
    char buf[256];
    snprintf(buf, sizeof buf, "%s: %s", what, nccl().GetErrorString ? nccl().GetErrorString(r) : "nccl error");
    return cc_internal_fail(CC_ERR_NCCL, buf);
}

}  // namespace

struct cc_comm_s {
    ncclComm_t comm = nullptr;
    int nranks = 0, rank = 0, device = 0;
};

#define NCCL_TRY(call, what)                                   \
    do {                                                       \
        ncclResult_t r_ = (call);                              \
        if (r_ != ncclSuccess) return nfail(r_, what);         \
    } while (0)
#define NEED_NCCL()                                                                       \
    do {                                                                                  \
        if (!nccl().ok) return cc_internal_fail(CC_ERR_UNSUPPORTED, nccl().why.c_str());  \
    } while (0)

extern "C" cc_status cc_comm_unique_id(void* id) {
    if (!id) return cc_internal_fail(CC_ERR_INVALID_ARG, "null id");
    NEED_NCCL();
    ncclUniqueId u;
    NCCL_TRY(nccl().GetUniqueId(&u), "ncclGetUniqueId");
    memcpy(id, &u, sizeof u);
    return CC_OK;
}

extern "C" cc_status cc_comm_init(const void* id, int32_t nranks, int32_t rank, int32_t device, cc_comm* out) {
    if (!id || !out || nranks < 1 || rank < 0 || rank >= nranks || device < 0)
        return cc_internal_fail(CC_ERR_INVALID_ARG, "bad communicator arguments");
    *out = nullptr;
    NEED_NCCL();
    int prev = 0;
    cudaGetDevice(&prev);
    if (cudaSetDevice(device) != cudaSuccess) return cc_internal_fail(CC_ERR_CUDA, "cudaSetDevice");
    ncclUniqueId u;
    memcpy(&u, id, sizeof u);
    cc_comm_s* c = new cc_comm_s();
    c->nranks = nranks; c->rank = rank; c->device = device;
    ncclResult_t r = nccl().CommInitRank(&c->comm, nranks, u, rank);
    cudaSetDevice(prev);
    if (r != ncclSuccess) { delete c; return nfail(r, "ncclCommInitRank"); }
    *out = c;
    return CC_OK;
}

extern "C" cc_status cc_comm_destroy(cc_comm c) {
    if (!c) return CC_OK;
    if (c->comm && nccl().ok) nccl().CommDestroy(c->comm);
    delete c;
    return CC_OK;
}

// Slab halo exchange (Jacobi / conv2d slab sharding): the local slab holds
// `rows` rows of leading dimension ld; rows [0, halo) mirror the previous
// rank's last owned rows and rows [rows-halo, rows) the next rank's first
// owned rows (none at the global edges).  One grouped send/recv pair per
// neighbour, row-contiguous when ld == cols, else row by row.
extern "C" cc_status cc_halo_exchange(cc_comm c, float* slab, int64_t ld, int32_t rows, int32_t cols,
                                      int32_t halo, void* stream) {
    if (!c || !slab || rows < 0 || cols < 0 || ld < cols || halo < 0 || rows < 2 * halo)
        return cc_internal_fail(CC_ERR_INVALID_ARG, "bad halo exchange arguments");
    if (c->nranks == 1 || halo == 0) return CC_OK;
    NEED_NCCL();
    cudaStream_t st = (cudaStream_t)stream;
    const bool up = c->rank > 0, dn = c->rank < c->nranks - 1;
    const int own0 = up ? halo : 0;                          // first owned local row
    const int own1 = dn ? rows - halo : rows;                // one past the last owned row
    NCCL_TRY(nccl().GroupStart(), "ncclGroupStart");
    for (int k = 0; k < halo; ++k) {
        const size_t n = (size_t)cols;
        if (up) {
            NCCL_TRY(nccl().Send(slab + (int64_t)(own0 + k) * ld, n, ncclFloat32, c->rank - 1, c->comm, st), "ncclSend");
            NCCL_TRY(nccl().Recv(slab + (int64_t)k * ld, n, ncclFloat32, c->rank - 1, c->comm, st), "ncclRecv");
        }
        if (dn) {
            NCCL_TRY(nccl().Send(slab + (int64_t)(own1 - halo + k) * ld, n, ncclFloat32, c->rank + 1, c->comm, st), "ncclSend");
            NCCL_TRY(nccl().Recv(slab + (int64_t)(own1 + k) * ld, n, ncclFloat32, c->rank + 1, c->comm, st), "ncclRecv");
        }
    }
    NCCL_TRY(nccl().GroupEnd(), "ncclGroupEnd");
    return CC_OK;
}

extern "C" cc_status cc_allreduce_sum(cc_comm c, float* buf, size_t count, void* stream) {
    if (!c || (!buf && count)) return cc_internal_fail(CC_ERR_INVALID_ARG, "bad all-reduce arguments");
    if (c->nranks == 1 || count == 0) return CC_OK;
    NEED_NCCL();
    NCCL_TRY(nccl().AllReduce(buf, buf, count, ncclFloat32, ncclSum, c->comm, (cudaStream_t)stream), "ncclAllReduce");
    return CC_OK;
}

extern "C" cc_status cc_allgather(cc_comm c, const float* send, float* recv, size_t count_per_rank, void* stream) {
    if (!c || ((!send || !recv) && count_per_rank)) return cc_internal_fail(CC_ERR_INVALID_ARG, "bad all-gather arguments");
    if (count_per_rank == 0) return CC_OK;
    if (c->nranks == 1) {
        if (send != recv && cudaMemcpyAsync(recv, send, count_per_rank * 4, cudaMemcpyDeviceToDevice, (cudaStream_t)stream) != cudaSuccess)
            return cc_internal_fail(CC_ERR_CUDA, "cudaMemcpyAsync");
        return CC_OK;
    }
    NEED_NCCL();
    NCCL_TRY(nccl().AllGather(send, recv, count_per_rank, ncclFloat32, c->comm, (cudaStream_t)stream), "ncclAllGather");
    return CC_OK;
}
