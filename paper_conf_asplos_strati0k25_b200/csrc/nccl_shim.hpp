// nccl_shim.hpp — the library's own NCCL communicator for the commit collective (C1 of
// SURVEY §2.3): an 8-byte ncclAllReduce (MIN / MAX, int64) over NVLink / NVSwitch.
// This replaces the paper's "send curr_counter to rank 0 and wait for the notify"
// (§4.1) with one allreduce (reading R9).
//
// libnccl.so.2 is dlopen'ed on first use so the library loads (and its CPU tests run)
// where NCCL or a GPU is absent; world == 1 never touches NCCL.
#pragma once
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <cstdint>
#include <cstring>

#include "../../include/pccheck.h"
#include "errors.hpp"

#ifndef PCC_NCCL_LIBDIR
#define PCC_NCCL_LIBDIR ""
#endif

namespace pcc {

struct NcclApi {
    void *h = nullptr;
    ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*AllReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*AllGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    const char *(*GetErrorString)(ncclResult_t) = nullptr;

    static NcclApi &get() {
        static NcclApi a;
        return a;
    }
    int load() {
        if (h) return PCC_OK;
        const char *cands[] = {"libnccl.so.2", PCC_NCCL_LIBDIR "/libnccl.so.2", "libnccl.so"};
        for (const char *p : cands) {
            if (!p || !*p) continue;
            h = dlopen(p, RTLD_NOW | RTLD_GLOBAL);
            if (h) break;
        }
        if (!h) return set_error(PCC_ENCCL, "cannot dlopen libnccl.so.2");
        GetUniqueId = (decltype(GetUniqueId))dlsym(h, "ncclGetUniqueId");
        CommInitRank = (decltype(CommInitRank))dlsym(h, "ncclCommInitRank");
        AllReduce = (decltype(AllReduce))dlsym(h, "ncclAllReduce");
        AllGather = (decltype(AllGather))dlsym(h, "ncclAllGather");
        CommDestroy = (decltype(CommDestroy))dlsym(h, "ncclCommDestroy");
        GetErrorString = (decltype(GetErrorString))dlsym(h, "ncclGetErrorString");
        if (!GetUniqueId || !CommInitRank || !AllReduce || !AllGather || !CommDestroy)
            return set_error(PCC_ENCCL, "libnccl.so.2 lacks symbols");
        return PCC_OK;
    }
};

struct NcclComm {
    ncclComm_t comm = nullptr;
    enum Op { kMin, kMax };

    int init(const void *uid, int world, int rank) {
        NcclApi &a = NcclApi::get();
        int rc = a.load();
        if (rc) return rc;
        ncclUniqueId id;
        std::memcpy(&id, uid, sizeof id);
        ncclResult_t r = a.CommInitRank(&comm, world, id, rank);
        if (r != ncclSuccess) return set_error(PCC_ENCCL, a.GetErrorString ? a.GetErrorString(r) : "init");
        return PCC_OK;
    }
    // in-place host vector v[count] -> allreduce -> v; synchronous on s
    int allreduce_i64(int64_t *v, size_t count, Op op, int64_t *dev, int64_t *pinned, cudaStream_t s) {
        NcclApi &a = NcclApi::get();
        std::memcpy(pinned, v, count * sizeof(int64_t));
        cudaMemcpyAsync(dev, pinned, count * sizeof(int64_t), cudaMemcpyHostToDevice, s);
        ncclResult_t r = a.AllReduce(dev, dev, count, ncclInt64, op == kMin ? ncclMin : ncclMax, comm, s);
        if (r != ncclSuccess) return set_error(PCC_ENCCL, a.GetErrorString ? a.GetErrorString(r) : "allreduce");
        cudaMemcpyAsync(pinned, dev, count * sizeof(int64_t), cudaMemcpyDeviceToHost, s);
        if (cudaStreamSynchronize(s) != cudaSuccess) return set_error(PCC_ECUDA, "allreduce sync");
        std::memcpy(v, pinned, count * sizeof(int64_t));
        return PCC_OK;
    }
    int allgather(const void *send, void *recv, size_t bytes, cudaStream_t s) {
        NcclApi &a = NcclApi::get();
        ncclResult_t r = a.AllGather(send, recv, bytes, ncclUint8, comm, s);
        if (r != ncclSuccess) return set_error(PCC_ENCCL, a.GetErrorString ? a.GetErrorString(r) : "allgather");
        return PCC_OK;
    }
    void destroy() {
        if (comm) NcclApi::get().CommDestroy(comm);
        comm = nullptr;
    }
};

}  // namespace pcc

extern "C" inline int pcc_nccl_unique_id_impl(void *out128) {
    pcc::NcclApi &a = pcc::NcclApi::get();
    int rc = a.load();
    if (rc) return rc;
    ncclUniqueId id;
    if (a.GetUniqueId(&id) != ncclSuccess) return pcc::set_error(PCC_ENCCL, "ncclGetUniqueId");
    std::memcpy(out128, &id, sizeof id);
    return PCC_OK;
}
