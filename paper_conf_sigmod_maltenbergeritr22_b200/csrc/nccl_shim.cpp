// nccl_shim.cpp - NCCL point-to-point for the swap of the P2P sort's merge
// stages (exchange mode 4: "the swap of pivot-split ranges
// between GPU pairs, using NCCL send/recv over NVLink"; paper §5.2
// swaps with cudaMemcpyPeer).  libnccl is opened at run time (dlopen of
// libnccl.so.2: the copy torch already loaded, else the system one), so the
// library has no link-time NCCL dependency; every failure is reported as
// MSORT_ERR_NCCL by the caller.
#include "nccl_shim.h"

#include <dlfcn.h>

#include <cstdlib>
#include <cstring>
#include <mutex>

namespace msort {

namespace {

struct NcclApi {
    bool ok = false;
    std::string err;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommInitAll)(ncclComm_t*, int, const int*) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
    ncclResult_t (*GetVersion)(int*) = nullptr;
};

NcclApi g_api;
std::once_flag g_once;

template <typename F>
bool sym(void* h, const char* name, F& f) {
    f = reinterpret_cast<F>(dlsym(h, name));
    return f != nullptr;
}

void load_api() {
    const char* env = std::getenv("MSORT_NCCL_LIB");
    const char* names[] = {env, "libnccl.so.2", "libnccl.so"};
    void* h = nullptr;
    for (const char* nm : names) {
        if (!nm) continue;
        h = dlopen(nm, RTLD_NOW | RTLD_GLOBAL);
        if (h) break;
    }
    if (!h) {
        const char* why = dlerror();  // (dlerror clears the message: read it once)
        g_api.err = std::string("dlopen libnccl.so.2 failed: ") + (why ? why : "?");
        return;
    }
    bool ok = sym(h, "ncclGetUniqueId", g_api.GetUniqueId) && sym(h, "ncclCommInitRank", g_api.CommInitRank) &&
              sym(h, "ncclCommInitAll", g_api.CommInitAll) && sym(h, "ncclCommDestroy", g_api.CommDestroy) &&
              sym(h, "ncclGroupStart", g_api.GroupStart) && sym(h, "ncclGroupEnd", g_api.GroupEnd) &&
              sym(h, "ncclSend", g_api.Send) && sym(h, "ncclRecv", g_api.Recv) &&
              sym(h, "ncclGetErrorString", g_api.GetErrorString) && sym(h, "ncclGetVersion", g_api.GetVersion);
    if (!ok) {
        g_api.err = "libnccl lacks a p2p symbol";
        return;
    }
    g_api.ok = true;
}

bool api(std::string* err) {
    std::call_once(g_once, load_api);
    if (!g_api.ok && err) *err = g_api.err;
    return g_api.ok;
}

bool check(ncclResult_t r, const char* what, std::string* err) {
    if (r == ncclSuccess) return true;
    if (err) *err = std::string(what) + ": " + (g_api.GetErrorString ? g_api.GetErrorString(r) : "nccl error");
    return false;
}

}  // namespace

int nccl_version() {
    int v = 0;
    if (!api(nullptr) || g_api.GetVersion(&v) != ncclSuccess) return 0;
    return v;
}

bool nccl_unique_id(void* out, std::string* err) {
    if (!api(err)) return false;
    ncclUniqueId id;
    if (!check(g_api.GetUniqueId(&id), "ncclGetUniqueId", err)) return false;
    std::memcpy(out, &id, sizeof(id));
    return true;
}

bool nccl_init_all(NcclState& s, const int* devs, int ndev, std::string* err) {
    if (!api(err)) return false;
    s.comms.assign(ndev, nullptr);
    if (!check(g_api.CommInitAll(s.comms.data(), ndev, devs), "ncclCommInitAll", err)) {
        s.comms.clear();
        return false;
    }
    return true;
}

bool nccl_init_rank(NcclState& s, int nranks, const void* id, int rank, std::string* err) {
    if (!api(err)) return false;
    ncclUniqueId uid;
    std::memcpy(&uid, id, sizeof(uid));
    s.comms.assign(1, nullptr);
    if (!check(g_api.CommInitRank(&s.comms[0], nranks, uid, rank), "ncclCommInitRank", err)) {
        s.comms.clear();
        return false;
    }
    return true;
}

void nccl_destroy(NcclState& s) {
    if (g_api.ok)
        for (ncclComm_t c : s.comms)
            if (c) g_api.CommDestroy(c);
    s.comms.clear();
}

bool nccl_group(const NcclState& s, const std::vector<P2POp>& ops, std::string* err) {
    if (!api(err)) return false;
    if (!check(g_api.GroupStart(), "ncclGroupStart", err)) return false;
    bool ok = true;
    for (const P2POp& op : ops) {
        if (!ok) break;
        ncclComm_t comm = s.comms[op.comm];
        if (op.send)
            ok = check(g_api.Send(op.buf, op.bytes, ncclUint8, op.peer, comm, op.stream), "ncclSend", err);
        else
            ok = check(g_api.Recv(const_cast<void*>(op.buf), op.bytes, ncclUint8, op.peer, comm, op.stream), "ncclRecv",
                       err);
    }
    const ncclResult_t r = g_api.GroupEnd();
    return check(r, "ncclGroupEnd", err) && ok;
}

}  // namespace msort
