// transport_nccl.cpp -- NCCL point-to-point transport over NVLink / NVSwitch.
//
// The communicator is borrowed (e.g. torch ProcessGroupNCCL._comm_ptr()), so
// libes must call into the SAME libnccl instance that created it: the
// library is resolved with dlopen(RTLD_NOLOAD) first, falling back to a
// normal dlopen of "libnccl.so.2".  Only ncclGroupStart/End + ncclSend/Recv
// are used (bytes as ncclUint8).
#include <dlfcn.h>

#include <vector>

#include "nccl.h"
#include "transport.h"

namespace es {
namespace {

struct NcclApi {
  bool ok = false;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  ncclResult_t (*Send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*CommCount)(const ncclComm_t, int *) = nullptr;
  ncclResult_t (*CommUserRank)(const ncclComm_t, int *) = nullptr;
  const char *(*GetErrorString)(ncclResult_t) = nullptr;
};

NcclApi *api(std::string *err) {
  static NcclApi a;
  static bool tried = false;
  if (tried) {
    if (!a.ok && err) *err = "libnccl.so.2 could not be loaded";
    return a.ok ? &a : nullptr;
  }
  tried = true;
  void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) {
    if (err) *err = std::string("dlopen libnccl.so.2 failed: ") + dlerror();
    return nullptr;
  }
#define ES_SYM(field, name)                                             \
  a.field = reinterpret_cast<decltype(a.field)>(dlsym(h, name));        \
  if (!a.field) {                                                       \
    if (err) *err = std::string("libnccl.so.2 lacks ") + name;          \
    return nullptr;                                                     \
  }
  ES_SYM(GroupStart, "ncclGroupStart");
  ES_SYM(GroupEnd, "ncclGroupEnd");
  ES_SYM(Send, "ncclSend");
  ES_SYM(Recv, "ncclRecv");
  ES_SYM(CommCount, "ncclCommCount");
  ES_SYM(CommUserRank, "ncclCommUserRank");
  ES_SYM(GetErrorString, "ncclGetErrorString");
#undef ES_SYM
  a.ok = true;
  return &a;
}

class NcclTransport : public Transport {
 public:
  NcclTransport(NcclApi *a, ncclComm_t c) : a_(a), comm_(c) {}
  es_status group_begin() override {
    ops_.clear();
    return ES_OK;
  }
  es_status send(const void *p, size_t bytes, int peer) override {
    ops_.push_back({true, const_cast<void *>(p), bytes, peer});
    return ES_OK;
  }
  es_status recv(void *p, size_t bytes, int peer) override {
    ops_.push_back({false, p, bytes, peer});
    return ES_OK;
  }
  es_status group_end(cudaStream_t s) override {
    if (ops_.empty()) return ES_OK;
    ncclResult_t r = a_->GroupStart();
    if (r != ncclSuccess) return fail(r);
    for (const P2P &o : ops_) {
      r = o.send ? a_->Send(o.p, o.bytes, ncclUint8, o.peer, comm_, s)
                 : a_->Recv(o.p, o.bytes, ncclUint8, o.peer, comm_, s);
      if (r != ncclSuccess) {
        a_->GroupEnd();
        return fail(r);
      }
    }
    r = a_->GroupEnd();
    ops_.clear();
    if (r != ncclSuccess) return fail(r);
    return ES_OK;
  }

 private:
  struct P2P {
    bool send;
    void *p;
    size_t bytes;
    int peer;
  };
  es_status fail(ncclResult_t r) {
    err = std::string("NCCL: ") + a_->GetErrorString(r);
    ops_.clear();
    return ES_ENCCL;
  }
  NcclApi *a_;
  ncclComm_t comm_;
  std::vector<P2P> ops_;
};

}  // namespace

Transport *make_nccl_transport(void *comm, int G, int rank, std::string *err) {
  NcclApi *a = api(err);
  if (!a) return nullptr;
  ncclComm_t c = reinterpret_cast<ncclComm_t>(comm);
  int n = -1, r = -1;
  if (a->CommCount(c, &n) != ncclSuccess || a->CommUserRank(c, &r) != ncclSuccess) {
    if (err) *err = "ncclCommCount/ncclCommUserRank failed on the given comm";
    return nullptr;
  }
  if (n != G || r != rank) {
    if (err) *err = "NCCL communicator size/rank does not match config G/rank";
    return nullptr;
  }
  return new NcclTransport(a, c);
}

}  // namespace es
