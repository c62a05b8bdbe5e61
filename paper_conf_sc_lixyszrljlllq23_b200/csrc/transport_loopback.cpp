// transport_loopback.cpp -- in-process transport for testing every G and
// EST->GPU mapping on ONE GPU.
//
// All G ranks live in one process, each driven by its own host thread, all
// on the same device.  Semantics follow NCCL point-to-point: messages
// between a (src, dst) pair match in posting order; a group's sends and
// receives progress together; a rank's stream does not pass group_end until
// the copies out of its send buffers have executed (so buffers may be
// reused afterwards, as with NCCL's rendezvous).  The copy itself is a
// cudaMemcpyAsync D2D on the receiver's stream, ordered after the sender's
// stream with events.
#include <chrono>
#include <condition_variable>
#include <deque>
#include <map>
#include <memory>
#include <mutex>
#include <vector>

#include "transport.h"

namespace es {
namespace {

struct Msg {
  const void *src = nullptr;
  size_t bytes = 0;
  cudaEvent_t ready = nullptr;   // sender stream position at group_end (shared)
  cudaEvent_t done = nullptr;    // receiver stream position after the copy
  bool matched = false;
  bool failed = false;
};

}  // namespace

struct LoopbackWorld {
  explicit LoopbackWorld(int g) : G(g) {}
  int G;
  std::mutex mu;
  std::condition_variable cv;
  std::map<std::pair<int, int>, std::deque<std::shared_ptr<Msg>>> box;  // (src, dst) -> FIFO
};

namespace {

constexpr auto kTimeout = std::chrono::seconds(120);

class LoopbackTransport : public Transport {
 public:
  LoopbackTransport(LoopbackWorld *w, int rank) : w_(w), rank_(rank) {}
  es_status group_begin() override {
    sends_.clear();
    recvs_.clear();
    return ES_OK;
  }
  es_status send(const void *p, size_t bytes, int peer) override {
    sends_.push_back({const_cast<void *>(p), bytes, peer});
    return ES_OK;
  }
  es_status recv(void *p, size_t bytes, int peer) override {
    recvs_.push_back({p, bytes, peer});
    return ES_OK;
  }
  es_status group_end(cudaStream_t s) override {
    if (sends_.empty() && recvs_.empty()) return ES_OK;
    // 1. post all sends (never blocks).
    std::vector<std::shared_ptr<Msg>> mine;
    cudaEvent_t ready = nullptr;
    if (!sends_.empty()) {
      if (cudaEventCreateWithFlags(&ready, cudaEventDisableTiming) != cudaSuccess ||
          cudaEventRecord(ready, s) != cudaSuccess)
        return cuda_fail("loopback: event record failed");
      std::lock_guard<std::mutex> lk(w_->mu);
      for (const P2P &o : sends_) {
        auto m = std::make_shared<Msg>();
        m->src = o.p;
        m->bytes = o.bytes;
        m->ready = ready;
        w_->box[{rank_, o.peer}].push_back(m);
        mine.push_back(m);
      }
      w_->cv.notify_all();
    }
    // 2. serve receives in posting order.
    es_status st = ES_OK;
    for (const P2P &o : recvs_) {
      std::shared_ptr<Msg> m;
      {
        std::unique_lock<std::mutex> lk(w_->mu);
        auto &q = w_->box[{o.peer, rank_}];
        if (!w_->cv.wait_for(lk, kTimeout, [&] { return !q.empty(); })) {
          err = "loopback: no matching send from peer (drive each rank from its own thread, same op order)";
          st = ES_ESTATE;
          break;
        }
        m = q.front();
        q.pop_front();
      }
      cudaEvent_t done = nullptr;
      bool ok = m->bytes == o.bytes;
      if (ok) {
        ok = cudaStreamWaitEvent(s, m->ready, 0) == cudaSuccess &&
             cudaMemcpyAsync(o.p, m->src, o.bytes, cudaMemcpyDeviceToDevice, s) == cudaSuccess &&
             cudaEventCreateWithFlags(&done, cudaEventDisableTiming) == cudaSuccess &&
             cudaEventRecord(done, s) == cudaSuccess;
      }
      {
        std::lock_guard<std::mutex> lk(w_->mu);
        m->done = done;
        m->failed = !ok;
        m->matched = true;
        w_->cv.notify_all();
      }
      if (!ok) {
        err = m->bytes == o.bytes ? "loopback: CUDA copy failed" : "loopback: send/recv size mismatch";
        st = m->bytes == o.bytes ? ES_ECUDA : ES_ESTATE;
        break;
      }
    }
    // 3. our stream may not run past the copies out of our send buffers.
    for (auto &m : mine) {
      std::unique_lock<std::mutex> lk(w_->mu);
      if (!w_->cv.wait_for(lk, kTimeout, [&] { return m->matched; })) {
        if (st == ES_OK) {
          err = "loopback: send never received by peer";
          st = ES_ESTATE;
        }
        continue;
      }
      lk.unlock();
      if (m->done) {
        if (cudaStreamWaitEvent(s, m->done, 0) != cudaSuccess && st == ES_OK) st = cuda_fail("loopback: wait failed");
        cudaEventDestroy(m->done);   // safe: destruction is deferred until the event completes
      } else if (st == ES_OK) {
        err = "loopback: peer failed to receive";
        st = ES_ESTATE;
      }
    }
    if (ready) cudaEventDestroy(ready);
    sends_.clear();
    recvs_.clear();
    return st;
  }

 private:
  struct P2P {
    void *p;
    size_t bytes;
    int peer;
  };
  es_status cuda_fail(const char *what) {
    err = what;
    return ES_ECUDA;
  }
  LoopbackWorld *w_;
  int rank_;
  std::vector<P2P> sends_, recvs_;
};

}  // namespace

Transport *make_loopback_transport(void *world, int G, int rank, std::string *err) {
  LoopbackWorld *w = reinterpret_cast<LoopbackWorld *>(world);
  if (w->G != G) {
    if (err) *err = "loopback world size does not match config G";
    return nullptr;
  }
  return new LoopbackTransport(w, rank);
}

}  // namespace es

extern "C" es_status es_loopback_create(int32_t G, void **world) {
  if (!world || G < 1 || G > 64) return ES_EINVAL;
  *world = new es::LoopbackWorld(G);
  return ES_OK;
}

extern "C" es_status es_loopback_destroy(void *world) {
  if (!world) return ES_EINVAL;
  delete reinterpret_cast<es::LoopbackWorld *>(world);
  return ES_OK;
}
