// transport.h -- byte exchange between the G ranks.
//
// Only point-to-point copies are ever requested: they are exact, so they can
// never change the canonical order the fold kernel fixes.  (An NCCL or NVLS
// reduction would impose its own order -- the non-determinism source of
// and is never used.)
#pragma once

#include <cuda_runtime.h>

#include <cstddef>
#include <string>

#include "../../include/es.h"

namespace es {

class Transport {
 public:
  virtual ~Transport() {}
  // A group is a set of sends/recvs that may progress concurrently; all
  // of them are enqueued on `s` at group_end.
  virtual es_status group_begin() = 0;
  virtual es_status send(const void *p, size_t bytes, int peer) = 0;
  virtual es_status recv(void *p, size_t bytes, int peer) = 0;
  virtual es_status group_end(cudaStream_t s) = 0;
  std::string err;
};

Transport *make_nccl_transport(void *comm, int G, int rank, std::string *err);
Transport *make_loopback_transport(void *world, int G, int rank, std::string *err);

}  // namespace es
