// Internal interface of the tensor-parallel collectives (comm.cpp).  Not part of the C-ABI.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>

#include "menos.h"

namespace menos {

struct Comm {
  int rank = 0, world = 1;
  menos_collective_fn fn = nullptr;
  void* user = nullptr;
  void* nccl = nullptr;      // ncclComm_t when the library drives NCCL itself
  long long calls = 0;       // collectives issued (evidence for tests / bench)
  double bytes = 0;          // payload bytes of those collectives (all-reduce: count; gather / scatter: world * count)
  int init(const menos_tp_cfg& tp, int device);
  void destroy();
  // op: MENOS_COLL_*; count = elements of ONE rank's share for ALLGATHER / REDUCE_SCATTER, of the buffer for ALLREDUCE
  int run(int op, const void* send, void* recv, size_t count, int dtype, cudaStream_t st);
};

}  // namespace menos
