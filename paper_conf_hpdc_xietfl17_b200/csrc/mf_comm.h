// mf_comm.h -- multi-GPU transport for the DSGD strata mode (north_star (5); section 6.1,
// P:L305-316, adapted): Q-segment rotation with NCCL send/recv, segment broadcasts for
// evaluation / gathering, and an fp64 all-reduce.  libnccl.so.2 is dlopen'ed at mf_create
// time (world > 1 only), so the library loads and its host-only entry points work without it.
#pragma once

#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>
#include <string>
#include <vector>

namespace mf {

struct Xfer {
  void* ptr;      // same offset on both ranks (the segment's rows of Q)
  size_t bytes;
  int src, dst;
};

struct LoopGroup;

// Two transports behind one interface:
//  * NCCL (transport 0): one process per GPU, libnccl.so.2 dlopen'ed.
//  * loopback (transport 1, tests): all ranks are ctxs of ONE process driven by one host thread
//    each (any devices, e.g. all on one GPU); transfers are stream-ordered device-to-device
//    copies, synchronised with CUDA events and a host barrier.  Same protocol and plan, so the
//    multi-rank path is testable on a single GPU.
class Comm {
 public:
  static Comm* create(const uint8_t id[128], int world, int rank, cudaStream_t st, std::string* why);
  static Comm* create_loopback(const uint8_t id[128], int world, int rank, cudaStream_t st,
                               std::string* why);
  static void destroy(Comm* c);

  // One grouped set of point-to-point transfers (ncclGroupStart/ncclSend/ncclRecv/ncclGroupEnd).
  bool exchange(const std::vector<Xfer>& xs, int me, std::string* why);
  // Broadcast `bytes` at ptr from root to all ranks.
  bool broadcast(void* ptr, size_t bytes, int root, std::string* why);
  // In-place sum of n doubles over all ranks.
  bool allreduce_sum(double* dptr, size_t n, std::string* why);
  // Row segments r in [0,a) of a rows x row_bytes matrix: broadcast each from its owner r/(a/G).
  bool gather_rows(void* base, int64_t rows, int a, int G, size_t row_bytes, std::string* why);

  // Holder (rank) of each Q segment's current valid copy; -1 = every rank holds it.
  const int32_t* holders(int a);
  void set_holders(const int32_t* h, int a);
  void reset_holders(int a);

  int world() const { return world_; }

 private:
  Comm() = default;
  void* comm_ = nullptr;
  LoopGroup* loop_ = nullptr;
  cudaEvent_t ev_ = nullptr;
  cudaStream_t st_ = nullptr;
  int world_ = 1, rank_ = 0;
  std::vector<int32_t> holders_;
};

}  // namespace mf
