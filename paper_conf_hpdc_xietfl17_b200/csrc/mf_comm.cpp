// mf_comm.cpp -- NCCL (dlopen'ed) transport for the strata mode; see mf_comm.h.
#include "mf_comm.h"

#include <dlfcn.h>
#include <nccl.h>

#include <chrono>
#include <condition_variable>
#include <cstdio>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>

namespace mf {
namespace {

struct Nccl {
  void* h = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Bcast)(const void*, void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*ErrStr)(ncclResult_t) = nullptr;
  ncclResult_t (*CommCount)(const ncclComm_t, int*) = nullptr;      // optional (logging)
  ncclResult_t (*CommCuDevice)(const ncclComm_t, int*) = nullptr;   // optional (logging)
  ncclResult_t (*GetVersion)(int*) = nullptr;                       // optional (logging)
};

Nccl* nccl(std::string* why) {
  static Nccl lib;
  static std::once_flag once;
  static bool ok = false;
  std::call_once(once, [] {
    const char* names[] = {"libnccl.so.2", "libnccl.so"};
    for (const char* nm : names) {
      lib.h = dlopen(nm, RTLD_NOW | RTLD_GLOBAL);
      if (lib.h) break;
    }
    if (!lib.h) return;
#define SYM(field, name) lib.field = reinterpret_cast<decltype(lib.field)>(dlsym(lib.h, name))
    SYM(CommInitRank, "ncclCommInitRank");
    SYM(CommDestroy, "ncclCommDestroy");
    SYM(Send, "ncclSend");
    SYM(Recv, "ncclRecv");
    SYM(Bcast, "ncclBroadcast");
    SYM(AllReduce, "ncclAllReduce");
    SYM(GroupStart, "ncclGroupStart");
    SYM(GroupEnd, "ncclGroupEnd");
    SYM(ErrStr, "ncclGetErrorString");
    SYM(CommCount, "ncclCommCount");
    SYM(CommCuDevice, "ncclCommCuDevice");
    SYM(GetVersion, "ncclGetVersion");
#undef SYM
    ok = lib.CommInitRank && lib.CommDestroy && lib.Send && lib.Recv && lib.Bcast &&
         lib.AllReduce && lib.GroupStart && lib.GroupEnd && lib.ErrStr;
  });
  if (!ok) {
    if (why) *why = "libnccl.so.2 not loadable or missing symbols";
    return nullptr;
  }
  return &lib;
}

bool check(Nccl* L, ncclResult_t r, const char* what, std::string* why) {
  if (r == ncclSuccess) return true;
  if (why) *why = std::string(what) + ": " + L->ErrStr(r);
  return false;
}

}  // namespace

// ---------------------------------------------------------------------------------------------
// loopback transport
// ---------------------------------------------------------------------------------------------
struct LoopGroup {
  int world = 0;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  int joined = 0;
  std::vector<cudaEvent_t> ev;                 // each rank's "my stream reached here" event
  std::vector<std::vector<void*>> ptrs;        // published device pointers per rank

  // Returns false if the other ranks do not arrive within 300 s (a rank failed mid-protocol);
  // the group is then poisoned so every later barrier fails fast instead of hanging.
  bool barrier() {
    std::unique_lock<std::mutex> l(mu);
    if (broken) return false;
    const uint64_t g = gen;
    if (++arrived == world) {
      arrived = 0;
      ++gen;
      cv.notify_all();
      return true;
    }
    if (!cv.wait_for(l, std::chrono::seconds(300), [&] { return gen != g || broken; }) || broken) {
      broken = true;
      cv.notify_all();
      return false;
    }
    return true;
  }
  bool broken = false;
};

namespace {
std::mutex g_reg_mu;
std::map<std::string, std::shared_ptr<LoopGroup>> g_reg;

bool lb_fail(std::string* why) {
  if (why) *why = "loopback: a rank did not reach the rendezvous (timeout or earlier failure)";
  return false;
}

bool cuda_ok(cudaError_t e, const char* what, std::string* why) {
  if (e == cudaSuccess) return true;
  if (why) *why = std::string(what) + ": " + cudaGetErrorString(e);
  return false;
}
}  // namespace

Comm* Comm::create_loopback(const uint8_t id[128], int world, int rank, cudaStream_t st,
                            std::string* why) {
  const std::string key(reinterpret_cast<const char*>(id), 128);
  std::shared_ptr<LoopGroup> g;
  {
    std::lock_guard<std::mutex> l(g_reg_mu);
    auto& slot = g_reg[key];
    if (!slot) {
      slot = std::make_shared<LoopGroup>();
      slot->world = world;
      slot->ev.assign((size_t)world, nullptr);
      slot->ptrs.assign((size_t)world, {});
    }
    g = slot;
    if (g->world != world) {
      if (why) *why = "loopback group world size mismatch";
      return nullptr;
    }
    ++g->joined;
  }
  Comm* c = new Comm();
  c->loop_ = g.get();
  c->st_ = st;
  c->world_ = world;
  c->rank_ = rank;
  if (!cuda_ok(cudaEventCreateWithFlags(&c->ev_, cudaEventDisableTiming), "cudaEventCreate", why)) {
    delete c;
    return nullptr;
  }
  g->ev[(size_t)rank] = c->ev_;
  if (!g->barrier()) {                         // all ranks joined (like ncclCommInitRank)
    if (why) *why = "loopback: not every rank joined within the timeout";
    destroy(c);
    return nullptr;
  }
  return c;
}

Comm* Comm::create(const uint8_t id[128], int world, int rank, cudaStream_t st, std::string* why) {
  Nccl* L = nccl(why);
  if (!L) return nullptr;
  ncclUniqueId uid;
  static_assert(sizeof(uid) == 128, "ncclUniqueId is 128 bytes");
  std::memcpy(&uid, id, 128);
  ncclComm_t cm = nullptr;
  if (!check(L, L->CommInitRank(&cm, world, uid, rank), "ncclCommInitRank", why)) return nullptr;
  // one line per rank on stderr: the communicator really spans `world` ranks (the driver's
  // multi-GPU record checks the count)
  int nranks = -1, dev = -1, ver = 0;
  if (L->CommCount) L->CommCount(cm, &nranks);
  if (L->CommCuDevice) L->CommCuDevice(cm, &dev);
  if (L->GetVersion) L->GetVersion(&ver);
  std::fprintf(stderr, "[mf_comm] NCCL communicator ready: rank %d of %d, ncclCommCount = %d, "
                       "cuda device %d, NCCL %d\n", rank, world, nranks, dev, ver);
  if (L->CommCount && nranks != world) {
    L->CommDestroy(cm);
    if (why) *why = "ncclCommCount differs from world";
    return nullptr;
  }
  Comm* c = new Comm();
  c->comm_ = cm;
  c->st_ = st;
  c->world_ = world;
  c->rank_ = rank;
  return c;
}

void Comm::destroy(Comm* c) {
  if (!c) return;
  if (c->loop_) {
    std::lock_guard<std::mutex> l(g_reg_mu);
    for (auto it = g_reg.begin(); it != g_reg.end(); ++it)
      if (it->second.get() == c->loop_ && --it->second->joined == 0) {
        g_reg.erase(it);
        break;
      }
    if (c->ev_) cudaEventDestroy(c->ev_);
    delete c;
    return;
  }
  Nccl* L = nccl(nullptr);
  if (L && c->comm_) L->CommDestroy(static_cast<ncclComm_t>(c->comm_));
  delete c;
}

bool Comm::exchange(const std::vector<Xfer>& xs, int me, std::string* why) {
  if (xs.empty()) return true;
  if (loop_) {
    LoopGroup& g = *loop_;
    std::vector<void*> mine;
    for (const Xfer& x : xs) mine.push_back(x.ptr);
    g.ptrs[(size_t)me] = mine;
    if (!cuda_ok(cudaEventRecord(ev_, st_), "cudaEventRecord", why)) return false;
    if (!g.barrier()) return lb_fail(why);         // every rank's segments are final on its stream
    for (size_t i = 0; i < xs.size(); ++i)
      if (xs[i].dst == me) {
        if (!cuda_ok(cudaStreamWaitEvent(st_, g.ev[(size_t)xs[i].src], 0), "wait", why)) return false;
        if (!cuda_ok(cudaMemcpyAsync(xs[i].ptr, g.ptrs[(size_t)xs[i].src][i], xs[i].bytes,
                                     cudaMemcpyDeviceToDevice, st_), "copy", why))
          return false;
      }
    if (!g.barrier()) return lb_fail(why);         // all copies enqueued before events are re-recorded
    if (!cuda_ok(cudaEventRecord(ev_, st_), "cudaEventRecord", why)) return false;
    if (!g.barrier()) return lb_fail(why);
    for (size_t i = 0; i < xs.size(); ++i)     // a source does not overwrite before the copy ran
      if (xs[i].src == me && !cuda_ok(cudaStreamWaitEvent(st_, g.ev[(size_t)xs[i].dst], 0), "wait", why))
        return false;
    if (!g.barrier()) return lb_fail(why);
    return true;
  }
  Nccl* L = nccl(why);
  if (!L) return false;
  ncclComm_t cm = static_cast<ncclComm_t>(comm_);
  if (!check(L, L->GroupStart(), "ncclGroupStart", why)) return false;
  bool ok = true;
  for (const Xfer& x : xs) {
    if (x.src == me) ok = ok && check(L, L->Send(x.ptr, x.bytes, ncclUint8, x.dst, cm, st_), "ncclSend", why);
    if (x.dst == me) ok = ok && check(L, L->Recv(x.ptr, x.bytes, ncclUint8, x.src, cm, st_), "ncclRecv", why);
  }
  const bool ended = check(L, L->GroupEnd(), "ncclGroupEnd", why);
  return ok && ended;
}

bool Comm::broadcast(void* ptr, size_t bytes, int root, std::string* why) {
  if (loop_) {
    std::vector<Xfer> xs;
    for (int r = 0; r < world_; ++r)
      if (r != root) xs.push_back(Xfer{ptr, bytes, root, r});
    return exchange(xs, rank_, why);
  }
  Nccl* L = nccl(why);
  if (!L) return false;
  return check(L, L->Bcast(ptr, ptr, bytes, ncclUint8, root, static_cast<ncclComm_t>(comm_), st_),
               "ncclBroadcast", why);
}

bool Comm::allreduce_sum(double* dptr, size_t n, std::string* why) {
  if (loop_) {
    LoopGroup& g = *loop_;
    g.ptrs[(size_t)rank_] = {dptr};
    if (!cuda_ok(cudaEventRecord(ev_, st_), "cudaEventRecord", why)) return false;
    if (!g.barrier()) return lb_fail(why);
    std::vector<double> acc(n, 0.0), tmp(n);
    for (int r = 0; r < world_; ++r) {         // fixed rank order: identical sum on every rank
      if (!cuda_ok(cudaStreamWaitEvent(st_, g.ev[(size_t)r], 0), "wait", why)) return false;
      if (!cuda_ok(cudaMemcpyAsync(tmp.data(), g.ptrs[(size_t)r][0], n * sizeof(double),
                                   cudaMemcpyDeviceToHost, st_), "copy", why) ||
          !cuda_ok(cudaStreamSynchronize(st_), "sync", why))
        return false;
      for (size_t i = 0; i < n; ++i) acc[i] += tmp[i];
    }
    if (!g.barrier()) return lb_fail(why);         // everyone read every input before overwriting
    if (!cuda_ok(cudaMemcpyAsync(dptr, acc.data(), n * sizeof(double), cudaMemcpyHostToDevice, st_),
                 "copy", why) ||
        !cuda_ok(cudaStreamSynchronize(st_), "sync", why))
      return false;
    if (!g.barrier()) return lb_fail(why);
    return true;
  }
  Nccl* L = nccl(why);
  if (!L) return false;
  return check(L, L->AllReduce(dptr, dptr, n, ncclFloat64, ncclSum, static_cast<ncclComm_t>(comm_), st_),
               "ncclAllReduce", why);
}

bool Comm::gather_rows(void* base, int64_t rows, int a, int G, size_t row_bytes, std::string* why) {
  const int per = a / G;
  for (int r = 0; r < a; ++r) {
    const int64_t lo = (static_cast<int64_t>(r) * rows + a - 1) / a;
    const int64_t hi = (static_cast<int64_t>(r + 1) * rows + a - 1) / a;
    if (hi <= lo) continue;
    if (!broadcast(static_cast<char*>(base) + static_cast<size_t>(lo) * row_bytes,
                   static_cast<size_t>(hi - lo) * row_bytes, r / per, why))
      return false;
  }
  return true;
}

const int32_t* Comm::holders(int a) {
  if (static_cast<int>(holders_.size()) != a) holders_.assign(static_cast<size_t>(a), -1);
  return holders_.data();
}
void Comm::set_holders(const int32_t* h, int a) { holders_.assign(h, h + a); }
void Comm::reset_holders(int a) { holders_.assign(static_cast<size_t>(a), -1); }

}  // namespace mf
