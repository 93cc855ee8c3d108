// mf_comm.cpp -- NCCL (dlopen'ed) transport for the strata mode; see mf_comm.h.
#include "mf_comm.h"

#include <dlfcn.h>
#include <nccl.h>

#include <cstring>
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

Comm* Comm::create(const uint8_t id[128], int world, int rank, cudaStream_t st, std::string* why) {
  Nccl* L = nccl(why);
  if (!L) return nullptr;
  ncclUniqueId uid;
  static_assert(sizeof(uid) == 128, "ncclUniqueId is 128 bytes");
  std::memcpy(&uid, id, 128);
  ncclComm_t cm = nullptr;
  if (!check(L, L->CommInitRank(&cm, world, uid, rank), "ncclCommInitRank", why)) return nullptr;
  Comm* c = new Comm();
  c->comm_ = cm;
  c->st_ = st;
  c->world_ = world;
  c->rank_ = rank;
  return c;
}

void Comm::destroy(Comm* c) {
  if (!c) return;
  Nccl* L = nccl(nullptr);
  if (L && c->comm_) L->CommDestroy(static_cast<ncclComm_t>(c->comm_));
  delete c;
}

bool Comm::exchange(const std::vector<Xfer>& xs, int me, std::string* why) {
  if (xs.empty()) return true;
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
  Nccl* L = nccl(why);
  if (!L) return false;
  return check(L, L->Bcast(ptr, ptr, bytes, ncclUint8, root, static_cast<ncclComm_t>(comm_), st_),
               "ncclBroadcast", why);
}

bool Comm::allreduce_sum(double* dptr, size_t n, std::string* why) {
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
