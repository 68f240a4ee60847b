// czc_comm.cu — NCCL plumbing for slab mode (see czc_comm.h).
#include "czc_comm.h"

#if defined(CZC_WITH_NCCL)
#include <nccl.h>
#include <string.h>

namespace czc {
struct CommState {
  ncclComm_t comm;      // collectives (slab table, P1 states, records)
  ncclComm_t halo;      // halo send / recv (split from comm: its own stream, overlapping P1)
  int rank, size;
  bool aborted;
};
int comm_available() { return 1; }
static bool ok(ncclResult_t r, const char* what, std::string* err) {
  if (r == ncclSuccess) return true;
  if (err) *err = std::string(what) + ": " + ncclGetErrorString(r);
  return false;
}
CommState* comm_create(const void* uid128, int rank, int nranks, std::string* err) {
  ncclUniqueId id;
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId must be 128 bytes");
  memcpy(&id, uid128, sizeof(id));
  CommState* c = new CommState();
  c->rank = rank;
  c->size = nranks;
  c->aborted = false;
  if (!ok(ncclCommInitRank(&c->comm, nranks, id, rank), "ncclCommInitRank", err)) {
    delete c;
    return nullptr;
  }
  if (!ok(ncclCommSplit(c->comm, 0, rank, &c->halo, nullptr), "ncclCommSplit", err)) {
    ncclCommDestroy(c->comm);
    delete c;
    return nullptr;
  }
  return c;
}
void comm_destroy(CommState* c) {
  if (!c) return;
  if (!c->aborted) {
    ncclCommDestroy(c->halo);
    ncclCommDestroy(c->comm);
  }
  delete c;
}
void comm_abort(CommState* c) {
  if (!c || c->aborted) return;
  c->aborted = true;
  ncclCommAbort(c->halo);                  // this rank's queued operations are dropped
  ncclCommAbort(c->comm);
}
bool comm_usable(const CommState* c) { return c && !c->aborted; }
int comm_rank(const CommState* c) { return c->rank; }
int comm_size(const CommState* c) { return c->size; }
bool comm_allgather(CommState* c, const void* send, void* recv, size_t bytes, cudaStream_t st, std::string* err) {
  return ok(ncclAllGather(send, recv, bytes, ncclUint8, c->comm, st), "ncclAllGather", err);
}
bool comm_group_begin(std::string* err) { return ok(ncclGroupStart(), "ncclGroupStart", err); }
bool comm_group_end(std::string* err) { return ok(ncclGroupEnd(), "ncclGroupEnd", err); }
bool comm_send(CommState* c, const void* buf, size_t bytes, int peer, cudaStream_t st, std::string* err) {
  return ok(ncclSend(buf, bytes, ncclUint8, peer, c->halo, st), "ncclSend", err);
}
bool comm_recv(CommState* c, void* buf, size_t bytes, int peer, cudaStream_t st, std::string* err) {
  return ok(ncclRecv(buf, bytes, ncclUint8, peer, c->halo, st), "ncclRecv", err);
}
}  // namespace czc
#else
namespace czc {
struct CommState { int rank, size; };
int comm_available() { return 0; }
CommState* comm_create(const void*, int, int, std::string* err) {
  if (err) *err = "built without NCCL";
  return nullptr;
}
void comm_destroy(CommState*) {}
void comm_abort(CommState*) {}
bool comm_usable(const CommState*) { return false; }
int comm_rank(const CommState* c) { return c ? c->rank : 0; }
int comm_size(const CommState* c) { return c ? c->size : 1; }
bool comm_allgather(CommState*, const void*, void*, size_t, cudaStream_t, std::string* err) { if (err) *err = "no NCCL"; return false; }
bool comm_group_begin(std::string* err) { if (err) *err = "no NCCL"; return false; }
bool comm_group_end(std::string* err) { if (err) *err = "no NCCL"; return false; }
bool comm_send(CommState*, const void*, size_t, int, cudaStream_t, std::string* err) { if (err) *err = "no NCCL"; return false; }
bool comm_recv(CommState*, void*, size_t, int, cudaStream_t, std::string* err) { if (err) *err = "no NCCL"; return false; }
}  // namespace czc
#endif
