// czc_comm.h — NCCL plumbing for slab mode (nranks > 1).  Only collectives live here; all
// assessment arithmetic stays in the kernels.  Built with -DCZC_WITH_NCCL, else a stub that
// reports CZC_ERR_UNSUPPORTED for nranks > 1.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>

#include <string>

namespace czc {
struct CommState;
int comm_available();
// Creates the rank's communicator and a second one split from it for the halo exchange, which
// runs on its own stream concurrently with the first one's collectives (the halo
// overlaps P1).  Every rank issues the operations of both in the same order.
CommState* comm_create(const void* uid128, int rank, int nranks, std::string* err);
void comm_destroy(CommState* c);
// Abort both communicators (a local failure after the first collective of a call: the peers'
// pending operations return with an error instead of waiting for this rank forever).
void comm_abort(CommState* c);
bool comm_usable(const CommState* c);
int comm_rank(const CommState* c);
int comm_size(const CommState* c);
// all ranks: recvbuf[nranks * bytes] <- sendbuf[bytes] of every rank (rank order)
bool comm_allgather(CommState* c, const void* send, void* recv, size_t bytes, cudaStream_t st, std::string* err);
// grouped point-to-point: send `sbytes` from sbuf to `peer_send` (if >= 0) and receive `rbytes`
// into rbuf from `peer_recv` (if >= 0); several calls between group_begin / group_end overlap.
bool comm_group_begin(std::string* err);
bool comm_group_end(std::string* err);
// point-to-point on the halo communicator
bool comm_send(CommState* c, const void* buf, size_t bytes, int peer, cudaStream_t st, std::string* err);
bool comm_recv(CommState* c, void* buf, size_t bytes, int peer, cudaStream_t st, std::string* err);
}  // namespace czc
