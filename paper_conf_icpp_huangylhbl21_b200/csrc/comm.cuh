// comm.cuh -- the data plane between shards: every exchange the
// library makes between ranks goes through this interface, whose production backend is
// NCCL (one process per GPU) and whose second backend is an in-process loopback (G
// handles on ONE device, one host thread each) so that one GPU runs the exact multi-rank
// data plane: the same call sites, the same buffers, the same stream/event ordering.
//
// Semantics follow NCCL's: operations are stream-ordered on the stream passed in; a
// send's buffer may be reused once the operation completes on that stream; send/recv (and
// broadcasts) issued between group_start() and group_end() are matched as one group, so a
// ring's simultaneous send-to-prev / recv-from-next cannot deadlock.  Every function
// returns 0 on success, else non-zero with the reason in err.
#pragma once

#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include <string>

#include "hccmf.h"

namespace hccmf {

enum class DType : int { f32 = 0, f64 = 1, f16 = 2, u8 = 3, i64 = 4, u64 = 5 };
enum class ROp : int { sum = 0, avg = 1 };

size_t dtype_size(DType t);

struct Comm {
  virtual ~Comm() {}
  virtual const char* backend() const = 0;
  int rank = 0, world = 1;
  std::string err;

  virtual int group_start() = 0;
  virtual int group_end() = 0;
  virtual int send(const void* buf, size_t bytes, int peer, cudaStream_t st) = 0;
  virtual int recv(void* buf, size_t bytes, int peer, cudaStream_t st) = 0;
  // may appear inside a group (grouped broadcasts with different roots)
  virtual int broadcast(const void* in, void* out, size_t bytes, int root, cudaStream_t st) = 0;
  // not inside a group
  virtual int allreduce(const void* in, void* out, size_t count, DType t, ROp op, cudaStream_t st) = 0;
  // out[r * bytes_per_rank ...] = rank r's in; in-place when in == out + rank * bytes_per_rank
  virtual int allgather(const void* in, void* out, size_t bytes_per_rank, cudaStream_t st) = 0;
  // host barrier (no device work): every rank's host thread reaches it
  virtual int barrier() = 0;
};

// NCCL backend: ncclCommInitRank over a 128-byte ncclUniqueId.  nullptr + *err on failure.
Comm* make_nccl_comm(const void* unique_id, int rank, int world, int device, std::string* err);
// Loopback backend on one device: every rank of `hub` is a handle in this process.
Comm* make_loopback_comm(hccmf_hub_t hub, int rank, int device, std::string* err);

// Call sites of the data plane (hccmf_comm_counts): how many times each one ran.
enum CommSite : int {
  SITE_RING_STAGE = 0,     // DET/stage-wise ring: one column group to rank-1, one from rank+1
  SITE_RING_BLOCK = 1,     // pipelined Hogwild ring: one column block per launch (comm stream)
  SITE_RING_WIRE16 = 2,    // either ring transfer in binary16 (Strategy 2)
  SITE_MATERIALIZE_Q = 3,  // broadcast of every ring group from its owner (after ring epochs)
  SITE_ALLREDUCE_Q = 4,    // fp32 ncclAvg of Q (server sync)
  SITE_ALLREDUCE_Q16 = 5,  // binary16 wire: all-to-all of chunks + fp64 mean + all-gather
  SITE_RMSE = 6,           // {sum, count} of the test squared errors
  SITE_EXPORT_P = 7,       // final push of P: every shard's rows to every rank
  SITE_INGEST_HIST = 8,    // sliced ingest: global permuted-row histogram + nnz
  SITE_INGEST_EXCHANGE = 9,// sliced ingest: ratings to their owner shard
  SITE_INGEST_BLOCKS = 10, // sliced ingest: global block offsets
  N_COMM_SITES = 11
};

}  // namespace hccmf
