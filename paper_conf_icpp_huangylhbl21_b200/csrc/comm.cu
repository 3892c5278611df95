// comm.cu -- the two backends of the shard data plane (comm.cuh).
//
// NCCL: the production backend, one process per GPU over NVLink / NVSwitch.
// Loopback: G handles of one process on one device.  A send posts {pointer, bytes,
// ready event} into the (src, dst) channel of a shared hub; the matching recv waits for
// the post, makes its stream wait on the ready event, copies with one cudaMemcpyAsync
// (device to device) and answers with an ack event; the sender's stream waits on the
// ack, so -- as with NCCL -- the send buffer is not overwritten before the receiver
// has it.  Sends of a group are posted before any of its receives block, so ring
// patterns cannot deadlock.  Host waits time out (HCCMF_LOOPBACK_TIMEOUT_S, default
// 300 s) and poison the hub instead of hanging.
#include <nccl.h>

#include <chrono>
#include <condition_variable>
#include <cstdlib>
#include <deque>
#include <memory>
#include <mutex>
#include <vector>

#include "comm.cuh"
#include "internal.cuh"

namespace hccmf {

size_t dtype_size(DType t) {
  switch (t) {
    case DType::f32: return 4;
    case DType::f64: return 8;
    case DType::f16: return 2;
    case DType::u8: return 1;
    case DType::i64: return 8;
    case DType::u64: return 8;
  }
  return 1;
}

// ================================================================== NCCL
namespace {

ncclDataType_t nccl_type(DType t) {
  switch (t) {
    case DType::f32: return ncclFloat;
    case DType::f64: return ncclDouble;
    case DType::f16: return ncclHalf;
    case DType::u8: return ncclUint8;
    case DType::i64: return ncclInt64;
    case DType::u64: return ncclUint64;
  }
  return ncclUint8;
}

struct NcclComm final : Comm {
  ncclComm_t c = nullptr;
  int device = 0;
  const char* backend() const override { return "nccl"; }
  ~NcclComm() override {
    if (c) ncclCommDestroy(c);
  }
  int chk(ncclResult_t r, const char* what) {
    if (r == ncclSuccess) return 0;
    err = std::string(what) + ": " + ncclGetErrorString(r);
    return 1;
  }
  int group_start() override { return chk(ncclGroupStart(), "ncclGroupStart"); }
  int group_end() override { return chk(ncclGroupEnd(), "ncclGroupEnd"); }
  int send(const void* buf, size_t bytes, int peer, cudaStream_t st) override {
    return chk(ncclSend(buf, bytes, ncclUint8, peer, c, st), "ncclSend");
  }
  int recv(void* buf, size_t bytes, int peer, cudaStream_t st) override {
    return chk(ncclRecv(buf, bytes, ncclUint8, peer, c, st), "ncclRecv");
  }
  int broadcast(const void* in, void* out, size_t bytes, int root, cudaStream_t st) override {
    return chk(ncclBroadcast(in, out, bytes, ncclUint8, root, c, st), "ncclBroadcast");
  }
  int allreduce(const void* in, void* out, size_t count, DType t, ROp op, cudaStream_t st) override {
    return chk(ncclAllReduce(in, out, count, nccl_type(t), op == ROp::avg ? ncclAvg : ncclSum, c, st),
               "ncclAllReduce");
  }
  int allgather(const void* in, void* out, size_t bpr, cudaStream_t st) override {
    return chk(ncclAllGather(in, out, bpr, ncclUint8, c, st), "ncclAllGather");
  }
  int barrier() override {
    cudaSetDevice(device);
    int* d = nullptr;
    cudaStream_t s;
    if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess) {
      err = "barrier: cudaStreamCreate failed";
      return 1;
    }
    int rc = 0;
    if (cudaMallocAsync((void**)&d, sizeof(int), s) != cudaSuccess || cudaMemsetAsync(d, 0, sizeof(int), s)) {
      err = "barrier: allocation failed";
      rc = 1;
    }
    if (!rc) rc = chk(ncclAllReduce(d, d, 1, ncclInt32, ncclSum, c, s), "ncclAllReduce(barrier)");
    if (d) cudaFreeAsync(d, s);
    cudaStreamSynchronize(s);
    cudaStreamDestroy(s);
    return rc;
  }
};

}  // namespace

Comm* make_nccl_comm(const void* unique_id, int rank, int world, int device, std::string* err) {
  auto* k = new NcclComm();
  k->rank = rank;
  k->world = world;
  k->device = device;
  ncclUniqueId id;
  memcpy(&id, unique_id, sizeof(id));
  cudaSetDevice(device);
  ncclResult_t r = ncclCommInitRank(&k->c, world, id, rank);
  if (r != ncclSuccess) {
    *err = std::string("ncclCommInitRank: ") + ncclGetErrorString(r);
    k->c = nullptr;
    delete k;
    return nullptr;
  }
  return k;
}

// ============================================================== loopback
namespace {

struct Post {
  const void* ptr = nullptr;
  size_t bytes = 0;
  cudaEvent_t ready = nullptr;
  cudaEvent_t ack = nullptr;
  bool acked = false;
};

// element-wise reduction of W gathered copies in rank order (fp64 / 64-bit integer accumulation)
template <typename T, typename Acc>
__global__ void reduce_gathered_kernel(const T* __restrict__ g, int W, int64_t count, int avg, T* __restrict__ out) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < count; e += (int64_t)gridDim.x * blockDim.x) {
    Acc s = 0;
    for (int r = 0; r < W; ++r) s += (Acc)g[(int64_t)r * count + e];
    if (avg) s = s / (Acc)W;
    out[e] = (T)s;
  }
}

template <typename T, typename Acc>
cudaError_t reduce_gathered(const void* g, int W, int64_t count, int avg, void* out, cudaStream_t st) {
  if (count <= 0) return cudaSuccess;
  const int threads = 256;
  const int64_t blocks = std::min<int64_t>((count + threads - 1) / threads, 148 * 8);
  (note_launch(), reduce_gathered_kernel<T, Acc><<<(unsigned)blocks, threads, 0, st>>>(
                      static_cast<const T*>(g), W, count, avg, static_cast<T*>(out)));
  return cudaGetLastError();
}

double loopback_timeout() {
  const char* s = getenv("HCCMF_LOOPBACK_TIMEOUT_S");
  const double t = s ? atof(s) : 300.0;
  return t > 0 ? t : 300.0;
}

}  // namespace
}  // namespace hccmf

struct hccmf_hub {
  int world = 1;
  std::mutex mu;
  std::condition_variable cv;
  std::vector<std::deque<std::shared_ptr<hccmf::Post>>> chan;  // [src * world + dst]
  int refs = 1;
  bool poisoned = false;
  int bar_count = 0;
  uint64_t bar_gen = 0;
  double timeout_s = 300.0;
};

namespace hccmf {
namespace {

void hub_release(hccmf_hub* hub) {
  bool last = false;
  {
    std::lock_guard<std::mutex> g(hub->mu);
    last = --hub->refs == 0;
  }
  if (last) delete hub;
}

struct LoopbackComm final : Comm {
  hccmf_hub* hub = nullptr;
  int device = 0;
  struct Op {
    int kind;  // 0 send, 1 recv, 2 local copy
    const void* src;
    void* dst;
    size_t bytes;
    int peer;
    cudaStream_t st;
  };
  std::vector<Op> ops;
  int depth = 0;

  const char* backend() const override { return "loopback"; }
  ~LoopbackComm() override {
    if (hub) hub_release(hub);
  }

  int fail(const std::string& m) {
    err = "loopback rank " + std::to_string(rank) + ": " + m;
    return 1;
  }
  int cu(cudaError_t e, const char* what) {
    if (e == cudaSuccess) return 0;
    return fail(std::string(what) + ": " + cudaGetErrorString(e));
  }
  // wait on the hub's condition variable for pred(); false on timeout / poisoned hub
  template <typename Pred>
  bool wait(std::unique_lock<std::mutex>& lk, Pred pred) {
    const auto deadline = std::chrono::steady_clock::now() + std::chrono::duration<double>(hub->timeout_s);
    while (!pred()) {
      if (hub->poisoned) return false;
      if (hub->cv.wait_until(lk, deadline) == std::cv_status::timeout && !pred()) {
        hub->poisoned = true;
        hub->cv.notify_all();
        return false;
      }
    }
    return true;
  }

  int flush() {
    std::vector<Op> mine;
    mine.swap(ops);
    if (mine.empty()) return 0;
    cudaStream_t st = mine[0].st;
    for (const Op& o : mine)
      if (o.st != st) return fail("one stream per group");
    if (cu(cudaSetDevice(device), "cudaSetDevice")) return 1;
    cudaEvent_t ready = nullptr;
    if (cu(cudaEventCreateWithFlags(&ready, cudaEventDisableTiming), "cudaEventCreate")) return 1;
    if (cu(cudaEventRecord(ready, st), "cudaEventRecord")) return 1;
    std::vector<std::shared_ptr<Post>> sent;
    {  // 1. post every send of the group
      std::lock_guard<std::mutex> g(hub->mu);
      for (const Op& o : mine)
        if (o.kind == 0) {
          auto p = std::make_shared<Post>();
          p->ptr = o.src;
          p->bytes = o.bytes;
          p->ready = ready;
          hub->chan[(size_t)rank * world + o.peer].push_back(p);
          sent.push_back(p);
        }
      hub->cv.notify_all();
    }
    // 2. receives: wait for the peer's post, copy after its ready event, acknowledge
    for (const Op& o : mine) {
      if (o.kind == 2) {
        if (o.bytes && o.dst != o.src && cu(cudaMemcpyAsync(o.dst, o.src, o.bytes, cudaMemcpyDeviceToDevice, st), "local copy"))
          return 1;
        continue;
      }
      if (o.kind != 1) continue;
      std::shared_ptr<Post> p;
      {
        std::unique_lock<std::mutex> lk(hub->mu);
        auto& q = hub->chan[(size_t)o.peer * world + rank];
        if (!wait(lk, [&] { return !q.empty(); }))
          return fail("no matching send from rank " + std::to_string(o.peer) + " (timeout or a failed peer)");
        p = q.front();
        q.pop_front();
      }
      if (p->bytes != o.bytes) {
        std::lock_guard<std::mutex> g(hub->mu);
        hub->poisoned = true;
        hub->cv.notify_all();
        return fail("send/recv size mismatch with rank " + std::to_string(o.peer) + ": " + std::to_string(p->bytes) +
                    " vs " + std::to_string(o.bytes) + " bytes");
      }
      if (cu(cudaStreamWaitEvent(st, p->ready, 0), "cudaStreamWaitEvent")) return 1;
      if (o.bytes && cu(cudaMemcpyAsync(o.dst, p->ptr, o.bytes, cudaMemcpyDeviceToDevice, st), "cudaMemcpyAsync"))
        return 1;
      cudaEvent_t ack = nullptr;
      if (cu(cudaEventCreateWithFlags(&ack, cudaEventDisableTiming), "cudaEventCreate")) return 1;
      if (cu(cudaEventRecord(ack, st), "cudaEventRecord")) return 1;
      std::lock_guard<std::mutex> g(hub->mu);
      p->ack = ack;
      p->acked = true;
      hub->cv.notify_all();
    }
    // 3. the stream continues only after every receiver copied what this rank sent
    for (auto& p : sent) {
      {
        std::unique_lock<std::mutex> lk(hub->mu);
        if (!wait(lk, [&] { return p->acked; })) return fail("send not received (timeout or a failed peer)");
      }
      if (cu(cudaStreamWaitEvent(st, p->ack, 0), "cudaStreamWaitEvent")) return 1;
      cudaEventDestroy(p->ack);  // released once complete
    }
    cudaEventDestroy(ready);
    return 0;
  }

  int group_start() override {
    ++depth;
    return 0;
  }
  int group_end() override {
    if (depth <= 0) return fail("group_end without group_start");
    return --depth == 0 ? flush() : 0;
  }
  int push(const Op& o) {
    if (o.kind != 2 && (o.peer < 0 || o.peer >= world)) return fail("bad peer");
    ops.push_back(o);
    return depth == 0 ? flush() : 0;
  }
  int send(const void* buf, size_t bytes, int peer, cudaStream_t st) override {
    return push(Op{0, buf, nullptr, bytes, peer, st});
  }
  int recv(void* buf, size_t bytes, int peer, cudaStream_t st) override {
    return push(Op{1, nullptr, buf, bytes, peer, st});
  }
  int broadcast(const void* in, void* out, size_t bytes, int root, cudaStream_t st) override {
    if (root < 0 || root >= world) return fail("bad root");
    group_start();
    int rc = 0;
    if (rank == root) {
      for (int p = 0; p < world && !rc; ++p)
        if (p != rank) rc = push(Op{0, in, nullptr, bytes, p, st});
      if (!rc) rc = push(Op{2, in, out, bytes, rank, st});
    } else {
      rc = push(Op{1, nullptr, out, bytes, root, st});
    }
    const int rc2 = group_end();
    return rc ? rc : rc2;
  }
  int allgather(const void* in, void* out, size_t bpr, cudaStream_t st) override {
    if (depth) return fail("allgather inside a group");
    group_start();
    int rc = 0;
    char* o = static_cast<char*>(out);
    for (int p = 0; p < world && !rc; ++p)
      if (p != rank) {
        rc = push(Op{0, in, nullptr, bpr, p, st});
        if (!rc) rc = push(Op{1, nullptr, o + (size_t)p * bpr, bpr, p, st});
      }
    if (!rc) rc = push(Op{2, in, o + (size_t)rank * bpr, bpr, rank, st});
    const int rc2 = group_end();
    return rc ? rc : rc2;
  }
  int allreduce(const void* in, void* out, size_t count, DType t, ROp op, cudaStream_t st) override {
    if (depth) return fail("allreduce inside a group");
    const size_t es = dtype_size(t), B = count * es;
    if (count == 0) return 0;
    if (cu(cudaSetDevice(device), "cudaSetDevice")) return 1;
    void* g = nullptr;
    if (cu(cudaMallocAsync(&g, B * world, st), "cudaMallocAsync")) return 1;
    int rc = allgather(in, g, B, st);
    if (!rc) {
      const int avg = op == ROp::avg;
      cudaError_t e = cudaErrorInvalidValue;
      switch (t) {
        case DType::f32: e = reduce_gathered<float, double>(g, world, (int64_t)count, avg, out, st); break;
        case DType::f64: e = reduce_gathered<double, double>(g, world, (int64_t)count, avg, out, st); break;
        case DType::i64: e = reduce_gathered<int64_t, int64_t>(g, world, (int64_t)count, avg, out, st); break;
        case DType::u64:
          e = reduce_gathered<unsigned long long, unsigned long long>(g, world, (int64_t)count, avg, out, st);
          break;
        default: break;
      }
      rc = cu(e, "loopback reduction");
    }
    cudaFreeAsync(g, st);
    return rc;
  }
  int barrier() override {
    std::unique_lock<std::mutex> lk(hub->mu);
    const uint64_t gen = hub->bar_gen;
    if (++hub->bar_count == world) {
      hub->bar_count = 0;
      ++hub->bar_gen;
      hub->cv.notify_all();
      return 0;
    }
    if (!wait(lk, [&] { return hub->bar_gen != gen; })) return fail("barrier timeout");
    return 0;
  }
};

}  // namespace

Comm* make_loopback_comm(hccmf_hub_t hub, int rank, int device, std::string* err) {
  if (!hub || rank < 0 || rank >= hub->world) {
    *err = "bad hub or rank";
    return nullptr;
  }
  auto* c = new LoopbackComm();
  c->rank = rank;
  c->world = hub->world;
  c->device = device;
  {
    std::lock_guard<std::mutex> g(hub->mu);
    ++hub->refs;
  }
  c->hub = hub;
  return c;
}

}  // namespace hccmf

extern "C" {

hccmf_status hccmf_hub_create(int32_t world, hccmf_hub_t* out) {
  if (!out || world < 1) return HCCMF_EINVAL;
  auto* h = new hccmf_hub();
  h->world = world;
  h->chan.resize((size_t)world * world);
  h->timeout_s = hccmf::loopback_timeout();
  *out = h;
  return HCCMF_OK;
}

void hccmf_hub_destroy(hccmf_hub_t hub) {
  if (hub) hccmf::hub_release(hub);
}

}  // extern "C"
