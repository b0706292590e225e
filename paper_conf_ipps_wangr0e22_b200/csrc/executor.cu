// executor.cu — replays the planner's op list on 1..64 (logical) GPUs.
//
//  * one CUDA stream per logical GPU; logical GPU g runs on device g % device_count, so the
//    multi-GPU scheduling / cache / P2P paths also run (as device-local copies) on one B200;
//  * tensors live in stream-ordered pool allocations (cudaMallocAsync), interleaved complex;
//  * H2D from the library's pinned node store, NVLink peer copies (cudaMemcpyPeerAsync) for
//    replicas held by another GPU, D2H spills of sole copies under memory pressure
//    (allocation and CPU↔GPU / GPU↔GPU movement are the memory
//    operations the scheduler trades against load balance);
//  * the tasks of one stage and GPU are batched into grouped GEMM launches (one per operand
//    layout class) and one grouped dot launch; descriptors are kernel parameters;
//  * rank-0 results land in a per-device scalar table [slot][t]; devices are combined by an
//    exact sum (each slot is nonzero on one device only): NCCL all-reduce in multi-process
//    mode, peer copies otherwise; then C(t) = Σ_g c_g Π_comp s_comp(t) on device 0.
// Multi-process mode (one process per GPU): every rank replays the same plan, executes only
// its own GPU's ops, and turns cross-GPU copies into matched ncclSend / ncclRecv.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>
#include <nvtx3/nvToolsExt.h>  // header-only NVTX v3: no cost unless a profiler injects itself

#include <algorithm>
#include <array>
#include <chrono>
#include <cstdlib>
#include <cstring>
#include <string>
#include <exception>
#include <thread>
#include <tuple>
#include <type_traits>
#include <unordered_map>

#include "executor.h"
#include "kernels.h"
#include "layout.h"

namespace micco {

#define CK(x)                                                                                       \
  do {                                                                                              \
    cudaError_t e_ = (x);                                                                           \
    if (e_ != cudaSuccess)                                                                          \
      fail(MICCO_ERR_CUDA, std::string("CUDA error: ") + cudaGetErrorString(e_) + " at " #x);       \
  } while (0)

// NVTX ranges (SURVEY.md §5 tracing): execute, planning, each flushed chunk of a stage, host
// and peer copies, so an nsys / ncu timeline shows the host-side structure of a step.
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange &) = delete;
  NvtxRange &operator=(const NvtxRange &) = delete;
};

// ------------------------------------------------------------------ NCCL (dlopen)

namespace {

struct NcclApi {
  bool ok = false;
  std::string why;
  ncclResult_t (*GetUniqueId)(ncclUniqueId *);
  ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int);
  ncclResult_t (*CommInitAll)(ncclComm_t *, int, const int *);
  ncclResult_t (*CommDestroy)(ncclComm_t);
  ncclResult_t (*AllReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t);
  ncclResult_t (*Send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
  ncclResult_t (*Recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
  ncclResult_t (*GroupStart)();
  ncclResult_t (*GroupEnd)();
  const char *(*GetErrorString)(ncclResult_t);
};

NcclApi &nccl() {
  static NcclApi api = [] {
    NcclApi a;
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) { a.why = "libnccl.so.2 not loadable"; return a; }
#define LOAD(name) a.name = reinterpret_cast<decltype(a.name)>(dlsym(h, "nccl" #name)); if (!a.name) { a.why = "missing nccl" #name; return a; }
    LOAD(GetUniqueId) LOAD(CommInitRank) LOAD(CommInitAll) LOAD(CommDestroy) LOAD(AllReduce)
    LOAD(Send) LOAD(Recv) LOAD(GroupStart) LOAD(GroupEnd) LOAD(GetErrorString)
#undef LOAD
    a.ok = true;
    return a;
  }();
  return api;
}

#define NK(x)                                                                                       \
  do {                                                                                              \
    ncclResult_t r_ = (x);                                                                          \
    if (r_ != ncclSuccess) fail(MICCO_ERR_NCCL, std::string("NCCL error: ") + nccl().GetErrorString(r_)); \
  } while (0)

}  // namespace

micco_status nccl_unique_id(uint8_t out[128]) {
  NcclApi &a = nccl();
  if (!a.ok) return MICCO_ERR_NCCL;
  ncclUniqueId id;
  if (a.GetUniqueId(&id) != ncclSuccess) return MICCO_ERR_NCCL;
  std::memcpy(out, &id, 128);
  return MICCO_OK;
}

// ------------------------------------------------------------------ executor state

namespace {

// chunks the H2D prefetch may run ahead (6: C4 e2e 122.2k graphs/s; 64: 129.7k; round 1)
constexpr int kLookahead = 64;
constexpr int64_t kPrefetchBytes = 8LL << 30;    // and at most this many bytes

struct EventPool {
  int dev = -1;
  unsigned flags = cudaEventDisableTiming;
  std::vector<cudaEvent_t> all;
  size_t used = 0;
  cudaEvent_t get() {
    if (used == all.size()) {
      cudaEvent_t e;
      CK(cudaSetDevice(dev));
      CK(cudaEventCreateWithFlags(&e, flags));
      all.push_back(e);
    }
    return all[used++];
  }
  void reset() { used = 0; }
  void destroy() {
    if (dev >= 0) cudaSetDevice(dev);
    for (auto e : all) cudaEventDestroy(e);
    all.clear();
    used = 0;
  }
};

struct DevState {
  int dev = -1;
  EventPool sync_events, timing_events;
  bool init = false;
};

// A scalar table [slot][t] (rank-0 results).  One per device by default; one per logical GPU
// with options.scalar_tables = 1, so that the cross-GPU combine (peer copy + exact
// accumulate) also runs when several logical GPUs share one device.
struct ScalarTable {
  int dev = -1;
  double2 *p = nullptr;
  size_t elems = 0;
};

struct Timed {
  cudaEvent_t a, b;
  int kind;  // 0 gemm, 1 dot (warp kernel: traces, fused-dot sums), 2 copy, 3 dot (CTA kernel)
  int dev;
};

struct LGpu {
  int idx = 0, dev = 0;
  bool local = true;
  cudaStream_t st = nullptr;   // compute stream: kernels, P2P, spills, frees
  cudaStream_t cst = nullptr;  // copy stream: H2D prefetch (async, overlaps the kernels)
  cudaStream_t pst = nullptr;  // peer stream: NVLink moves (peer copies / NCCL send-recv)
  // side stream of a flushed chunk (forked from st, joined back into it): the chunk's GEMM
  // launches alternate between st and kst[0], so one persistent launch's last, partly empty
  // wave overlaps the next launch's first (a chunk's tasks are independent).  The dots stay on
  // st after the join: run beside the GEMMs they only stretched the GEMM launches (C3: same
  // step time, 42.8 → 39.6 TF/s of GEMM device time).
  cudaStream_t kst[1] = {nullptr};
  std::vector<cudaEvent_t> flush_ev;  // compute-stream event after each flushed chunk
  std::vector<int64_t> chunk_fetch;   // bytes fetched for each flushed chunk
  std::vector<int64_t> fetch_bytes_since;
  int64_t pending_fetch = 0;          // bytes fetched for the chunk being built
  std::vector<double2 *> ptr;                                  // tensor → replica
  std::unordered_map<int32_t, std::vector<cudaEvent_t>> readers;  // peer reads to wait for before free
  std::vector<GemmDesc> gemm;
  std::vector<std::array<CUtensorMap, 2>> gemm_maps;  // per gemm entry (TMA classes only)
  std::vector<DotDesc> dot;
  std::vector<double2 *> part_allocs;  // fused-dot partials of the pending batch
  long long gemm_tiles = 0, dot_ctas = 0;
  // bytes the H2D prefetch may run ahead of the compute stream: the device memory left outside
  // the planned budgets, shared by the logical GPUs on this device (budgets())
  int64_t prefetch_cap = kPrefetchBytes;
};

}  // namespace

struct Executor::Impl {
  Context &c;
  int ndev = 0;
  int n = 0;  // logical GPUs
  std::vector<LGpu> g;
  std::vector<DevState> devs;
  std::vector<ScalarTable> tables;  // indexed by table_of(logical GPU)
  std::vector<Timed> timed;
  std::vector<cudaEvent_t> time_ref;  // per device: origin of the timed intervals
  std::unordered_map<int32_t, double *> spill_host;
  std::unordered_map<int32_t, std::pair<int, cudaEvent_t>> spill_ev;
  HostArena spill_arena;
  ncclComm_t comm = nullptr;
  std::vector<ncclComm_t> comms_all;  // single-process multi-device
  std::vector<int64_t> budget_cache;
  int budget_cache_n = 0;
  std::vector<std::pair<int32_t, uint64_t>> cached_nodes;
  std::vector<int32_t> fused_dot;  // of the plan being replayed
  std::unique_ptr<GemmBatch> gemm_batch{new GemmBatch};  // kernel-parameter staging
  std::unique_ptr<GemmTmaBatch> tma_batch{new GemmTmaBatch};
  std::unique_ptr<DotBatch> dot_batch{new DotBatch};
  std::unique_ptr<DotGroupBatch> dot_group_batch{new DotGroupBatch};
  int32_t chosen_bd[3] = {0, 0, 0};
  int chosen_bd_n = 0;
  int stream_ok_n = 0;  // GPU count of the last completed execute (its nodes are materialised)
  int32_t chosen_w = 256;  // window chosen by choose_window for chosen_w_n GPUs
  int chosen_w_n = 0;
  int64_t cache_dag_key = -1;
  // results on device 0
  double2 *d_vals = nullptr;
  size_t vals_elems = 0;
  int vals_dev = 0;
  double2 *h_corr = nullptr;
  int64_t launches = 0, tma_launches = 0, oom_retries = 0;
  int launch_seq = 0;  // launches of the chunk being flushed (side-stream choice)
  bool use_tma = true;  // TMA GEMM for the contractions that fit it (see execute)
  bool dist() const { return c.opt.dist_world > 0; }
  int table_of(int i) const { return c.opt.scalar_tables ? i : g[i].dev; }
  double2 *table_row(const LGpu &l, int32_t slot) const {
    return tables[table_of(l.idx)].p + (size_t)slot * c.Lt;
  }
  int my_rank() const { return c.opt.dist_rank; }

  explicit Impl(Context &ctx) : c(ctx) {}
  ~Impl() { teardown(); }

  void teardown() {
    for (auto &l : g) free_lgpu(l, true);
    g.clear();
    n = 0;
    for (auto &d : devs) {
      if (d.dev < 0) continue;
      cudaSetDevice(d.dev);
      if (d.init) {  // hand the pool's cached blocks back, so the next setup's budget (from the
        cudaMemPool_t pool;  // device's free memory) does not count them as used
        if (cudaDeviceGetDefaultMemPool(&pool, d.dev) == cudaSuccess) {
          cudaDeviceSynchronize();
          cudaMemPoolTrimTo(pool, 0);
        }
      }
      d.sync_events.destroy();
      d.timing_events.destroy();
    }
    for (auto &t : tables)
      if (t.p) { cudaSetDevice(t.dev); cudaFree(t.p); }
    tables.clear();
    if (d_vals) { cudaSetDevice(vals_dev); cudaFree(d_vals); d_vals = nullptr; }
    vals_elems = 0;  // (a re-setup for another GPU count must reallocate the value table)
    if (h_corr) { cudaFreeHost(h_corr); h_corr = nullptr; }
    if (comm && nccl().ok) nccl().CommDestroy(comm);
    comm = nullptr;
    for (auto cm : comms_all) if (cm && nccl().ok) nccl().CommDestroy(cm);
    comms_all.clear();
  }

  void free_lgpu(LGpu &l, bool destroy_stream) {
    if (!l.local || !l.st) return;
    cudaSetDevice(l.dev);
    for (auto &p : l.ptr)
      if (p) { cudaFreeAsync(p, l.st); p = nullptr; }
    cudaStreamSynchronize(l.st);
    if (l.cst) cudaStreamSynchronize(l.cst);
    if (l.pst) cudaStreamSynchronize(l.pst);
    for (cudaStream_t k : l.kst)
      if (k) cudaStreamSynchronize(k);
    l.readers.clear();
    if (destroy_stream) {
      cudaStreamDestroy(l.st);
      cudaStreamDestroy(l.cst);
      cudaStreamDestroy(l.pst);
      for (cudaStream_t &k : l.kst) {
        if (k) cudaStreamDestroy(k);
        k = nullptr;
      }
      l.pst = nullptr;
      l.st = nullptr;
      l.cst = nullptr;
    }
  }

  void setup(int n_gpus) {
    CK(cudaGetDeviceCount(&ndev));
    if (ndev < 1) fail(MICCO_ERR_CUDA, "no CUDA device (micco has no CPU fallback)");
    if (n_gpus == n && !g.empty()) return;
    teardown();
    cached_nodes.clear();
    n = n_gpus;
    devs.assign(ndev, DevState{});
    for (int d = 0; d < ndev; ++d) {
      devs[d].dev = d;
      devs[d].sync_events.dev = d;
      devs[d].timing_events.dev = d;
      devs[d].timing_events.flags = cudaEventDefault;
    }
    g.assign(n, LGpu{});
    for (int i = 0; i < n; ++i) {
      LGpu &l = g[i];
      l.idx = i;
      l.dev = i % ndev;
      l.local = !dist() || i == my_rank();
      if (!l.local) continue;
      CK(cudaSetDevice(l.dev));
      if (!devs[l.dev].init) {
        cudaMemPool_t pool;
        CK(cudaDeviceGetDefaultMemPool(&pool, l.dev));
        uint64_t thr = UINT64_MAX;
        CK(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
        // never let an allocation on one stream wait for a free on another: the H2D prefetch
        // on the copy stream must not be serialised behind the compute stream (the driver
        // would otherwise insert a dependency to reuse a block freed by the compute stream)
        int no = 0;
        CK(cudaMemPoolSetAttribute(pool, cudaMemPoolReuseAllowInternalDependencies, &no));
        for (int p = 0; p < ndev; ++p) {  // NVLink peer access for P2P replicas
          if (p == l.dev) continue;
          int can = 0;
          cudaDeviceCanAccessPeer(&can, l.dev, p);
          if (can) {
            cudaError_t e = cudaDeviceEnablePeerAccess(p, 0);
            if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) CK(e);
            cudaGetLastError();
          }
        }
        devs[l.dev].init = true;
      }
      CK(cudaStreamCreateWithFlags(&l.st, cudaStreamNonBlocking));
      CK(cudaStreamCreateWithFlags(&l.cst, cudaStreamNonBlocking));
      CK(cudaStreamCreateWithFlags(&l.pst, cudaStreamNonBlocking));
      for (cudaStream_t &k : l.kst) CK(cudaStreamCreateWithFlags(&k, cudaStreamNonBlocking));
    }
    // Peer access to stream-ordered pool memory is granted per pool (cudaDeviceEnablePeerAccess
    // covers cudaMalloc memory only): every device in use may read every other's pool, so a
    // peer copy of a replica is a direct NVLink transfer.
    for (int d = 0; d < ndev; ++d) {
      if (!devs[d].init) continue;
      cudaMemPool_t pool;
      CK(cudaDeviceGetDefaultMemPool(&pool, d));
      for (int p = 0; p < ndev; ++p) {
        if (p == d || !devs[p].init) continue;
        int can = 0;
        cudaDeviceCanAccessPeer(&can, p, d);
        if (!can) continue;
        cudaMemAccessDesc acc{};
        acc.location.type = cudaMemLocationTypeDevice;
        acc.location.id = p;
        acc.flags = cudaMemAccessFlagsProtReadWrite;
        CK(cudaMemPoolSetAccess(pool, &acc, 1));
      }
    }
    if (dist()) {
      if (!c.have_nccl_id) fail(MICCO_ERR_STATE, "multi-process mode needs micco_set_nccl_id before execute");
      if (!nccl().ok) fail(MICCO_ERR_NCCL, "NCCL unavailable: " + nccl().why);
      ncclUniqueId id;
      std::memcpy(&id, c.nccl_id, 128);
      CK(cudaSetDevice(g[my_rank()].dev));
      NK(nccl().CommInitRank(&comm, n, id, my_rank()));
    }
    budget_cache_n = 0;
  }

  std::vector<int64_t> budgets() {
    if (budget_cache_n == n) return budget_cache;
    std::vector<int64_t> b(n);
    std::vector<int> per_dev(ndev, 0);
    for (int i = 0; i < n; ++i) per_dev[g[i].dev]++;
    for (int i = 0; i < n; ++i) {
      size_t fr = 0, tot = 0;
      if (g[i].local || !dist()) {
        CK(cudaSetDevice(g[i].dev));
        CK(cudaMemGetInfo(&fr, &tot));
      } else {
        // remote ranks: assume the same device model as ours (identical plan on every rank)
        CK(cudaSetDevice(g[my_rank()].dev));
        CK(cudaMemGetInfo(&fr, &tot));
      }
      const int k = dist() ? 1 : per_dev[g[i].dev];
      if (c.opt.mem_budget_bytes > 0) {
        b[i] = c.opt.mem_budget_bytes;
      } else {
        int64_t usable = (int64_t)(fr * 0.92) - (2LL << 30);
        b[i] = std::max<int64_t>(usable / k, 1LL << 28);
      }
      // The prefetch (and peer look-ahead) allocate beyond what the plan has freed so far:
      // keep them inside the memory the budgets leave free on this device, minus a reserve
      // for the fused-dot partials and the allocator's rounding (with several
      // logical GPUs per device or a caller budget near capacity the pool could run out).
      const int64_t slack = ((int64_t)fr - k * b[i] - (1LL << 30)) / k;
      g[i].prefetch_cap = std::min<int64_t>(kPrefetchBytes, std::max<int64_t>(slack, 0));
    }
    if (dist()) {  // every rank must plan with identical budgets: the minimum over ranks
      int64_t mn = *std::min_element(b.begin(), b.end());
      if (c.opt.mem_budget_bytes <= 0 && comm) {
        LGpu &l = g[my_rank()];
        CK(cudaSetDevice(l.dev));
        int64_t *d = nullptr;
        CK(cudaMallocAsync((void **)&d, sizeof(int64_t), l.st));
        CK(cudaMemcpyAsync(d, &mn, sizeof(int64_t), cudaMemcpyHostToDevice, l.st));
        NK(nccl().AllReduce(d, d, 1, ncclInt64, ncclMin, comm, l.st));
        CK(cudaMemcpyAsync(&mn, d, sizeof(int64_t), cudaMemcpyDeviceToHost, l.st));
        CK(cudaFreeAsync(d, l.st));
        CK(cudaStreamSynchronize(l.st));
      }
      std::fill(b.begin(), b.end(), mn);
    }
    budget_cache = b;
    budget_cache_n = n;
    return b;
  }

  // ---------------------------------------------------------------- op replay

  cudaEvent_t record(int gi) { return record_on(gi, g[gi].st); }
  cudaEvent_t record_on(int gi, cudaStream_t s) {
    LGpu &l = g[gi];
    cudaEvent_t e = devs[l.dev].sync_events.get();
    CK(cudaSetDevice(l.dev));
    CK(cudaEventRecord(e, s));
    return e;
  }
  // Peer moves run on their own stream, ordered with the kernels by events only: the
  // transfer overlaps the kernels of earlier stages, and in multi-process mode an ncclSend
  // does not hold the sender's compute stream until the receiver's stream reaches the
  // matching ncclRecv.  All NCCL calls of a rank stay on one
  // stream in the global plan order (the pairing argument of the op list is unchanged).
  // A peer move for the chunk being built may start once the compute stream has finished the
  // chunk before the last flushed one: the peer stream runs at most ~2 stages ahead, so
  // replicas are not allocated far ahead of the frees the plan's budget assumed.
  void pace_peer(LGpu &l) {
    const size_t nf = l.flush_ev.size();
    if (nf >= 2) CK(cudaStreamWaitEvent(l.pst, l.flush_ev[nf - 2], 0));
  }

  double2 *alloc(LGpu &l, int64_t bytes) { return (double2 *)alloc_on(l, bytes, l.st); }

  // A stream-ordered allocation that survives transient pool pressure.  The plan keeps each
  // GPU's live set inside its budget in plan order, but the copy and peer streams run ahead of
  // the compute stream, so an allocation can be made while frees the plan placed before it are
  // still queued behind kernels, and the pool cannot hand their blocks out yet; with very large
  // tensors (C5's 17.2 GB rank-4 intermediates) and a budget near the device size that can
  // exhaust the device.  On an out-of-memory error: drain this device's streams (the queued
  // frees complete), retry; then return the pool's cached blocks to the driver, retry; only then
  // fail (MICCO_ERR_OOM).
  void *alloc_on(LGpu &l, int64_t bytes, cudaStream_t s) {
    void *p = nullptr;
    cudaError_t e = cudaMallocAsync(&p, (size_t)bytes, s);
    if (e == cudaErrorMemoryAllocation) {
      cudaGetLastError();  // (not sticky)
      for (auto &o : g)
        if (o.local && o.dev == l.dev) {
          CK(cudaStreamSynchronize(o.st));
          CK(cudaStreamSynchronize(o.cst));
          CK(cudaStreamSynchronize(o.pst));
        }
      ++oom_retries;
      e = cudaMallocAsync(&p, (size_t)bytes, s);
      if (e == cudaErrorMemoryAllocation) {
        cudaGetLastError();
        cudaMemPool_t pool;
        CK(cudaDeviceGetDefaultMemPool(&pool, l.dev));
        CK(cudaMemPoolTrimTo(pool, 0));
        e = cudaMallocAsync(&p, (size_t)bytes, s);
      }
      if (e == cudaErrorMemoryAllocation) {
        cudaGetLastError();
        fail(MICCO_ERR_OOM, "device allocation of " + std::to_string(bytes) + " B failed after draining the streams");
      }
    }
    CK(e);
    return p;
  }

  int64_t bytes_of(int32_t x) const { return c.tensors[x].bytes(c.Lt); }

  const double *host_src(int32_t x) const {
    const TensorRec &t = c.tensors[x];
    if (t.node >= 0) {
      if (!c.nodes[t.node].host) materialize_nodes(c, {t.node});  // (streamed plans only)
      if (!c.nodes[t.node].host) fail(MICCO_ERR_STATE, "executor: node data not materialised");
      return c.nodes[t.node].host;
    }
    auto it = spill_host.find(x);
    if (it == spill_host.end()) fail(MICCO_ERR_STATE, "executor: missing host copy");
    return it->second;
  }

  template <typename D, typename Batch, typename Prefix>
  void launch_batch(LGpu &l, std::vector<D> &v, int kind, int cls, Batch &b, int cap, Prefix &&prefix,
                    cudaStream_t (*pick)(LGpu &, int) = nullptr) {
    if (v.empty()) return;
    for (size_t i0 = 0; i0 < v.size(); i0 += (size_t)cap) {
      const int cnt = (int)std::min((size_t)cap, v.size() - i0);
      b.n = cnt;
      std::memcpy(b.d, &v[i0], cnt * sizeof(D));
      const long long total = prefix(b.d, cnt);  // grid offsets of this launch
      const cudaStream_t s = pick ? pick(l, launch_seq++) : l.st;
      Timed tm{devs[l.dev].timing_events.get(), devs[l.dev].timing_events.get(), kind, l.dev};
      CK(cudaEventRecord(tm.a, s));
      if constexpr (std::is_same<D, GemmDesc>::value) CK(launch_gemm_group(&b, total, cls, s));
      else CK(launch_dot_group(&b, total, cls, s));
      CK(cudaEventRecord(tm.b, s));
      timed.push_back(tm);
      ++launches;
    }
    v.clear();
  }

  // Small dots that share their A operand go to the shared-operand kernel (kernels.h
  // DotGroupBatch).  Batches keep the plan order (so a launch covers the same operands as an
  // ungrouped one); inside a batch the descriptors are ordered by A (stable) and consecutive
  // equal A's form groups of up to kDotGroupPartners (splitting is exact: a dot's value does
  // not depend on its group).
  void launch_shared_groups(LGpu &l, std::vector<DotDesc> &v) {
    auto key = [](const DotDesc &d) {
      return std::make_tuple((uintptr_t)d.A, d.sAt, d.sAy, d.X, d.Y, d.mode, d.sBt, d.sBx, d.sBy);
    };
    DotGroupBatch &b = *dot_group_batch;
    for (size_t i0 = 0; i0 < v.size(); i0 += kDotGroupBatch) {
      const int cnt = (int)std::min((size_t)kDotGroupBatch, v.size() - i0);
      std::stable_sort(v.begin() + i0, v.begin() + i0 + cnt,
                       [&](const DotDesc &x, const DotDesc &y) { return key(x) < key(y); });
      b.n = cnt;
      b.n_groups = 0;
      for (int k = 0; k < cnt; ++k) {
        b.d[k] = v[i0 + k];
        if (k == 0 || key(b.d[k]) != key(b.d[k - 1]) || k - b.first[b.n_groups - 1] == kDotGroupPartners)
          b.first[b.n_groups++] = (short)k;
      }
      b.first[b.n_groups] = (short)cnt;
      Timed tm{devs[l.dev].timing_events.get(), devs[l.dev].timing_events.get(), 3, l.dev};
      CK(cudaEventRecord(tm.a, l.st));
      CK(launch_dot_shared_group(&b, c.Lt, l.st));
      CK(cudaEventRecord(tm.b, l.st));
      timed.push_back(tm);
      ++launches;
    }
    v.clear();
  }

  static cudaStream_t pick_gemm(LGpu &l, int seq) { return (seq & 1) ? l.kst[0] : l.st; }

  void flush(LGpu &l) {
    NvtxRange nr("micco flush");
    CK(cudaSetDevice(l.dev));
    if (l.gemm.empty() && l.dot.empty()) return;
    launch_seq = 0;
    if (!l.gemm.empty()) {  // one grouped launch per operand-layout class
      // fork the side stream off the compute stream (after this chunk's allocations and copy
      // waits); the launches alternate between the two, joined back below before the dots
      const cudaEvent_t fork = record_on(l.idx, l.st);
      for (cudaStream_t k : l.kst) CK(cudaStreamWaitEvent(k, fork, 0));
      std::vector<GemmDesc> by[kGemmClasses];
      std::vector<size_t> tma_idx[kGemmClasses];
      for (size_t i = 0; i < l.gemm.size(); ++i) {
        const GemmDesc &d = l.gemm[i];
        if (d.cls >= kGemmClassTMA) tma_idx[d.cls].push_back(i);
        else by[d.cls].push_back(d);
      }
      for (int c = kGemmClassTMA; c < kGemmClasses; ++c) {  // TMA kernel: descriptors + tensor maps
        const std::vector<size_t> &ix = tma_idx[c];
        for (size_t i0 = 0; i0 < ix.size(); i0 += kGemmTmaBatch) {
          const int cnt = (int)std::min((size_t)kGemmTmaBatch, ix.size() - i0);
          GemmTmaBatch &b = *tma_batch;
          b.n = cnt;
          long long acc = 0;
          for (int k = 0; k < cnt; ++k) {
            b.d[k] = l.gemm[ix[i0 + k]];
            b.map[2 * k] = l.gemm_maps[ix[i0 + k]][0];
            b.map[2 * k + 1] = l.gemm_maps[ix[i0 + k]][1];
            b.d[k].tile_begin = acc;
            acc += (long long)b.d[k].Lt * b.d[k].Mo * b.d[k].No * b.d[k].tilesM * b.d[k].tilesN;
          }
          const cudaStream_t s = pick_gemm(l, launch_seq++);
          Timed tm{devs[l.dev].timing_events.get(), devs[l.dev].timing_events.get(), 0, l.dev};
          CK(cudaEventRecord(tm.a, s));
          CK(launch_gemm_tma_group(&b, acc, c, s));
          CK(cudaEventRecord(tm.b, s));
          timed.push_back(tm);
          ++launches;
          ++tma_launches;
        }
      }
      l.gemm.clear();
      l.gemm_maps.clear();
      for (int c = 0; c < kGemmClassTMA; ++c)
        launch_batch(l, by[c], 0, c, *gemm_batch, kGemmBatch, [](GemmDesc *d, int cnt) {
          long long acc = 0;
          for (int i = 0; i < cnt; ++i) {
            d[i].tile_begin = acc;
            acc += (long long)d[i].Lt * d[i].Mo * d[i].No * d[i].tilesM * d[i].tilesN;
          }
          return acc;
        }, pick_gemm);
    }
    if (launch_seq > 1)  // join (with one launch the side stream got no work)
      for (cudaStream_t k : l.kst) CK(cudaStreamWaitEvent(l.st, record_on(l.idx, k), 0));
    if (!l.dot.empty()) {  // one launch group per dot kernel (kernels.h dot_class)
      std::vector<DotDesc> by[2], grp;
      for (const DotDesc &d : l.dot) {
        if (dot_class(d.mode) == 1 && dot_groupable(d)) grp.push_back(d);
        else by[dot_class(d.mode)].push_back(d);
      }
      l.dot.clear();
      launch_shared_groups(l, grp);
      for (int c = 0; c < 2; ++c) {
        launch_batch(l, by[c], c == 0 ? 1 : 3, c, *dot_batch, kDotBatch, [](DotDesc *d, int cnt) {
          long long acc = 0;
          for (int i = 0; i < cnt; ++i) {
            d[i].cta_begin = acc;
            acc += d[i].Lt;
          }
          return acc;
        });
      }
    }
    for (double2 *p : l.part_allocs) CK(cudaFreeAsync(p, l.st));
    l.part_allocs.clear();
  }

  void compute(LGpu &l, int32_t task, micco_stats &st) {
    const TaskRec &tk = c.tasks[task];
    const TensorRec &A = c.tensors[tk.a];
    double2 *pa = l.ptr[tk.a];
    if (!pa) fail(MICCO_ERR_STATE, "executor: operand not resident");
    if (tk.kind == TASK_GEMM) {
      const TensorRec &B = c.tensors[tk.b];
      double2 *pb = l.ptr[tk.b];
      if (!pb) fail(MICCO_ERR_STATE, "executor: operand not resident");
      GemmLayout L;
      if (!gemm_layout(A.rank, A.dim, B.rank, B.dim, tk.c, tk.pa, tk.pb, L))
        fail(MICCO_ERR_UNSUPPORTED, "executor: GEMM layout");
      const long long lim = (1LL << 31) - 1;  // the GEMM keeps per-slice offsets in 32 bits
      if (L.sliceA > lim || L.sliceB > lim || L.sliceC > lim)
        fail(MICCO_ERR_UNSUPPORTED, "executor: tensor slice exceeds 2^31 elements");
      const int32_t fd = fused_dot.empty() ? -1 : fused_dot[task];
      double2 *pc = fd >= 0 ? nullptr : alloc(l, bytes_of(tk.out));
      l.ptr[tk.out] = pc;
      GemmDesc d{};
      d.A = pa; d.B = pb; d.C = pc;
      d.sAt = L.sliceA; d.sBt = L.sliceB; d.sCt = L.sliceC;
      d.Mo = L.Mo; d.Mi = L.Mi; d.No = L.No; d.Ni = L.Ni; d.Ko = L.Ko; d.Ki = L.Ki;
      d.sAmo = L.sAmo; d.sAmi = L.sAmi; d.sAko = L.sAko; d.sAki = L.sAki;
      d.sBko = L.sBko; d.sBki = L.sBki; d.sBno = L.sBno; d.sBni = L.sBni;
      d.sCmo = L.sCmo; d.sCmi = L.sCmi; d.sCno = L.sCno; d.sCni = L.sCni;
      d.Lt = c.Lt;
      d.cls = gemm_kernel_class(gemm_class(L), L.Ko);
      std::array<CUtensorMap, 2> maps;
      {
        int tcls;  // the TMA kernel when the operands fit its tensor maps (kernels.cu gemm_tma_class)
        if (use_tma && gemm_tma_class(d, &tcls) && gemm_tma_encode(d, tcls, &maps[0], &maps[1])) d.cls = tcls;
      }
      int tbm, tbn;
      gemm_tile_shape(d.cls, &tbm, &tbn);
      d.tilesM = (L.Mi + tbm - 1) / tbm;
      d.tilesN = (L.Ni + tbn - 1) / tbn;
      if ((long long)c.Lt * L.Mo * L.No * d.tilesM * d.tilesN >= (1LL << 32))
        fail(MICCO_ERR_UNSUPPORTED, "executor: more than 2^32 tiles in one contraction");
      if (fd >= 0) {  // final dot in the epilogue: C is never materialised
        const TaskRec &dk = c.tasks[fd];
        const int32_t X = tk.out, Y = dk.a == X ? dk.b : dk.a;
        const TensorRec &YT = c.tensors[Y];
        int q[2] = {0, 1};  // Y leg paired with X leg 0 (M) and X leg 1 (N)
        for (int i = 0; i < dk.c; ++i) {
          if (dk.a == X) q[dk.pa[i]] = dk.pb[i]; else q[dk.pb[i]] = dk.pa[i];
        }
        const long long sY[2] = {YT.dim[1], 1};
        d.D = l.ptr[Y];
        if (!d.D) fail(MICCO_ERR_STATE, "executor: fused dot partner not resident");
        d.sDt = YT.slice_elems;
        d.sDmo = d.sDno = 0;
        d.sDmi = sY[q[0]];
        d.sDni = sY[q[1]];
        const long long tps = (long long)L.Mo * L.No * d.tilesM * d.tilesN * gemm_warps_per_tile(d.cls);  // partials per slice
        d.part = alloc(l, tps * c.Lt * 16);
        l.part_allocs.push_back(d.part);
        DotDesc r{};
        r.A = d.part; r.B = nullptr;
        r.out = table_row(l, c.tensors[dk.out].scalar_slot);
        r.sAt = tps; r.mode = 3; r.X = (int)tps; r.Lt = c.Lt;
        for (int i = 0; i < 3; ++i) r.O[i] = 1;
        l.dot.push_back(r);
        st.dot_bytes += (double)YT.slice_elems * 16.0 * c.Lt;
      }
      l.gemm.push_back(d);
      l.gemm_maps.push_back(maps);
      st.gemm_flops += tk.flops;
      const bool m3 = gemm_uses_3m(d.cls);
      st.gemm_dmma_flops += m3 ? tk.flops * 0.75 : tk.flops;
      if (m3) st.gemm_3m = 1;
    } else {
      DotLayout L;
      double2 *pb = nullptr;
      bool ok;
      if (tk.kind == TASK_TRACE) {
        ok = dot_layout(A.rank, A.dim, 0, nullptr, 1, tk.pa, tk.pb, L);
      } else {
        const TensorRec &B = c.tensors[tk.b];
        pb = l.ptr[tk.b];
        if (!pb) fail(MICCO_ERR_STATE, "executor: operand not resident");
        ok = dot_layout(A.rank, A.dim, B.rank, B.dim, tk.c, tk.pa, tk.pb, L);
      }
      if (!ok) fail(MICCO_ERR_UNSUPPORTED, "executor: dot layout");
      if (L.sliceA > (1LL << 31) - 1)  // the dot kernel's short-run path indexes a slice in 32 bits
        fail(MICCO_ERR_UNSUPPORTED, "executor: tensor slice exceeds 2^31 elements");
      DotDesc d{};
      d.A = pa; d.B = pb;
      d.out = table_row(l, c.tensors[tk.out].scalar_slot);
      d.sAt = L.sliceA; d.sBt = L.sliceB;
      d.mode = L.mode; d.nO = L.nO; d.X = L.X; d.Y = L.Y;
      d.sAx = L.sAx; d.sAy = L.sAy; d.sBx = L.sBx; d.sBy = L.sBy;
      for (int i = 0; i < 3; ++i) { d.O[i] = L.O[i]; d.sAo[i] = L.sAo[i]; d.sBo[i] = L.sBo[i]; }
      d.Lt = c.Lt;
      l.dot.push_back(d);
      st.dot_bytes += (double)(L.sliceA + L.sliceB) * 16.0 * c.Lt;
      if (dot_class(L.mode) == 1) st.dot_main_bytes += (double)(L.sliceA + L.sliceB) * 16.0 * c.Lt;
    }
  }

  void run_op(const PlanOp &op, micco_stats &st) {
    switch (op.kind) {
      case PlanOp::H2D: {
        NvtxRange nr("micco h2d");
        // Prefetch on the copy stream (NEXT #1 of SURVEY.md §8(f); "asynchronous
        // data copy and prefetching"): the copy for chunk k+1 may start once chunk k-1 has
        // finished (bounded look-ahead: at most prefetch_cap bytes beyond the planned budget);
        // the compute stream waits for the copy right away, so everything it enqueues later
        // (kernels, peer reads) sees the data, while already-enqueued kernels keep running.
        LGpu &l = g[op.gpu];
        if (!l.local) return;
        CK(cudaSetDevice(l.dev));
        // look-ahead: the copy for stage s may run while stages s-1 .. s-kLookahead compute;
        // bounded by bytes so the pool stays within the device memory the budgets leave free
        {
          const int64_t nb = bytes_of(op.id);
          l.fetch_bytes_since.push_back(nb);
          size_t nf = l.flush_ev.size();
          int64_t ahead = 0;
          int depth = 0;
          // walk back over flushed chunks while the prefetch window stays small
          while (depth < kLookahead && depth < (int)nf) {
            ahead += l.chunk_fetch[nf - 1 - depth];
            if (ahead > l.prefetch_cap) break;
            ++depth;
          }
          if ((int)nf > depth) CK(cudaStreamWaitEvent(l.cst, l.flush_ev[nf - 1 - depth], 0));
          l.pending_fetch += nb;
        }
        auto it = spill_ev.find(op.id);  // a spilled intermediate: wait for its D2H
        if (it != spill_ev.end() && c.tensors[op.id].node < 0) CK(cudaStreamWaitEvent(l.cst, it->second.second, 0));
        void *p = nullptr;
        p = alloc_on(l, bytes_of(op.id), l.cst);
        Timed tm{devs[l.dev].timing_events.get(), devs[l.dev].timing_events.get(), 2, l.dev};
        CK(cudaEventRecord(tm.a, l.cst));
        CK(cudaMemcpyAsync(p, host_src(op.id), bytes_of(op.id), cudaMemcpyHostToDevice, l.cst));
        CK(cudaEventRecord(tm.b, l.cst));
        timed.push_back(tm);
        cudaEvent_t done = devs[l.dev].sync_events.get();
        CK(cudaEventRecord(done, l.cst));
        CK(cudaStreamWaitEvent(l.st, done, 0));
        l.ptr[op.id] = (double2 *)p;
        st.bytes_h2d += bytes_of(op.id);
        return;
      }
      case PlanOp::P2P: {  // on the peer stream, ordered with the kernels by events (pace_peer)
        NvtxRange nr("micco p2p");
        LGpu &dst = g[op.gpu];
        LGpu &src = g[op.src];
        const int64_t nb = bytes_of(op.id);
        if (dist()) {
          if (dst.local) {
            CK(cudaSetDevice(dst.dev));
            cudaStream_t s = dst.pst;
            pace_peer(dst);
            void *p = alloc_on(dst, nb, s);
            NK(nccl().Recv(p, (size_t)nb / 8, ncclDouble, op.src, comm, s));
            CK(cudaStreamWaitEvent(dst.st, record_on(op.gpu, s), 0));  // consumers wait
            dst.ptr[op.id] = (double2 *)p;
            st.bytes_p2p += nb;
          } else if (src.local) {
            CK(cudaSetDevice(src.dev));
            CK(cudaStreamWaitEvent(src.pst, record(op.src), 0));  // the replica is complete
            NK(nccl().Send(src.ptr[op.id], (size_t)nb / 8, ncclDouble, op.gpu, comm, src.pst));
            src.readers[op.id].push_back(record_on(op.src, src.pst));  // a free waits for the send
          }
          return;
        }
        cudaEvent_t ready = record(op.src);  // the replica on src is complete
        CK(cudaSetDevice(dst.dev));
        cudaStream_t s = dst.pst;
        CK(cudaStreamWaitEvent(s, ready, 0));
        pace_peer(dst);
        double2 *p = (double2 *)alloc_on(dst, nb, s);
        if (dst.dev == src.dev)
          CK(cudaMemcpyAsync(p, src.ptr[op.id], nb, cudaMemcpyDeviceToDevice, s));
        else
          CK(cudaMemcpyPeerAsync(p, dst.dev, src.ptr[op.id], src.dev, nb, s));
        cudaEvent_t done = record_on(op.gpu, s);
        CK(cudaStreamWaitEvent(dst.st, done, 0));
        dst.ptr[op.id] = p;
        src.readers[op.id].push_back(done);
        st.bytes_p2p += nb;
        return;
      }
      case PlanOp::SPILL: {
        LGpu &l = g[op.gpu];
        if (!l.local) return;
        CK(cudaSetDevice(l.dev));
        double *h = spill_arena.alloc(bytes_of(op.id));
        CK(cudaMemcpyAsync(h, l.ptr[op.id], bytes_of(op.id), cudaMemcpyDeviceToHost, l.st));
        spill_host[op.id] = h;
        spill_ev[op.id] = {l.dev, record(op.gpu)};
        st.bytes_d2h += bytes_of(op.id);
        return;
      }
      case PlanOp::FREE: {
        if (op.gpu < 0) { spill_host.erase(op.id); spill_ev.erase(op.id); return; }
        LGpu &l = g[op.gpu];
        if (!l.local) return;
        CK(cudaSetDevice(l.dev));
        auto it = l.readers.find(op.id);
        if (it != l.readers.end()) {
          for (cudaEvent_t e : it->second) CK(cudaStreamWaitEvent(l.st, e, 0));
          l.readers.erase(it);
        }
        if (l.ptr[op.id]) CK(cudaFreeAsync(l.ptr[op.id], l.st));
        l.ptr[op.id] = nullptr;
        return;
      }
      case PlanOp::COMPUTE: {
        LGpu &l = g[op.gpu];
        if (!l.local) return;
        CK(cudaSetDevice(l.dev));
        compute(l, op.id, st);
        return;
      }
      case PlanOp::FLUSH: {
        LGpu &l = g[op.gpu];
        if (!l.local) return;
        flush(l);
        l.flush_ev.push_back(record(op.gpu));
        l.chunk_fetch.push_back(l.pending_fetch);
        l.pending_fetch = 0;
        return;
      }
    }
  }

  // ---------------------------------------------------------------- execute

  // Any failure inside an execute (a CUDA error, a planner exception rethrown mid-replay)
  // leaves per-GPU state that the next execute must not see: pending descriptors whose
  // output pointers may point into a freed table, replicas the cache bookkeeping no longer
  // matches.  Drain the streams and drop all of it, then rethrow.
  void execute(int n_gpus, const int32_t *bd) {
    try {
      execute_impl(n_gpus, bd);
    } catch (...) {
      recover();
      throw;
    }
  }

  void recover() noexcept {
    for (auto &l : g) {
      if (!l.local || !l.st) continue;
      cudaSetDevice(l.dev);
      cudaStreamSynchronize(l.st);
      if (l.cst) cudaStreamSynchronize(l.cst);
      if (l.pst) cudaStreamSynchronize(l.pst);
      for (cudaStream_t k : l.kst)
        if (k) cudaStreamSynchronize(k);
      for (auto &p : l.ptr)
        if (p) { cudaFree(p); p = nullptr; }
      for (double2 *p : l.part_allocs) cudaFree(p);
      l.part_allocs.clear();
      l.gemm.clear();
      l.gemm_maps.clear();
      l.dot.clear();
      l.readers.clear();
      l.flush_ev.clear();
      l.chunk_fetch.clear();
      l.fetch_bytes_since.clear();
      l.pending_fetch = 0;
    }
    cudaGetLastError();  // (a non-sticky error must not leak into the next call)
    cached_nodes.clear();
    stream_ok_n = 0;
    spill_host.clear();
    spill_ev.clear();
    spill_arena.rewind();
  }

  void execute_impl(int n_gpus, const int32_t *bd) {
    NvtxRange nr("micco_execute");
    auto t0 = std::chrono::steady_clock::now();
    setup(n_gpus);
    for (auto &l : g)
      if (l.local && l.ptr.size() < c.tensors.size()) l.ptr.resize(c.tensors.size(), nullptr);
    launches = 0;
    tma_launches = 0;
    oom_retries = 0;
    timed.clear();
    for (auto &l : g) {
      l.flush_ev.clear();
      l.chunk_fetch.clear();
      l.fetch_bytes_since.clear();
      l.pending_fetch = 0;
    }
    for (auto &d : devs) { d.sync_events.reset(); d.timing_events.reset(); }
    // per-device time origin of the kernel/copy intervals (the streams are idle here, so every
    // later launch on any stream of the device starts after it)
    time_ref.assign(ndev, nullptr);
    for (auto &l : g)
      if (l.local && !time_ref[l.dev]) {
        time_ref[l.dev] = devs[l.dev].timing_events.get();
        CK(cudaSetDevice(l.dev));
        CK(cudaEventRecord(time_ref[l.dev], l.st));
      }

    PlanInput in;
    in.n_gpus = n;
    in.policy = c.opt.policy;
    in.budget = budgets();
    in.window_graphs = c.opt.window_graphs;
    in.keep_inputs = c.opt.keep_inputs_resident != 0;
    in.fuse = true;  // GEMM → final dot in the GEMM epilogue when legal (every GEMM kernel has it)
    {  // MICCO_GEMM_TMA=0: keep every contraction on the cp.async kernels (read per execute; the
       // parity suite runs both paths)
      const char *e = getenv("MICCO_GEMM_TMA");
      use_tma = !(e && e[0] == '0');
    }
    in.peer_gbs = (ndev > 1 && !dist()) || dist() ? kModelPeerGBs : kModelLocalCopyGBs;
    in.host_gbs = kModelHostGBs;
    in.flops_per_s = kModelFlopsPerS;
    // node replicas cached by the previous execute: the previous plan's final residency,
    // identical on every rank (the local pointers must agree with it)
    in.initial_nodes.assign(n, {});
    if (in.keep_inputs)
      for (const auto &fn : cached_nodes)
        for (int i = 0; i < n; ++i)
          if ((fn.second >> i) & 1) {
            if (g[i].local && !g[i].ptr[fn.first]) fail(MICCO_ERR_STATE, "executor: cache out of sync");
            in.initial_nodes[i].push_back(fn.first);
          }
    Plan plan;
    bool sweep = false;  // whole-plan bound sweep (27 plans): synchronous
    // choices cached across executes are valid for this GPU count and this DAG
    const int64_t dag_key = ((int64_t)c.tasks.size() * 1000003 + (int64_t)c.graphs.size()) * 8 + c.opt.policy;
    if (dag_key != cache_dag_key) {
      chosen_bd_n = chosen_w_n = 0;
      cache_dag_key = dag_key;
    }
    for (int i = 0; i < 3; ++i) in.reuse_bound[i] = 0;
    if (!bd && c.opt.bound_model != BOUNDS_FIXED) {  // per-vector bounds (sweep or regression)
      in.bound_mode = c.opt.bound_model;
    } else if (bd) {
      for (int i = 0; i < 3; ++i) in.reuse_bound[i] = bd[i];
    } else if (chosen_bd_n == n) {  // bounds chosen by an earlier sweep for this GPU count
      for (int i = 0; i < 3; ++i) in.reuse_bound[i] = chosen_bd[i];
    } else {
      sweep = true;
    }
    if (in.window_graphs <= 0) {  // options.window_graphs == 0: sized to the budget
      if (chosen_w_n != n) {
        chosen_w = choose_window(c, in);
        chosen_w_n = n;
      }
      in.window_graphs = chosen_w;
    }
    // Streamed planning: once an execute on this GPU count has materialised the synthetic
    // nodes this process uploads, later executes plan on a host thread and replay each stage
    // as soon as it is final (PlanStream), so the GPU starts after the first stage is planned
    // instead of the whole DAG (every rank plans the whole DAG: the plan grows with n).
    const char *nps = getenv("MICCO_NO_PLAN_STREAM");
    const bool streaming = !sweep && stream_ok_n == n && !(nps && nps[0] == '1');
    PlanStream ps;
    std::thread planner;
    std::exception_ptr plan_err;
    double plan_ms = 0;
    if (streaming) {
      in.stream = &ps;
      planner = std::thread([&] {
        NvtxRange pr("micco plan (streamed)");
        auto p0 = std::chrono::steady_clock::now();
        try {
          plan = make_plan(c, in);
          ps.publish_ops(plan.ops);
        } catch (...) {
          plan_err = std::current_exception();
        }
        plan_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - p0).count();
        ps.finish();
      });
    } else {
      NvtxRange pr(sweep ? "micco plan (bound sweep)" : "micco plan");
      if (sweep) {
        plan = make_plan_auto(c, in);
        for (int i = 0; i < 3; ++i) chosen_bd[i] = plan.reuse_bound[i];
        chosen_bd_n = n;
      } else {
        plan = make_plan(c, in);
      }
      cached_nodes = plan.final_nodes;
      fused_dot = plan.fused_dot;
      // synthetic nodes this process uploads must have host data (lazy in multi-process mode)
      std::vector<int32_t> need;
      for (const PlanOp &op : plan.ops)
        if (op.kind == PlanOp::H2D && g[op.gpu].local && c.tensors[op.id].node >= 0 &&
            !c.nodes[c.tensors[op.id].node].host)
          need.push_back(c.tensors[op.id].node);
      materialize_nodes(c, need);
      plan_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    }
    // the planner thread must be joined on every exit path
    struct Joiner {
      std::thread &t;
      ~Joiner() { if (t.joinable()) t.join(); }
    } joiner{planner};

    micco_stats st{};
    st.struct_size = sizeof(st);
    // scalar tables (one per device in use, or one per logical GPU), zeroed before any dot
    // writes; every logical GPU writing a table waits for its zeroing
    const size_t selems = (size_t)std::max(1, c.n_scalar_slots) * c.Lt;
    const int ntab = c.opt.scalar_tables ? n : ndev;
    if ((int)tables.size() < ntab) tables.resize(ntab);
    std::vector<int> first_lgpu(ntab, -1);  // the logical GPU that zeroes (and owns) table k
    for (int i = 0; i < n; ++i)
      if (g[i].local && first_lgpu[table_of(i)] < 0) first_lgpu[table_of(i)] = i;
    for (int k = 0; k < ntab; ++k) {
      if (first_lgpu[k] < 0) continue;
      LGpu &l = g[first_lgpu[k]];
      ScalarTable &T = tables[k];
      CK(cudaSetDevice(l.dev));
      if (T.elems < selems || T.dev != l.dev) {
        CK(cudaStreamSynchronize(l.st));
        if (T.p) { CK(cudaSetDevice(T.dev)); CK(cudaFree(T.p)); CK(cudaSetDevice(l.dev)); }
        CK(cudaMalloc((void **)&T.p, selems * sizeof(double2)));
        T.elems = selems;
        T.dev = l.dev;
      }
      CK(cudaMemsetAsync(T.p, 0, selems * sizeof(double2), l.st));
      cudaEvent_t e = record(first_lgpu[k]);
      for (int i = 0; i < n; ++i)
        if (g[i].local && table_of(i) == k && i != first_lgpu[k]) CK(cudaStreamWaitEvent(g[i].st, e, 0));
    }
    auto tq0 = std::chrono::steady_clock::now();
    if (streaming) {
      {
        std::unique_lock<std::mutex> lk(ps.m);
        ps.cv.wait(lk, [&] { return ps.have_fused; });
        fused_dot = ps.fused_dot;
      }
      std::vector<PlanOp> batch;
      for (;;) {
        bool fin;
        {
          std::unique_lock<std::mutex> lk(ps.m);
          ps.cv.wait(lk, [&] { return !ps.q.empty() || ps.done; });
          batch.swap(ps.q);
          fin = ps.done;  // finish() follows the last publish: nothing can arrive after this
        }
        for (const PlanOp &op : batch) run_op(op, st);
        batch.clear();
        if (fin) break;
      }
      planner.join();
      if (plan_err) std::rethrow_exception(plan_err);
      cached_nodes = plan.final_nodes;
    } else {
      for (const PlanOp &op : plan.ops) run_op(op, st);
    }
    st.enqueue_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - tq0).count();
    st.host_pinned = c.arena.pinned() ? 1 : 0;
    for (auto &l : g)
      if (l.local && (!l.gemm.empty() || !l.dot.empty())) flush(l);
    // intermediates must all be released by now; drop leftovers defensively
    for (auto &l : g) {
      if (!l.local) continue;
      CK(cudaSetDevice(l.dev));
      for (size_t x = 0; x < l.ptr.size(); ++x)
        if (l.ptr[x] && !(in.keep_inputs && c.tensors[x].node >= 0)) {
          auto it = l.readers.find((int32_t)x);
          if (it != l.readers.end())
            for (cudaEvent_t e : it->second) CK(cudaStreamWaitEvent(l.st, e, 0));
          CK(cudaFreeAsync(l.ptr[x], l.st));
          l.ptr[x] = nullptr;
        }
      l.readers.clear();
    }

    // combine devices, finalize on the "home" GPU
    const int home = dist() ? my_rank() : 0;
    LGpu &H = g[home];
    CK(cudaSetDevice(H.dev));
    for (int i = 0; i < n; ++i)
      if (i != home && g[i].local) CK(cudaStreamWaitEvent(H.st, record(i), 0));
    double2 *S = tables[table_of(home)].p;
    if (dist()) {
      // every NCCL call of this rank in one order: the all-reduce after the last send/recv
      if (H.pst) CK(cudaStreamWaitEvent(H.st, record_on(home, H.pst), 0));
      NK(nccl().AllReduce(S, S, selems * 2, ncclDouble, ncclSum, comm, H.st));
    } else {
      // Exact combine: every slot is nonzero in exactly one table (the producing GPU's), so
      // S += T adds zeros everywhere else, and the result is bitwise independent of the GPU
      // count and of the order of the tables (north_star: final cross-GPU reduce).
      for (int k = 0; k < ntab; ++k) {
        if (k == table_of(home) || first_lgpu[k] < 0) continue;
        const ScalarTable &T = tables[k];
        double2 *tmp = alloc(H, (int64_t)(selems * sizeof(double2)));
        if (T.dev == H.dev)
          CK(cudaMemcpyAsync(tmp, T.p, selems * sizeof(double2), cudaMemcpyDeviceToDevice, H.st));
        else
          CK(cudaMemcpyPeerAsync(tmp, H.dev, T.p, T.dev, selems * sizeof(double2), H.st));
        CK(launch_accumulate(S, tmp, (long long)selems, H.st));
        ++launches;
        CK(cudaFreeAsync(tmp, H.st));
      }
    }
    const int G = (int)c.graphs.size();
    std::vector<int> comp_off(G + 1), comp_slot;
    std::vector<double2> coefs(G);
    for (int gi = 0; gi < G; ++gi) {
      const GraphRec &gr = c.graphs[gi];
      comp_off[gi] = (int)comp_slot.size();
      for (int k = gr.comp_begin; k < gr.comp_end; ++k) comp_slot.push_back(c.tensors[c.graph_scalars[k]].scalar_slot);
      coefs[gi] = make_double2(gr.coef_re, gr.coef_im);
    }
    comp_off[G] = (int)comp_slot.size();
    if (comp_slot.empty()) comp_slot.push_back(0);
    int *d_off = (int *)alloc(H, (int64_t)comp_off.size() * 4);
    int *d_slot = (int *)alloc(H, (int64_t)comp_slot.size() * 4);
    double2 *d_coef = alloc(H, (int64_t)G * 16);
    CK(cudaMemcpyAsync(d_off, comp_off.data(), comp_off.size() * 4, cudaMemcpyHostToDevice, H.st));
    CK(cudaMemcpyAsync(d_slot, comp_slot.data(), comp_slot.size() * 4, cudaMemcpyHostToDevice, H.st));
    CK(cudaMemcpyAsync(d_coef, coefs.data(), (size_t)G * 16, cudaMemcpyHostToDevice, H.st));
    if (vals_elems < (size_t)G * c.Lt) {
      CK(cudaStreamSynchronize(H.st));
      if (d_vals) CK(cudaFree(d_vals));
      CK(cudaMalloc((void **)&d_vals, (size_t)G * c.Lt * sizeof(double2)));
      vals_elems = (size_t)G * c.Lt;
      vals_dev = H.dev;
    }
    if (!h_corr) CK(cudaHostAlloc((void **)&h_corr, 1 << 20, cudaHostAllocPortable));
    double2 *d_corr = alloc(H, (int64_t)c.Lt * 16);
    CK(launch_finalize(G, c.Lt, d_off, d_slot, S, d_vals, H.st));
    CK(launch_correlator_sum(G, c.Lt, d_coef, d_vals, d_corr, H.st));
    launches += 2;
    if ((size_t)c.Lt * 16 > (1 << 20)) fail(MICCO_ERR_ARG, "Lt too large");
    CK(cudaMemcpyAsync(h_corr, d_corr, (size_t)c.Lt * 16, cudaMemcpyDeviceToHost, H.st));
    CK(cudaFreeAsync(d_off, H.st));
    CK(cudaFreeAsync(d_slot, H.st));
    CK(cudaFreeAsync(d_coef, H.st));
    CK(cudaFreeAsync(d_corr, H.st));
    for (auto &l : g)
      if (l.local) {
        CK(cudaSetDevice(l.dev));
        CK(cudaStreamSynchronize(l.st));
        CK(cudaStreamSynchronize(l.cst));
        CK(cudaStreamSynchronize(l.pst));
      }
    auto t2 = std::chrono::steady_clock::now();

    c.corr.assign(2 * (size_t)c.Lt, 0.0);
    std::memcpy(c.corr.data(), h_corr, (size_t)c.Lt * 16);
    spill_host.clear();
    spill_ev.clear();
    spill_arena.rewind();  // keep the pinned spill chunks for the next execute

    // statistics: device time per kind = the union of its launches' intervals on each device
    // (launches of one chunk overlap on the side streams, so a plain sum would count the
    // overlap twice), summed over devices
    {
      std::vector<std::pair<float, float>> iv[5];  // gemm, dot (warp), copy, dot (CTA), all kernels
      auto union_ms = [](std::vector<std::pair<float, float>> &v) {
        std::sort(v.begin(), v.end());
        double tot = 0, a = 0, b = -1;
        for (const auto &x : v) {
          if (x.first > b) { if (b > a) tot += b - a; a = x.first; b = x.second; }
          else b = std::max(b, (double)x.second);
        }
        if (b > a) tot += b - a;
        v.clear();
        return tot;
      };
      for (int d = 0; d < ndev; ++d) {
        if (d >= (int)time_ref.size() || !time_ref[d]) continue;
        CK(cudaSetDevice(d));
        for (const Timed &tm : timed) {
          if (tm.dev != d) continue;
          float a = 0, b = 0;
          CK(cudaEventElapsedTime(&a, time_ref[d], tm.a));
          CK(cudaEventElapsedTime(&b, time_ref[d], tm.b));
          iv[tm.kind].push_back({a, b});
          if (tm.kind != 2) iv[4].push_back({a, b});
          if (tm.kind == 0) ++st.gemm_launches;
          else if (tm.kind == 1) ++st.dot_launches;
          else if (tm.kind == 3) { ++st.dot_launches; ++st.dot_main_launches; }
        }
        st.gemm_kernel_ms += union_ms(iv[0]);
        st.copy_ms += union_ms(iv[2]);
        iv[1].insert(iv[1].end(), iv[3].begin(), iv[3].end());
        st.dot_main_ms += union_ms(iv[3]);
        st.dot_kernel_ms += union_ms(iv[1]);
        st.kernel_ms += union_ms(iv[4]);
      }
    }
    st.wall_ms = std::chrono::duration<double, std::milli>(t2 - t0).count();
    st.sched_ms = plan_ms;  // planning time (overlapped with the replay when streamed)
    st.plan_ms = plan_ms;
    stream_ok_n = n;
    st.evictions = plan.evictions;
    st.cache_hits = plan.cache_hits;
    st.unique_tasks = (int64_t)c.tasks.size();
    st.dedup_hits = c.dedup_hits;
    st.component_dedup_hits = c.component_dedup_hits;
    for (const TaskRec &t : c.tasks) (t.kind == TASK_GEMM ? st.n_gemm : st.n_dot)++;
    st.n_stages = plan.n_stages;
    st.kernel_launches = launches;
    st.gemm_tma_launches = tma_launches;
    st.alloc_retries = oom_retries;
    st.flops = plan.flops;
    for (const GraphRec &gr : c.graphs) st.flops_no_dedup += gr.flops_no_dedup;
    st.max_over_mean_load = plan.max_over_mean_load;
    st.model_s = plan.predicted_s;
    for (int64_t b : plan.gpu_peak_bytes) st.peak_bytes = std::max(st.peak_bytes, b);
    st.window_graphs = plan.window_graphs;
    st.model_overlap_s = plan.predicted_overlap_s;
    for (int i = 0; i < 3; ++i) st.reuse_bound[i] = plan.reuse_bound[i];
    st.n_gpus = n;
    if (dist()) {  // plan-level byte counts are global; report them
      st.bytes_h2d = plan.bytes_h2d;
      st.bytes_p2p = plan.bytes_p2p;
      st.bytes_d2h = plan.bytes_d2h;
    }
    c.stats = st;
  }

  void fetch_graph_values() {
    const int G = (int)c.graphs.size();
    c.graph_vals.assign((size_t)G * c.Lt * 2, 0.0);
    const int home = dist() ? my_rank() : 0;
    CK(cudaSetDevice(g[home].dev));
    CK(cudaMemcpy(c.graph_vals.data(), d_vals, (size_t)G * c.Lt * 16, cudaMemcpyDeviceToHost));
    c.graph_vals_valid = true;
  }

  void release_cache() {
    for (auto &l : g) free_lgpu(l, false);
    cached_nodes.clear();
  }
};

Executor::Executor(Context &c) : p_(new Impl(c)) {}
Executor::~Executor() = default;
void Executor::execute(int n_gpus, const int32_t *bd) { p_->execute(n_gpus, bd); }
void Executor::fetch_graph_values() { p_->fetch_graph_values(); }
void Executor::release_cache() { p_->release_cache(); }

}  // namespace micco
