// proclus_api.cu -- the C ABI of include/proclus.h and the host driver of
// the B200 PROCLUS hot path.  The host only draws the sample (Alg 1 l.2) and
// the initial MCur, allocates everything up front and launches; the
// iterative phase (Alg 1 l.5-14) including its control runs on the device,
// by default as one CUDA graph whose while-node loops until the device-side
// control clears the condition (no host round trip per iteration).
#include <cuda_runtime.h>
#include <nccl.h>

#include <condition_variable>
#include <mutex>
#include <new>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <unordered_map>
#include <vector>

#include "../../include/proclus.h"
#include "proclus_kernels.h"

using namespace pc;

// ------------------------------------------------------------------ errors
static thread_local std::string g_err;

static proclus_status fail(proclus_status st, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return st;
}

#define CK(call)                                                              \
  do {                                                                        \
    cudaError_t e_ = (call);                                                  \
    if (e_ != cudaSuccess)                                                    \
      return fail(PROCLUS_ECUDA, "%s failed: %s (%s:%d)", #call,              \
                  cudaGetErrorString(e_), __FILE__, __LINE__);                \
  } while (0)

#define CKN(call)                                                             \
  do {                                                                        \
    ncclResult_t r_ = (call);                                                 \
    if (r_ != ncclSuccess)                                                    \
      return fail(PROCLUS_ENCCL, "%s failed: %s", #call,                      \
                  ncclGetErrorString(r_));                                    \
  } while (0)

#define TRY(expr)                                                             \
  do {                                                                        \
    proclus_status s_ = (expr);                                               \
    if (s_ != PROCLUS_OK) return s_;                                          \
  } while (0)

// ------------------------------------------------------------------ RNG
// SplitMix64 streams (reading R2).  Host side of the library; the oracle has
// its own independent implementation.
static uint64_t sm_next(uint64_t* s) {
  uint64_t z = (*s += 0x9E3779B97F4A7C15ULL);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
static uint64_t sm_uniform(uint64_t* s, uint64_t m) {
  return (uint64_t)(((unsigned __int128)sm_next(s) * m) >> 64);
}
static uint64_t sm_once(uint64_t x) { return sm_next(&x); }
static uint64_t stream_sm(uint64_t seed, int64_t k_sm) {
  return sm_once(sm_once(seed) + (uint64_t)k_sm);
}
static uint64_t stream_it(uint64_t seed, int64_t k, int64_t l) {
  return sm_once(sm_once(sm_once(seed) + (uint64_t)k) + (uint64_t)l + 4294967296ULL);
}

// ------------------------------------------------------------------ handle
template <class T>
struct DBuf {
  T* p = nullptr;
  size_t cap = 0;
  cudaError_t ensure(size_t count) {
    if (count <= cap && p) return cudaSuccess;
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
    cudaError_t e = cudaMalloc(&p, sizeof(T) * (count ? count : 1));
    if (e == cudaSuccess) cap = count;
    return e;
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
  }
};

enum Kind {
  K_PACK = 0, K_GATHER, K_GREEDY, K_PREPARE, K_LOC, K_ASG, K_COST, K_REF, K_FIN, K_SPLIT
};

// In-process communicator of `world` handles (test layer F): the
// shards' partial sums are combined by a host-staged reduction in fixed rank
// order, so the row-sharded schedule runs with G logical shards on one GPU
// and no NCCL.  Every rank calls the collectives from its own host thread;
// they rendezvous at a generation-counted barrier.
struct proclus_group {
  int world = 0;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  long long gen = 0;
  std::vector<std::vector<unsigned char>> slot;  // per rank: this collective's bytes
  void barrier() {
    std::unique_lock<std::mutex> lk(mu);
    const long long g = gen;
    if (++arrived == world) {
      arrived = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != g; });
    }
  }
};

struct proclus_handle {
  int dev = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int64_t n = 0, n_pad = 0, n_total = 0, row_offset = 0;
  int d = 0;
  int metric = 0, max_iter = 10000;
  bool data_on_device = false, trace = false, stats = false;
  int variant = 0;  // proclus_variant
  int world = 1, rank = 0;
  ncclComm_t comm = nullptr;
  proclus_group* group = nullptr;  // in-process communicator (instead of comm)
  int num_sms = 148;
  int64_t launches = 0;

  DBuf<float> xs, staging;
  // proclus_prefetch: H2D of the next dataset into `staging` on cstream
  cudaStream_t cstream = nullptr;
  cudaEvent_t pf_done = nullptr, pack_done = nullptr;
  const float* pf_src = nullptr;
  DBuf<int> flag;
  DBuf<unsigned> colmax;
  DBuf<double> scale, iscale;
  DBuf<int> qflag;  // device: quant_sum fma flag (RunParams::qflag)
  // init-phase products
  DBuf<long long> sids, mids;
  DBuf<float> srows, mrows;
  DBuf<int> spos;
  DBuf<double> pickdist, gscratch;
  int64_t nS = 0, nM = 0;
  bool m_valid = false;
  uint64_t m_seed = 0;
  int m_ksm = 0, m_A = 0, m_B = 0;
  // caches of GPU-FAST-PROCLUS (persist across settings of run_multi)
  DBuf<float> dist;
  DBuf<long long> Hq;
  DBuf<double> dprev;
  DBuf<long long> nL;
  DBuf<unsigned char> found, used;
  // per-run buffers
  DBuf<unsigned char> lab;
  DBuf<double> med, X, Z, mu, Delta;
  DBuf<int> dlist, pool, out_labels;
  DBuf<unsigned char> dmask;
  DBuf<long long> accg, cntg;
  DBuf<DevState> st;
  DevState* h_st = nullptr;  // pinned
  // pinned staging of the small mid-run / result reads (M ids, D mask): a
  // pageable D2H would wait behind a prefetch's H2D of the next dataset
  unsigned char* h_pin = nullptr;
  size_t h_pin_bytes = 0;
  // graph of one run (prepare -> while{loc, asg, cost} -> refine, final)
  // instantiated graphs by (RunParams, PassShape): a multi-parameter sweep
  // builds one per (k, l) setting (~0.7 ms of host capture + instantiation
  // with the GPU idle) and later sweeps of the same handle reuse them
  struct GraphEntry {
    RunParams key;
    PassShape shape;
    cudaGraphExec_t exec;
    unsigned long long used;
  };
  std::vector<GraphEntry> graphs;
  unsigned long long graph_tick = 0;
  cudaGraphExec_t gexec = nullptr;  // the graph of the current run (owned by graphs)
  // trace
  int tr_cap = 0;
  DBuf<int> t_mcur;
  DBuf<double> t_delta, t_cost, t_X;
  DBuf<long long> t_nL, t_sizes;
  DBuf<unsigned char> t_dims, t_improved, t_bad;
  int last_k = 0, tr_count = 0;
  // per-launch CUDA events (options.stats)
  struct Rec {
    int kind, iter;
    cudaEvent_t a, b;
  };
  std::vector<cudaEvent_t> evpool;
  size_t evnext = 0;
  std::vector<Rec> recs;
  size_t rec_done = 0;
  proclus_stats last_stats{};
};

static cudaEvent_t ev_get(proclus_handle* h) {
  if (h->evnext == h->evpool.size()) {
    cudaEvent_t e;
    cudaEventCreate(&e);
    h->evpool.push_back(e);
  }
  return h->evpool[h->evnext++];
}

// Launch `f` on the handle's stream, bracketed by events when stats are on.
template <class F>
static void launch(proclus_handle* h, int kind, int iter, F&& f) {
  h->launches += 1;
  if (!h->stats) {
    f();
    return;
  }
  cudaEvent_t a = ev_get(h), b = ev_get(h);
  cudaEventRecord(a, h->stream);
  f();
  cudaEventRecord(b, h->stream);
  h->recs.push_back({kind, iter, a, b});
}

static proclus_status set_device(proclus_handle* h) {
  CK(cudaSetDevice(h->dev));
  return PROCLUS_OK;
}

// Element-wise reduction of the ranks' slots in rank order 0, 1, ... (sum or
// max; the int64 cell sums are exact, the float sum adds one non-zero row).
template <class T>
static void group_reduce(proclus_group* g, size_t count, bool is_max, T* out) {
  for (size_t e = 0; e < count; ++e) {
    T acc = reinterpret_cast<const T*>(g->slot[0].data())[e];
    for (int r = 1; r < g->world; ++r) {
      const T v = reinterpret_cast<const T*>(g->slot[(size_t)r].data())[e];
      acc = is_max ? (v > acc ? v : acc) : (T)(acc + v);
    }
    out[e] = acc;
  }
}

static proclus_status allreduce(proclus_handle* h, void* buf, size_t count, ncclDataType_t t,
                                ncclRedOp_t op = ncclSum) {
  if (h->world <= 1) return PROCLUS_OK;
  if (!h->group) {
    CKN(ncclAllReduce(buf, buf, count, t, op, h->comm, h->stream));
    return PROCLUS_OK;
  }
  size_t es = 0;
  switch (t) {
    case ncclInt64: es = 8; break;
    case ncclUint32: case ncclInt32: case ncclFloat: es = 4; break;
    default: return fail(PROCLUS_EINTERNAL, "group allreduce: unsupported type");
  }
  proclus_group* g = h->group;
  std::vector<unsigned char> res(count * es);
  g->slot[(size_t)h->rank].resize(count * es);
  CK(cudaMemcpyAsync(g->slot[(size_t)h->rank].data(), buf, count * es, cudaMemcpyDeviceToHost,
                     h->stream));
  CK(cudaStreamSynchronize(h->stream));
  g->barrier();  // every rank's slot is filled
  const bool mx = op == ncclMax;
  if (t == ncclInt64) group_reduce(g, count, mx, reinterpret_cast<long long*>(res.data()));
  else if (t == ncclUint32) group_reduce(g, count, mx, reinterpret_cast<unsigned*>(res.data()));
  else if (t == ncclInt32) group_reduce(g, count, mx, reinterpret_cast<int*>(res.data()));
  else group_reduce(g, count, mx, reinterpret_cast<float*>(res.data()));
  g->barrier();  // every rank has read every slot
  CK(cudaMemcpyAsync(buf, res.data(), count * es, cudaMemcpyHostToDevice, h->stream));
  CK(cudaStreamSynchronize(h->stream));
  return PROCLUS_OK;
}

extern "C" {

const char* proclus_last_error(void) { return g_err.c_str(); }
int32_t proclus_abi_version(void) { return PROCLUS_ABI_VERSION; }
int32_t proclus_target_sm(void) { return 100; }

proclus_status proclus_group_create(int32_t world, proclus_group** out) {
  if (!out) return fail(PROCLUS_EINVAL, "out is NULL");
  *out = nullptr;
  if (world < 1 || world > 1024) return fail(PROCLUS_EINVAL, "world must be in [1, 1024]");
  proclus_group* g = new (std::nothrow) proclus_group;
  if (!g) return fail(PROCLUS_ENOMEM, "group allocation");
  g->world = world;
  g->slot.resize((size_t)world);
  *out = g;
  return PROCLUS_OK;
}

void proclus_group_destroy(proclus_group* g) { delete g; }

proclus_status proclus_options_init(proclus_options* opt) {
  if (!opt) return fail(PROCLUS_EINVAL, "opt is NULL");
  memset(opt, 0, sizeof(*opt));
  opt->device = -1;
  opt->metric = PROCLUS_METRIC_L2;
  opt->max_iter = 10000;
  opt->world_size = 1;
  return PROCLUS_OK;
}

}  // extern "C"

static proclus_status pin_ensure(proclus_handle* h, size_t bytes) {
  if (bytes <= h->h_pin_bytes) return PROCLUS_OK;
  if (h->h_pin) cudaFreeHost(h->h_pin);
  h->h_pin = nullptr;
  h->h_pin_bytes = 0;
  const size_t want = std::max<size_t>(bytes, 4096);
  if (cudaMallocHost((void**)&h->h_pin, want) != cudaSuccess)
    return fail(PROCLUS_ENOMEM, "cudaMallocHost(%zu) failed", want);
  h->h_pin_bytes = want;
  return PROCLUS_OK;
}

// Exact ceil(log2 x) for x > 0 from the binary exponent (the device's
// k_scales uses the same rule, so both load paths give identical scales).
static int ceil_log2(double x) {
  int ex;
  const double f = std::frexp(x, &ex);
  return f == 0.5 ? ex - 1 : ex;
}

// N0 pack + per-dimension fixed-point scales.  Cell sums of dimension j are
// bounded by 2 * n_total * max|x_j| (|x - c| with c inside the column range,
// or |x|), so e_j = 61 - ceil(log2(bound)) keeps every total below 2^61.
// sync = false (proclus_load on one GPU): the scales are computed on the
// device (k_scales) and nothing waits for the host; a non-finite value makes
// the next proclus_run return EINVAL (k_prepare stops it at once).
static proclus_status upload_data(proclus_handle* h, const float* data, bool sync) {
  const size_t bytes = sizeof(float) * (size_t)h->n * h->d;
  const float* src = data;
  if (!h->data_on_device) {
    CK(h->staging.ensure((size_t)h->n * h->d));
    if (h->pf_src) CK(cudaStreamWaitEvent(h->stream, h->pf_done, 0));  // staging is being filled
    if (h->pf_src != data)
      CK(cudaMemcpyAsync(h->staging.p, data, bytes, cudaMemcpyHostToDevice, h->stream));
    h->pf_src = nullptr;
    src = h->staging.p;
  }
  CK(cudaMemsetAsync(h->flag.p, 0, sizeof(int), h->stream));
  CK(cudaMemsetAsync(h->colmax.p, 0, sizeof(unsigned) * PACK_COPIES * h->d, h->stream));
  launch(h, K_PACK, -1, [&] {
    launch_pack_soa(src, h->n, h->d, h->n_pad, h->xs.p, h->flag.p, h->colmax.p, h->stream);
  });
  CK(cudaGetLastError());
  if (h->pack_done) CK(cudaEventRecord(h->pack_done, h->stream));  // staging read
  h->m_valid = false;  // cached M / Dist rows refer to old data
  if (!sync && h->world == 1) {
    launch_scales(h->colmax.p, h->d, h->n_total, h->scale.p, h->iscale.p, h->qflag.p, h->stream);
    CK(cudaGetLastError());
    return PROCLUS_OK;
  }
  TRY(allreduce(h, h->colmax.p, h->d, ncclUint32, ncclMax));
  TRY(allreduce(h, h->flag.p, 1, ncclInt32, ncclMax));
  int bad = 0;
  std::vector<unsigned> cm((size_t)h->d);
  CK(cudaMemcpyAsync(&bad, h->flag.p, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
  CK(cudaMemcpyAsync(cm.data(), h->colmax.p, sizeof(unsigned) * h->d, cudaMemcpyDeviceToHost,
                     h->stream));
  CK(cudaStreamSynchronize(h->stream));
  if (bad) return fail(PROCLUS_EINVAL, "data contains non-finite values");
  std::vector<double> sc((size_t)h->d), isc((size_t)h->d);
  int qmagic = 1;
  for (int j = 0; j < h->d; ++j) {
    float m;
    memcpy(&m, &cm[(size_t)j], sizeof(float));
    int e = 0;
    if (m > 0.f) {
      e = 61 - ceil_log2(2.0 * (double)h->n_total * (double)m);
      // one term (<= 2 max|x_j|) stays below 2^51: the per-term quantisation
      // of the lane-private passes keeps it in the low mantissa bits of a double
      e = std::min(e, 50 - ceil_log2(2.0 * (double)m));
      e = std::max(-1000, std::min(1000, e));
      // a band sum of <= 256 terms (<= 512 max|x_j|, one chunk of the wide
      // locality consumer) below 2^51: quant_sum's fma path
      if (std::ldexp(512.0 * (double)m, e) >= std::ldexp(1.0, 51)) qmagic = 0;
    }
    sc[(size_t)j] = std::ldexp(1.0, e);
    isc[(size_t)j] = std::ldexp(1.0, -e);
  }
  CK(cudaMemcpyAsync(h->scale.p, sc.data(), sizeof(double) * h->d, cudaMemcpyHostToDevice,
                     h->stream));
  CK(cudaMemcpyAsync(h->iscale.p, isc.data(), sizeof(double) * h->d, cudaMemcpyHostToDevice,
                     h->stream));
  CK(cudaMemcpyAsync(h->qflag.p, &qmagic, sizeof(int), cudaMemcpyHostToDevice, h->stream));
  CK(cudaStreamSynchronize(h->stream));
  return PROCLUS_OK;
}

extern "C" {

proclus_status proclus_create_ex(const float* data, int64_t n, int32_t d,
                                 const proclus_options* opt, proclus_handle** out) {
  if (!out) return fail(PROCLUS_EINVAL, "out is NULL");
  *out = nullptr;
  proclus_options o;
  if (opt)
    o = *opt;
  else
    proclus_options_init(&o);
  if (!data) return fail(PROCLUS_EINVAL, "data is NULL");
  if (n < 1) return fail(PROCLUS_EINVAL, "n must be >= 1 (got %lld)", (long long)n);
  if (d < 2 || d > PROCLUS_D_MAX)
    return fail(PROCLUS_EINVAL, "d must be in [2, %d] (got %d)", PROCLUS_D_MAX, d);
  if (o.metric != PROCLUS_METRIC_L2 && o.metric != PROCLUS_METRIC_L1)
    return fail(PROCLUS_EINVAL, "unknown metric %d", o.metric);
  if (o.variant < PROCLUS_VARIANT_FAST || o.variant > PROCLUS_VARIANT_FAST_STAR)
    return fail(PROCLUS_EINVAL, "unknown variant %d", o.variant);
  if (o.world_size < 1 || o.rank < 0 || o.rank >= o.world_size)
    return fail(PROCLUS_EINVAL, "bad world_size/rank");
  const int64_t n_total = o.n_global > 0 ? o.n_global : n;
  if (o.world_size == 1 && (n_total != n || o.row_offset != 0))
    return fail(PROCLUS_EINVAL, "n_global/row_offset need world_size > 1");
  if (o.row_offset < 0 || o.row_offset + n > n_total)
    return fail(PROCLUS_EINVAL, "shard [row_offset, row_offset+n) outside n_global");
  if (n_total >= (int64_t)1 << 40) return fail(PROCLUS_EINVAL, "n_global too large");
  int ndev = 0;
  CK(cudaGetDeviceCount(&ndev));
  int dev = o.device;
  if (dev < 0) CK(cudaGetDevice(&dev));
  if (dev >= ndev) return fail(PROCLUS_EINVAL, "device %d >= device count %d", dev, ndev);
  auto* h = new proclus_handle();
  h->dev = dev;
  h->n = n;
  h->d = d;
  h->n_pad = ((n + PAD_ALIGN - 1) / PAD_ALIGN) * PAD_ALIGN;
  h->n_total = n_total;
  h->row_offset = o.row_offset;
  h->metric = o.metric;
  h->max_iter = o.max_iter > 0 ? o.max_iter : 10000;
  h->data_on_device = o.data_on_device != 0;
  h->trace = o.trace != 0;
  h->stats = o.stats != 0;
  h->variant = o.variant;
  h->world = o.world_size;
  h->rank = o.rank;
  proclus_status st = PROCLUS_OK;
  auto cleanup = [&](proclus_status s) {
    proclus_destroy(h);
    return s;
  };
  if ((st = set_device(h)) != PROCLUS_OK) return cleanup(st);
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, dev) != cudaSuccess)
    return cleanup(fail(PROCLUS_ECUDA, "cudaGetDeviceProperties failed"));
  h->num_sms = prop.multiProcessorCount;
  if (o.stream) {
    h->stream = (cudaStream_t)o.stream;
  } else {
    if (cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking) != cudaSuccess)
      return cleanup(fail(PROCLUS_ECUDA, "cudaStreamCreate failed"));
    h->own_stream = true;
  }
  if (h->world > 1 && o.group) {
    proclus_group* g = reinterpret_cast<proclus_group*>(o.group);
    if (g->world != h->world)
      return cleanup(fail(PROCLUS_EINVAL, "group of %d ranks, world_size %d", g->world, h->world));
    h->group = g;
  } else if (h->world > 1) {
    if (!o.nccl_unique_id) return cleanup(fail(PROCLUS_EINVAL, "nccl_unique_id required"));
    ncclUniqueId id;
    memcpy(&id, o.nccl_unique_id, sizeof(id));
    ncclResult_t r = ncclCommInitRank(&h->comm, h->world, id, h->rank);
    if (r != ncclSuccess)
      return cleanup(fail(PROCLUS_ENCCL, "ncclCommInitRank: %s", ncclGetErrorString(r)));
  }
  if (h->xs.ensure((size_t)h->n_pad * d) != cudaSuccess || h->flag.ensure(1) != cudaSuccess ||
      h->qflag.ensure(1) != cudaSuccess ||
      h->colmax.ensure((size_t)PACK_COPIES * d) != cudaSuccess || h->scale.ensure((size_t)d) != cudaSuccess ||
      h->iscale.ensure((size_t)d) != cudaSuccess)
    return cleanup(
        fail(PROCLUS_ENOMEM, "device allocation of %lld x %d failed", (long long)n, d));
  if (cudaMallocHost(&h->h_st, sizeof(DevState)) != cudaSuccess)
    return cleanup(fail(PROCLUS_ENOMEM, "pinned allocation failed"));
  if ((st = upload_data(h, data, true)) != PROCLUS_OK) return cleanup(st);
  *out = h;
  return PROCLUS_OK;
}

proclus_status proclus_create(const float* data, int64_t n, int32_t d, proclus_handle** out) {
  return proclus_create_ex(data, n, d, nullptr, out);
}

proclus_status proclus_load(proclus_handle* h, const float* data) {
  if (!h || !data) return fail(PROCLUS_EINVAL, "NULL argument");
  TRY(set_device(h));
  return upload_data(h, data, false);
}

proclus_status proclus_prefetch(proclus_handle* h, const float* data) {
  if (!h || !data) return fail(PROCLUS_EINVAL, "NULL argument");
  if (h->data_on_device) return fail(PROCLUS_EINVAL, "prefetch needs host-resident data");
  TRY(set_device(h));
  if (!h->cstream) {
    CK(cudaStreamCreateWithFlags(&h->cstream, cudaStreamNonBlocking));
    CK(cudaEventCreateWithFlags(&h->pf_done, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&h->pack_done, cudaEventDisableTiming));
    CK(cudaEventRecord(h->pack_done, h->stream));
  }
  CK(h->staging.ensure((size_t)h->n * h->d));
  if (h->pf_src) CK(cudaStreamWaitEvent(h->cstream, h->pf_done, 0));
  CK(cudaStreamWaitEvent(h->cstream, h->pack_done, 0));  // the last pack has read staging
  CK(cudaMemcpyAsync(h->staging.p, data, sizeof(float) * (size_t)h->n * h->d,
                     cudaMemcpyHostToDevice, h->cstream));
  CK(cudaEventRecord(h->pf_done, h->cstream));
  h->pf_src = data;
  return PROCLUS_OK;
}

void proclus_destroy(proclus_handle* h) {
  if (!h) return;
  cudaSetDevice(h->dev);
  if (h->stream) cudaStreamSynchronize(h->stream);
  if (h->cstream) {
    cudaStreamSynchronize(h->cstream);
    cudaStreamDestroy(h->cstream);
    cudaEventDestroy(h->pf_done);
    cudaEventDestroy(h->pack_done);
  }
  for (auto& ge : h->graphs) cudaGraphExecDestroy(ge.exec);
  h->graphs.clear();
  h->gexec = nullptr;
  h->xs.release();
  h->staging.release();
  h->flag.release();
  h->qflag.release();
  h->colmax.release();
  h->scale.release();
  h->iscale.release();
  h->sids.release();
  h->mids.release();
  h->srows.release();
  h->mrows.release();
  h->spos.release();
  h->pickdist.release();
  h->gscratch.release();
  h->dist.release();
  h->Hq.release();
  h->dprev.release();
  h->nL.release();
  h->found.release();
  h->used.release();
  h->lab.release();
  h->med.release();
  h->X.release();
  h->Z.release();
  h->mu.release();
  h->Delta.release();
  h->dlist.release();
  h->pool.release();
  h->out_labels.release();
  h->dmask.release();
  h->accg.release();
  h->cntg.release();
  h->st.release();
  h->t_mcur.release();
  h->t_delta.release();
  h->t_cost.release();
  h->t_X.release();
  h->t_nL.release();
  h->t_sizes.release();
  h->t_dims.release();
  h->t_improved.release();
  h->t_bad.release();
  for (cudaEvent_t e : h->evpool) cudaEventDestroy(e);
  if (h->h_st) cudaFreeHost(h->h_st);
  if (h->h_pin) cudaFreeHost(h->h_pin);
  if (h->comm) ncclCommDestroy(h->comm);
  if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
  delete h;
}

int64_t proclus_last_launches(proclus_handle* h) { return h ? h->launches : -1; }

}  // extern "C"

// ------------------------------------------------------------------ driver
static proclus_status validate_setting(const proclus_handle* h, int k, int l, int A, int B,
                                       double minDev, int itrPat) {
  if (k < 2 || k > PROCLUS_K_MAX)
    return fail(PROCLUS_EINVAL, "k must be in [2, %d] (got %d)", PROCLUS_K_MAX, k);
  if (l < 2 || l > h->d) return fail(PROCLUS_EINVAL, "l must be in [2, d=%d] (got %d)", h->d, l);
  if (A < 1 || B < 1) return fail(PROCLUS_EINVAL, "A and B must be >= 1");
  if (!(minDev > 0.0) || !std::isfinite(minDev))
    return fail(PROCLUS_EINVAL, "minDev must be finite and > 0");
  if (itrPat < 1) return fail(PROCLUS_EINVAL, "itrPat must be >= 1");
  int64_t nS = std::min<int64_t>((int64_t)A * k, h->n_total);
  int64_t nM = std::min<int64_t>((int64_t)B * k, nS);
  if (nM < k) return fail(PROCLUS_EINVAL, "#M = %lld < k = %d", (long long)nM, k);
  return PROCLUS_OK;
}

static void reset_stats(proclus_handle* h) {
  h->launches = 0;
  h->evnext = 0;
  h->recs.clear();
  h->rec_done = 0;
  memset(&h->last_stats, 0, sizeof(h->last_stats));
}

// Initialization phase (Alg 1 l.2-3): Data' by partial Fisher-Yates over
// [0, n_total) (reading R13), Greedy on the GPU (Alg 2).  Keyed by
// (seed, k_sm, A, B) so that run_multi can reuse it.
static proclus_status init_phase(proclus_handle* h, int k_sm, int A, int B, uint64_t seed) {
  if (h->m_valid && h->m_seed == seed && h->m_ksm == k_sm && h->m_A == A && h->m_B == B)
    return PROCLUS_OK;
  const int64_t nS = std::min<int64_t>((int64_t)A * k_sm, h->n_total);
  const int64_t nM = std::min<int64_t>((int64_t)B * k_sm, nS);
  uint64_t st = stream_sm(seed, k_sm);
  std::vector<long long> S((size_t)nS);
  {
    std::unordered_map<int64_t, int64_t> v;
    v.reserve((size_t)(2 * nS + 1));
    auto get = [&](int64_t i) {
      auto it = v.find(i);
      return it == v.end() ? i : it->second;
    };
    for (int64_t t = 0; t < nS; ++t) {
      int64_t r = t + (int64_t)sm_uniform(&st, (uint64_t)(h->n_total - t));
      int64_t vt = get(t), vr = get(r);
      v[t] = vr;
      v[r] = vt;
      S[(size_t)t] = vr;
    }
  }
  const int q0 = (int)sm_uniform(&st, (uint64_t)nS);
  const int d = h->d;
  CK(h->sids.ensure((size_t)nS));
  CK(h->srows.ensure((size_t)nS * d));
  CK(h->spos.ensure((size_t)nM));
  CK(h->pickdist.ensure((size_t)nM));
  CK(h->gscratch.ensure(greedy_scratch_doubles((int)nS)));
  CK(h->mrows.ensure((size_t)nM * d));
  CK(h->mids.ensure((size_t)nM));
  launch_put(h->sids.p, S.data(), sizeof(long long) * nS, h->stream);
  CK(cudaGetLastError());
  launch(h, K_GATHER, -1, [&] {
    launch_gather_rows(h->xs.p, h->n_pad, d, h->sids.p, h->row_offset, h->n, (int)nS,
                       h->srows.p, h->stream);
  });
  CK(cudaGetLastError());
  TRY(allreduce(h, h->srows.p, (size_t)nS * d, ncclFloat));
  cudaError_t ge = cudaSuccess;
  launch(h, K_GREEDY, -1, [&] {
    ge = launch_greedy(h->srows.p, (int)nS, d, (int)nM, q0, h->metric, h->gscratch.p,
                       h->spos.p, h->pickdist.p, h->stream);
  });
  CK(ge);
  launch(h, K_GATHER, -1, [&] {
    launch_gather_m(h->srows.p, h->sids.p, h->spos.p, (int)nM, d, h->mrows.p, h->mids.p,
                    h->stream);
  });
  CK(cudaGetLastError());
  // no host round trip here: the ids of M are read back with the results
  // (a mid-run D2H would queue behind a prefetch's H2D on the copy engine)
  h->nS = nS;
  h->nM = nM;
  h->m_valid = true;
  h->m_seed = seed;
  h->m_ksm = k_sm;
  h->m_A = A;
  h->m_B = B;
  // new M: the Dist / H caches (keyed by M position) start empty.  FAST*
  // keeps k rows (allocated per setting), plain GPU-PROCLUS none.
  if (h->variant == PROCLUS_VARIANT_FAST) CK(h->dist.ensure((size_t)nM * h->n_pad));
  CK(h->Hq.ensure((size_t)nM * d));
  CK(h->dprev.ensure((size_t)nM));
  CK(h->nL.ensure((size_t)nM));
  CK(h->found.ensure((size_t)nM));
  CK(h->used.ensure((size_t)nM));
  CK(cudaMemsetAsync(h->Hq.p, 0, sizeof(long long) * nM * d, h->stream));
  CK(cudaMemsetAsync(h->nL.p, 0, sizeof(long long) * nM, h->stream));
  CK(cudaMemsetAsync(h->dprev.p, 0, sizeof(double) * nM, h->stream));  // read only if used
  CK(cudaMemsetAsync(h->found.p, 0, nM, h->stream));
  CK(cudaMemsetAsync(h->used.p, 0, nM, h->stream));
  return PROCLUS_OK;
}

// world_size > 1: allreduce the fixed-point cell sums (exact in int64) over
// NVLink (NCCL), then finalise on every rank.
static proclus_status split_tail(proclus_handle* h, const RunParams& p, int tail, int iter) {
  // every one of the NCOPY accumulator copies (blocks add into copy
  // blockIdx % NCOPY; the tail sums the copies), element-wise over ranks
  TRY(allreduce(h, p.accg, (size_t)NCOPY * p.k * p.d, ncclInt64));
  TRY(allreduce(h, p.cntg, (size_t)NCOPY * KMAX, ncclInt64));
  launch(h, K_SPLIT, iter, [&] { launch_tail(p, tail, h->stream); });
  return PROCLUS_OK;
}

// One run as a CUDA graph: prepare -> while(cond){locality, assign, cost} ->
// refine_x -> final.  The cost tail sets the condition.  Rebuilt only when
// the kernel parameters change (new buffers or setting).
static proclus_status build_graph(proclus_handle* h, RunParams p, const PassShape& ps) {
  for (auto& ge : h->graphs)
    if (memcmp(&ge.key, &p, sizeof(RunParams)) == 0 && memcmp(&ge.shape, &ps, sizeof(PassShape)) == 0) {
      ge.used = ++h->graph_tick;
      h->gexec = ge.exec;
      return PROCLUS_OK;
    }
  constexpr size_t kMaxGraphs = 256;  // the C5 grid has 128 settings
  if (h->graphs.size() >= kMaxGraphs) {  // evict the least recently used
    size_t lru = 0;
    for (size_t i = 1; i < h->graphs.size(); ++i)
      if (h->graphs[i].used < h->graphs[lru].used) lru = i;
    cudaGraphExecDestroy(h->graphs[lru].exec);
    h->graphs.erase(h->graphs.begin() + (long)lru);
  }
  h->gexec = nullptr;
  const RunParams key = p;
  cudaGraph_t g;
  CK(cudaGraphCreate(&g, 0));
  cudaGraphConditionalHandle cond;
  CK(cudaGraphConditionalHandleCreate(&cond, g, 1, cudaGraphCondAssignDefault));
  p.use_cond = 1;
  p.cond = (unsigned long long)cond;
  cudaStream_t cs;
  CK(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
  cudaGraph_t tmp;
  // prepare
  CK(cudaStreamBeginCaptureToGraph(cs, g, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed));
  launch_prepare(p, cs);
  CK(cudaStreamEndCapture(cs, &tmp));
  size_t nn = 0;
  CK(cudaGraphGetNodes(g, nullptr, &nn));
  std::vector<cudaGraphNode_t> nodes(nn);
  CK(cudaGraphGetNodes(g, nodes.data(), &nn));
  cudaGraphNode_t prep = nodes.back();
  // while node
  cudaGraphNodeParams cp = {};
  cp.type = cudaGraphNodeTypeConditional;
  cp.conditional.handle = cond;
  cp.conditional.type = cudaGraphCondTypeWhile;
  cp.conditional.size = 1;
  cudaGraphNode_t wnode;
  CK(cudaGraphAddNode(&wnode, g, &prep, 1, &cp));
  cudaGraph_t body = cp.conditional.phGraph_out[0];
  CK(cudaStreamBeginCaptureToGraph(cs, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed));
  launch_locality(p, ps, cs);
  if (!p.fuse_tail) launch_tail(p, TAIL_LOC, cs);
  launch_assign(p, ps, cs);
  if (!p.fuse_tail) launch_tail(p, TAIL_ASG, cs);
  launch_cost(p, ps, cs);
  if (!p.fuse_tail) launch_tail(p, TAIL_COST, cs);
  CK(cudaStreamEndCapture(cs, &tmp));
  // refinement after the loop
  CK(cudaStreamBeginCaptureToGraph(cs, g, &wnode, nullptr, 1, cudaStreamCaptureModeRelaxed));
  launch_refine_x(p, ps, cs);
  if (!p.fuse_tail) launch_tail(p, TAIL_REF, cs);
  launch_final(p, ps, cs);
  CK(cudaStreamEndCapture(cs, &tmp));
  CK(cudaStreamDestroy(cs));
  cudaGraphExec_t ge = nullptr;
  cudaError_t e = cudaGraphInstantiate(&ge, g, 0);
  cudaGraphDestroy(g);
  CK(e);
  h->graphs.push_back({key, ps, ge, ++h->graph_tick});
  h->gexec = ge;
  return PROCLUS_OK;
}

static proclus_status run_setting(proclus_handle* h, int k, int l, double minDev, int itrPat,
                                  uint64_t seed, proclus_result* out,
                                  const std::vector<int>* warm = nullptr) {
  const int d = h->d;
  const int nM = (int)h->nM;
  const PassShape ps = pass_shape(d, k, l, nM, h->num_sms);
  CK(configure_kernels(ps));
  CK(h->lab.ensure((size_t)2 * h->n_pad));
  if (h->variant == PROCLUS_VARIANT_FAST_STAR) CK(h->dist.ensure((size_t)k * h->n_pad));
  if (h->variant == PROCLUS_VARIANT_PLAIN) CK(h->dist.ensure(1));
  CK(h->med.ensure((size_t)KMAX * d));
  CK(h->X.ensure((size_t)KMAX * d));
  CK(h->Z.ensure((size_t)KMAX * d));
  CK(h->mu.ensure((size_t)KMAX * d));
  CK(h->dlist.ensure((size_t)KMAX * d));
  // the rows' tails beyond |D_i| are copied by the passes but never used
  CK(cudaMemsetAsync(h->dlist.p, 0, sizeof(int) * KMAX * d, h->stream));
  CK(h->dmask.ensure((size_t)KMAX * d));
  CK(h->accg.ensure((size_t)NCOPY * KMAX * d));
  CK(h->cntg.ensure((size_t)NCOPY * KMAX));
  CK(h->pool.ensure((size_t)std::max<int64_t>(h->nM, 1024)));
  CK(h->Delta.ensure(KMAX));
  CK(h->st.ensure(1));
  CK(h->out_labels.ensure((size_t)h->n));
  if (h->trace) {
    const int cap = std::min(h->max_iter, 4096);
    h->tr_cap = cap;
    CK(h->t_mcur.ensure((size_t)cap * KMAX));
    CK(h->t_delta.ensure((size_t)cap * KMAX));
    CK(h->t_nL.ensure((size_t)cap * KMAX));
    CK(h->t_sizes.ensure((size_t)cap * KMAX));
    CK(h->t_bad.ensure((size_t)cap * KMAX));
    CK(h->t_dims.ensure((size_t)cap * KMAX * d));
    CK(h->t_X.ensure((size_t)cap * KMAX * d));
    CK(h->t_cost.ensure((size_t)cap));
    CK(h->t_improved.ensure((size_t)cap));
  }
  // initial MCur: k distinct positions of M (partial Fisher-Yates, stream IT)
  uint64_t it = stream_it(seed, k, l);
  std::vector<int> pool((size_t)nM);
  DevState& s = *h->h_st;
  memset(&s, 0, sizeof(s));
  if (warm && !warm->empty()) {
    // multi-param level 3 (reading R21): a random subset of the
    // previous setting's MBest (slot order), topped up from M \ MBest_prev
    const int nw = (int)warm->size(), m = std::min(k, nw);
    std::vector<int> wp(*warm);
    for (int i = 0; i < m; ++i) {
      int r = i + (int)sm_uniform(&it, (uint64_t)(nw - i));
      std::swap(wp[(size_t)i], wp[(size_t)r]);
      s.mcur[i] = wp[(size_t)i];
    }
    if (k > nw) {
      std::vector<char> in((size_t)nM, 1);
      for (int v : *warm) in[(size_t)v] = 0;
      int np2 = 0;
      for (int t = 0; t < nM; ++t)
        if (in[(size_t)t]) pool[(size_t)np2++] = t;
      for (int i = nw; i < k; ++i) {
        const int u = i - nw;
        int r = u + (int)sm_uniform(&it, (uint64_t)(np2 - u));
        std::swap(pool[(size_t)u], pool[(size_t)r]);
        s.mcur[i] = pool[(size_t)u];
      }
    }
    for (int i = 0; i < k; ++i) s.mbest[i] = s.mcur[i];
  } else {
    for (int t = 0; t < nM; ++t) pool[(size_t)t] = t;
    for (int i = 0; i < k; ++i) {
      int r = i + (int)sm_uniform(&it, (uint64_t)(nM - i));
      std::swap(pool[(size_t)i], pool[(size_t)r]);
      s.mcur[i] = pool[(size_t)i];
      s.mbest[i] = pool[(size_t)i];
    }
  }
  s.rng = it;
  for (int i = 0; i < KMAX; ++i) s.cown[i] = -1;
  s.cost_best = INFINITY;
  s.dbg_t[0] = ~0ull;  // min-reduced entry time of the profiled locality launch
  s.cur_buf = 0;
  s.best_buf = 1;
  launch_put(h->st.p, &s, sizeof(DevState), h->stream);
  CK(cudaGetLastError());
  CK(cudaMemsetAsync(h->accg.p, 0, sizeof(long long) * NCOPY * KMAX * d, h->stream));
  CK(cudaMemsetAsync(h->cntg.p, 0, sizeof(long long) * NCOPY * KMAX, h->stream));

  RunParams p;
  memset(&p, 0, sizeof(p));
  p.n = h->n;
  p.n_pad = h->n_pad;
  p.n_total = h->n_total;
  p.d = d;
  p.k = k;
  p.l = l;
  p.nM = nM;
  p.itrPat = itrPat;
  p.max_iter = h->max_iter;
  p.metric = h->metric;
  p.minDev = minDev;
  p.xs = h->xs.p;
  p.mrows = h->mrows.p;
  p.dist = h->dist.p;
  p.lab0 = h->lab.p;
  p.lab1 = h->lab.p + h->n_pad;
  p.Hq = h->Hq.p;
  p.dprev = h->dprev.p;
  p.nL = h->nL.p;
  p.found = h->found.p;
  p.used = h->used.p;
  p.med = h->med.p;
  p.dlist = h->dlist.p;
  p.dmask = h->dmask.p;
  p.X = h->X.p;
  p.Z = h->Z.p;
  p.mu = h->mu.p;
  p.accg = h->accg.p;
  p.cntg = h->cntg.p;
  p.scale = h->scale.p;
  p.iscale = h->iscale.p;
  p.pool = h->pool.p;
  p.st = h->st.p;
  p.P = ps.P;
  p.stages = ps.stages;
  for (int q = 0; q < NLAY; ++q) p.lay[q] = ps.lay[q];
  p.tl = ps.tl;
  p.tail_smem = ps.tail_smem;
  p.nchunks = (h->n + ps.P - 1) / ps.P;
  // PROCLUS_SPLIT_TAIL=1: the multi-GPU schedule (pass, allreduce, separate
  // tail kernel) on one GPU, so that single-GPU tests cover that path
  const char* split_env = getenv("PROCLUS_SPLIT_TAIL");
  const bool force_split = split_env && split_env[0] == '1';
  // PROCLUS_TAIL_KERNELS=1: single GPU with the single-block tails as kernels
  // of their own (the north_star's separate Z-score / selection kernel)
  // instead of the last block of each pass; graph mode still applies
  const char* tk_env = getenv("PROCLUS_TAIL_KERNELS");
  const bool tail_kernels =
      h->world == 1 && (ps.split_tails || (tk_env && tk_env[0] == '1')) &&
      !(tk_env && tk_env[0] == '0');
  p.fuse_tail = (h->world == 1 && !force_split && !tail_kernels) ? 1 : 0;
  p.cost1 = ps.cost1;
  p.qflag = h->qflag.p;
  p.badflag = h->flag.p;
  p.variant = h->variant;
  p.out_labels = h->out_labels.p;
  p.Delta = h->Delta.p;
  if (h->trace) {
    p.tr.cap = h->tr_cap;
    p.tr.mcur = h->t_mcur.p;
    p.tr.delta = h->t_delta.p;
    p.tr.nL = h->t_nL.p;
    p.tr.dims = h->t_dims.p;
    p.tr.sizes = h->t_sizes.p;
    p.tr.cost = h->t_cost.p;
    p.tr.improved = h->t_improved.p;
    p.tr.bad = h->t_bad.p;
    p.tr.X = h->t_X.p;
  }
  if (out && out->labels_on_device && out->labels) p.out_labels = out->labels;

  // graph mode unless per-launch events are wanted, multi-GPU (NCCL between
  // kernels), or PROCLUS_GRAPH=0 (ncu cannot profile kernels of graphs that
  // contain conditional nodes)
  const char* genv = getenv("PROCLUS_GRAPH");
  const bool graph_env = !(genv && genv[0] == '0');
  const bool use_graph = (p.fuse_tail || tail_kernels) && !h->stats && graph_env;
  if (use_graph) {
    // one graph launch: the whole iterative + refinement phase on the device
    TRY(build_graph(h, p, ps));
    CK(cudaGraphLaunch(h->gexec, h->stream));
    h->launches += 0;  // counted below from the iteration count
  } else {
    launch(h, K_PREPARE, -1, [&] { launch_prepare(p, h->stream); });
    CK(cudaGetLastError());
    // Kernels exit immediately once the device sets `done`, so iterations
    // are enqueued speculatively in batches and the flag is read once per
    // batch (the minimum run length is itrPat + 1).
    int launched = 0;
    int batch = itrPat + 1;
    for (;;) {
      for (int b = 0; b < batch; ++b) {
        const int iter = launched + b;
        launch(h, K_LOC, iter, [&] { launch_locality(p, ps, h->stream); });
        if (!p.fuse_tail) TRY(split_tail(h, p, TAIL_LOC, iter));
        launch(h, K_ASG, iter, [&] { launch_assign(p, ps, h->stream); });
        if (!p.fuse_tail) TRY(split_tail(h, p, TAIL_ASG, iter));
        launch(h, K_COST, iter, [&] { launch_cost(p, ps, h->stream); });
        if (!p.fuse_tail) TRY(split_tail(h, p, TAIL_COST, iter));
      }
      CK(cudaGetLastError());
      launched += batch;
      CK(cudaMemcpyAsync(h->h_st, h->st.p, sizeof(DevState), cudaMemcpyDeviceToHost,
                         h->stream));
      CK(cudaStreamSynchronize(h->stream));
      if (h->h_st->done) break;
      if (launched >= h->max_iter) break;
      batch = 2;
    }
    // Refinement phase (Alg 1 l.16-19)
    launch(h, K_REF, -1, [&] { launch_refine_x(p, ps, h->stream); });
    if (!p.fuse_tail) TRY(split_tail(h, p, TAIL_REF, -1));
    launch(h, K_FIN, -1, [&] { launch_final(p, ps, h->stream); });
    CK(cudaGetLastError());
  }
  CK(cudaMemcpyAsync(h->h_st, h->st.p, sizeof(DevState), cudaMemcpyDeviceToHost, h->stream));
  if (out) {
    if (out->labels && !out->labels_on_device)
      CK(cudaMemcpyAsync(out->labels, p.out_labels, sizeof(int32_t) * h->n,
                         cudaMemcpyDeviceToHost, h->stream));
    // pinned staging: [ids of M (int64, #M)][D mask (k x d bytes)]
    TRY(pin_ensure(h, sizeof(long long) * h->nM + (size_t)k * d));
    CK(cudaMemcpyAsync(h->h_pin, h->mids.p, sizeof(long long) * h->nM, cudaMemcpyDeviceToHost,
                       h->stream));
    if (out->dims)
      CK(cudaMemcpyAsync(h->h_pin + sizeof(long long) * h->nM, h->dmask.p, (size_t)k * d,
                         cudaMemcpyDeviceToHost, h->stream));
  }
  CK(cudaStreamSynchronize(h->stream));
  if (out && out->dims) memcpy(out->dims, h->h_pin + sizeof(long long) * h->nM, (size_t)k * d);
  if (h->h_st->err == ERR_NONFINITE)
    return fail(PROCLUS_EINVAL, "data contains non-finite values (found by the last load)");
  if (h->h_st->err) return fail(PROCLUS_EINTERNAL, "device reported error %d", h->h_st->err);
  const int T = h->h_st->iterations;
  if (use_graph) h->launches += p.fuse_tail ? 1 + 3 * (int64_t)T + 2 : 1 + 6 * (int64_t)T + 3;
  if (out) {
    for (int i = 0; i < k; ++i)
      if (out->medoids)
        out->medoids[i] = reinterpret_cast<const long long*>(h->h_pin)[h->h_st->mbest[i]];
    out->cost = h->h_st->cost_best;
    out->iterations = T;
  }
  h->last_k = k;
  h->tr_count = h->trace ? std::min(T, h->tr_cap) : 0;
  if (h->stats) {
    proclus_stats& S = h->last_stats;
    const double bytes_pass = 4.0 * (double)h->n * d + (double)h->n;  // data + u8 labels
    float last = 0.f;
    for (size_t r = h->rec_done; r < h->recs.size(); ++r) {
      const auto& R = h->recs[r];
      if (R.iter >= T) continue;  // speculative launch after the stop: no work
      float ms = 0.f;
      CK(cudaEventElapsedTime(&ms, R.a, R.b));
      S.launches[R.kind] += 1;
      S.ms[R.kind] += ms;
      float from0 = 0.f;
      CK(cudaEventElapsedTime(&from0, h->recs[0].a, R.b));
      if (from0 > last) last = from0;
    }
    h->rec_done = h->recs.size();
    if (last > S.run_ms) S.run_ms = last;
    S.alg_bytes[K_LOC] += h->h_st->bytes_loc;
    S.alg_bytes[K_ASG] += T * bytes_pass;
    S.alg_bytes[K_COST] += T * bytes_pass;
    S.alg_bytes[K_REF] += bytes_pass;
    S.alg_bytes[K_FIN] += 4.0 * (double)h->n * d + 4.0 * (double)h->n;
    S.total_launches = h->launches;
    for (int t = 0; t < 4; ++t) {
      S.tail_ms[t] += (double)h->h_st->tail_ns[t] * 1e-6;
      S.fallbacks[t] += h->h_st->fallback[t];
    }
    if (getenv("PROCLUS_TAIL_PROFILE")) {
      fprintf(stderr, "tail_cycles");
      for (int t = 0; t < 24; ++t) fprintf(stderr, " %llu", h->h_st->dbg_cyc[t]);
      fprintf(stderr, "\n");
      fprintf(stderr, "loc_phase_ns launches %llu prologue %llu chunks %llu flush %llu tail_start %llu\n",
              h->h_st->dbg_ts[0], h->h_st->dbg_ts[1], h->h_st->dbg_ts[2], h->h_st->dbg_ts[3],
              h->h_st->dbg_ts[4]);
    }
  }
  return PROCLUS_OK;
}

extern "C" {

proclus_status proclus_run(proclus_handle* h, int32_t k, int32_t l, int32_t A, int32_t B,
                           double minDev, int32_t itrPat, uint64_t seed, proclus_result* out) {
  if (!h) return fail(PROCLUS_EINVAL, "handle is NULL");
  if (!out || !out->medoids || !out->dims || !out->labels)
    return fail(PROCLUS_EINVAL, "out and its labels/medoids/dims arrays are required");
  TRY(validate_setting(h, k, l, A, B, minDev, itrPat));
  TRY(set_device(h));
  reset_stats(h);
  TRY(init_phase(h, k, A, B, seed));
  return run_setting(h, k, l, minDev, itrPat, seed, out);
}

proclus_status proclus_run_multi(proclus_handle* h, const int32_t* ks, int32_t nk,
                                 const int32_t* ls, int32_t nl, int32_t A, int32_t B,
                                 double minDev, int32_t itrPat, uint64_t seed,
                                 int32_t reuse_level, proclus_result* outs) {
  if (!h || !ks || !ls || !outs) return fail(PROCLUS_EINVAL, "NULL argument");
  if (nk < 1 || nl < 1) return fail(PROCLUS_EINVAL, "empty parameter grid");
  if (reuse_level < 1 || reuse_level > 3)
    return fail(PROCLUS_EINVAL, "reuse_level must be 1, 2 or 3");
  int kmax = 0;
  for (int a = 0; a < nk; ++a) {
    kmax = std::max(kmax, ks[a]);
    for (int b = 0; b < nl; ++b) {
      TRY(validate_setting(h, ks[a], ls[b], A, B, minDev, itrPat));
      proclus_result* o = &outs[a * nl + b];
      if (!o->labels || !o->medoids || !o->dims)
        return fail(PROCLUS_EINVAL, "outs[%d] arrays are required", a * nl + b);
    }
  }
  TRY(set_device(h));
  reset_stats(h);
  if (reuse_level >= 2) TRY(init_phase(h, kmax, A, B, seed));
  std::vector<int> warm;  // level 3: MBest (positions in M) of the previous setting
  for (int a = 0; a < nk; ++a)
    for (int b = 0; b < nl; ++b) {
      if (reuse_level == 1) TRY(init_phase(h, ks[a], A, B, seed));
      TRY(run_setting(h, ks[a], ls[b], minDev, itrPat, seed, &outs[a * nl + b],
                      reuse_level == 3 ? &warm : nullptr));
      if (reuse_level == 3) warm.assign(h->h_st->mbest, h->h_st->mbest + ks[a]);
    }
  return PROCLUS_OK;
}

proclus_status proclus_run_list(proclus_handle* h, const int32_t* ks, const int32_t* ls,
                                int32_t nset, int32_t k_sample, int32_t A, int32_t B,
                                double minDev, int32_t itrPat, uint64_t seed,
                                int32_t reuse_level, proclus_result* outs) {
  if (!h || !ks || !ls || !outs) return fail(PROCLUS_EINVAL, "NULL argument");
  if (nset < 1) return fail(PROCLUS_EINVAL, "empty settings list");
  if (reuse_level != 1 && reuse_level != 2)
    return fail(PROCLUS_EINVAL, "reuse_level must be 1 or 2 (level 3 is sequential)");
  for (int s = 0; s < nset; ++s) {
    TRY(validate_setting(h, ks[s], ls[s], A, B, minDev, itrPat));
    if (reuse_level == 2 && ks[s] > k_sample)
      return fail(PROCLUS_EINVAL, "k_sample %d < k = %d of setting %d", k_sample, ks[s], s);
    if (!outs[s].labels || !outs[s].medoids || !outs[s].dims)
      return fail(PROCLUS_EINVAL, "outs[%d] arrays are required", s);
  }
  if (reuse_level == 2 && (k_sample < 2 || k_sample > PROCLUS_K_MAX))
    return fail(PROCLUS_EINVAL, "k_sample must be in [2, %d]", PROCLUS_K_MAX);
  TRY(set_device(h));
  reset_stats(h);
  if (reuse_level == 2) TRY(init_phase(h, k_sample, A, B, seed));
  for (int s = 0; s < nset; ++s) {
    if (reuse_level == 1) TRY(init_phase(h, ks[s], A, B, seed));
    TRY(run_setting(h, ks[s], ls[s], minDev, itrPat, seed, &outs[s]));
  }
  return PROCLUS_OK;
}

proclus_status proclus_get_stats(proclus_handle* h, proclus_stats* st) {
  if (!h || !st) return fail(PROCLUS_EINVAL, "NULL argument");
  if (!h->stats) return fail(PROCLUS_EINVAL, "handle created without options.stats");
  *st = h->last_stats;
  return PROCLUS_OK;
}

proclus_status proclus_get_trace(proclus_handle* h, proclus_trace* tr) {
  if (!h || !tr) return fail(PROCLUS_EINVAL, "NULL argument");
  if (!h->trace) return fail(PROCLUS_EINVAL, "handle created without options.trace");
  TRY(set_device(h));
  const int c = std::min(tr->cap, h->tr_count);
  const int k = h->last_k, d = h->d;
  tr->count = c;
  auto cp = [&](void* dst, const void* src, size_t bytes) -> proclus_status {
    if (dst && bytes) CK(cudaMemcpy(dst, src, bytes, cudaMemcpyDeviceToHost));
    return PROCLUS_OK;
  };
  TRY(cp(tr->mcur, h->t_mcur.p, sizeof(int) * c * k));
  TRY(cp(tr->delta, h->t_delta.p, sizeof(double) * c * k));
  TRY(cp(tr->nL, h->t_nL.p, sizeof(long long) * c * k));
  TRY(cp(tr->dims, h->t_dims.p, (size_t)c * k * d));
  TRY(cp(tr->sizes, h->t_sizes.p, sizeof(long long) * c * k));
  TRY(cp(tr->cost, h->t_cost.p, sizeof(double) * c));
  TRY(cp(tr->improved, h->t_improved.p, (size_t)c));
  TRY(cp(tr->bad, h->t_bad.p, (size_t)c * k));
  TRY(cp(tr->X, h->t_X.p, sizeof(double) * c * k * d));
  return PROCLUS_OK;
}

}  // extern "C"
