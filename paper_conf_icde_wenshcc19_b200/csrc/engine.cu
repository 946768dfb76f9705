// engine.cu -- host orchestration of the hot path (Algorithm 2, and the
// prediction procedure L259-L273 / L331-L363) on one GPU.  Every arithmetic step runs in the
// kernels of stage.cu / krow.cu / solver.cu / predict.cu; this file allocates, launches,
// polls the per-pair stop flags once per outer iteration, and assembles the model.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <functional>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "model.h"

namespace gmpsvm {

std::atomic<uint64_t> g_launches{0};

[[noreturn]] void throw_cuda(cudaError_t e, const char* what, const char* file, int line) {
  std::string msg = std::string("CUDA error ") + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ") at " + file +
                    ":" + std::to_string(line) + ": " + what;
  if (e == cudaErrorMemoryAllocation) throw Error(GMPSVM_ENOMEM, msg);
  throw Error(GMPSVM_ECUDA, msg);
}

void set_max_dyn_smem(const void* func, size_t bytes) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, size_t> done;
  int dev = 0;
  GM_CUDA(cudaGetDevice(&dev));
  std::lock_guard<std::mutex> lk(mu);
  size_t& cur = done[{func, dev}];
  if (bytes <= cur) return;
  GM_CUDA(cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes));
  cur = bytes;
}

namespace {

constexpr int kMaxK = 64;          // label-rank shared memory bound
constexpr int kMaxCoupleK = 40;    // coupling shared memory bound
constexpr int kItemTiles = 4;      // SV tiles per dec_contract work item
constexpr int64_t kPredictChunk = 32768;
constexpr int kMaxGroups = 4;      // solver graphs per call (lead mode: the lead pairs + up to 3 groups)
constexpr int kMaxStreams = kMaxGroups + 1;  // solver streams: one graph launch per group + graph capture
constexpr int kDefaultB = 192;     // working-set rows (tuned on MNIST-shaped data; the tile of K_ws,ws stays in shared memory for B <= 224)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    GM_CUDA(cudaGetDevice(&prev));
    if (dev != prev) GM_CUDA(cudaSetDevice(dev));
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

std::mutex g_stream_mu;
cudaStream_t g_streams[64] = {};
bool g_pool_cfg[64] = {};

cudaStream_t get_stream(const gmpsvm_options& opt) {
  int dev = opt.device;
  std::lock_guard<std::mutex> lk(g_stream_mu);
  if (dev >= 0 && dev < 64 && !g_pool_cfg[dev]) {
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
      uint64_t thr = UINT64_MAX;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    g_pool_cfg[dev] = true;
  }
  if (opt.stream) return (cudaStream_t)opt.stream;
  if (dev < 0 || dev >= 64) throw Error(GMPSVM_EINVAL, "device ordinal out of range");
  if (!g_streams[dev]) GM_CUDA(cudaStreamCreateWithFlags(&g_streams[dev], cudaStreamNonBlocking));
  return g_streams[dev];
}

size_t device_total_mem(int dev) {
  static std::mutex mu;
  static size_t total[64] = {};
  std::lock_guard<std::mutex> lk(mu);
  if (!total[dev]) {
    cudaDeviceProp p;
    GM_CUDA(cudaGetDeviceProperties(&p, dev));
    total[dev] = p.totalGlobalMem;
  }
  return total[dev];
}

// Per-device pool of non-blocking streams for the concurrent pair groups.
std::mutex g_pool_mu;
std::vector<cudaStream_t> g_pools[64];
// The solver's streams have the highest priority: when the kernel-value waves share the GPU with
// the lead pairs' solver (lead mode), the block scheduler dispatches solver CTAs first.
const std::vector<cudaStream_t>& stream_pool(int dev) {
  std::lock_guard<std::mutex> lk(g_pool_mu);
  auto& v = g_pools[dev];
  int least = 0, greatest = 0;
  if (v.size() < (size_t)kMaxStreams) GM_CUDA(cudaDeviceGetStreamPriorityRange(&least, &greatest));
  // pool[g]: the graph of pair group g (lead mode; else pool[0] alone), pool.back(): capture
  while ((int)v.size() < kMaxStreams) {
    cudaStream_t s;
    GM_CUDA(cudaStreamCreateWithPriority(&s, cudaStreamNonBlocking, greatest));
    v.push_back(s);
  }
  return v;
}

// Low-priority stream for the kernel-value waves of lead mode.
cudaStream_t krow_stream(int dev) {
  static std::mutex mu;
  static cudaStream_t s[64] = {};
  std::lock_guard<std::mutex> lk(mu);
  if (!s[dev]) {
    int least = 0, greatest = 0;
    GM_CUDA(cudaDeviceGetStreamPriorityRange(&least, &greatest));
    GM_CUDA(cudaStreamCreateWithPriority(&s[dev], cudaStreamNonBlocking, least));
  }
  return s[dev];
}

// Events created on demand and destroyed with the pool (timing-free unless asked).
struct EventPool {
  std::vector<cudaEvent_t> evs;
  cudaEvent_t get(bool timing = false) {
    cudaEvent_t e;
    GM_CUDA(cudaEventCreateWithFlags(&e, timing ? cudaEventDefault : cudaEventDisableTiming));
    evs.push_back(e);
    return e;
  }
  ~EventPool() {
    for (auto e : evs) cudaEventDestroy(e);
  }
};

// Kernel-matrix workspace cache (FULL_K regime): the n^2 x 4 B buffer is the largest
// allocation of a training run; growing a stream-ordered pool by 14.4 GB costs 0.1-0.5 s, so
// the buffer is kept per device and reused by later runs.  A buffer is handed out to one run
// at a time; the next user's stream waits on an event recorded when the previous run ended.
struct KCacheEntry {
  float* p = nullptr;
  size_t bytes = 0;
  cudaEvent_t done = nullptr;
  bool busy = false;
};
std::mutex g_kcache_mu;
std::vector<KCacheEntry> g_kcache[64];

// bytes of the cached kernel-matrix workspaces of a device (reusable by the next run)
size_t kcache_bytes(int dev) {
  std::lock_guard<std::mutex> lk(g_kcache_mu);
  size_t b = 0;
  for (const auto& e : g_kcache[dev])
    if (!e.busy) b += e.bytes;
  return b;
}

struct KWorkspace {
  int dev;
  size_t slot = (size_t)-1;
  cudaStream_t st;
  float* p = nullptr;
  KWorkspace(int device, size_t bytes, cudaStream_t s) : dev(device), st(s) {
    std::lock_guard<std::mutex> lk(g_kcache_mu);
    auto& v = g_kcache[dev];
    for (size_t i = 0; i < v.size(); ++i)
      if (!v[i].busy && v[i].bytes >= bytes) {
        slot = i;
        break;
      }
    if (slot == (size_t)-1) {
      for (size_t i = 0; i < v.size(); ++i)  // drop idle buffers that are too small
        if (!v[i].busy && v[i].p) {
          GM_CUDA(cudaEventSynchronize(v[i].done));
          cudaFree(v[i].p);
          v[i].p = nullptr;
          v[i].bytes = 0;
        }
      KCacheEntry e;
      GM_CUDA(cudaMalloc((void**)&e.p, bytes));
      e.bytes = bytes;
      GM_CUDA(cudaEventCreateWithFlags(&e.done, cudaEventDisableTiming));
      GM_CUDA(cudaEventRecord(e.done, st));
      size_t i = 0;
      for (; i < v.size(); ++i)
        if (!v[i].busy && !v[i].p) break;
      if (i == v.size()) v.push_back(e);
      else v[i] = e;
      slot = i;
    }
    v[slot].busy = true;
    GM_CUDA(cudaStreamWaitEvent(st, v[slot].done, 0));
    p = v[slot].p;
  }
  ~KWorkspace() {
    std::lock_guard<std::mutex> lk(g_kcache_mu);
    auto& e = g_kcache[dev][slot];
    cudaEventRecord(e.done, st);
    e.busy = false;
  }
  float* get() const { return p; }
};

// Destroying the solver's executable graph (hundreds of nodes) takes ~3 ms of host time and holds
// the driver while it runs, so a finished graph is not destroyed when its training call returns:
// it is parked here and destroyed by the next training call right after that call has launched
// its own solver graph (the GPU then has tens of ms of queued work to hide it behind).
std::mutex g_parked_mu;
std::vector<std::pair<cudaGraphExec_t, cudaGraph_t>> g_parked;

void destroy_parked_graphs() {
  std::vector<std::pair<cudaGraphExec_t, cudaGraph_t>> v;
  {
    std::lock_guard<std::mutex> lk(g_parked_mu);
    v.swap(g_parked);
  }
  for (auto& e : v) {
    if (e.first) cudaGraphExecDestroy(e.first);
    if (e.second) cudaGraphDestroy(e.second);
  }
}

struct GraphGuard {
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t exec = nullptr;
  ~GraphGuard() {
    if (exec || graph) {
      std::lock_guard<std::mutex> lk(g_parked_mu);
      g_parked.emplace_back(exec, graph);
    }
  }
};

// Solver-state arena: pointers carved from one allocation at fixed offsets (same sizes -> same
// pointers, so a cached graph's kernel arguments stay valid).
template <class T>
struct ArenaPtr {
  T* p = nullptr;
  T* get() const { return p; }
};
struct ArenaLayout {
  size_t bytes = 0;
  std::vector<std::function<void(char*)>> set;
  template <class T>
  void add(ArenaPtr<T>& a, size_t count) {
    bytes = (bytes + 255) & ~(size_t)255;
    const size_t off = bytes;
    set.push_back([&a, off](char* base) { a.p = reinterpret_cast<T*>(base + off); });
    bytes += std::max<size_t>(count, 1) * sizeof(T);
  }
  void place(void* base) {
    for (auto& f : set) f(static_cast<char*>(base));
  }
};

// Per-device solver workspace kept across training calls: the arena and the instantiated solver
// graphs (lead graph + the rest) with the signature of what they were captured with.
struct SolverWs {
  void* base = nullptr;
  size_t cap = 0;
  bool busy = false;
  cudaEvent_t done = nullptr;  // end of the last call's use of the arena
  std::vector<uint8_t> sig;
  std::vector<cudaGraph_t> graph;  // one per pair group
  std::vector<cudaGraphExec_t> exec;
  std::vector<int64_t> body_per_pair;
  int final_selects = 0;
  // kernel-value tile list of the last call (FULL_K on tcgen05): key, device copy, wave split
  std::vector<int64_t> tkey;
  int2* tiles = nullptr;
  size_t n_tiles = 0;
  std::vector<size_t> wave_off;
  double kv_subset = -1;
  void park_graphs() {  // destroyed later by destroy_parked_graphs (it blocks until the device idles)
    std::lock_guard<std::mutex> lk(g_parked_mu);
    for (size_t i = 0; i < exec.size(); ++i)
      if (exec[i] || graph[i]) g_parked.emplace_back(exec[i], graph[i]);
    exec.clear();
    graph.clear();
    sig.clear();
  }
};
std::mutex g_sws_mu;
SolverWs g_sws[64];

// A training call's hold on its device's SolverWs (ws == nullptr: not cacheable, or in use by a
// concurrent call -- the caller then allocates its own arena and tiles and builds its own graphs).
struct SolverCacheLease {
  SolverWs* ws = nullptr;
  cudaStream_t st = nullptr;
  SolverCacheLease(int dev, cudaStream_t s) : st(s) {
    if (dev < 0 || dev >= 64) return;
    std::lock_guard<std::mutex> lk(g_sws_mu);
    SolverWs& w = g_sws[dev];
    if (w.busy) return;
    if (w.done) GM_CUDA(cudaStreamWaitEvent(st, w.done, 0));  // the previous call is done with it
    w.busy = true;
    ws = &w;
  }
  // the cached arena, (re)allocated for `bytes` (same size as before: same base)
  void* arena(size_t bytes) {
    SolverWs& w = *ws;
    if (w.cap < bytes || w.cap > 2 * bytes + ((size_t)64 << 20)) {
      w.park_graphs();  // their kernel arguments point into the old arena
      if (w.base) cudaFreeAsync(w.base, st);
      w.base = nullptr;
      w.cap = 0;
      GM_CUDA(cudaMallocAsync(&w.base, bytes, st));
      w.cap = bytes;
    }
    return w.base;
  }
  ~SolverCacheLease() {
    if (!ws) return;
    std::lock_guard<std::mutex> lk(g_sws_mu);
    if (!ws->done) cudaEventCreateWithFlags(&ws->done, cudaEventDisableTiming);
    if (ws->done) cudaEventRecord(ws->done, st);
    ws->busy = false;
  }
  SolverCacheLease(const SolverCacheLease&) = delete;
  SolverCacheLease& operator=(const SolverCacheLease&) = delete;
};

template <class T>
struct PinnedBuf {
  T* p = nullptr;
  explicit PinnedBuf(size_t count) {
    if (count) GM_CUDA(cudaMallocHost((void**)&p, count * sizeof(T)));
  }
  ~PinnedBuf() {
    if (p) cudaFreeHost(p);
  }
};

// Device buffers of a model (DevModel).  A model is freed on the library stream while the next
// one is typically allocated on the caller's stream; the stream-ordered pool then cannot hand the
// freed blocks straight to the new allocation, and a cudaMallocAsync of the ~90 MB int8 SV planes
// was measured blocking the host for 2-28 ms per training call (GMPSVM_SLOW_API).  So a freed
// model's buffers go to a small per-device cache instead, each with an event marking the end of
// its last use; an allocation of a size within 25 % of a cached block takes it and makes its
// stream wait on that event (no host block).  Bounded: beyond kModelCacheBytes the oldest cached
// blocks are released to the pool.
constexpr size_t kModelCacheBytes = (size_t)2 << 30;
struct CachedBlock {
  void* p;
  size_t bytes;
  cudaEvent_t ev;
};
std::mutex g_mcache_mu;
std::deque<CachedBlock> g_mcache[64];
std::map<void*, size_t> g_msize[64];  // live and cached model blocks: bytes

void* model_alloc(size_t bytes, cudaStream_t st, int dev) {
  if (!bytes) return nullptr;
  {
    std::lock_guard<std::mutex> lk(g_mcache_mu);
    auto& c = g_mcache[dev];
    int best = -1;
    for (int i = 0; i < (int)c.size(); ++i)
      if (c[i].bytes >= bytes && c[i].bytes - bytes <= bytes / 4 && (best < 0 || c[i].bytes < c[best].bytes)) best = i;
    if (best >= 0) {
      const CachedBlock b = c[best];
      c.erase(c.begin() + best);
      GM_CUDA(cudaStreamWaitEvent(st, b.ev, 0));
      cudaEventDestroy(b.ev);
      return b.p;
    }
  }
  void* p = nullptr;
  GM_CUDA(cudaMallocAsync(&p, bytes, st));
  std::lock_guard<std::mutex> lk(g_mcache_mu);
  g_msize[dev][p] = bytes;
  return p;
}

// ls: a stream ordered after the block's last use
void model_free(void* p, cudaStream_t ls, int dev) {
  if (!p) return;
  std::lock_guard<std::mutex> lk(g_mcache_mu);
  auto it = g_msize[dev].find(p);
  if (!ls || it == g_msize[dev].end()) {  // no stream (device gone?) or not ours: plain free
    if (it != g_msize[dev].end()) g_msize[dev].erase(it);
    cudaFree(p);
    return;
  }
  cudaEvent_t ev = nullptr;
  if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess || cudaEventRecord(ev, ls) != cudaSuccess) {
    if (ev) cudaEventDestroy(ev);
    g_msize[dev].erase(it);
    cudaFreeAsync(p, ls);
    return;
  }
  auto& c = g_mcache[dev];
  c.push_back(CachedBlock{p, it->second, ev});
  size_t tot = 0;
  for (const auto& b : c) tot += b.bytes;
  while (tot > kModelCacheBytes && !c.empty()) {  // release the oldest
    const CachedBlock b = c.front();
    c.pop_front();
    tot -= b.bytes;
    cudaStreamWaitEvent(ls, b.ev, 0);
    cudaEventDestroy(b.ev);
    g_msize[dev].erase(b.p);
    cudaFreeAsync(b.p, ls);
  }
}

template <class T>
T* dev_alloc(size_t count, cudaStream_t st, int dev) {
  return static_cast<T*>(model_alloc(count * sizeof(T), st, dev));
}

// Per-thread cached pinned host staging (cudaMallocHost / cudaFreeHost are slow and the
// latter synchronises the device, so they are not called per training run).
template <class T>
T* pinned_scratch(size_t count, int slot = 0) {
  static thread_local void* bufs[3] = {nullptr, nullptr, nullptr};
  static thread_local size_t caps[3] = {0, 0, 0};
  void*& buf = bufs[slot];
  size_t& cap = caps[slot];
  const size_t bytes = count * sizeof(T);
  if (bytes > cap) {
    if (buf) cudaFreeHost(buf);
    buf = nullptr;
    cap = 0;
    GM_CUDA(cudaMallocHost(&buf, bytes));
    cap = bytes;
  }
  return static_cast<T*>(buf);
}

enum { PH_STAGE, PH_KERNEL, PH_SELECT, PH_SUB, PH_FUP, PH_FIN, PH_DEC, PH_COUPLE, PH_D2H, PH_SOLVER, PH_N };

// timing events of lead mode's kernel-value waves (destroyed with the scope)
struct TimedEvents {
  cudaEvent_t a = nullptr, b = nullptr;
  TimedEvents() {
    GM_CUDA(cudaEventCreate(&a));
    GM_CUDA(cudaEventCreate(&b));
  }
  ~TimedEvents() {
    cudaEventDestroy(a);
    cudaEventDestroy(b);
  }
};

struct PhaseTimer {
  cudaStream_t st;
  std::vector<cudaEvent_t> evs[PH_N];
  explicit PhaseTimer(cudaStream_t s) : st(s) {}
  void mark(int ph) {
    cudaEvent_t e;
    GM_CUDA(cudaEventCreate(&e));
    GM_CUDA(cudaEventRecord(e, st));
    evs[ph].push_back(e);
  }
  double ms(int ph) {
    double t = 0.0;
    for (size_t i = 0; i + 1 < evs[ph].size(); i += 2) {
      float x = 0.f;
      GM_CUDA(cudaEventElapsedTime(&x, evs[ph][i], evs[ph][i + 1]));
      t += x;
    }
    return t;
  }
  ~PhaseTimer() {
    for (auto& v : evs)
      for (auto e : v) cudaEventDestroy(e);
  }
};

double host_ms_since(std::chrono::steady_clock::time_point t0) {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

bool finite_pos(double v) { return std::isfinite(v) && v > 0.0; }

}  // namespace

// ------------------------------------------------------------------------------------------
DevModel::~DevModel() {
  int prev = -1;
  cudaGetDevice(&prev);
  if (device >= 0) cudaSetDevice(device);
  gmpsvm_options o;
  gmpsvm_options_init(&o);
  o.device = device;
  cudaStream_t ls = nullptr;
  try {
    ls = get_stream(o);
  } catch (...) {
  }
  if (ls && last_use) cudaStreamWaitEvent(ls, last_use, 0);
  void* ptrs[] = {SvT,   nsv,      coef, items,     item_begin, item_end, b,    A,    B,     SvHi,
                  SvLo,  nsvc,     mu,   alpha_dev, coef64,     nsv64,    SvI8, sv_e, sv_n64};
  for (void* p : ptrs) model_free(p, ls, device >= 0 && device < 64 ? device : 0);
  if (last_use) cudaEventDestroy(last_use);
  if (prev >= 0) cudaSetDevice(prev);
}

std::vector<int64_t> Model::class_off() const {
  std::vector<int64_t> off(k + 1, 0);
  for (int c = 0; c < k; ++c) off[c + 1] = off[c] + class_count[c];
  return off;
}

std::vector<int64_t> Model::pair_offsets() const {
  std::vector<int64_t> po(P() + 1, 0);
  int p = 0;
  for (int s = 0; s < k; ++s)
    for (int t = s + 1; t < k; ++t, ++p) po[p + 1] = po[p] + class_count[s] + class_count[t];
  return po;
}

int Model::n_trained() const {
  int c = 0;
  for (auto t : trained) c += t ? 1 : 0;
  return c;
}

gmpsvm_predict_stats& tls_predict_stats() {
  static thread_local gmpsvm_predict_stats s{};
  return s;
}

// Build the device prediction structures from SV rows already on the device.
// rows: device pointer to rows (stride d); row_of_sv[i] = row of SV i (SV order = sv_pos order).
// pair index -> (s, t), the inverse of pair_index
static int ps_of(int p, int k) {
  int s = 0, rem = p;
  while (rem >= k - 1 - s) rem -= k - 1 - s++;
  return s;
}
static int pt_of(int p, int k) {
  int s = 0, rem = p;
  while (rem >= k - 1 - s) rem -= k - 1 - s++;
  return s + 1 + rem;
}
// Decision-value routing: a model predicts through the fastest path whose
// worst-case probability error kCoupleAmp * max_p |A_p|/4 * sum_j |alpha_pj| * E_K stays within
// kDecProbBound, half the 1e-4 contract.  dP/d dec = A P (1 - P) <= |A|/4 (Eq 12); |d dec| <=
// sum_j |alpha_j| |dK_j| (Eq 11); kCoupleAmp bounds max |dp| / max |dr| of the coupling (Eq 15:
// measured <= 1.97 over 1,500 random r matrices, k = 2..26).  E_K: the path's bound on |K~ - K|.
constexpr double kDecProbBound = 5e-5;
constexpr double kCoupleAmp = 2.0;
constexpr double kF16KErr = 4e-5;   // FP16 hi/lo split, FP32 K: 2x the measured max relative error (§6.1)
constexpr double kTestRange = 4.0;  // int8 bound assumes test rows within 4x the SVs' max |x| (checked per call)
enum { kDecF64 = 0, kDecI8 = 1, kDecF16 = 2 };

static void choose_dec_path(DevModel& dm, const Model& m) {
  const int P = m.P();
  dm.wsum = 0.0;
  for (int p = 0; p < P; ++p)
    if (m.trained[p] && p < (int)dm.abs_sum.size()) dm.wsum = std::max(dm.wsum, std::fabs(m.A[p]) * dm.abs_sum[p]);
  const double amp = kCoupleAmp * dm.wsum / 4.0;
  dm.cond_f16 = amp * kF16KErr;
  dm.cond_i8 = dm.SvI8 ? amp * dec_i8_kernel_err(dm.amax_sv, kTestRange * dm.amax_sv, m.d, m.gamma) : HUGE_VAL;
  static const char* dec_env = getenv("GMPSVM_DEC");  // forcing: f64 | i8 | f16 (tests, measurements)
  const std::string mode = dec_env ? dec_env : "";
  if (mode == "f64") dm.path = kDecF64;
  else if (mode == "f16" && dm.tc) dm.path = kDecF16;
  else if (mode == "i8" && dm.SvI8) dm.path = kDecI8;
  else if (dm.SvI8 && dm.cond_i8 <= kDecProbBound) dm.path = kDecI8;
  else dm.path = kDecF64;
  dm.f64 = dm.path == kDecF64;
}

// mu_in / sc_in: a given centre and split scale for the SV rows; nullptr = compute them from the
// SV rows
// alpha_hp / alpha_off: the training call's device alpha (solver pair order) and each model
// pair's offset into it; the coefficients are then built on the device and the DevModel keeps
// a copy of alpha (Model::alpha stays on the device until asked for).  nullptr: from m.alpha.
static std::unique_ptr<DevModel> build_dev_model(const Model& m, const float* rows, const std::vector<int64_t>& row_of_sv,
                                                 int device, cudaStream_t st, const float* mu_in = nullptr,
                                                 float sc_in = 0.f, const double* alpha_hp = nullptr,
                                                 int64_t alpha_tot = 0, const std::vector<int64_t>* alpha_off = nullptr) {
  auto dm = std::make_unique<DevModel>();
  static const bool ht = getenv("GMPSVM_HOST_TIMING") != nullptr;
  auto t_last = std::chrono::steady_clock::now();
  std::string line;
  auto HT = [&](const char* what) {
    if (!ht) return;
    GM_CUDA(cudaStreamSynchronize(st));
    const auto now = std::chrono::steady_clock::now();
    line += std::string(" ") + what + "=" +
            std::to_string(std::chrono::duration<double, std::milli>(now - t_last).count()).substr(0, 6);
    t_last = now;
  };
  dm->device = device;
  const int k = m.k, P = m.P();
  dm->km1 = k - 1;
  dm->km1_pad = (int)round_up(k - 1, 4);
  dm->d_pad = (int)round_up(m.d, kBK);
  const auto off = m.class_off();
  const auto po = m.pair_offsets();
  const int64_t nsv = (int64_t)m.sv_pos.size();
  // per-class SV ranges (sv_pos ascending => class order)
  std::vector<int64_t> sv_cls_begin(k + 1, 0);
  {
    int64_t i = 0;
    for (int c = 0; c < k; ++c) {
      sv_cls_begin[c] = i;
      while (i < nsv && m.sv_pos[i] < off[c + 1]) ++i;
    }
    sv_cls_begin[k] = nsv;
  }
  std::vector<int64_t> slot_begin(k + 1, 0);
  for (int c = 0; c < k; ++c)
    slot_begin[c + 1] = slot_begin[c] + round_up(sv_cls_begin[c + 1] - sv_cls_begin[c], kTile);
  dm->nsv_pad = std::max<int64_t>(slot_begin[k], kTile);
  dm->slot_sv.assign(dm->nsv_pad, -1);
  std::vector<int64_t> slot_src(dm->nsv_pad, -1);
  const bool dev_coef = alpha_hp != nullptr;
  std::vector<float> coef(dev_coef ? 0 : (size_t)dm->nsv_pad * dm->km1_pad, 0.f);
  std::vector<double> coef64(dev_coef ? 0 : (size_t)dm->nsv_pad * dm->km1_pad, 0.0);
  std::vector<int64_t> slot_g(dev_coef ? dm->nsv_pad : 0, -1);  // device coef: class-sorted position per slot
  std::vector<DecItem> items;
  std::vector<int32_t> ib(k, 0), ie(k, 0);
  for (int c = 0; c < k; ++c) {
    for (int64_t i = sv_cls_begin[c]; i < sv_cls_begin[c + 1]; ++i) {
      const int64_t slot = slot_begin[c] + (i - sv_cls_begin[c]);
      dm->slot_sv[slot] = i;
      slot_src[slot] = row_of_sv[i];
      const int64_t g = m.sv_pos[i];
      if (dev_coef) {
        slot_g[slot] = g;
        continue;
      }
      for (int u = 0; u < k; ++u) {
        if (u == c) continue;
        const int s = std::min(c, u), t = std::max(c, u);
        const int p = pair_index(s, t, k);
        const int64_t j = (c == s) ? (g - off[s]) : (m.class_count[s] + (g - off[t]));
        const double a = m.alpha[po[p] + j];
        const int col = u < c ? u : u - 1;
        coef[(size_t)slot * dm->km1_pad + col] = (float)((c == s) ? a : -a);
        coef64[(size_t)slot * dm->km1_pad + col] = (c == s) ? a : -a;
      }
    }
    ib[c] = (int32_t)items.size();
    const int t0 = (int)(slot_begin[c] / kTile), t1 = (int)(slot_begin[c + 1] / kTile);
    for (int t = t0; t < t1; t += kItemTiles) items.push_back(DecItem{c, t, std::min(t1, t + kItemTiles), 0});
    ie[c] = (int32_t)items.size();
  }
  if (items.empty()) items.push_back(DecItem{0, 0, 0, 0});  // no SV at all: zero contribution
  dm->n_items = (int)items.size();
  HT("host_coef");
  dm->SvT = dev_alloc<float>((size_t)dm->d_pad * dm->nsv_pad, st, device);
  dm->nsv = dev_alloc<float>(dm->nsv_pad, st, device);
  dm->coef = dev_alloc<float>((size_t)dm->nsv_pad * dm->km1_pad, st, device);
  dm->items = dev_alloc<DecItem>(items.size(), st, device);
  dm->item_begin = dev_alloc<int32_t>(k, st, device);
  dm->item_end = dev_alloc<int32_t>(k, st, device);
  dm->b = dev_alloc<double>(P, st, device);
  dm->A = dev_alloc<double>(P, st, device);
  dm->B = dev_alloc<double>(P, st, device);
  DevBuf<int64_t> d_src(slot_src.size(), st);
  GM_CUDA(cudaMemcpyAsync(d_src.get(), slot_src.data(), slot_src.size() * 8, cudaMemcpyHostToDevice, st));
  // conditioning of the decision values: sum_j |alpha_pj| per trained pair
  std::vector<double> abs_sum(P, 0.0);
  double* abs_pin = nullptr;  // device path: read after the call's last synchronisation
  if (dev_coef) {
    std::vector<int64_t> npv(P, 0);
    for (int p = 0; p < P; ++p) npv[p] = m.class_count[ps_of(p, k)] + m.class_count[pt_of(p, k)];
    DevBuf<int64_t> d_ao(P, st), d_np(P, st);
    DevBuf<double> d_sum(P, st);
    GM_CUDA(cudaMemcpyAsync(d_ao.get(), alpha_off->data(), (size_t)P * 8, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(d_np.get(), npv.data(), (size_t)P * 8, cudaMemcpyHostToDevice, st));
    launch_alpha_abs_sum(alpha_hp, d_ao.get(), d_np.get(), P, d_sum.get(), st);
    abs_pin = pinned_scratch<double>((size_t)P, 2);
    GM_CUDA(cudaMemcpyAsync(abs_pin, d_sum.get(), (size_t)P * 8, cudaMemcpyDeviceToHost, st));
  } else {
    for (int p = 0; p < P; ++p)
      for (int64_t j = po[p]; j < po[p + 1]; ++j) abs_sum[p] += std::fabs(m.alpha[j]);
  }
  static const char* dec_env = getenv("GMPSVM_DEC");
  const std::string dec_mode = dec_env ? dec_env : "";
  // FP64 coefficients: the int8 and FP64 paths contract in FP64
  dm->coef64 = dev_alloc<double>((size_t)dm->nsv_pad * dm->km1_pad, st, device);
  if (dev_coef) {
    dm->alpha_dev = dev_alloc<double>(std::max<int64_t>(alpha_tot, 1), st, device);
    if (alpha_tot) GM_CUDA(cudaMemcpyAsync(dm->alpha_dev, alpha_hp, (size_t)alpha_tot * 8, cudaMemcpyDeviceToDevice, st));
    dm->alpha_dev_off = *alpha_off;
    DevBuf<int64_t> d_g(slot_g.size(), st), d_aoff(P, st), d_off(k + 1, st), d_cc(k, st);
    GM_CUDA(cudaMemcpyAsync(d_g.get(), slot_g.data(), slot_g.size() * 8, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(d_aoff.get(), alpha_off->data(), (size_t)P * 8, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(d_off.get(), off.data(), (size_t)(k + 1) * 8, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(d_cc.get(), m.class_count.data(), (size_t)k * 8, cudaMemcpyHostToDevice, st));
    launch_build_coef(dm->alpha_dev, d_aoff.get(), d_g.get(), d_off.get(), d_cc.get(), k, dm->nsv_pad, dm->km1_pad,
                      dm->coef, dm->coef64, st);
  } else {
    GM_CUDA(cudaMemcpyAsync(dm->coef, coef.data(), coef.size() * 4, cudaMemcpyHostToDevice, st));
    if (dm->coef64) GM_CUDA(cudaMemcpyAsync(dm->coef64, coef64.data(), coef64.size() * 8, cudaMemcpyHostToDevice, st));
  }
  GM_CUDA(cudaMemcpyAsync(dm->items, items.data(), items.size() * sizeof(DecItem), cudaMemcpyHostToDevice, st));
  GM_CUDA(cudaMemcpyAsync(dm->item_begin, ib.data(), k * 4, cudaMemcpyHostToDevice, st));
  GM_CUDA(cudaMemcpyAsync(dm->item_end, ie.data(), k * 4, cudaMemcpyHostToDevice, st));
  GM_CUDA(cudaMemcpyAsync(dm->b, m.b.data(), P * 8, cudaMemcpyHostToDevice, st));
  GM_CUDA(cudaMemcpyAsync(dm->A, m.A.data(), P * 8, cudaMemcpyHostToDevice, st));
  GM_CUDA(cudaMemcpyAsync(dm->B, m.B.data(), P * 8, cudaMemcpyHostToDevice, st));
  launch_stage_features(rows, dm->nsv_pad, m.d, d_src.get(), dm->SvT, dm->nsv_pad, dm->d_pad, dm->nsv_pad, dm->nsv,
                        nullptr, st);
  HT("h2d_svt");
  dm->nsv64 = dev_alloc<double>(dm->nsv_pad, st, device);
  launch_col_norms64(dm->SvT, dm->nsv_pad, dm->nsv_pad, dm->d_pad, dm->nsv64, st);
  dm->h_items = items;
  // int8-digit SV planes (the default RBF path, dec_i8.cu)
  uint32_t amax_bits = 0;
  if (m.kernel == 0 && dm->km1_pad <= dec_i8_max_km1()) {
    dm->SvI8 = dev_alloc<int8_t>(dec_i8_plane_bytes(dm->nsv_pad, m.d), st, device);
    dm->sv_e = dev_alloc<int32_t>(dm->nsv_pad, st, device);
    dm->sv_n64 = dev_alloc<double>(dm->nsv_pad, st, device);
    DevBuf<unsigned> d_amax(1, st);
    GM_CUDA(cudaMemsetAsync(d_amax.get(), 0, 4, st));
    launch_stage_i8(rows, dm->nsv_pad, m.d, d_src.get(), dm->SvI8, dm->nsv_pad, dm->sv_e, dm->sv_n64, d_amax.get(), st);
    GM_CUDA(cudaMemcpyAsync(&amax_bits, d_amax.get(), 4, cudaMemcpyDeviceToHost, st));
    HT("stage_i8");
  }
  // FP16-split tensor-core decision values (forced with GMPSVM_DEC=f16): centre = mean of the SV
  // rows, hi/lo split of the SV slots
  dm->tc = dec_mode == "f16" && krow_use_tc() && krow_split_f16() && dm->km1_pad <= (m.kernel != 0 ? 12 : dec_tc_max_km1());
  if (dm->tc) {
    dm->dpt = krow_tc_d_pad(m.d);
    dm->mu = dev_alloc<float>(m.d, st, device);
    dm->SvHi = dev_alloc<float>(krow_tc_buf_floats(dm->nsv_pad, dm->dpt), st, device);
    dm->SvLo = dev_alloc<float>(krow_tc_buf_floats(dm->nsv_pad, dm->dpt), st, device);
    dm->nsvc = dev_alloc<float>(dm->nsv_pad, st, device);
    if (mu_in) {
      GM_CUDA(cudaMemcpyAsync(dm->mu, mu_in, (size_t)m.d * 4, cudaMemcpyDeviceToDevice, st));
      dm->sc = sc_in;
    } else if (m.kernel != 0) {  // dot-product kernels: uncentred rows (x . y itself)
      GM_CUDA(cudaMemsetAsync(dm->mu, 0, (size_t)m.d * 4, st));
      dm->sc = krow_split_scale(launch_maxabs(rows, dm->nsv_pad, m.d, d_src.get(), dm->mu, st));
    } else {
      launch_gather_col_mean(rows, m.d, d_src.get(), dm->nsv_pad, nsv, dm->mu, st);
      HT("mean");
      dm->sc = krow_split_scale(launch_maxabs(rows, dm->nsv_pad, m.d, d_src.get(), dm->mu, st));
      HT("maxabs");
    }
    launch_split_hilo_mu(rows, dm->nsv_pad, m.d, d_src.get(), dm->mu, dm->sc, dm->SvHi, dm->SvLo, dm->nsvc, dm->nsv_pad,
                         dm->dpt, st);
    HT("split");
  }
  GM_CUDA(cudaEventCreateWithFlags(&dm->last_use, cudaEventDisableTiming));
  GM_CUDA(cudaEventRecord(dm->last_use, st));
  GM_CUDA(cudaStreamSynchronize(st));  // host vectors above go out of scope
  if (abs_pin) std::copy(abs_pin, abs_pin + P, abs_sum.begin());
  dm->abs_sum = abs_sum;
  std::memcpy(&dm->amax_sv, &amax_bits, 4);
  choose_dec_path(*dm, m);
  if (ht)
    fprintf(stderr, "[gmpsvm devmodel ms]%s path=%d cond_i8=%.3e cond_f16=%.3e\n", line.c_str(), dm->path, dm->cond_i8,
            dm->cond_f16);
  return dm;
}

void ensure_host_sv(const Model& mdl) {
  Model& m = const_cast<Model&>(mdl);
  if (m.sv_X_ready) return;
  const int64_t nsv = (int64_t)m.sv_pos.size();
  m.sv_X.assign((size_t)nsv * m.d, 0.f);
  if (nsv > 0) {
    if (!m.dev) throw Error(GMPSVM_EINVAL, "model has no SV rows on host or device");
    DeviceGuard dg(m.dev->device);
    std::vector<float> t((size_t)m.dev->d_pad * m.dev->nsv_pad);
    GM_CUDA(cudaMemcpy(t.data(), m.dev->SvT, t.size() * 4, cudaMemcpyDeviceToHost));
    for (int64_t slot = 0; slot < m.dev->nsv_pad; ++slot) {
      const int64_t i = m.dev->slot_sv[slot];
      if (i < 0) continue;
      for (int c = 0; c < m.d; ++c) m.sv_X[(size_t)i * m.d + c] = t[(size_t)c * m.dev->nsv_pad + slot];
    }
  }
  m.sv_X_ready = true;
}

void ensure_host_alpha(const Model& mdl) {
  Model& m = const_cast<Model&>(mdl);
  if (m.alpha_ready) return;
  const auto po = m.pair_offsets();
  const int P = m.P();
  m.alpha.assign(po[P], 0.0);
  if (!m.dev || !m.dev->alpha_dev) throw Error(GMPSVM_EINVAL, "model alpha is on neither host nor device");
  DeviceGuard dg(m.dev->device);
  for (int p = 0; p < P; ++p) {
    const int64_t o = m.dev->alpha_dev_off[p];
    if (o >= 0 && po[p + 1] > po[p])
      GM_CUDA(cudaMemcpy(&m.alpha[po[p]], m.dev->alpha_dev + o, (size_t)(po[p + 1] - po[p]) * 8, cudaMemcpyDeviceToHost));
  }
  m.alpha_ready = true;
}

// ------------------------------------------------------------------------------------------
static int engine_train_core(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C, double gamma,
                             double eps, const gmpsvm_options& opt, Model** out, const CsrSrc* csr = nullptr);

// NEXT-2, LibSVM's probability training (ref [15]; the paper fits on in-sample values, R10):
// F-fold cross-validated decision values.  Fold of instance i = (its rank within its class,
// original order) mod F.  For each fold: train on the other folds (all pairs), decision values of
// the held-out rows (Eq 11) scattered into the pairs' pair-local layout; then every pair's
// sigmoid (Eq 12-13) is fitted on its out-of-fold values, and the final model (trained on all
// rows) gets those A, B.  All steps are the library's own kernels; F + 1 trainings.
static int engine_train_cv(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C, double gamma,
                           double eps, const gmpsvm_options& opt, Model** out) {
  const auto t_start = std::chrono::steady_clock::now();
  const int F = opt.prob_folds;
  if (F < 2 || F > 64) throw Error(GMPSVM_EINVAL, "prob_folds must be 0 or in [2, 64]");
  if (opt.pair_ids)
    throw Error(GMPSVM_ENOTIMPL, "cross-validated sigmoids need all pairs (no pair_ids)");
  if (!X || !y || !out) throw Error(GMPSVM_EINVAL, "null argument");
  if (n < 2 || d < 1 || k < 2) throw Error(GMPSVM_EINVAL, "need n >= 2, d >= 1, k >= 2");
  DeviceGuard dg(opt.device);
  cudaStream_t st = get_stream(opt);
  std::vector<int32_t> hy(n);
  if (opt.inputs_on_device) GM_CUDA(cudaMemcpy(hy.data(), y, (size_t)n * 4, cudaMemcpyDeviceToHost));
  else std::memcpy(hy.data(), y, (size_t)n * 4);
  std::vector<int64_t> rank(n), cnt(k, 0);
  for (int64_t i = 0; i < n; ++i) {
    if (hy[i] < 0 || hy[i] >= k) throw Error(GMPSVM_EINVAL, "labels must be in [0, k)");
    rank[i] = cnt[hy[i]]++;
  }
  for (int c = 0; c < k; ++c)
    if (cnt[c] < F) throw Error(GMPSVM_EINVAL, "prob_folds: every class needs at least `prob_folds` instances");
  DevBuf<float> bufX(opt.inputs_on_device ? 0 : (size_t)n * d, st);
  const float* dX = X;
  if (!opt.inputs_on_device) {
    GM_CUDA(cudaMemcpyAsync(bufX.get(), X, (size_t)n * d * 4, cudaMemcpyHostToDevice, st));
    dX = bufX.get();
  }
  gmpsvm_options o2 = opt;
  o2.prob_folds = 0;
  o2.inputs_on_device = 1;
  o2.stream = st;
  const int P = k * (k - 1) / 2;
  std::vector<PairDesc> pdv(P);
  int64_t tot = 0;
  for (int p = 0; p < P; ++p) {
    PairDesc& x = pdv[p];
    std::memset(&x, 0, sizeof(x));
    x.s = ps_of(p, k);
    x.t = pt_of(p, k);
    x.n_s = (int32_t)cnt[x.s];
    x.n_t = (int32_t)cnt[x.t];
    x.a_off = tot;
    x.pid = p;
    tot += x.n_s + x.n_t;
  }
  DevBuf<PairDesc> d_pairs(P, st);
  GM_CUDA(cudaMemcpyAsync(d_pairs.get(), pdv.data(), (size_t)P * sizeof(PairDesc), cudaMemcpyHostToDevice, st));
  DevBuf<double> d_v(tot, st);
  GM_CUDA(cudaMemsetAsync(d_v.get(), 0, (size_t)tot * 8, st));
  for (int f = 0; f < F; ++f) {
    std::vector<int64_t> tr, ho;
    std::vector<int32_t> ytr, cls;
    std::vector<int64_t> rk;
    for (int64_t i = 0; i < n; ++i) {
      if (rank[i] % F != f) {
        tr.push_back(i);
        ytr.push_back(hy[i]);
      } else {
        ho.push_back(i);
        cls.push_back(hy[i]);
        rk.push_back(rank[i]);
      }
    }
    const int64_t ntr = (int64_t)tr.size(), nho = (int64_t)ho.size();
    DevBuf<int64_t> d_tr(ntr, st), d_ho(nho, st), d_rk(nho, st);
    DevBuf<int32_t> d_ytr(ntr, st), d_cls(nho, st);
    DevBuf<float> Xtr((size_t)ntr * d, st), Xho((size_t)nho * d, st);
    DevBuf<double> dec((size_t)nho * P, st);
    GM_CUDA(cudaMemcpyAsync(d_tr.get(), tr.data(), (size_t)ntr * 8, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(d_ho.get(), ho.data(), (size_t)nho * 8, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(d_rk.get(), rk.data(), (size_t)nho * 8, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(d_ytr.get(), ytr.data(), (size_t)ntr * 4, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(d_cls.get(), cls.data(), (size_t)nho * 4, cudaMemcpyHostToDevice, st));
    launch_gather_rows(dX, d, d_tr.get(), ntr, Xtr.get(), st);
    launch_gather_rows(dX, d, d_ho.get(), nho, Xho.get(), st);
    Model* mf = nullptr;
    engine_train_core(Xtr.get(), d_ytr.get(), ntr, d, k, C, gamma, eps, o2, &mf);
    std::unique_ptr<Model> gf(mf);
    engine_predict(*mf, Xho.get(), nho, nullptr, dec.get(), o2);
    launch_scatter_oof(dec.get(), nho, P, d_cls.get(), d_rk.get(), d_pairs.get(), d_v.get(), st);
    GM_CUDA(cudaStreamSynchronize(st));  // fold buffers go out of scope
  }
  DevBuf<double> dA(P, st), dB(P, st);
  DevBuf<int32_t> dS(P, st);
  launch_sigmoid_fit_on(d_pairs.get(), P, d_v.get(), dA.get(), dB.get(), dS.get(), st);
  std::vector<double> hA(P), hB(P);
  std::vector<int32_t> hS(P);
  GM_CUDA(cudaMemcpyAsync(hA.data(), dA.get(), (size_t)P * 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaMemcpyAsync(hB.data(), dB.get(), (size_t)P * 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaMemcpyAsync(hS.data(), dS.get(), (size_t)P * 4, cudaMemcpyDeviceToHost, st));
  DevBuf<int32_t> bufY(opt.inputs_on_device ? 0 : (size_t)n, st);
  const int32_t* dy = y;
  if (!opt.inputs_on_device) {
    GM_CUDA(cudaMemcpyAsync(bufY.get(), hy.data(), (size_t)n * 4, cudaMemcpyHostToDevice, st));
    dy = bufY.get();
  }
  Model* m = nullptr;
  int rc = engine_train_core(dX, dy, n, d, k, C, gamma, eps, o2, &m);
  std::unique_ptr<Model> gm(m);
  GM_CUDA(cudaStreamSynchronize(st));
  for (int p = 0; p < P; ++p) {  // the cross-validated sigmoids replace the in-sample ones
    m->A[p] = hA[p];
    m->B[p] = hB[p];
    m->status[p] = (m->status[p] & 0xff) | (hS[p] << 8);
    if (hS[p] == 1) rc = GMPSVM_WARN_MAXITER;
  }
  if (m->dev) {
    GM_CUDA(cudaMemcpy(m->dev->A, hA.data(), (size_t)P * 8, cudaMemcpyHostToDevice));
    GM_CUDA(cudaMemcpy(m->dev->B, hB.data(), (size_t)P * 8, cudaMemcpyHostToDevice));
    choose_dec_path(*m->dev, *m);  // the routing bound depends on A (re-evaluated)
  }
  m->stats.t_total_ms = host_ms_since(t_start);
  *out = gm.release();
  return rc;
}

int engine_train(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C, double gamma, double eps,
                 const gmpsvm_options& opt, Model** out) {
  if (opt.prob_folds != 0) return engine_train_cv(X, y, n, d, k, C, gamma, eps, opt, out);
  return engine_train_core(X, y, n, d, k, C, gamma, eps, opt, out);
}

static int engine_train_core(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C, double gamma,
                             double eps, const gmpsvm_options& opt, Model** out, const CsrSrc* csr) {
  const auto t_start = std::chrono::steady_clock::now();
  // GMPSVM_HOST_TIMING=1: host-clock checkpoints of the training call on stderr
  static const bool host_timing = getenv("GMPSVM_HOST_TIMING") != nullptr;
  auto t_last = t_start;
  std::string ht_line;
  auto HT = [&](const char* what) {
    if (!host_timing) return;
    const auto now = std::chrono::steady_clock::now();
    ht_line += std::string(" ") + what + "=" +
               std::to_string(std::chrono::duration<double, std::milli>(now - t_last).count()).substr(0, 6);
    t_last = now;
  };
  if ((!X && !csr) || !y || !out) throw Error(GMPSVM_EINVAL, "null argument");
  if (csr && (!opt.inputs_on_device || opt.kernel != 0 || opt.prob_folds != 0))
    throw Error(GMPSVM_ENOTIMPL, "sparse kernel values: device CSR rows, the Gaussian kernel, no CV sigmoids");
  if (n < 2 || d < 1 || k < 2) throw Error(GMPSVM_EINVAL, "need n >= 2, d >= 1, k >= 2");
  if (k > kMaxK) throw Error(GMPSVM_ENOTIMPL, "k > 64 classes not supported by this build");
  if (n >= (int64_t)1 << 31) throw Error(GMPSVM_ENOTIMPL, "n >= 2^31 not supported");
  if (!finite_pos(C) || !finite_pos(gamma) || !finite_pos(eps)) throw Error(GMPSVM_EINVAL, "C, gamma, eps must be finite and > 0");
  const int ktype = opt.kernel;  // GMPSVM_KERNEL_*: the paper's RBF or one of its other kernels (L76-L78)
  const double kcoef0 = opt.coef0;
  const int kdegree = opt.degree ? opt.degree : 3;
  if (ktype < 0 || ktype > 3 || kdegree < 1 || kdegree > 16 || !std::isfinite(kcoef0))
    throw Error(GMPSVM_EINVAL, "kernel must be 0..3, degree 1..16, coef0 finite");
  int B = opt.ws_size ? opt.ws_size : kDefaultB;
  if (B < 2 || B > 1024 || (B & 1)) throw Error(GMPSVM_EINVAL, "ws_size must be even and in [2, 1024]");
  int q = opt.q ? opt.q : B / 2;
  if (q < 2 || q > B) throw Error(GMPSVM_EINVAL, "q must be in [2, ws_size]");
  DeviceGuard dg(opt.device);
  cudaStream_t st = get_stream(opt);
  const uint64_t launches0 = g_launches.load();
  PhaseTimer tm(st);
  static const bool lead_dbg = getenv("GMPSVM_LEAD_DEBUG") != nullptr;  // diagnostics: device timeline
  TimedEvents dbg0, dbg1;  // call entry (a), solver done on st (b); finalize done (dbg1.a)
  if (lead_dbg) GM_CUDA(cudaEventRecord(dbg0.a, st));

  // ---------------- a1 staging
  HT("stage0");
  tm.mark(PH_STAGE);
  DevBuf<float> bufX(opt.inputs_on_device ? 0 : (size_t)n * d, st);
  DevBuf<int32_t> bufY(opt.inputs_on_device ? 0 : (size_t)n, st);
  const float* dX = X;
  const int32_t* dy = y;
  if (!opt.inputs_on_device) {
    GM_CUDA(cudaMemcpyAsync(bufX.get(), X, (size_t)n * d * 4, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(bufY.get(), y, (size_t)n * 4, cudaMemcpyHostToDevice, st));
    dX = bufX.get();
    dy = bufY.get();
  }
  const int nb = (int)ceil_div(n, 1024);
  DevBuf<int32_t> blk_counts((size_t)nb * (k + 1), st), blk_off((size_t)nb * k, st);
  DevBuf<int64_t> d_count(k + 1, st), d_off(k + 1, st), d_perm(n, st);
  launch_class_sort(dy, n, k, blk_counts.get(), blk_off.get(), d_count.get(), d_off.get(), st);
  std::vector<int64_t> cc(k + 1);
  GM_CUDA(cudaMemcpyAsync(cc.data(), d_count.get(), (k + 1) * 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaStreamSynchronize(st));
  if (cc[k] != 0) throw Error(GMPSVM_EINVAL, "labels must be in [0, k)");
  for (int c = 0; c < k; ++c)
    if (cc[c] == 0) throw Error(GMPSVM_EINVAL, "every class must have at least one instance");
  launch_class_rank(dy, n, k, blk_off.get(), d_off.get(), d_perm.get(), st);
  // a2 regime: FULL_K keeps the whole class-sorted n x n kernel matrix
  // resident when it fits the cache budget; otherwise ROW_CACHE computes the rows of each
  // pair's new working-set entries per outer iteration into a B-row buffer per pair.
  const int64_t ldk = round_up(n, 4);
  const double bytes_K = (double)n * ldk * 4.0;
  // default budget: 85% of the device memory (cached per device; cudaMemGetInfo can take
  // tens of milliseconds, so it is not queried per call)
  const double budget = opt.cache_bytes > 0 ? (double)opt.cache_bytes : 0.85 * (double)device_total_mem(opt.device);
  const bool full_k = bytes_K <= budget;
  if (csr && !full_k) throw Error(GMPSVM_ENOTIMPL, "sparse kernel values: the n x n kernel matrix must fit (FULL_K)");
  // tensor cores for the kernel values: FULL_K always; ROW_CACHE rows for the Gaussian with the
  // FP16 split (rows_tc_kernel); the SIMT contraction otherwise (GMPSVM_KROW=simt)
  const bool use_tc = !csr && krow_use_tc() && (full_k || (ktype == 0 && krow_split_f16()));
  if (ktype != 0 && !(use_tc && krow_split_f16()))
    throw Error(GMPSVM_ENOTIMPL, "the linear / polynomial / sigmoid kernels need the FULL_K regime on the tensor cores");
  const int d_pad = use_tc ? krow_tc_d_pad(d) : (int)round_up(d, kBK);
  // ROW_CACHE column tiles start at 4-aligned segment starts and may run 127 columns past n
  const int64_t n_pad = use_tc ? krow_tc_rows_pad(n) : round_up(n, kTile) + (full_k ? 0 : kTile);
  // SIMT path: class-sorted feature-major copy; tensor-core path: row-major FP16 hi/lo split
  // (TF32 with GMPSVM_SPLIT=tf32).
  // norms: + one tile of zeros (ROW_CACHE column tiles run up to 127 columns past n)
  DevBuf<float> XT(use_tc || csr ? 0 : (size_t)d_pad * n_pad, st), norms(n_pad + kTile, st);
  // NEXT-3: class-sorted CSR rows (sptr on the host from the input row pointers and the order)
  DevBuf<int64_t> c_ptr(csr ? (size_t)n + 1 : 0, st);
  DevBuf<int32_t> c_idx(csr ? (size_t)std::max<int64_t>(csr->nnz, 1) : 0, st);
  DevBuf<float> c_val(csr ? (size_t)std::max<int64_t>(csr->nnz, 1) : 0, st);
  GM_CUDA(cudaMemsetAsync(norms.get() + n_pad, 0, kTile * sizeof(float), st));
  DevBuf<float> Xhi(use_tc ? krow_tc_buf_floats(n_pad, d_pad) : 0, st), Xlo(use_tc ? krow_tc_buf_floats(n_pad, d_pad) : 0, st);
  float ksc = 1.f;  // scale of the split (FP16: exact power of two)
  DevBuf<int32_t> bad(1, st);
  GM_CUDA(cudaMemsetAsync(bad.get(), 0, 4, st));
  DevBuf<uint8_t> tc_scratch(use_tc ? krow_tc_scratch_bytes(n, d) : 0, st);
  if (use_tc) {
    launch_row_norms(dX, n, d, d_perm.get(), norms.get(), n_pad, bad.get(), st);  // validation (non-finite rows)
    ksc = launch_split_hilo(dX, n, d, d_perm.get(), Xhi.get(), Xlo.get(), norms.get(), n_pad, d_pad, tc_scratch.get(), st,
                            ktype == 0);
  } else if (csr) {
    std::vector<int64_t> hptr((size_t)n + 1), hperm(n), sptr((size_t)n + 1, 0);
    GM_CUDA(cudaMemcpyAsync(hptr.data(), csr->indptr, ((size_t)n + 1) * 8, cudaMemcpyDeviceToHost, st));
    GM_CUDA(cudaMemcpyAsync(hperm.data(), d_perm.get(), (size_t)n * 8, cudaMemcpyDeviceToHost, st));
    GM_CUDA(cudaStreamSynchronize(st));
    for (int64_t i = 0; i < n; ++i) {
      const int64_t len = hptr[hperm[i] + 1] - hptr[hperm[i]];
      if (len < 0) throw Error(GMPSVM_EINVAL, "CSR row pointers must be non-decreasing");
      sptr[i + 1] = sptr[i] + len;
    }
    if (sptr[n] != csr->nnz) throw Error(GMPSVM_EINVAL, "CSR row pointers do not match nnz");
    GM_CUDA(cudaMemcpyAsync(c_ptr.get(), sptr.data(), ((size_t)n + 1) * 8, cudaMemcpyHostToDevice, st));
    launch_csr_stage(csr->indptr, csr->indices, csr->values, d_perm.get(), n, d, c_ptr.get(), c_idx.get(), c_val.get(),
                     norms.get(), bad.get(), st);
  } else {
    launch_stage_features(dX, n, d, d_perm.get(), XT.get(), n_pad, d_pad, n_pad, norms.get(), bad.get(), st);
  }
  int32_t hbad = 0;
  GM_CUDA(cudaMemcpyAsync(&hbad, bad.get(), 4, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaStreamSynchronize(st));
  if (hbad) throw Error(GMPSVM_EINVAL, "X contains non-finite values");
  tm.mark(PH_STAGE);
  HT("stage1");
  // class means and spreads of the staged rows: the pairs whose classes overlap most -- smallest
  // Fisher ratio |mu_s - mu_t|^2 / (tr S_s + tr S_t) -- are expected to need the most solver work
  // (measured, MNIST-shaped: Spearman 0.85 against the pairs' inner SMO steps, the hardest pair
  // (0,8) ranked first; tools/pair_difficulty.py), so they come first: their own graph branches
  // and, in lead mode below, their kernel values first
  std::vector<double> fisher;  // per pair index (tc path)
  if (use_tc) {
    DevBuf<float> d_mu((size_t)k * d_pad, st), d_m2((size_t)k * d_pad, st);
    launch_class_means(Xhi.get(), d_pad, d_off.get(), k, d_mu.get(), d_m2.get(), st);
    std::vector<float> mu((size_t)k * d_pad), m2((size_t)k * d_pad);
    GM_CUDA(cudaMemcpyAsync(mu.data(), d_mu.get(), mu.size() * 4, cudaMemcpyDeviceToHost, st));
    GM_CUDA(cudaMemcpyAsync(m2.data(), d_m2.get(), m2.size() * 4, cudaMemcpyDeviceToHost, st));
    GM_CUDA(cudaStreamSynchronize(st));
    std::vector<double> var(k, 0.0);
    for (int c = 0; c < k; ++c)
      for (int f = 0; f < d_pad; ++f) {
        const double m = mu[(size_t)c * d_pad + f];
        var[c] += std::max(0.0, (double)m2[(size_t)c * d_pad + f] - m * m);
      }
    fisher.assign((size_t)k * (k - 1) / 2, 0.0);
    for (int s0 = 0; s0 < k; ++s0)
      for (int t0 = s0 + 1; t0 < k; ++t0) {
        double acc = 0.0;
        for (int f = 0; f < d_pad; ++f) {
          const double df = (double)mu[(size_t)s0 * d_pad + f] - mu[(size_t)t0 * d_pad + f];
          acc += df * df;
        }
        fisher[pair_index(s0, t0, k)] = acc / std::max(var[s0] + var[t0], 1e-30);
      }
  }

  // ---------------- pairs to train
  const int P = k * (k - 1) / 2;
  std::vector<int> pids;
  // an explicit but empty subset is an error, not "all pairs" (a multi-GPU rank with no pair
  // must skip training; dist.train_predict does)
  if (opt.pair_ids && opt.n_pair_ids <= 0) throw Error(GMPSVM_EINVAL, "pair_ids given with n_pair_ids <= 0");
  if (opt.pair_ids && opt.n_pair_ids > 0) {
    std::vector<uint8_t> seen(P, 0);
    for (int i = 0; i < opt.n_pair_ids; ++i) {
      const int p = opt.pair_ids[i];
      if (p < 0 || p >= P || seen[p]) throw Error(GMPSVM_EINVAL, "pair_ids out of range or repeated");
      seen[p] = 1;
      pids.push_back(p);
    }
  } else {
    for (int p = 0; p < P; ++p) pids.push_back(p);
  }
  const int Pl = (int)pids.size();
  std::vector<int64_t> coff(k + 1, 0);
  for (int c = 0; c < k; ++c) coff[c + 1] = coff[c] + cc[c];
  std::vector<int> ps(P), pt(P);
  for (int s = 0; s < k; ++s)
    for (int t = s + 1; t < k; ++t) {
      ps[pair_index(s, t, k)] = s;
      pt[pair_index(s, t, k)] = t;
    }
  // largest pairs first (smallest Fisher ratio first on the tensor-core path, see above): they
  // start first and share streams with pairs of similar cost
  if (!fisher.empty())
    std::stable_sort(pids.begin(), pids.end(), [&](int x, int y) { return fisher[x] < fisher[y]; });
  else
    std::stable_sort(pids.begin(), pids.end(),
                     [&](int x, int y) { return cc[ps[x]] + cc[pt[x]] > cc[ps[y]] + cc[pt[y]]; });
  std::vector<PairDesc> hp(Pl);
  int64_t tot = 0, np_max = 0;
  for (int i = 0; i < Pl; ++i) {
    const int p = pids[i];
    PairDesc& x = hp[i];
    x.s = ps[p];
    x.t = pt[p];
    x.n_s = (int32_t)cc[x.s];
    x.n_t = (int32_t)cc[x.t];
    x.off_s = coff[x.s];
    x.off_t = coff[x.t];
    x.a_off = tot;
    x.pid = p;
    x.pad = 0;
    tot += x.n_s + x.n_t;
    np_max = std::max<int64_t>(np_max, x.n_s + x.n_t);
  }

  // Default working-set size: B = 192 (the shared-memory local solver, tuned on MNIST-shaped
  // data) when every pair fits the wsolve.cu path; pairs beyond it (n_p > 16,384) run the
  // solver.cu kernels, where the paper's B = 1024, q = 512 (L377) cuts the outer iterations 4-40x
  // (measured: covtype-shaped 581k 0.41 -> 0.20 s, MNIST8M-shaped 1M 15.9 -> 5.1 s): the largest
  // of 1024 / 512 / 256 whose ROW_CACHE row buffers fit the budget (else 192).
  // ROW_CACHE: the row buffers must fit next to what is already allocated (X, its staged copy):
  // the free device memory now (+ a cached kernel-matrix workspace this call may reuse), less a
  // 4 GB margin for the solver's other buffers
  double rc_avail = 0.0;
  if (!full_k) {
    size_t fr = 0, tt = 0;
    cudaMemPool_t pool;  // memory the stream-ordered pool holds but does not use goes back first
    GM_CUDA(cudaStreamSynchronize(st));
    GM_CUDA(cudaDeviceGetDefaultMemPool(&pool, opt.device));
    GM_CUDA(cudaMemPoolTrimTo(pool, 0));
    GM_CUDA(cudaMemGetInfo(&fr, &tt));
    rc_avail = std::min((double)fr + (double)kcache_bytes(opt.device) - 4e9, 0.85 * (double)device_total_mem(opt.device));
  }
  if (!opt.ws_size && np_max > kWsMaxNp) {
    for (int cand : {1024, 512, 256, 128}) {
      double r = 0;
      for (const auto& x : hp) r += (double)cand * round_up(x.n_s + x.n_t, 4) * 4.0;
      if (full_k || r + (double)Pl * d_pad * round_up(cand, kTile) * 4.0 <= rc_avail) {
        B = cand;
        break;
      }
    }
    if (!opt.q) q = B / 2;
  }

  // ---------------- a2 kernel values
  HT("memgetinfo");
  const int ldat = (int)round_up(B, kTile);
  double bytes_R = 0;
  for (auto& x : hp) {
    x.r_off = (int64_t)(bytes_R / 4);
    bytes_R += (double)B * round_up(x.n_s + x.n_t, 4) * 4.0;
  }
  if (!full_k) {
    const double rc_total = bytes_R + (double)Pl * d_pad * ldat * 4.0;
    if (rc_total > rc_avail)
      throw Error(GMPSVM_ENOTIMPL, "ROW_CACHE buffers (" + std::to_string(rc_total / 1e9) +
                                       " GB) exceed the device memory; train the pairs in parts (pair_ids) and merge");
  }
  // FULL_K: the n x ldk matrix; ROW_CACHE: the per-pair B x round_up(n_p, 4) row buffers
  KWorkspace K(opt.device, full_k ? (size_t)n * ldk * sizeof(float) : (size_t)bytes_R, st);
  HT("k_alloc");
  // The solver's state, its graphs and the kernel-value tile list are kept per device and reused by
  // the next call of the same shape in the default regime (FULL_K, every pair on the wsolve.cu
  // kernels, no diagnostics); see the arena below.
  static const bool smo_prof = getenv("GMPSVM_SMO_PHASES") != nullptr;
  // GMPSVM_TRACE=<pair position>: kernel timeline of that pair (entries sorted largest pair first)
  static const int trace_pos = getenv("GMPSVM_TRACE") ? atoi(getenv("GMPSVM_TRACE")) : -1;
  static const bool no_reuse = getenv("GMPSVM_GRAPH_REUSE") && std::string(getenv("GMPSVM_GRAPH_REUSE")) == "0";
  const bool cacheable = !no_reuse && full_k && !smo_prof && trace_pos < 0 && ws_solve_supported(B, np_max);
  SolverCacheLease lease(cacheable ? opt.device : -1, st);  // cached arena, graphs, tiles -- or none
  DevBuf<int2> d_tiles_own;
  const int2* d_tiles = nullptr;
  size_t n_tiles = 0;
  // Lead mode (default on the tensor-core FULL_K path with the device-driven solver): the pairs
  // are split into groups in their order (the predicted hardest first, above) -- the lead pairs,
  // one graph branch each, then GMPSVM_GROUPS groups of the rest -- and each group is a graph of
  // its own that starts as soon as the kernel values of its pairs' class blocks (s,s), (s,t), (t,t)
  // are done.  The kernel matrix is computed in that order, one wave per group: wave 0 (the lead
  // blocks) on every SM, the later waves on all but `reserve` SMs, where the started groups' solver
  // chains run.  The solver's critical path -- the hardest pairs' chains of outer iterations --
  // so overlaps the kernel-value contraction instead of following it.  GMPSVM_LEAD=<pairs>
  // (0: off), GMPSVM_LEAD_RESERVE=<SMs>, GMPSVM_GROUPS=<groups of the rest> (measured on
  // MNIST-shaped data: 1 group best -- more groups start more chains beside the lead chain and
  // slow it down: 33.3 / 34.4 / 34.8 ms per bench step for 1 / 2 / 3 groups; 1 / 2 / 4 lead pairs
  // and 4 / 8 / 12 / 16 reserved SMs within 0.3 ms of each other).
  const bool fk_tc = full_k && use_tc;  // the FULL_K contraction on tcgen05
  static const int lead_env = getenv("GMPSVM_LEAD") ? std::max(0, atoi(getenv("GMPSVM_LEAD"))) : 1;
  static const int reserve_env = getenv("GMPSVM_LEAD_RESERVE") ? std::max(0, atoi(getenv("GMPSVM_LEAD_RESERVE"))) : 8;
  static const int groups_env =
      std::max(1, std::min(kMaxGroups - 1, getenv("GMPSVM_GROUPS") ? atoi(getenv("GMPSVM_GROUPS")) : 1));
  // Solver graph branches (below): the runtime runs at most CUDA_DEVICE_MAX_CONNECTIONS branches
  // concurrently -- a branch beyond that shares a hardware queue with another and waits for it --
  // so the pairs are packed into that many branches: the first pairs alone, the last two (or more)
  // to a branch in lockstep.  Lead mode keeps a queue free per graph launch stream and one for the
  // kernel-value stream: measured, a branch otherwise queued behind the lead chain.
  const int conn = connections_in_effect();
  int n_lead = (fk_tc && lead_env > 0 && Pl > lead_env && ws_solve_supported(B, np_max)) ? lead_env : 0;
  int ng = 1;  // pair groups (graphs)
  if (n_lead) {
    ng = 1 + std::min(groups_env, Pl - n_lead);
    if (conn - n_lead - ng - 1 < ng - 1) n_lead = 0, ng = 1;  // not enough queues
  }
  const bool lead = n_lead > 0;
  std::vector<int> gpos(ng + 1, 0), gbr(ng + 1, 0);  // per group: pair positions, branches
  std::vector<int> bb(1, 0);                          // per branch: pair positions [bb[b], bb[b+1])
  auto pack = [&](int p0, int cnt, int nb) {          // cnt pairs from position p0 into nb branches
    const int m = cnt / nb, r = cnt % nb;             // the last r branches take m + 1 pairs
    for (int b = 0; b < nb; ++b) bb.push_back(bb.back() + m + (b >= nb - r ? 1 : 0));
    (void)p0;
  };
  if (!lead) {
    gpos[1] = Pl;
    pack(0, Pl, std::min(Pl, conn));
    gbr[1] = (int)bb.size() - 1;
  } else {
    gpos[1] = n_lead;
    pack(0, n_lead, n_lead);
    gbr[1] = n_lead;
    const int rest = Pl - n_lead, ngr = ng - 1, budget = conn - n_lead - ng - 1;
    for (int g = 1; g < ng; ++g) {
      const int cnt = rest / ngr + (g - 1 < rest % ngr ? 1 : 0);
      gpos[g + 1] = gpos[g] + cnt;
      const int nb = std::max(1, std::min(cnt, (int)((double)budget * cnt / rest)));
      pack(gpos[g], cnt, nb);
      gbr[g + 1] = (int)bb.size() - 1;
    }
  }
  const int nbr = (int)bb.size() - 1;
  cudaStream_t kst = krow_stream(opt.device);
  TimedEvents kev;
  cudaEvent_t ev_k0 = kev.a, ev_k1 = kev.b;
  EventPool evk;
  static const bool lead_dbg_t = getenv("GMPSVM_LEAD_DEBUG") != nullptr;
  std::vector<cudaEvent_t> ev_wave(ng, nullptr), ev_gst(ng, nullptr), ev_gend(ng, nullptr);  // per group
  std::vector<size_t> wave_off(ng + 1, 0);  // lead mode: tile range of wave g
  const bool two_cta = fk_tc && !lead && ktype == 0 && krow_tc_2cta();  // lead waves: single-CTA tiles
  double kv_subset = -1;  // >= 0: kernel values computed for a pair subset (tiles skipped)
  // 2-CTA clusters sharing the row operand by TMA multicast (the Gaussian kernel, FP16 split)
  const bool kmc = fk_tc && !two_cta && ktype == 0 && krow_tc_mc();
  if (fk_tc) {
    // class range [cr[2i], cr[2i+1]] of the rows of tile row / column i
    const int nti = (int)ceil_div(n, kKrowTileRows);
    std::vector<int> cr(2 * (size_t)nti);
    for (int i = 0, c = 0; i < nti; ++i) {
      const int64_t r0 = (int64_t)i * kKrowTileRows, r1 = std::min<int64_t>(n, r0 + kKrowTileRows) - 1;
      while (coff[c + 1] <= r0) ++c;
      int e = c;
      while (coff[e + 1] <= r1) ++e;
      cr[2 * i] = c;
      cr[2 * i + 1] = e;
    }
    // does tile tl overlap a class block marked in blk (k x k, upper triangle)?
    auto touches = [&](const int2 tl, const std::vector<uint8_t>& blk) {
      for (int a0 = cr[2 * tl.x]; a0 <= cr[2 * tl.x + 1]; ++a0)
        for (int b0 = cr[2 * tl.y]; b0 <= cr[2 * tl.y + 1]; ++b0)
          if (blk[(size_t)std::min(a0, b0) * k + std::max(a0, b0)]) return true;
      return false;
    };
    auto blocks_of = [&](int i0, int i1) {  // class blocks of the pairs at positions [i0, i1)
      std::vector<uint8_t> blk((size_t)k * k, 0);
      for (int i = i0; i < i1; ++i) {
        blk[(size_t)hp[i].s * k + hp[i].s] = blk[(size_t)hp[i].t * k + hp[i].t] = 1;
        blk[(size_t)std::min(hp[i].s, hp[i].t) * k + std::max(hp[i].s, hp[i].t)] = 1;
      }
      return blk;
    };
    const bool subset = !two_cta && Pl < P;
    const std::vector<uint8_t> need = subset ? blocks_of(0, Pl) : std::vector<uint8_t>();
    std::vector<std::vector<uint8_t>> gmask;  // lead mode: class blocks per group
    if (lead)
      for (int g = 0; g < ng; ++g) gmask.push_back(blocks_of(gpos[g], gpos[g + 1]));
    std::vector<int64_t> tkey = {n, two_cta ? 1 : 0, k, kmc ? 1 : 0};  // what the tile list depends on
    tkey.insert(tkey.end(), coff.begin(), coff.end());
    for (const uint8_t v : need) tkey.push_back(v);
    for (const auto& gm : gmask) {
      tkey.push_back(-1);
      for (const uint8_t v : gm) tkey.push_back(v);
    }
    SolverWs* ws = lease.ws;
    if (ws && ws->tiles && ws->tkey == tkey) {  // the last call's list
      d_tiles = ws->tiles;
      n_tiles = ws->n_tiles;
      wave_off = ws->wave_off;
      kv_subset = ws->kv_subset;
    } else {
      std::vector<int2> tiles = krow_tc_tiles(n, two_cta);
      if (subset) {
        // pair subset (multi-GPU shard, pair_ids): only the tiles overlapping a class block
        // (s,s), (s,t), (t,t) of a trained pair are computed (PAPER.md L313-L325 sharing, per rank)
        std::vector<int2> kept;
        for (const int2 tl : tiles)
          if (touches(tl, need)) kept.push_back(tl);
        tiles.swap(kept);
        kv_subset = 0;  // kernel values (r <= c) the kept tiles compute
        for (const int2 tl : tiles) {
          const int64_t r0 = (int64_t)tl.x * kKrowTileRows, c0 = (int64_t)tl.y * kKrowTileRows;
          const int64_t nr = std::min<int64_t>(n, r0 + kKrowTileRows) - r0, nc = std::min<int64_t>(n, c0 + kKrowTileRows) - c0;
          kv_subset += tl.x == tl.y ? (double)nr * (double)(nr + 1) / 2.0 : (double)nr * (double)nc;
        }
      }
      if (lead) {  // wave g: the tiles first needed by group g (blocked order kept within a wave)
        std::vector<std::vector<int2>> w(ng);
        for (const int2 tl : tiles) {
          int g = 0;
          while (g < ng - 1 && !touches(tl, gmask[g])) ++g;
          w[g].push_back(tl);
        }
        tiles.clear();
        for (int g = 0; g < ng; ++g) {
          if (kmc) w[g] = krow_tc_mc_pairs(w[g]);
          tiles.insert(tiles.end(), w[g].begin(), w[g].end());
          wave_off[g + 1] = tiles.size();
        }
      } else if (kmc) {
        tiles = krow_tc_mc_pairs(tiles);
      }
      n_tiles = tiles.size();
      int2* dt = nullptr;
      if (ws) {
        if (ws->tiles) cudaFreeAsync(ws->tiles, st);
        ws->tiles = nullptr;
        ws->tkey.clear();
        GM_CUDA(cudaMallocAsync((void**)&ws->tiles, std::max<size_t>(n_tiles, 1) * sizeof(int2), st));
        dt = ws->tiles;
        ws->tkey = tkey;
        ws->n_tiles = n_tiles;
        ws->wave_off = wave_off;
        ws->kv_subset = kv_subset;
      } else {
        new (&d_tiles_own) DevBuf<int2>(n_tiles, st);
        dt = d_tiles_own.get();
      }
      GM_CUDA(cudaMemcpyAsync(dt, tiles.data(), n_tiles * sizeof(int2), cudaMemcpyHostToDevice, st));
      d_tiles = dt;
    }
  }
  tm.mark(PH_KERNEL);
  // lead mode: CTAs of the kernel-value wave beside the lead group that have started (the
  // persistent lead group's workers launch only once they all hold their SMs)
  DevBuf<unsigned long long> d_kres(fk_tc && lead ? 1 : 0, st);
  int kres_wait = 0;
  const KrowKernel kk{ktype, (float)gamma, (float)kcoef0, 0.f, kdegree, nullptr};
  const KrowKernel* kkp = ktype != 0 ? &kk : nullptr;
  if (fk_tc && !lead) {
    launch_krow_tc(Xhi.get(), Xlo.get(), n_pad, d_pad, d_tiles, (int)n_tiles, norms.get(), n, gamma, ksc, K.get(), ldk, st,
                   two_cta, kkp, 0, nullptr, kmc, (int)d);
  } else if (fk_tc) {  // the waves on the low-priority stream: the solver's CTAs are dispatched first
    GM_CUDA(cudaMemsetAsync(d_kres.get(), 0, sizeof(unsigned long long), st));
    cudaEvent_t ev_staged = evk.get();
    GM_CUDA(cudaEventRecord(ev_staged, st));
    GM_CUDA(cudaStreamWaitEvent(kst, ev_staged, 0));
    GM_CUDA(cudaEventRecord(ev_k0, kst));
    for (int g = 0; g < ng; ++g) {
      const size_t cnt = wave_off[g + 1] - wave_off[g];
      if (cnt && g == 1) kres_wait = krow_tc_grid((int)cnt, reserve_env, kmc);  // the wave beside the lead group
      if (cnt)
        launch_krow_tc(Xhi.get(), Xlo.get(), n_pad, d_pad, d_tiles + wave_off[g], (int)cnt, norms.get(), n, gamma, ksc,
                       K.get(), ldk, kst, false, kkp, g == 0 ? 0 : reserve_env, g == 1 ? d_kres.get() : nullptr, kmc,
                       (int)d);
      ev_wave[g] = evk.get(lead_dbg_t);
      GM_CUDA(cudaEventRecord(ev_wave[g], kst));
    }
    GM_CUDA(cudaEventRecord(ev_k1, kst));
  } else if (full_k && csr) {  // NEXT-3: sparse x dense from the class-sorted CSR rows
    launch_krow_csr(c_ptr.get(), c_idx.get(), c_val.get(), norms.get(), n, d, gamma, K.get(), ldk, st);
  } else if (full_k && !use_tc) {
    launch_krow_full_sym(XT.get(), n_pad, norms.get(), n, d_pad, gamma, K.get(), ldk, st);
  }
  tm.mark(PH_KERNEL);
  HT("krow_launched");

  // ---------------- a4-a6 batched working-set solver, all pairs concurrently
  const int Bw = B;
  // The solver's state lives in one arena.  In the default regime (FULL_K, every pair on the
  // wsolve.cu kernels, no diagnostics) the arena and the instantiated solver graphs are kept per
  // device and reused by the next call of the same shape: same buffers, same kernel arguments,
  // so the graphs are relaunched as they are -- no per-call capture / instantiation (~4.7 ms of
  // host time) and no graph destruction, which blocks the host until the device is idle and then
  // takes another ~3.4 ms (measured, GMPSVM_HOST_TIMING / GMPSVM_LEAD_DEBUG).  The per-call state
  // is re-initialised by launch_init_pairs as before; the kernels never read state they have not
  // written in this call (the same holds for fresh pool memory).
  ArenaPtr<PairDesc> d_pairs;
  ArenaPtr<double> d_alpha, d_f, d_v, d_dcoef, d_gap, d_b, d_A, d_B;
  ArenaPtr<uint32_t> d_stamp;
  ArenaPtr<uint8_t> d_ulf;
  ArenaPtr<int32_t> d_ws, d_wsn, d_wst, d_status, d_outer, d_sig;
  ArenaPtr<int64_t> d_inner, d_cyc, d_body;
  ArenaPtr<float> d_Kws;
  ArenaLayout lay;
  lay.add(d_pairs, Pl);
  lay.add(d_alpha, tot);
  lay.add(d_f, tot);
  lay.add(d_v, tot);
  lay.add(d_dcoef, (size_t)Pl * Bw);
  lay.add(d_gap, Pl);
  lay.add(d_b, Pl);
  lay.add(d_A, Pl);
  lay.add(d_B, Pl);
  lay.add(d_stamp, tot);
  lay.add(d_ulf, tot);
  lay.add(d_ws, (size_t)Pl * Bw);
  lay.add(d_wsn, Pl);
  lay.add(d_wst, (size_t)Pl * Bw);
  lay.add(d_status, Pl);
  lay.add(d_outer, Pl);
  lay.add(d_sig, Pl);
  lay.add(d_inner, Pl);
  lay.add(d_cyc, Pl);
  lay.add(d_body, Pl);
  lay.add(d_Kws, (size_t)Pl * kws_pair_stride(Bw));
  DevBuf<uint8_t> arena_own(lease.ws ? 0 : lay.bytes, st);
  lay.place(lease.ws ? lease.arena(lay.bytes) : arena_own.get());
  GM_CUDA(cudaMemcpyAsync(d_pairs.get(), hp.data(), Pl * sizeof(PairDesc), cudaMemcpyHostToDevice, st));
  const bool rc = !full_k;
  const bool rc_tc = rc && use_tc;  // ROW_CACHE rows on tcgen05
  DevBuf<float> d_Ahi(rc_tc ? krow_tc_buf_floats((int64_t)Pl * ldat, d_pad) : 0, st),
      d_Alo(rc_tc ? krow_tc_buf_floats((int64_t)Pl * ldat, d_pad) : 0, st);
  DevBuf<int32_t> d_slot(rc ? (size_t)Pl * Bw : 0, st), d_slot_tmp(rc ? (size_t)Pl * Bw : 0, st), d_keep(rc ? Pl : 0, st);
  DevBuf<float> d_ATnew(rc && !rc_tc ? (size_t)Pl * d_pad * ldat : 0, st);
  DevBuf<int64_t> d_rows(rc ? Pl : 0, st);
  if (rc) GM_CUDA(cudaMemsetAsync(d_rows.get(), 0, Pl * 8, st));
  SolverArgs a{};
  std::memset(&a, 0, sizeof a);  // padding included: the bytes are the cached graphs' signature
  a.pairs = d_pairs.get();
  a.K = full_k ? K.get() : nullptr;
  a.ldk = ldk;
  a.R = rc ? K.get() : nullptr;
  a.ws_slot = d_slot.get();
  a.ws_slot_tmp = d_slot_tmp.get();
  a.ws_keep = d_keep.get();
  a.rows_done = d_rows.get();
  a.XT = rc ? XT.get() : nullptr;  // ROW_CACHE operands only (FULL_K: no per-call pointers in the graph)
  a.ldx = n_pad;
  a.norms = rc ? norms.get() : nullptr;
  a.ATnew = d_ATnew.get();
  a.d_pad = d_pad;
  a.ldat = ldat;
  if (rc_tc) {
    a.Xhi = Xhi.get();
    a.Xlo = Xlo.get();
    a.Ahi = d_Ahi.get();
    a.Alo = d_Alo.get();
    a.dpt = d_pad;
    a.n_pad = n_pad;
    a.kscale = (float)(-gamma * 1.4426950408889634 / ((double)ksc * (double)ksc));
  }
  a.gamma = gamma;
  a.alpha = d_alpha.get();
  a.f = d_f.get();
  a.v = d_v.get();
  a.stamp = d_stamp.get();
  a.ws = d_ws.get();
  a.ws_n = d_wsn.get();
  a.ws_tmp = d_wst.get();
  a.Kws = d_Kws.get();
  a.dcoef = d_dcoef.get();
  a.status = d_status.get();
  a.gap = d_gap.get();
  a.inner_iters = d_inner.get();
  a.smo_cycles = d_cyc.get();
  DevBuf<int64_t> d_phase(smo_prof ? (size_t)Pl * 5 : 0, st);
  if (smo_prof) GM_CUDA(cudaMemsetAsync(d_phase.get(), 0, (size_t)Pl * 5 * 8, st));
  a.smo_phase = smo_prof ? d_phase.get() : nullptr;
  DevBuf<int64_t> d_sphase(smo_prof ? (size_t)(Pl + 8192) * 5 : 0, st);
  if (smo_prof) GM_CUDA(cudaMemsetAsync(d_sphase.get(), 0, (size_t)(Pl + 8192) * 5 * 8, st));
  a.sel_phase = smo_prof ? d_sphase.get() : nullptr;
  const int trace_cap = 1 << 16;
  DevBuf<int64_t> d_trace(trace_pos >= 0 ? (size_t)trace_cap * 3 + 2 * (size_t)Pl : 0, st);
  if (trace_pos >= 0) GM_CUDA(cudaMemsetAsync(d_trace.get(), 0, ((size_t)trace_cap * 3 + 2 * (size_t)Pl) * 8, st));
  DevBuf<int32_t> d_trace_n(trace_pos >= 0 ? 4 : 0, st);
  if (trace_pos >= 0) GM_CUDA(cudaMemsetAsync(d_trace_n.get(), 0, 16, st));
  GM_CUDA(cudaMemsetAsync(d_body.get(), 0, Pl * 8, st));
  a.body_iters = d_body.get();
  a.trace = d_trace.get();
  a.trace_n = d_trace_n.get();
  a.trace_pair = trace_pos;
  a.trace_cap = trace_cap;
  static const int fu_chunks = getenv("GMPSVM_FU_CHUNKS") ? std::max(1, atoi(getenv("GMPSVM_FU_CHUNKS"))) : 1;
  a.fu_chunks = fu_chunks;
  static const bool ulf_off = getenv("GMPSVM_ULF") && std::string(getenv("GMPSVM_ULF")) == "0";
  a.ulf = ulf_off ? nullptr : d_ulf.get();  // selection reads membership bits instead of alpha
  static const bool smo_f64_env = getenv("GMPSVM_SMO_F32") && std::string(getenv("GMPSVM_SMO_F32")) == "0";
  a.smo_f32 = (!smo_f64_env && ktype == 0) ? 1 : 0;  // the Gaussian kernel's QP is convex: FP32 local f
  a.outer_iters = d_outer.get();
  a.b = d_b.get();
  a.A = d_A.get();
  a.Bs = d_B.get();
  a.sig_status = d_sig.get();
  a.B = Bw;
  a.q = q;
  // local SMO steps per outer iteration (R20): B / 2 on the shared-memory solver (measured,
  // MNIST-shaped: cap 64 / 80 / 96 / 112 / none: 31.5 / 30.2 / 29.8 / 29.8 / 30.1-30.3 ms -- the
  // long first local solves of the hardest pairs stop early and the next outer iteration, with the
  // exact f, continues), else 100 B.  The Gaussian kernel only: the dot-product kernels' duals need
  // not have a unique alpha (linear: rank <= d), so their path decides the alpha reached
  a.inner_cap = opt.inner_iter_cap > 0 ? opt.inner_iter_cap
                                       : (ktype == 0 && Bw <= ws_smo_max_b() ? std::max(16, Bw / 2) : 100 * Bw);
  a.C = C;
  a.eps = eps;
  static const double env_ratio = getenv("GMPSVM_LOCAL_RATIO") ? atof(getenv("GMPSVM_LOCAL_RATIO")) : 0.1;
  a.local_ratio = env_ratio;
  HT("solver_alloc");
  launch_init_pairs(a, Pl, tot, st);
  const int64_t max_outer = opt.max_outer_iter > 0 ? opt.max_outer_iter : 1000000;
  const std::vector<cudaStream_t>& pool = stream_pool(opt.device);
  EventPool evp;
  cudaEvent_t ev_ready = evp.get();
  GM_CUDA(cudaEventRecord(ev_ready, st));
  tm.mark(PH_SOLVER);
  HT("init");
  int64_t rc_launches = 0;  // ROW_CACHE row-contraction launches
  DevBuf<int4> d_rtiles;  // ROW_CACHE tcgen05 row tiles of every branch (outlives the graph run)
  int64_t body_launches = 0;
  std::vector<int64_t> body_per_pair(Pl, 0);  // kernels per loop-body run of the pair's branch
  int n_branches = 0, final_selects = 0;
  bool fin_in_graph = false;  // finalize + sigmoid fit captured at the end of each graph branch
  // Persistent solver (default where it applies: FULL_K, every pair on the wsolve.cu kernels, at
  // most two pair groups): one launch per group -- its pairs' leaders plus workers on the SMs the
  // group may use (lead mode: the lead group on the `reserve` SMs beside the kernel-value waves,
  // the rest on the others) -- instead of the graphs of per-step kernels below.
  int n_sm = 0;
  GM_CUDA(cudaDeviceGetAttribute(&n_sm, cudaDevAttrMultiProcessorCount, opt.device));
  bool persist = !rc && ng <= 2 && !smo_prof && ws_persist_supported(Bw, np_max);
  // GMPSVM_PERSIST=lead: only the lead group persistent (its handoffs are flag round trips, its
  // workers on its reserved SMs); the other groups run the graphs below
  static const bool persist_lead_env = getenv("GMPSVM_PERSIST") && std::string(getenv("GMPSVM_PERSIST")) == "lead";
  bool plead = persist && persist_lead_env && lead && ng >= 2;
  if (plead) persist = false;
  int npg = plead ? 1 : (persist ? ng : 0);  // groups on the persistent solver: [0, npg)
  std::vector<int> pgrid(ng, 0);
  std::vector<size_t> pq_off(ng + 1, 0);
  if (npg > 0) {
    const int wps = ws_persist_workers_per_sm();
    for (int g = 0; g < npg; ++g) {
      const int pg = gpos[g + 1] - gpos[g];
      // the group's SMs: lead mode -- the lead group beside the last kernel-value wave on the
      // `reserve` SMs, the rest on the others; workers fill the SMs around the leaders
      const int sms = !lead ? n_sm : (g == 0 ? std::max(2, std::min(reserve_env, n_sm / 2)) : n_sm - std::max(2, std::min(reserve_env, n_sm / 2)));
      pgrid[g] = std::max(0, sms - pg) * wps + pg;  // workers
      if (pg >= sms || wps < 1) persist = plead = false;
      pq_off[g + 1] = pq_off[g] + ws_persist_ring_bytes() + ws_persist_ctr_words(pg) * 8;
    }
    if (!persist && !plead) npg = 0;
  }
  const bool pq_on = persist || plead;
  DevBuf<uint8_t> d_pq(pq_on ? pq_off[npg] : 0, st);
  if (pq_on) GM_CUDA(cudaMemsetAsync(d_pq.get(), 0, pq_off[npg], st));
  auto pq_ctr = [&](int g) {
    return reinterpret_cast<unsigned long long*>(d_pq.get() + pq_off[g] + ws_persist_ring_bytes());
  };
  // GMPSVM_NOGRAPH=1 (profiling only: ncu does not see the kernels of the conditional graphs): the
  // same per-iteration kernels launched from the host on `st`, all pairs per launch, the host
  // polling the pairs' status every 8 iterations -- the same arithmetic, far slower
  static const bool nograph = getenv("GMPSVM_NOGRAPH") && std::string(getenv("GMPSVM_NOGRAPH")) == "1";
  if (nograph && !persist && !rc && ws_solve_supported(Bw, np_max)) {
    std::vector<int32_t> hst(Pl);
    for (int g = 0; lead && g < ng; ++g) GM_CUDA(cudaStreamWaitEvent(st, ev_wave[g], 0));
    for (int64_t it = 0;; ++it) {
      launch_ws_iteration(a, Pl, np_max, cudaGraphConditionalHandle{}, 0, max_outer, st, false);
      if (it % 8 == 7) {
        GM_CUDA(cudaMemcpyAsync(hst.data(), d_status.get(), Pl * 4, cudaMemcpyDeviceToHost, st));
        GM_CUDA(cudaStreamSynchronize(st));
        bool more = false;
        for (int i = 0; i < Pl; ++i) more = more || hst[i] == 0;
        if (!more) break;
      }
    }
    n_branches = 1;
  } else if (persist) {
    GM_CUDA(cudaEventRecord(ev_ready, st));
    for (int g = 0; g < ng; ++g) {
      cudaStream_t ls = pool[g];
      GM_CUDA(cudaStreamWaitEvent(ls, ev_ready, 0));
      if (lead) GM_CUDA(cudaStreamWaitEvent(ls, ev_wave[g], 0));
      if (lead_dbg_t) {
        ev_gst[g] = evk.get(true);
        ev_gend[g] = evk.get(true);
        GM_CUDA(cudaEventRecord(ev_gst[g], ls));
      }
      SolverArgs ag = a;
      ag.pair_base = gpos[g];
      launch_ws_persist(ag, gpos[g + 1] - gpos[g], pgrid[g], max_outer, d_pq.get() + pq_off[g], pq_ctr(g), ls,
                        lead && g == 0 ? d_kres.get() : nullptr, lead && g == 0 ? kres_wait : 0);
      cudaEvent_t ev = ev_gend[g] ? ev_gend[g] : evp.get();
      GM_CUDA(cudaEventRecord(ev, ls));
      GM_CUDA(cudaStreamWaitEvent(st, ev, 0));
    }
    n_branches = ng;
    destroy_parked_graphs();
  } else {
    // Device-driven outer loops: one CUDA graph holding, per branch (packing above), a
    // conditional WHILE node whose body is that branch's select -> [rows] -> gather -> local SMO ->
    // f-update chain (the f-update kernel sets the loop condition), followed by one last selection
    // (the stop test on the final alpha) on the split path.  The branches are independent, so no
    // pair waits for another at a kernel boundary and the host is not involved until the end.
    // ROW_CACHE rows on tcgen05: each branch's static tile list (its pairs x row tiles x column tiles)
    std::vector<int> rtile_off(nbr + 1, 0);
    std::vector<int4> rtiles;
    if (rc_tc)
      for (int br = 0; br < nbr; ++br) {
        const std::vector<int4> t = rows_tc_tiles(hp, bb[br], bb[br + 1] - bb[br], Bw);
        rtiles.insert(rtiles.end(), t.begin(), t.end());
        rtile_off[br + 1] = (int)rtiles.size();
      }
    new (&d_rtiles) DevBuf<int4>(std::max<size_t>(rtiles.size(), 1), st);
    if (!rtiles.empty())
      GM_CUDA(cudaMemcpyAsync(d_rtiles.get(), rtiles.data(), rtiles.size() * sizeof(int4), cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaEventRecord(ev_ready, st));
    cudaStream_t cs = pool.back();  // capture stream
    // iterations per conditional-body run (measured, round 2: 2 / 4 / 8 -> 30.67 / 30.28 / 30.06 ms)
    static const int unroll = getenv("GMPSVM_UNROLL") ? std::max(1, atoi(getenv("GMPSVM_UNROLL"))) : 8;
    auto build = [&](int br0, int br1, GraphGuard& g) {  // branches [br0, br1), instantiated
      const uint64_t l0 = g_launches.load();
      GM_CUDA(cudaGraphCreate(&g.graph, 0));
      for (int br = br0; br < br1; ++br) {
        const int i = bb[br], gn = bb[br + 1] - bb[br];
        int64_t npi = 0;
        for (int j = bb[br]; j < bb[br + 1]; ++j) npi = std::max<int64_t>(npi, hp[j].n_s + hp[j].n_t);
        cudaGraphConditionalHandle h;
        GM_CUDA(cudaGraphConditionalHandleCreate(&h, g.graph, 1, cudaGraphCondAssignDefault));
        cudaGraphNodeParams cp = {};
        cp.type = cudaGraphNodeTypeConditional;
        cp.conditional.handle = h;
        cp.conditional.type = cudaGraphCondTypeWhile;
        cp.conditional.size = 1;
        cudaGraphNode_t wnode;
        GM_CUDA(cudaGraphAddNode(&wnode, g.graph, nullptr, 0, &cp));
        SolverArgs ag = a;
        ag.pair_base = i;
        const bool wsp = !rc && ws_solve_supported(Bw, npi);
        const uint64_t b0 = g_launches.load();
        cudaGraph_t cap;
        GM_CUDA(cudaStreamBeginCaptureToGraph(cs, cp.conditional.phGraph_out[0], nullptr, nullptr, 0,
                                              cudaStreamCaptureModeRelaxed));
        if (wsp) {  // default kernels (wsolve.cu): selection -> gather -> local SMO -> f-update, unrolled:
                    // the conditional node's re-launch (~10 us) is paid every `unroll` iterations
          for (int u = 0; u < unroll; ++u) launch_ws_iteration(ag, gn, npi, h, u == unroll - 1, max_outer, cs, u > 0);
        } else {
          launch_select_ws(ag, gn, 0, -1, cs);
          if (rc_tc)
            launch_rows_compute_tc(ag, gn, d_rtiles.get() + rtile_off[br], rtile_off[br + 1] - rtile_off[br], Pl, cs);
          else if (rc)
            launch_rows_compute(ag, gn, npi, cs);
          launch_gather_kws(ag, gn, -1, cs);
          launch_local_smo(ag, gn, cs);
          launch_f_update_loop(ag, gn, npi, h, max_outer, cs);
        }
        GM_CUDA(cudaStreamEndCapture(cs, &cap));
        body_launches = (int64_t)(g_launches.load() - b0);
        body_per_pair[i] = body_launches;
        // after the loop, in the branch: the stop test on the final alpha (split path; the default
        // path tests in every f-update), then the branch's bias / in-sample values (a7) and sigmoid
        // fits (a8) -- they overlap the pairs still iterating instead of following the last one
        GM_CUDA(cudaStreamBeginCaptureToGraph(cs, g.graph, &wnode, nullptr, 1, cudaStreamCaptureModeRelaxed));
        if (!wsp) {
          launch_select_ws(ag, gn, 0, -1, cs);
          ++final_selects;
        }
        launch_finalize(ag, gn, cs);
        launch_sigmoid_fit(ag, gn, cs);
        final_selects += 2;  // counted with the final selections: one run per graph launch
        GM_CUDA(cudaStreamEndCapture(cs, &cap));
      }
      g_launches.fetch_sub(g_launches.load() - l0);  // captured, not executed: counted after the run
      GM_CUDA(cudaGraphInstantiate(&g.exec, g.graph, 0));
    };
    auto launch_after = [&](cudaGraphExec_t ex, cudaStream_t ls, cudaEvent_t extra, cudaEvent_t done, cudaEvent_t start) {
      GM_CUDA(cudaStreamWaitEvent(ls, ev_ready, 0));
      if (extra) GM_CUDA(cudaStreamWaitEvent(ls, extra, 0));
      if (start) GM_CUDA(cudaEventRecord(start, ls));
      GM_CUDA(cudaGraphLaunch(ex, ls));
      cudaEvent_t ev = done ? done : evp.get();
      GM_CUDA(cudaEventRecord(ev, ls));
      GM_CUDA(cudaStreamWaitEvent(st, ev, 0));
    };
    // the cached graphs fit this call if they were captured with the same kernel arguments,
    // branch packing and per-branch launch shapes
    std::vector<uint8_t> sig;
    SolverWs* ws = lease.ws;
    if (ws) {
      auto put = [&](const void* p, size_t nb) {
        sig.insert(sig.end(), static_cast<const uint8_t*>(p), static_cast<const uint8_t*>(p) + nb);
      };
      put(&a, sizeof a);
      put(bb.data(), bb.size() * sizeof(int));
      put(gbr.data(), gbr.size() * sizeof(int));
      put(&max_outer, sizeof max_outer);
      put(&unroll, sizeof unroll);
      for (int br = 0; br < nbr; ++br) {
        int64_t npi = 0;
        for (int j = bb[br]; j < bb[br + 1]; ++j) npi = std::max<int64_t>(npi, hp[j].n_s + hp[j].n_t);
        put(&npi, sizeof npi);
      }
    }
    const bool reuse = ws && (int)ws->exec.size() == ng && ws->sig == sig;
    std::vector<GraphGuard> gg(ng);  // this call's graphs (uncached, or to be kept)
    std::vector<cudaGraphExec_t> ex(ng, nullptr);
    if (reuse) {
      ex = ws->exec;
      body_per_pair = ws->body_per_pair;
      final_selects = ws->final_selects;
    }
    // group g's graph on pool[g]; lead mode: after its wave (the lead graph is small and built in
    // well under wave 0's time; the others are built while their waves run)
    for (int g = 0; g < ng; ++g) {
      if (!reuse) {
        build(gbr[g], gbr[g + 1], gg[g]);
        ex[g] = gg[g].exec;
      }
      if (lead_dbg_t) {
        ev_gst[g] = evk.get(true);
        ev_gend[g] = evk.get(true);
      }
      if (plead && g == 0) {  // the lead group's graph stays unlaunched (cached with the others)
        cudaStream_t ls = pool[0];
        GM_CUDA(cudaStreamWaitEvent(ls, ev_ready, 0));
        GM_CUDA(cudaStreamWaitEvent(ls, ev_wave[0], 0));
        if (ev_gst[0]) GM_CUDA(cudaEventRecord(ev_gst[0], ls));
        SolverArgs ag = a;
        ag.pair_base = gpos[0];
        const int pg = gpos[1] - gpos[0];
        launch_ws_persist(ag, pg, pgrid[0], max_outer, d_pq.get(), pq_ctr(0), ls, d_kres.get(), kres_wait);
        launch_finalize(ag, pg, ls);
        launch_sigmoid_fit(ag, pg, ls);
        cudaEvent_t ev = ev_gend[0] ? ev_gend[0] : evp.get();
        GM_CUDA(cudaEventRecord(ev, ls));
        GM_CUDA(cudaStreamWaitEvent(st, ev, 0));
        continue;
      }
      launch_after(ex[g], pool[g], lead ? ev_wave[g] : nullptr, ev_gend[g], ev_gst[g]);
    }
    if (ws && !reuse) {  // the freshly built graphs become the device's cached ones
      ws->park_graphs();
      for (int g = 0; g < ng; ++g) {
        ws->graph.push_back(gg[g].graph);
        ws->exec.push_back(gg[g].exec);
        gg[g].graph = nullptr;
        gg[g].exec = nullptr;
      }
      ws->sig = sig;
      ws->body_per_pair = body_per_pair;
      ws->final_selects = final_selects;
    }
    HT("graph_build");
    n_branches = nbr;
    fin_in_graph = true;
    // graphs no call will launch again (uncached calls, replaced cached ones): destroying one
    // blocks the host until the device is idle, so it is done here, behind the running solver
    destroy_parked_graphs();
    HT("destroy");
  }
  if (lead_dbg) GM_CUDA(cudaEventRecord(dbg0.b, st));
  tm.mark(PH_SOLVER);
  HT("solver_loop");
  bool cap_hit = false;

  // ---------------- a7-a9 bias, decision values, sigmoid, SV union
  tm.mark(PH_FIN);
  HT("fin0");
  if (host_timing) {  // synchronised checkpoints: the solver's end, then each finalize step
    GM_CUDA(cudaStreamSynchronize(st));
    HT("solver_wait");
  }
  if (!fin_in_graph) {  // the graph path ran them per branch
    launch_finalize(a, Pl, st);
    launch_sigmoid_fit(a, Pl, st);
  }
  DevBuf<uint8_t> d_flags(n, st);
  GM_CUDA(cudaMemsetAsync(d_flags.get(), 0, n, st));
  launch_sv_flags(a, Pl, np_max, d_flags.get(), st);
  if (host_timing) {
    GM_CUDA(cudaStreamSynchronize(st));
    HT("fin_kernels");
  }
  std::vector<double> hb(Pl), hA(Pl), hB(Pl);
  std::vector<int32_t> h_sig(Pl), h_st(Pl), h_outer(Pl);
  std::vector<int64_t> h_inner(Pl), h_cyc(Pl), h_body(Pl);
  // every read-back lands in pinned memory (async DMA, one synchronisation; a copy into pageable
  // memory would wait for the stream each time): the permutation, the SV flags and the per-pair
  // results; alpha stays on the device (the model's host copy is materialised on demand,
  // ensure_host_alpha)
  const size_t o_flags = (size_t)n * 8, o_small = round_up((int64_t)(o_flags + (size_t)n), 8);
  uint8_t* pin = pinned_scratch<uint8_t>(o_small + (size_t)Pl * (6 * 8 + 3 * 4) + 64, 1);
  int64_t* h_permp = reinterpret_cast<int64_t*>(pin);
  uint8_t* h_flags = pin + o_flags;
  uint8_t* sp = pin + o_small;
  struct Rb {
    void* host;
    const void* dev;
    size_t bytes;
  };
  const Rb rb[] = {{hb.data(), d_b.get(), (size_t)Pl * 8},         {hA.data(), d_A.get(), (size_t)Pl * 8},
                   {hB.data(), d_B.get(), (size_t)Pl * 8},         {h_inner.data(), d_inner.get(), (size_t)Pl * 8},
                   {h_cyc.data(), d_cyc.get(), (size_t)Pl * 8},    {h_body.data(), d_body.get(), (size_t)Pl * 8},
                   {h_sig.data(), d_sig.get(), (size_t)Pl * 4},    {h_st.data(), d_status.get(), (size_t)Pl * 4},
                   {h_outer.data(), d_outer.get(), (size_t)Pl * 4}};
  {
    size_t o = 0;
    for (const Rb& r : rb) {
      GM_CUDA(cudaMemcpyAsync(sp + o, r.dev, r.bytes, cudaMemcpyDeviceToHost, st));
      o += r.bytes;
    }
  }
  GM_CUDA(cudaMemcpyAsync(h_permp, d_perm.get(), n * 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaMemcpyAsync(h_flags, d_flags.get(), n, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaStreamSynchronize(st));
  {
    size_t o = 0;
    for (const Rb& r : rb) {
      std::memcpy(r.host, sp + o, r.bytes);
      o += r.bytes;
    }
  }
  HT("fin_d2h");
  for (int g = 0; g < npg; ++g) {
    unsigned long long perr = 0;
    GM_CUDA(cudaMemcpy(&perr, pq_ctr(g) + 3, 8, cudaMemcpyDeviceToHost));
    if (perr) throw Error(GMPSVM_ECUDA, "persistent solver: a wait timed out (group " + std::to_string(g) + ")");
  }
  {  // kernels the graph executed: every body run launches body_launches kernels, + final selects
    int64_t ex = final_selects;  // one final selection per split-path branch
    if (plead) {  // the lead group ran persistent: its launches were counted at launch
      ex -= 2 * (gbr[1] - gbr[0]);
      for (int i = gpos[0]; i < gpos[1]; ++i) body_per_pair[i] = 0;
    }
    for (int i = 0; i < Pl; ++i) ex += h_body[i] * body_per_pair[i];  // counted at each branch's first pair
    g_launches.fetch_add((uint64_t)ex);
    if (rc) {
      rc_launches = 0;
      for (int i = 0; i < Pl; ++i) rc_launches += h_body[i];
    }
  }

  if (trace_pos >= 0 && trace_pos < Pl) {
    int32_t nt = 0;
    GM_CUDA(cudaMemcpy(&nt, d_trace_n.get(), 4, cudaMemcpyDeviceToHost));
    nt = std::min(nt, trace_cap);
    std::vector<int64_t> tr((size_t)nt * 3);
    GM_CUDA(cudaMemcpy(tr.data(), d_trace.get(), tr.size() * 8, cudaMemcpyDeviceToHost));
    std::vector<int> order(nt);
    for (int i = 0; i < nt; ++i) order[i] = i;
    std::sort(order.begin(), order.end(), [&](int x, int y) { return tr[3 * x + 1] < tr[3 * y + 1]; });
    const char* names[11] = {"select", "gather", "smo", "fupdate", "rows_gather", "rows_contract", "ws_solve",
                             "fu_end_to_select", "select_resident_wait", "gather_task", "fupdate_task"};
    double dur[11] = {0}, cnt[11] = {0}, gap_before[11] = {0};
    int prev = -1;
    for (int j = 0; j < nt; ++j) {
      const int i = order[j];
      const int kd = (int)tr[3 * i];
      dur[kd] += (double)(tr[3 * i + 2] - tr[3 * i + 1]);
      cnt[kd] += 1;
      if (kd >= 7) continue;  // handoff records: not part of the kernel chain
      if (prev >= 0) gap_before[kd] += (double)(tr[3 * i + 1] - tr[3 * prev + 2]);
      prev = i;
    }
    int64_t s_lo = INT64_MAX, s_hi = 0;  // span of the kernel chain (kinds 0-6)
    for (int i = 0; i < nt; ++i)
      if (tr[3 * i] < 7) {
        s_lo = std::min(s_lo, tr[3 * i + 1]);
        s_hi = std::max(s_hi, tr[3 * i + 2]);
      }
    const double span = s_hi > 0 ? (double)(s_hi - s_lo) : 0.0;
    std::string line;
    for (int kd = 0; kd < 11; ++kd)
      if (cnt[kd] > 0)
        line += std::string(" ") + names[kd] + " n=" + std::to_string((int)cnt[kd]) +
                " mean_us=" + std::to_string(dur[kd] / cnt[kd] / 1e3).substr(0, 6) +
                " gap_before_us=" + std::to_string(gap_before[kd] / cnt[kd] / 1e3).substr(0, 6) + ";";
    std::vector<int64_t> win((size_t)2 * Pl);
    GM_CUDA(cudaMemcpy(win.data(), d_trace.get() + (size_t)trace_cap * 3, win.size() * 8, cudaMemcpyDeviceToHost));
    int64_t t_min = INT64_MAX;
    for (int i = 0; i < Pl; ++i)
      if (win[2 * i]) t_min = std::min(t_min, win[2 * i]);
    std::string wl;
    for (int i = 0; i < Pl; ++i)
      wl += " " + std::to_string(i) + ":" + std::to_string((win[2 * i] - t_min) / 100000 / 10.0).substr(0, 4) + "-" +
            std::to_string((win[2 * i + 1] - t_min) / 100000 / 10.0).substr(0, 4);
    fprintf(stderr, "[gmpsvm trace] pair windows (ms from first start):%s\n", wl.c_str());
    fprintf(stderr, "[gmpsvm trace] pair (%d,%d) outer %d span %.2f ms:%s\n", hp[trace_pos].s, hp[trace_pos].t,
            h_outer[trace_pos], span / 1e6, line.c_str());
  }
  if (smo_prof) {
    std::vector<int64_t> ph((size_t)Pl * 5);
    GM_CUDA(cudaMemcpy(ph.data(), d_phase.get(), ph.size() * 8, cudaMemcpyDeviceToHost));
    double tot[5] = {0, 0, 0, 0, 0};
    for (int i = 0; i < Pl; ++i)
      for (int q = 0; q < 5; ++q) tot[q] += (double)ph[i * 5 + q];
    int64_t steps = 0, outer = 0;
    for (int i = 0; i < Pl; ++i) {
      steps += h_inner[i];
      outer += h_outer[i];
    }
    fprintf(stderr,
            "[gmpsvm] local_smo cycles/step: u-reduce %.0f  row-u %.0f  l-reduce %.0f  step+row-l %.0f | "
            "prologue cycles/launch %.0f\n",
            tot[0] / steps, tot[1] / steps, tot[2] / steps, tot[3] / steps, tot[4] / outer);
    GM_CUDA(cudaMemcpy(ph.data(), d_sphase.get(), ph.size() * 8, cudaMemcpyDeviceToHost));
    double sp[5] = {0, 0, 0, 0, 0};
    for (int i = 0; i < Pl; ++i)
      for (int q = 0; q < 5; ++q) sp[q] += (double)ph[i * 5 + q];
    fprintf(stderr, "[gmpsvm] select_ws cycles/launch: staging %.0f  reduce %.0f  retain %.0f  pick %.0f  copy %.0f\n",
            sp[0] / outer, sp[1] / outer, sp[2] / outer, sp[3] / outer, sp[4] / outer);
    std::vector<int64_t> fq((size_t)Pl * 5);
    GM_CUDA(cudaMemcpy(fq.data(), d_sphase.get() + (size_t)4096 * 5, fq.size() * 8, cudaMemcpyDeviceToHost));
    double fs[5] = {0, 0, 0, 0, 0};
    for (int i = 0; i < Pl; ++i)
      for (int q = 0; q < 5; ++q) fs[q] += (double)fq[i * 5 + q];
    fprintf(stderr, "[gmpsvm] fast select cycles/launch: staging %.0f  thresholds %.0f  compact %.0f  ranks %.0f  write-out %.0f (fallbacks x1e6)\n",
            fs[0] / outer, fs[1] / outer, fs[2] / outer, fs[3] / outer, fs[4] / outer);
    GM_CUDA(cudaMemcpy(fq.data(), d_sphase.get() + (size_t)8192 * 5, fq.size() * 8, cudaMemcpyDeviceToHost));
    double wo[5] = {0, 0, 0, 0, 0};
    for (int i = 0; i < Pl; ++i)
      for (int q = 0; q < 5; ++q) wo[q] += (double)fq[i * 5 + q];
    fprintf(stderr, "[gmpsvm] select write-out cycles/launch: bitmap %.0f  prefix %.0f  stores %.0f\n", wo[0] / outer,
            wo[1] / outer, wo[2] / outer);
    std::string per;
    for (int i = 0; i < Pl; ++i)
      per += " (" + std::to_string(hp[i].s) + "," + std::to_string(hp[i].t) + "):" + std::to_string(h_outer[i]) + "/" +
             std::to_string(h_inner[i]);
    fprintf(stderr, "[gmpsvm] per pair outer/inner:%s\n", per.c_str());
  }
  auto* mdl = new Model();
  std::unique_ptr<Model> guard(mdl);
  mdl->k = k;
  mdl->d = d;
  mdl->C = C;
  mdl->gamma = gamma;
  mdl->eps = eps;
  mdl->kernel = ktype;
  mdl->coef0 = kcoef0;
  mdl->degree = kdegree;
  mdl->n = n;
  mdl->class_count.assign(cc.begin(), cc.begin() + k);
  mdl->perm.assign(h_permp, h_permp + n);
  mdl->trained.assign(P, 0);
  mdl->b.assign(P, 0.0);
  mdl->A.assign(P, 0.0);
  mdl->B.assign(P, 0.0);
  mdl->status.assign(P, 0);
  mdl->pair_outer.assign(P, 0);
  mdl->pair_inner.assign(P, 0);
  mdl->pair_rows.assign(P, 0);
  const auto po = mdl->pair_offsets();
  mdl->alpha_ready = false;
  std::vector<int64_t> alpha_off(P, -1);  // model pair -> offset into the solver's device alpha
  int64_t outer_max = 0, outer_sum = 0, inner_sum = 0, cyc_sum = 0;
  for (int i = 0; i < Pl; ++i) {
    const int p = pids[i];
    mdl->trained[p] = 1;
    mdl->b[p] = hb[i];
    mdl->A[p] = hA[i];
    mdl->B[p] = hB[i];
    if (h_st[i] == 0 || h_st[i] == 2) {  // still active / capped in-kernel: the outer-iteration cap stopped it
      h_st[i] = 2;
      cap_hit = true;
    }
    mdl->status[p] = (h_st[i] == 1 ? 0 : h_st[i]) | (h_sig[i] << 8);
    mdl->pair_outer[p] = h_outer[i];
    mdl->pair_inner[p] = h_inner[i];
    alpha_off[p] = hp[i].a_off;
    outer_max = std::max<int64_t>(outer_max, h_outer[i]);
    outer_sum += h_outer[i];
    inner_sum += h_inner[i];
    cyc_sum += h_cyc[i];
  }
  {  // the SV positions: count, then a branchless compaction (~1/3 of the flags are set, at random)
    int64_t cnt = 0;
    for (int64_t g = 0; g < n; ++g) cnt += h_flags[g] != 0;
    mdl->sv_pos.resize((size_t)cnt + 1);
    int64_t* o = mdl->sv_pos.data();
    int64_t j = 0;
    for (int64_t g = 0; g < n; ++g) {
      o[j] = g;
      j += h_flags[g] != 0;
    }
    mdl->sv_pos.resize((size_t)cnt);
  }
  HT("asm_svpos");
  std::vector<int64_t> row_of_sv(mdl->sv_pos.size());
  for (size_t i = 0; i < row_of_sv.size(); ++i) row_of_sv[i] = mdl->perm[mdl->sv_pos[i]];
  HT("assembled");
  // the SV-row centre and scale are recomputed from the SV rows (not the training call's), so a
  // model merged from partial trainings predicts bitwise like the single-call model
  DevBuf<float> sv_dense(csr ? (size_t)std::max<size_t>(row_of_sv.size(), 1) * d : 0, st);
  if (csr) {  // the model's support-vector rows, densified (prediction contracts dense SV tiles)
    DevBuf<int64_t> d_rows(std::max<size_t>(row_of_sv.size(), 1), st);
    if (!row_of_sv.empty())
      GM_CUDA(cudaMemcpyAsync(d_rows.get(), row_of_sv.data(), row_of_sv.size() * 8, cudaMemcpyHostToDevice, st));
    launch_csr_densify_rows(csr->indptr, csr->indices, csr->values, d_rows.get(), (int64_t)row_of_sv.size(), d,
                            sv_dense.get(), st);
    for (size_t i = 0; i < row_of_sv.size(); ++i) row_of_sv[i] = (int64_t)i;
    GM_CUDA(cudaStreamSynchronize(st));  // d_rows goes out of scope
  }
  mdl->dev = build_dev_model(*mdl, csr ? sv_dense.get() : dX, row_of_sv, opt.device, st, nullptr, 0.f, d_alpha.get(),
                             tot, &alpha_off);
  tm.mark(PH_FIN);
  HT("devmodel");
  if (lead_dbg) GM_CUDA(cudaEventRecord(dbg1.a, st));
  GM_CUDA(cudaStreamSynchronize(st));
  if (lead_dbg) {
    float sv = 0.f, en = 0.f, k0 = -1.f;
    GM_CUDA(cudaEventElapsedTime(&sv, dbg0.a, dbg0.b));
    GM_CUDA(cudaEventElapsedTime(&en, dbg0.a, dbg1.a));
    if (lead) GM_CUDA(cudaEventElapsedTime(&k0, dbg0.a, ev_k0));
    fprintf(stderr, "[gmpsvm timeline ms] from the call: first wave %.3f  solver done (st) %.3f  end %.3f\n", k0, sv, en);
  }

  gmpsvm_train_stats& s = mdl->stats;
  s.t_stage_ms = tm.ms(PH_STAGE);
  if (lead) {  // span of the kernel-value waves (they share the GPU with the lead pairs' solver)
    float x = 0.f;
    GM_CUDA(cudaEventElapsedTime(&x, ev_k0, ev_k1));
    s.t_kernel_ms = x;
    if (lead_dbg) {
      std::string line;
      for (int g = 0; g < ng; ++g) {
        float w = 0.f, g0 = 0.f, g1 = 0.f;
        GM_CUDA(cudaEventElapsedTime(&w, ev_k0, ev_wave[g]));
        GM_CUDA(cudaEventElapsedTime(&g0, ev_k0, ev_gst[g]));
        GM_CUDA(cudaEventElapsedTime(&g1, ev_k0, ev_gend[g]));
        char buf[160];
        snprintf(buf, sizeof buf, "  g%d[%d pairs] wave %.3f graph %.3f-%.3f", g, gpos[g + 1] - gpos[g], w, g0, g1);
        line += buf;
      }
      fprintf(stderr, "[gmpsvm lead ms] from the first wave:%s (tiles %zu)\n", line.c_str(), n_tiles);
    }
  } else {
    s.t_kernel_ms = tm.ms(PH_KERNEL);
  }
  s.t_select_ms = tm.ms(PH_SELECT);
  s.t_subproblem_ms = tm.ms(PH_SUB);
  s.t_fupdate_ms = tm.ms(PH_FUP);
  s.t_finalize_ms = tm.ms(PH_FIN);
  s.t_solver_ms = tm.ms(PH_SOLVER);
  s.n_streams = n_branches;
  if (full_k) {
    s.kernel_values = kv_subset >= 0 ? kv_subset : (double)n * (double)(n + 1) / 2.0;
    s.krow_launches = 1;
  } else {
    std::vector<int64_t> rows(Pl);
    GM_CUDA(cudaMemcpy(rows.data(), d_rows.get(), Pl * 8, cudaMemcpyDeviceToHost));
    for (int i = 0; i < Pl; ++i) mdl->pair_rows[hp[i].pid] = rows[i];
    s.kernel_values = 0;
    for (int i = 0; i < Pl; ++i) s.kernel_values += (double)rows[i] * (double)(hp[i].n_s + hp[i].n_t);
    s.krow_launches = rc_launches;
  }
  s.kernel_flops = s.kernel_values * (2.0 * d + 3.0);
  s.outer_iters_max = outer_max;
  s.outer_iters_sum = outer_sum;
  s.inner_iters_sum = inner_sum;
  s.smo_cycles_sum = cyc_sum;
  s.n_sv = (int64_t)mdl->sv_pos.size();
  s.cache_regime = full_k ? 0 : 1;
  s.kernel_path = csr ? 2 : (use_tc ? 0 : 1);
  s.n_pairs_trained = Pl;
  s.launches = (int64_t)(g_launches.load() - launches0);
  s.t_total_ms = host_ms_since(t_start);
  if (host_timing) fprintf(stderr, "[gmpsvm host ms]%s\n", ht_line.c_str());
  *out = guard.release();
  bool warn = cap_hit;
  for (int i = 0; i < Pl; ++i) warn = warn || h_sig[i] == 1;
  return warn ? GMPSVM_WARN_MAXITER : GMPSVM_OK;
}

// ------------------------------------------------------------------------------------------
// The complete model from per-pair solutions computed elsewhere (multi-GPU: each rank trains a
// pair subset; the ranks all-reduce the disjoint alpha / b / A / B vectors and every rank
// rebuilds the model from its own replicated X -- only O(sum n_p) doubles cross NVLink instead
// of serialized SV rows).  alpha: sum_p n_p doubles, pairs in index order, pair-local order (the
// gmpsvm_model_pair layout); b, A, B: P doubles; status: P int32 or NULL.  Host pointers.
int engine_model_from_alpha(const float* X, const int32_t* y, int64_t n, int32_t d, int32_t k, double C, double gamma,
                            const double* alpha, const double* b, const double* A, const double* B,
                            const int32_t* status, const gmpsvm_options& opt, Model** out) {
  if (!X || !y || !alpha || !b || !A || !B || !out) throw Error(GMPSVM_EINVAL, "null argument");
  if (n < 2 || d < 1 || k < 2) throw Error(GMPSVM_EINVAL, "need n >= 2, d >= 1, k >= 2");
  if (k > kMaxK) throw Error(GMPSVM_ENOTIMPL, "k > 64 classes not supported by this build");
  if (!finite_pos(C) || !finite_pos(gamma)) throw Error(GMPSVM_EINVAL, "C, gamma must be finite and > 0");
  DeviceGuard dg(opt.device);
  cudaStream_t st = get_stream(opt);
  DevBuf<float> bufX(opt.inputs_on_device ? 0 : (size_t)n * d, st);
  DevBuf<int32_t> bufY(opt.inputs_on_device ? 0 : (size_t)n, st);
  const float* dX = X;
  const int32_t* dy = y;
  if (!opt.inputs_on_device) {
    GM_CUDA(cudaMemcpyAsync(bufX.get(), X, (size_t)n * d * 4, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(bufY.get(), y, (size_t)n * 4, cudaMemcpyHostToDevice, st));
    dX = bufX.get();
    dy = bufY.get();
  }
  // a1: the same stable class sort as training (class-sorted positions <-> original rows)
  const int nb = (int)ceil_div(n, 1024);
  DevBuf<int32_t> blk_counts((size_t)nb * (k + 1), st), blk_off((size_t)nb * k, st);
  DevBuf<int64_t> d_count(k + 1, st), d_off(k + 1, st), d_perm(n, st);
  launch_class_sort(dy, n, k, blk_counts.get(), blk_off.get(), d_count.get(), d_off.get(), st);
  std::vector<int64_t> cc(k + 1);
  GM_CUDA(cudaMemcpyAsync(cc.data(), d_count.get(), (k + 1) * 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaStreamSynchronize(st));
  if (cc[k] != 0) throw Error(GMPSVM_EINVAL, "labels must be in [0, k)");
  for (int c = 0; c < k; ++c)
    if (cc[c] == 0) throw Error(GMPSVM_EINVAL, "every class must have at least one instance");
  launch_class_rank(dy, n, k, blk_off.get(), d_off.get(), d_perm.get(), st);
  auto* mdl = new Model();
  std::unique_ptr<Model> guard(mdl);
  mdl->k = k;
  mdl->d = d;
  mdl->C = C;
  mdl->gamma = gamma;
  mdl->kernel = opt.kernel;
  mdl->coef0 = opt.coef0;
  mdl->degree = opt.degree ? opt.degree : 3;
  if (mdl->kernel < 0 || mdl->kernel > 3 || mdl->degree < 1 || mdl->degree > 16 || !std::isfinite(mdl->coef0))
    throw Error(GMPSVM_EINVAL, "kernel must be 0..3, degree 1..16, coef0 finite");
  mdl->n = n;
  mdl->class_count.assign(cc.begin(), cc.begin() + k);
  mdl->perm.resize(n);
  GM_CUDA(cudaMemcpyAsync(mdl->perm.data(), d_perm.get(), (size_t)n * 8, cudaMemcpyDeviceToHost, st));
  const int P = k * (k - 1) / 2;
  const auto po = mdl->pair_offsets();
  mdl->trained.assign(P, 1);
  mdl->b.assign(b, b + P);
  mdl->A.assign(A, A + P);
  mdl->B.assign(B, B + P);
  mdl->status.assign(P, 0);
  mdl->pair_outer.assign(P, 0);
  mdl->pair_inner.assign(P, 0);
  mdl->pair_rows.assign(P, 0);
  if (status) mdl->status.assign(status, status + P);
  mdl->alpha.assign(alpha, alpha + po[P]);
  for (int64_t j = 0; j < po[P]; ++j)
    if (!(alpha[j] >= 0.0 && alpha[j] <= C)) throw Error(GMPSVM_EINVAL, "alpha outside [0, C]");
  // a9: the SV union over the pairs, ascending class-sorted position (Alg 2 l.16, L363)
  std::vector<int64_t> off(k + 1, 0);
  for (int c = 0; c < k; ++c) off[c + 1] = off[c] + cc[c];
  std::vector<uint8_t> is_sv(n, 0);
  for (int p = 0; p < P; ++p) {
    const int s = ps_of(p, k), t = pt_of(p, k);
    for (int64_t j = 0; j < cc[s] + cc[t]; ++j)
      if (alpha[po[p] + j] > 0.0) is_sv[j < cc[s] ? off[s] + j : off[t] + (j - cc[s])] = 1;
  }
  GM_CUDA(cudaStreamSynchronize(st));  // perm on the host
  for (int64_t g = 0; g < n; ++g)
    if (is_sv[g]) mdl->sv_pos.push_back(g);
  std::vector<int64_t> row_of_sv(mdl->sv_pos.size());
  for (size_t i = 0; i < row_of_sv.size(); ++i) row_of_sv[i] = mdl->perm[mdl->sv_pos[i]];
  mdl->stats = gmpsvm_train_stats{};
  mdl->stats.n_sv = (int64_t)mdl->sv_pos.size();
  mdl->stats.n_pairs_trained = P;
  mdl->dev = build_dev_model(*mdl, dX, row_of_sv, opt.device, st);
  *out = guard.release();
  return GMPSVM_OK;
}

// ------------------------------------------------------------------------------------------
// CSR input (NEXT-3, the format of the paper's datasets): densified on the device, then the dense
// path (the kernel-value contraction runs on the dense rows).  indptr [n+1] int64, indices [nnz]
// int32, values [nnz] float; host or device pointers per opt.inputs_on_device.
struct CsrDev {  // the CSR arrays on the device (uploaded, or the caller's device pointers)
  DevBuf<int64_t> ip;
  DevBuf<int32_t> ix;
  DevBuf<float> vv;
  CsrSrc src{};
  CsrDev(const int64_t* indptr, const int32_t* indices, const float* values, int64_t n, int32_t d,
         const gmpsvm_options& opt, cudaStream_t st) {
    if (n < 0 || d < 1 || !indptr) throw Error(GMPSVM_EINVAL, "bad CSR arguments");
    int64_t nnz = 0;
    if (opt.inputs_on_device) GM_CUDA(cudaMemcpy(&nnz, indptr + n, 8, cudaMemcpyDeviceToHost));
    else nnz = indptr[n];
    if (nnz < 0 || (nnz > 0 && (!indices || !values))) throw Error(GMPSVM_EINVAL, "bad CSR arguments");
    src = CsrSrc{indptr, indices, values, nnz};
    if (!opt.inputs_on_device) {
      new (&ip) DevBuf<int64_t>((size_t)n + 1, st);
      new (&ix) DevBuf<int32_t>((size_t)std::max<int64_t>(nnz, 1), st);
      new (&vv) DevBuf<float>((size_t)std::max<int64_t>(nnz, 1), st);
      GM_CUDA(cudaMemcpyAsync(ip.get(), indptr, ((size_t)n + 1) * 8, cudaMemcpyHostToDevice, st));
      if (nnz) {
        GM_CUDA(cudaMemcpyAsync(ix.get(), indices, (size_t)nnz * 4, cudaMemcpyHostToDevice, st));
        GM_CUDA(cudaMemcpyAsync(vv.get(), values, (size_t)nnz * 4, cudaMemcpyHostToDevice, st));
      }
      src = CsrSrc{ip.get(), ix.get(), vv.get(), nnz};
    }
  }
};

struct CsrDense {  // densified on the device (the dense path's input)
  DevBuf<float> X;
  CsrDense(const CsrSrc& c, int64_t n, int32_t d, cudaStream_t st) : X((size_t)std::max<int64_t>(n, 1) * d, st) {
    DevBuf<int32_t> bad(1, st);
    GM_CUDA(cudaMemsetAsync(bad.get(), 0, 4, st));
    launch_csr_densify(c.indptr, c.indices, c.values, n, d, X.get(), bad.get(), st);
    int32_t hb = 0;
    GM_CUDA(cudaMemcpyAsync(&hb, bad.get(), 4, cudaMemcpyDeviceToHost, st));
    GM_CUDA(cudaStreamSynchronize(st));
    if (hb) throw Error(GMPSVM_EINVAL, "CSR column index outside [0, d)");
  }
};

// Sparse kernel values (NEXT-3, csr.cu): GMPSVM_CSR=sparse forces them (read per call), =dense
// the densified path.  By default the rows are densified -- on the news20-shaped data the dense
// tcgen05 contraction is faster (n = 20k, d = 5000, 1 % non-zero: 4.4 vs 8.1 ms) --
// unless the dense copy would take more than a quarter of the device memory.  The sparse path
// needs the Gaussian kernel, FULL_K, no CV sigmoids and one dense row in shared memory (d <= 56k).
static bool csr_sparse_path(const CsrSrc& c, int64_t n, int32_t d, const gmpsvm_options& opt) {
  const char* env = getenv("GMPSVM_CSR");
  const std::string mode = env ? env : "";
  if (mode == "dense") return false;
  const double mem = (double)device_total_mem(opt.device);
  const double budget = opt.cache_bytes > 0 ? (double)opt.cache_bytes : 0.85 * mem;
  const bool ok = opt.kernel == 0 && opt.prob_folds == 0 && krow_csr_rows_per_cta(d) >= 1 &&
                  (double)n * round_up(n, 4) * 4.0 <= budget;
  if (mode == "sparse") {
    if (!ok) throw Error(GMPSVM_ENOTIMPL, "GMPSVM_CSR=sparse: needs the Gaussian kernel, FULL_K, no CV sigmoids, d <= 56k");
    return true;
  }
  (void)c;
  return ok && (double)n * (double)d * 4.0 > 0.25 * mem;
}

int engine_train_csr(const int64_t* indptr, const int32_t* indices, const float* values, const int32_t* y, int64_t n,
                     int32_t d, int32_t k, double C, double gamma, double eps, const gmpsvm_options& opt, Model** out) {
  DeviceGuard dg(opt.device);
  cudaStream_t st = get_stream(opt);
  CsrDev cdev(indptr, indices, values, n, d, opt, st);
  gmpsvm_options o2 = opt;
  DevBuf<int32_t> yb(opt.inputs_on_device ? 0 : (size_t)n, st);
  const int32_t* dy = y;
  if (!opt.inputs_on_device) {
    if (!y) throw Error(GMPSVM_EINVAL, "null argument");
    GM_CUDA(cudaMemcpyAsync(yb.get(), y, (size_t)n * 4, cudaMemcpyHostToDevice, st));
    dy = yb.get();
  }
  o2.inputs_on_device = 1;
  o2.stream = st;
  if (csr_sparse_path(cdev.src, n, d, opt)) return engine_train_core(nullptr, dy, n, d, k, C, gamma, eps, o2, out, &cdev.src);
  CsrDense cd(cdev.src, n, d, st);
  return engine_train(cd.X.get(), dy, n, d, k, C, gamma, eps, o2, out);
}

int engine_predict_csr(const Model& mdl, const int64_t* indptr, const int32_t* indices, const float* values, int64_t m,
                       double* prob_out, const gmpsvm_options& opt) {
  if (m == 0) return GMPSVM_OK;
  DeviceGuard dg(opt.device);
  cudaStream_t st = get_stream(opt);
  CsrDev cdev(indptr, indices, values, m, mdl.d, opt, st);
  CsrDense cd(cdev.src, m, mdl.d, st);
  gmpsvm_options o2 = opt;
  o2.stream = st;
  if (opt.inputs_on_device) return engine_predict(mdl, cd.X.get(), m, prob_out, nullptr, o2);
  DevBuf<double> pb((size_t)m * mdl.k, st);
  o2.inputs_on_device = 1;
  const int rc = engine_predict(mdl, cd.X.get(), m, pb.get(), nullptr, o2);
  GM_CUDA(cudaMemcpyAsync(prob_out, pb.get(), (size_t)m * mdl.k * 8, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaStreamSynchronize(st));
  return rc;
}

// ------------------------------------------------------------------------------------------
static std::shared_ptr<DevModel> ensure_dev_model(const Model& mdl, int device, cudaStream_t st) {
  std::lock_guard<std::mutex> lk(mdl.mu);
  if (mdl.dev && mdl.dev->device == device) return mdl.dev;
  if (mdl.dev) {  // moving to another device: the host copies are the source of the new one
    ensure_host_sv(mdl);
    ensure_host_alpha(mdl);
  }
  const int64_t nsv = (int64_t)mdl.sv_pos.size();
  DevBuf<float> rows((size_t)std::max<int64_t>(nsv, 1) * mdl.d, st);
  if (nsv > 0) {
    if (!mdl.sv_X_ready) throw Error(GMPSVM_EINVAL, "model has no SV rows");
    GM_CUDA(cudaMemcpyAsync(rows.get(), mdl.sv_X.data(), (size_t)nsv * mdl.d * 4, cudaMemcpyHostToDevice, st));
  }
  std::vector<int64_t> row_of_sv(nsv);
  for (int64_t i = 0; i < nsv; ++i) row_of_sv[i] = i;
  mdl.dev = build_dev_model(mdl, rows.get(), row_of_sv, device, st);
  return mdl.dev;
}

static int engine_predict_path(const Model& mdl, const float* Xt, int64_t m, double* prob_out, double* dec_out,
                               const gmpsvm_options& opt, int force_path);

int engine_predict(const Model& mdl, const float* Xt, int64_t m, double* prob_out, double* dec_out,
                   const gmpsvm_options& opt) {
  return engine_predict_path(mdl, Xt, m, prob_out, dec_out, opt, -1);
}

static int engine_predict_path(const Model& mdl, const float* Xt, int64_t m, double* prob_out, double* dec_out,
                               const gmpsvm_options& opt, int force_path) {
  const auto t_start = std::chrono::steady_clock::now();
  gmpsvm_predict_stats& ps = tls_predict_stats();
  ps = gmpsvm_predict_stats{};
  if (m < 0 || (m > 0 && (!Xt || (!prob_out && !dec_out)))) throw Error(GMPSVM_EINVAL, "bad predict arguments");
  if (mdl.n_trained() != mdl.P()) throw Error(GMPSVM_EINVAL, "model does not contain every pair (merge the parts first)");
  if (prob_out && mdl.k > kMaxCoupleK) throw Error(GMPSVM_ENOTIMPL, "coupling supports k <= 40");
  if (m == 0) return GMPSVM_OK;
  DeviceGuard dg(opt.device);
  cudaStream_t st = get_stream(opt);
  const uint64_t launches0 = g_launches.load();
  const std::shared_ptr<DevModel> dm_ref = ensure_dev_model(mdl, opt.device, st);  // held for the whole call
  const DevModel& dm = *dm_ref;
  const int k = mdl.k, d = mdl.d, P = mdl.P();
  const int path = force_path >= 0 ? force_path : dm.path;
  PhaseTimer tm(st);
  const int64_t mc_max = std::min<int64_t>(m, kPredictChunk);
  const int64_t mc_pad = round_up(mc_max, kTile);
  const bool p_i8 = path == kDecI8, p_f16 = path == kDecF16;
  DevBuf<float> xin(opt.inputs_on_device ? 0 : (size_t)mc_max * d, st);
  // feature-major test rows: the FP64 path (and the FP16 path's fallback for rows outside its range)
  DevBuf<float> XtT(p_i8 ? 0 : (size_t)dm.d_pad * mc_pad, st), nt(mc_pad, st);
  DevBuf<float> Xhi(p_f16 ? krow_tc_buf_floats(mc_pad, dm.dpt) : 0, st), Xlo(p_f16 ? krow_tc_buf_floats(mc_pad, dm.dpt) : 0, st);
  DevBuf<float> part(p_f16 ? (size_t)dm.n_items * mc_pad * dm.km1_pad : 0, st);
  DevBuf<double> part64((size_t)dm.n_items * mc_pad * dm.km1_pad, st), nt64(mc_pad, st);
  DevBuf<int8_t> tI8(p_i8 ? dec_i8_plane_bytes(mc_pad, d) : 0, st);
  DevBuf<int32_t> t_e(p_i8 ? mc_pad : 0, st);
  DevBuf<unsigned> d_amax(1, st);
  GM_CUDA(cudaMemsetAsync(d_amax.get(), 0, 4, st));
  DevBuf<double> dec_buf(opt.inputs_on_device ? 0 : (size_t)mc_max * P, st);
  DevBuf<double> prob_buf((opt.inputs_on_device || !prob_out) ? 0 : (size_t)mc_max * k, st);
  DevBuf<double> dec_tmp((opt.inputs_on_device && !dec_out) ? (size_t)mc_max * P : 0, st);
  DevBuf<int32_t> bad(1, st);
  GM_CUDA(cudaMemsetAsync(bad.get(), 0, 4, st));
  for (int64_t i0 = 0; i0 < m; i0 += mc_max) {
    const int64_t mc = std::min(mc_max, m - i0);
    const int64_t mcp = round_up(mc, kTile);
    tm.mark(PH_STAGE);
    const float* src = Xt + i0 * d;
    if (!opt.inputs_on_device) {
      GM_CUDA(cudaMemcpyAsync(xin.get(), src, (size_t)mc * d * 4, cudaMemcpyHostToDevice, st));
      src = xin.get();
    }
    DevBuf<int2> d_dtiles;
    DevBuf<int32_t> d_uoff, d_uitem;
    int n_units = 0;
    // FP16 split: test rows far outside the SVs' range would overflow half precision -> FP64
    const bool use_tc = p_f16 && launch_maxabs(src, mc, d, nullptr, dm.mu, st) * dm.sc < 60000.f;
    const bool f64 = !p_i8 && !use_tc;
    if (!f64) {
      // work units: (item, test tile), test tiles fastest; unit = the item's SV tiles for that test tile
      const int ntt = (int)(mcp / kTile);
      std::vector<int2> dt;
      std::vector<int32_t> uoff(1, 0), uitem;
      for (int it = 0; it < dm.n_items; ++it)
        for (int tt = 0; tt < ntt; ++tt) {
          for (int sv = dm.h_items[it].tile_begin; sv < dm.h_items[it].tile_end; ++sv) dt.push_back(make_int2(tt, sv));
          uoff.push_back((int32_t)dt.size());
          uitem.push_back(it);
        }
      n_units = (int)uitem.size();
      new (&d_dtiles) DevBuf<int2>(std::max<size_t>(dt.size(), 1), st);
      new (&d_uoff) DevBuf<int32_t>(uoff.size(), st);
      new (&d_uitem) DevBuf<int32_t>(std::max<size_t>(uitem.size(), 1), st);
      if (!dt.empty())
        GM_CUDA(cudaMemcpyAsync(d_dtiles.get(), dt.data(), dt.size() * sizeof(int2), cudaMemcpyHostToDevice, st));
      GM_CUDA(cudaMemcpyAsync(d_uoff.get(), uoff.data(), uoff.size() * 4, cudaMemcpyHostToDevice, st));
      if (!uitem.empty())
        GM_CUDA(cudaMemcpyAsync(d_uitem.get(), uitem.data(), uitem.size() * 4, cudaMemcpyHostToDevice, st));
    }
    if (p_i8) {
      launch_row_norms(src, mc, d, nullptr, nt.get(), mcp, bad.get(), st);  // validation (non-finite rows)
      launch_stage_i8(src, mc, d, nullptr, tI8.get(), mcp, t_e.get(), nt64.get(), d_amax.get(), st);
    } else if (use_tc) {
      launch_row_norms(src, mc, d, nullptr, nt.get(), mcp, bad.get(), st);  // validation (non-finite rows)
      launch_split_hilo_mu(src, mc, d, nullptr, dm.mu, dm.sc, Xhi.get(), Xlo.get(), nt.get(), mcp, dm.dpt, st);
    } else {
      launch_stage_features(src, mc, d, nullptr, XtT.get(), mcp, dm.d_pad, mcp, nt.get(), bad.get(), st);
    }
    tm.mark(PH_STAGE);
    double* dec_d = opt.inputs_on_device ? (dec_out ? dec_out + i0 * P : dec_tmp.get()) : dec_buf.get();
    tm.mark(PH_DEC);
    if (f64) {  // FP64 decision values (SIMT; any kernel)
      launch_col_norms64(XtT.get(), mcp, mcp, dm.d_pad, nt64.get(), st);
      GM_CUDA(cudaMemsetAsync(part64.get(), 0, (size_t)dm.n_items * mcp * dm.km1_pad * 8, st));
      launch_dec_f64(XtT.get(), mcp, nt64.get(), mcp, dm.SvT, dm.nsv_pad, dm.nsv64, dm.coef64, dm.km1, dm.km1_pad, dm.items,
                     dm.n_items, dm.d_pad, mdl.gamma, part64.get(), st, mdl.kernel, mdl.coef0, mdl.degree);
      launch_dec_reduce64(part64.get(), mc, mcp, k, dm.km1_pad, dm.item_begin, dm.item_end, dm.b, dec_d, st);
    } else if (p_i8) {  // exact int8-digit dot products, FP64 kernel values (dec_i8.cu)
      GM_CUDA(cudaMemsetAsync(part64.get(), 0, (size_t)dm.n_items * mcp * dm.km1_pad * 8, st));  // items without tiles
      if (n_units > 0)
        launch_dec_i8(tI8.get(), mcp, t_e.get(), nt64.get(), dm.SvI8, dm.nsv_pad, dm.sv_e, dm.sv_n64, d,
                      d_dtiles.get(), d_uoff.get(), d_uitem.get(), n_units, dm.coef64, dm.km1, dm.km1_pad, mdl.gamma,
                      part64.get(), st);
      launch_dec_reduce64(part64.get(), mc, mcp, k, dm.km1_pad, dm.item_begin, dm.item_end, dm.b, dec_d, st);
    } else {
      GM_CUDA(cudaMemsetAsync(part.get(), 0, (size_t)dm.n_items * mcp * dm.km1_pad * 4, st));  // items without tiles
      if (n_units > 0) {
        const KrowKernel kk{mdl.kernel, (float)mdl.gamma, (float)mdl.coef0, 0.f, mdl.degree};
        launch_dec_tc(Xhi.get(), Xlo.get(), mcp, dm.SvHi, dm.SvLo, dm.nsv_pad, dm.dpt, d_dtiles.get(), d_uoff.get(),
                      d_uitem.get(), n_units, nt.get(), dm.nsvc, dm.coef, dm.km1, dm.km1_pad, mdl.gamma, dm.sc, part.get(),
                      st, mdl.kernel != 0 ? &kk : nullptr);
      }
      launch_dec_reduce(part.get(), mc, mcp, k, dm.km1_pad, dm.item_begin, dm.item_end, dm.b, dec_d, st);
    }
    ps.dec_launches += 1;
    tm.mark(PH_DEC);
    double* prob_d = nullptr;
    if (prob_out) {
      prob_d = opt.inputs_on_device ? prob_out + i0 * k : prob_buf.get();
      tm.mark(PH_COUPLE);
      launch_couple(dec_d, mc, k, dm.A, dm.B, prob_d, st);
      tm.mark(PH_COUPLE);
    }
    if (!opt.inputs_on_device) {
      tm.mark(PH_D2H);
      if (prob_out)
        GM_CUDA(cudaMemcpyAsync(prob_out + i0 * k, prob_d, (size_t)mc * k * 8, cudaMemcpyDeviceToHost, st));
      if (dec_out) GM_CUDA(cudaMemcpyAsync(dec_out + i0 * P, dec_d, (size_t)mc * P * 8, cudaMemcpyDeviceToHost, st));
      tm.mark(PH_D2H);
    }
  }
  GM_CUDA(cudaEventRecord(dm.last_use, st));
  int32_t hbad = 0;
  uint32_t amax_bits = 0;
  GM_CUDA(cudaMemcpyAsync(&hbad, bad.get(), 4, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaMemcpyAsync(&amax_bits, d_amax.get(), 4, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaStreamSynchronize(st));
  if (hbad) throw Error(GMPSVM_EINVAL, "Xtest contains non-finite values");
  float amax_t = 0.f;
  std::memcpy(&amax_t, &amax_bits, 4);
  if (p_i8 && force_path < 0 && amax_t > kTestRange * dm.amax_sv)  // outside the range the routing bound assumed
    return engine_predict_path(mdl, Xt, m, prob_out, dec_out, opt, kDecF64);
  ps.t_stage_ms = tm.ms(PH_STAGE);
  ps.t_decision_ms = tm.ms(PH_DEC);
  ps.t_couple_ms = tm.ms(PH_COUPLE);
  ps.t_d2h_ms = tm.ms(PH_D2H);
  ps.dec_flops = (double)m * (double)mdl.sv_pos.size() * (2.0 * d + 3.0 + 2.0 * (k - 1));
  ps.launches = (int64_t)(g_launches.load() - launches0);
  ps.dec_path = path;
  ps.t_total_ms = host_ms_since(t_start);
  return GMPSVM_OK;
}

// ------------------------------------------------------------------------------------------
int engine_rbf_kernel(const float* X, int64_t n, const float* Y, int64_t m, int32_t d, double gamma, float* K_out,
                      const gmpsvm_options& opt) {
  if (n < 0 || m < 0 || d < 1 || !finite_pos(gamma)) throw Error(GMPSVM_EINVAL, "bad rbf_kernel arguments");
  if (opt.kernel != 0) throw Error(GMPSVM_ENOTIMPL, "gmpsvm_rbf_kernel computes the Gaussian kernel only");
  if (n == 0 || m == 0) return GMPSVM_OK;
  if (!X || !Y || !K_out) throw Error(GMPSVM_EINVAL, "null argument");
  DeviceGuard dg(opt.device);
  cudaStream_t st = get_stream(opt);
  const int d_pad = (int)round_up(d, kBK);
  const int64_t n_pad = round_up(n, kTile), m_pad = round_up(m, kTile);
  DevBuf<float> bx(opt.inputs_on_device ? 0 : (size_t)n * d, st), by(opt.inputs_on_device ? 0 : (size_t)m * d, st);
  const float* dX = X;
  const float* dY = Y;
  if (!opt.inputs_on_device) {
    GM_CUDA(cudaMemcpyAsync(bx.get(), X, (size_t)n * d * 4, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(by.get(), Y, (size_t)m * d * 4, cudaMemcpyHostToDevice, st));
    dX = bx.get();
    dY = by.get();
  }
  // X == Y (same buffer, same size): the symmetric FULL_K launch that training uses (K_ii = 1)
  const bool sym = (X == Y && n == m);
  if (sym && krow_use_tc()) {
    const int dp = krow_tc_d_pad(d);
    const int64_t np2 = krow_tc_rows_pad(n);
    DevBuf<float> hi(krow_tc_buf_floats(np2, dp), st), lo(krow_tc_buf_floats(np2, dp), st), nx2(np2, st);
    DevBuf<uint8_t> scr(krow_tc_scratch_bytes(n, d), st);
    const float ksc = launch_split_hilo(dX, n, d, nullptr, hi.get(), lo.get(), nx2.get(), np2, dp, scr.get(), st);
    DevBuf<float> kb2(opt.inputs_on_device ? 0 : (size_t)n * m, st);
    float* dK2 = opt.inputs_on_device ? K_out : kb2.get();
    const bool two_cta = krow_tc_2cta() && (m % 4) == 0 && (reinterpret_cast<uintptr_t>(dK2) & 15) == 0;
    const std::vector<int2> tl = krow_tc_tiles(n, two_cta);
    DevBuf<int2> dt(tl.size(), st);
    GM_CUDA(cudaMemcpyAsync(dt.get(), tl.data(), tl.size() * sizeof(int2), cudaMemcpyHostToDevice, st));
    launch_krow_tc(hi.get(), lo.get(), np2, dp, dt.get(), (int)tl.size(), nx2.get(), n, gamma, ksc, dK2, m, st, two_cta);
    if (!opt.inputs_on_device) GM_CUDA(cudaMemcpyAsync(K_out, dK2, (size_t)n * m * 4, cudaMemcpyDeviceToHost, st));
    GM_CUDA(cudaStreamSynchronize(st));
    return GMPSVM_OK;
  }
  DevBuf<float> XT((size_t)d_pad * n_pad, st), YT(sym ? 0 : (size_t)d_pad * m_pad, st), nx(n_pad, st),
      ny(sym ? 0 : m_pad, st);
  launch_stage_features(dX, n, d, nullptr, XT.get(), n_pad, d_pad, n_pad, nx.get(), nullptr, st);
  if (!sym) launch_stage_features(dY, m, d, nullptr, YT.get(), m_pad, d_pad, m_pad, ny.get(), nullptr, st);
  DevBuf<float> kb(opt.inputs_on_device ? 0 : (size_t)n * m, st);
  float* dK = opt.inputs_on_device ? K_out : kb.get();
  if (sym)
    launch_krow_full_sym(XT.get(), n_pad, nx.get(), n, d_pad, gamma, dK, m, st);
  else
    launch_krow_rect(XT.get(), n_pad, nx.get(), n, YT.get(), m_pad, ny.get(), m, d_pad, gamma, dK, m, st);
  if (!opt.inputs_on_device) GM_CUDA(cudaMemcpyAsync(K_out, dK, (size_t)n * m * 4, cudaMemcpyDeviceToHost, st));
  GM_CUDA(cudaStreamSynchronize(st));
  return GMPSVM_OK;
}

int engine_couple(const double* dec, int64_t m, int32_t k, const double* A, const double* B, double* prob_out,
                  const gmpsvm_options& opt) {
  if (m < 0 || k < 2 || !dec || !A || !B || !prob_out) throw Error(GMPSVM_EINVAL, "bad couple arguments");
  if (k > kMaxCoupleK) throw Error(GMPSVM_ENOTIMPL, "coupling supports k <= 40");
  if (m == 0) return GMPSVM_OK;
  DeviceGuard dg(opt.device);
  cudaStream_t st = get_stream(opt);
  const int P = k * (k - 1) / 2;
  if (opt.inputs_on_device) {
    launch_couple(dec, m, k, A, B, prob_out, st);
  } else {
    DevBuf<double> dd((size_t)m * P, st), dA(P, st), dB(P, st), dp((size_t)m * k, st);
    GM_CUDA(cudaMemcpyAsync(dd.get(), dec, (size_t)m * P * 8, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(dA.get(), A, P * 8, cudaMemcpyHostToDevice, st));
    GM_CUDA(cudaMemcpyAsync(dB.get(), B, P * 8, cudaMemcpyHostToDevice, st));
    launch_couple(dd.get(), m, k, dA.get(), dB.get(), dp.get(), st);
    GM_CUDA(cudaMemcpyAsync(prob_out, dp.get(), (size_t)m * k * 8, cudaMemcpyDeviceToHost, st));
  }
  GM_CUDA(cudaStreamSynchronize(st));
  return GMPSVM_OK;
}

}  // namespace gmpsvm
