// ratel_runtime.cu -- the C ABI (include/ratel.h): registration, the per-step
// state machine of active gradient offloading, the pinned-host tile ring, the
// optional global-norm clip and the multi-GPU range partition.
//
// PAPER.md anchors: AGO's "active message" -- the optimizer handler for a
// tensor runs "upon main memory receiving the offloaded gradients"
// (P:L1017-1031); gradients arrive "sequentially with a decreasing index"
// (P:L1038-1041); naive AGO serialises state-in, compute, state-out
// (Fig. 3a) while optimized AGO overlaps the write-back of
// tensor i with the compute of tensor i-1 (Fig. 3b).  Here the
// "message" is a CUDA event recorded on the caller's backward stream, the
// handler is the K1 kernel on a low-priority optimizer stream, and for
// pinned-host states the state-in / write-back run on two copy streams (the
// host link is duplex, unlike the paper's SSD link).
#include <cuda_runtime.h>

#include <fcntl.h>
#include <sys/stat.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <cerrno>
#include <condition_variable>
#include <deque>
#include <mutex>
#include <new>
#include <string>
#include <thread>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "nccl_dl.h"
#include "ratel.h"
#include "ratel_host_adam.h"
#include "ratel_plan_impl.h"
#include "ratel_uring.h"
#include "ratel_kernels.cuh"

namespace {

using namespace ratel;

thread_local char t_err[1024] = "";

// NVTX ranges around the API calls, tile stages and host handlers (header-only
// nvtx3: free unless a profiler is attached; nsys/ncu show the AGO schedule).
struct Nvtx {
  explicit Nvtx(const char* fmt, ...) {
    char buf[96];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    nvtxRangePushA(buf);
  }
  ~Nvtx() { nvtxRangePop(); }
};

int set_error(int code, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(t_err, sizeof t_err, fmt, ap);
  va_end(ap);
  return code;
}

struct Slice {
  uint64_t begin = 0, end = 0;
};

struct Block {
  bool registered = false;
  int residency = RATEL_DEVICE;
  int order = -1;  // registration index (fixes the clip reduction order)
  std::vector<ratel_range> ranges;
  std::vector<Slice> slices;
  cudaEvent_t ev_grad = nullptr;  // "gradient arrived" -- recorded on the caller's stream
  cudaEvent_t ev_done = nullptr;  // this rank's P16 slices written -- on s_opt (s_hc_h2d for HOST_COMPUTE)
  cudaEvent_t ev_gh = nullptr;    // HOST_COMPUTE: G16 slices landed in host staging
  cudaEvent_t ev_hc = nullptr;    // HOST_COMPUTE: the CPU update of this block finished (on s_host)
  std::vector<uint16_t*> h_g, h_p;  // HOST_COMPUTE: pinned G16 / P16 staging per range (rank slice)
  std::vector<std::vector<uint16_t*>> peers;  // per range: every rank's P16 base as mapped here (fused all-gather)
  // Fused data-parallel gradient reduction (R17): per range, every rank's
  // full-range G16 base as mapped here (empty = plain rank-slice gradient).
  std::vector<std::vector<const uint16_t*>> rgrads;
  std::vector<double> rscale;
  bool rs = false;                  // some range of this block has peer grads
  bool pp = false;                  // some range of this block has peer params (fused all-gather)
  // RS or PP + NCCL: every rank has handed this block off -- its G16 is complete
  // everywhere, and no rank's backward still reads the P16 the peers will overwrite
  cudaEvent_t ev_ready = nullptr;
  cudaEvent_t ev_rel = nullptr;     // RS + NCCL: every rank finished reading this block's G16
  bool handed_off = false, enqueued = false;
  // SSD residency: per range, the state file and where the slice's arrays are
  struct SsdRange {
    int fd = -1;
    uint64_t off = 0, stride = 0;  // theta at off, m at off + stride, v at off + 2*stride (bytes)
  };
  std::vector<SsdRange> ssd;
  uint64_t ssd_seq = 0;  // engine job number of this block's last submission
  bool ssd_cpu = false;  // RATEL_SSD_HOST_COMPUTE: the CPU handler updates the tiles (residency stays RATEL_SSD)
};

// The SSD tier's reader/writer threads (RATEL_SSD).  Shared with the main
// thread through `mu`; GPU work is issued by the reader on its own streams.
constexpr int kMaxDepth = 16;  // tile ring slots (pinned-host and SSD)
struct SsdJob {
  int block = -1;
  std::vector<cudaEvent_t> wait;  // host-waited before the block's states are read
};
struct SsdTile {
  uint64_t seq = 0;  // ring order (E.ring_k at its read)
  int slot = 0, fd = -1;
  uint64_t foff = 0, stride = 0, bytes = 0;
  bool host = false;  // updated by the CPU handler in the staging slot (no D2H to wait for)
};
struct SsdEngine {
  std::thread reader, writer;
  std::mutex mu;
  std::condition_variable cv;
  std::deque<SsdJob> jobs;
  std::deque<SsdTile> wq;
  int slot_busy[kMaxDepth] = {};  // a tile in this slot still awaits its write-back
  bool stop = false;
  bool reader_done = false;  // the writer drains until the reader can queue no more tiles
  // RATEL_SSD_SIMPLEX: one file transfer at a time (disk_busy), and tile k's
  // write-back waits for tile k+1's read (tiles_read > k+1) unless no read is
  // pending (reader idle with an empty job queue).
  bool disk_busy = false;
  bool reader_idle = true;
  uint64_t tiles_read = 0;   // tiles whose three arrays have been read (ring order)
  uint64_t jobs_in = 0, jobs_out = 0, tiles_in = 0, tiles_out = 0;
  int err = 0;
  std::string msg;
  IoRing rd_ring, wr_ring;   // RATEL_SSD_IO_URING: the reader's and the writer's io_uring
  float* h_ring = nullptr;  // pinned: depth x {theta, m, v} x tile
  float* d_ring = nullptr;  // device: the same shape
  cudaStream_t s_in = nullptr, s_k = nullptr, s_out = nullptr;
  cudaEvent_t ev_h2d[kMaxDepth] = {}, ev_d2h[kMaxDepth] = {}, ev_k1[kMaxDepth] = {};
  uint64_t ring_k = 0;
  double read_s = 0, write_s = 0;  // host seconds inside pread / pwrite
  uint64_t read_bytes = 0, write_bytes = 0;
};

// One host-handler invocation (owned by the callback, deleted when done).
struct HostTask {
  std::vector<HostAdamArgs> ranges;
  const double* sumsq = nullptr;  // clip: pinned copy of the global sum of squares
  double max_norm = 0.0;
  int threads = 0;
};

struct TimingPair {
  cudaEvent_t a = nullptr, b = nullptr;
};

struct Ctx {
  bool inited = false;
  std::atomic<int> sticky{0};
  char sticky_msg[1024] = "";
  int device = 0, rank = 0, world = 1;
  ratel_config cfg{};
  int sms = 0, k1_grid = 0, k2_grid = 0, rs_grid = 0, lite_grid = 0;
  cudaStream_t s_opt = nullptr, s_h2d = nullptr, s_d2h = nullptr, s_comm = nullptr, s_host = nullptr,
               s_tile = nullptr;
  // HOST_COMPUTE's own copy streams (G16 down, P16 up): kept apart from the
  // tile ring's s_h2d/s_d2h so CPU-handler blocks and GPU-streamed blocks in
  // one step do not queue behind each other's copies.
  cudaStream_t s_hc_d2h = nullptr, s_hc_h2d = nullptr;
  // Device-residency update kernels alternate over s_k[0..update_streams-1];
  // s_opt joins each (ev_done) so it stays ordered after every grad read.
  cudaStream_t s_k[2] = {nullptr, nullptr};
  unsigned k_next = 0;
  static constexpr int kNS = 13;  // every stream (10 + the SSD engine's 3), for the sync cross-waits
  cudaEvent_t ev_end[kNS] = {};
  cudaEvent_t ev_norm = nullptr;  // clip: global norm final (on s_opt)
  double* h_sumsq = nullptr;      // clip + HOST_COMPUTE: pinned copy of the norm
  double hp_lr = 0, hp_b1 = 0, hp_b2 = 0, hp_eps = 0, hp_wd = 0, hp_bc1 = 1, hp_bc2 = 1;
  std::vector<Block> blocks;
  std::vector<int> reg;      // registered ids, registration order
  std::vector<int> pending;  // handed off before arming (deferred), hand-off order
  int n_handed = 0;
  bool armed = false;
  int64_t last_step = 0;
  AdamScalars scal{};
  // clip
  double* d_partials = nullptr;
  size_t partial_cap = 0;  // slots
  double* d_sumsq = nullptr;  // [0] this rank, [1] all ranks, [2] barrier scratch
  double* d_barrier = nullptr;
  // TMA update kernel's dynamic tile counters, one per launching stream
  // (s_k[0], s_k[1], s_tile, s_opt): launches on one stream are serialised,
  // so each counter's value at a launch is known on the host (ctr_base).
  unsigned long long* d_ctr = nullptr;
  unsigned long long ctr_base[5] = {0, 0, 0, 0, 0};  // + the SSD reader's kernel stream
  int n_peer_ranges = 0;      // ranges using the fused (peer-store) all-gather
  int n_rs_blocks = 0;        // blocks using the fused gradient reduction
  int* h_flag = nullptr;      // mapped pinned: non-finite norm seen
  int* d_flag = nullptr;
  // pinned-host tile ring
  float* d_tiles = nullptr;  // depth x {theta, m, v} x tile
  cudaEvent_t ev_h2d[kMaxDepth] = {}, ev_k1[kMaxDepth] = {}, ev_d2h[kMaxDepth] = {};
  uint64_t ring_k = 0;
  // NCCL
  ncclComm_t comm = nullptr;
  // stats
  std::atomic<int64_t> launches{0};
  std::vector<TimingPair> tpool;
  size_t tused = 0;
  SsdEngine* ssd = nullptr;  // created by the first RATEL_SSD registration
};

Ctx G;
NcclApi g_nccl;

int sticky_fail(int code, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(G.sticky_msg, sizeof G.sticky_msg, fmt, ap);
  va_end(ap);
  G.sticky = code;
  snprintf(t_err, sizeof t_err, "%s", G.sticky_msg);
  return code;
}

#define CK(call)                                                                                 \
  do {                                                                                           \
    cudaError_t e_ = (call);                                                                     \
    if (e_ != cudaSuccess)                                                                       \
      return sticky_fail(e_ == cudaErrorMemoryAllocation ? RATEL_ENOMEM : RATEL_ECUDA,           \
                         "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
  } while (0)

#define NK(call)                                                                                  \
  do {                                                                                            \
    ncclResult_t r_ = (call);                                                                     \
    if (r_ != ncclSuccess)                                                                        \
      return sticky_fail(RATEL_ENCCL, "%s failed: %s (%s:%d)", #call, g_nccl.GetErrorString(r_), \
                         __FILE__, __LINE__);                                                     \
  } while (0)

#define RK(call)              \
  do {                        \
    int rc_ = (call);         \
    if (rc_ != RATEL_OK) return rc_; \
  } while (0)

std::mutex g_launch_mu;  // launch bookkeeping (timing pool, tile counters): main + SSD reader thread

int entry() {
  if (!G.inited) return set_error(RATEL_ESTATE, "ratel: not initialised (call ratel_init first)");
  if (G.sticky) return set_error(G.sticky, "ratel: sticky error: %s", G.sticky_msg);
  CK(cudaSetDevice(G.device));
  return RATEL_OK;
}

uint64_t padded(uint64_t n, int world) {
  const uint64_t q = 8ull * static_cast<uint64_t>(world);
  return (n + q - 1) / q * q;
}

Slice slice_of(uint64_t n, int world, int rank) {
  const uint64_t s = padded(n, world) / world;
  Slice r;
  r.begin = std::min<uint64_t>(n, s * rank);
  r.end = std::min<uint64_t>(n, r.begin + s);
  return r;
}

const uint16_t* grad_ptr(const ratel_range& r, const Slice& s) {
  return static_cast<const uint16_t*>(r.grad_bf16) + (r.grad_is_rank_slice ? 0 : s.begin);
}

// ------------------------------------------------------------------ launches
#ifndef RATEL_K1_TMA
#define RATEL_K1_TMA 1
#endif

#ifndef RATEL_TMA_DYNAMIC
#define RATEL_TMA_DYNAMIC 1
#endif

int ctr_slot(cudaStream_t st) {
  if (G.ssd != nullptr && st == G.ssd->s_k) return 4;
  return st == G.s_k[0] ? 0 : st == G.s_k[1] ? 1 : st == G.s_tile ? 2 : 3;
}

template <int MODE, bool CLIP>
void launch_k1(UpdateParams& P, unsigned grid, cudaStream_t st, int kernel) {
  if (kernel == RATEL_UPDATE_LDG) {
    adam_update_kernel<MODE, CLIP><<<grid, kThreads, 0, st>>>(P);
    return;
  }
  if (kernel == RATEL_UPDATE_LDG_LITE) {
    uint64_t max8 = 0;
    for (int r = 0; r < P.nr; ++r) max8 = std::max<uint64_t>(max8, (P.r[r].n + 7) / 8);
    const uint64_t want = std::max<uint64_t>(1, (max8 + kThreads - 1) / kThreads);
    const unsigned g = static_cast<unsigned>(std::min<uint64_t>(want, static_cast<uint64_t>(G.lite_grid)));
    adam_update_kernel<MODE, CLIP, 1, 4><<<g, kThreads, 0, st>>>(P);
    return;
  }
#if RATEL_K1_TMA
  (void)grid;
  uint64_t tiles = 0;
  for (int r = 0; r < P.nr; ++r) tiles += ((P.r[r].n & ~7ull) + kTmaTile - 1) / kTmaTile;
  uint64_t cap = static_cast<uint64_t>(G.sms) * RATEL_TMA_CTAS_PER_SM;
  if (G.cfg.max_ctas > 0) cap = std::min<uint64_t>(cap, static_cast<uint64_t>(G.cfg.max_ctas));
  unsigned g = static_cast<unsigned>(std::max<uint64_t>(1, std::min<uint64_t>(tiles, cap)));
  if (G.cfg.cta_tiles > 0) {  // non-persistent: CTA b takes tiles [b*Y, b*Y+Y), then retires
    const uint64_t Y = static_cast<uint64_t>(G.cfg.cta_tiles);
    P.cta_tiles = static_cast<uint32_t>(Y);
    P.tile_ctr = nullptr;
    g = static_cast<unsigned>(std::max<uint64_t>(1, (tiles + Y - 1) / Y));
  } else {
#if RATEL_TMA_DYNAMIC
    const int slot = ctr_slot(st);
    P.tile_ctr = G.d_ctr + slot;
    P.tile_base = G.ctr_base[slot];
    G.ctr_base[slot] += tiles + g;  // every tile taken once + one final grab per CTA
#endif
  }
  adam_update_tma_kernel<MODE, CLIP><<<g, kTmaThreads, kTmaSmemBytes, st>>>(P);
#else
  adam_update_kernel<MODE, CLIP><<<grid, kThreads, 0, st>>>(P);
#endif
}

template <int MODE, bool CLIP>
cudaError_t prepare_k1() {
#if RATEL_K1_TMA
  const cudaError_t e = cudaFuncSetAttribute(adam_update_rs_tma_kernel<MODE, CLIP>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             static_cast<int>(std::max(rs_tma_smem_bytes(1),
                                                                       rs_tma_smem_bytes(kMaxRanks))));
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(adam_update_tma_kernel<MODE, CLIP>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              static_cast<int>(kTmaSmemBytes));
#else
  return cudaSuccess;
#endif
}

template <int MODE, bool CLIP>
void launch_k1_rs(RsUpdateParams& Q, unsigned grid, cudaStream_t st) {
  (void)grid;
#if RATEL_K1_TMA
  if (G.cfg.k1_kernel == RATEL_UPDATE_TMA) {  // TMA-staged fused reduction (one CTA per SM, persistent)
    uint64_t tiles = 0;
    int nmax = 1;
    for (int r = 0; r < Q.u.nr; ++r) {
      tiles += ((Q.u.r[r].n & ~7ull) + kRsTmaTile - 1) / kRsTmaTile;
      nmax = std::max(nmax, Q.gp[r].n);
    }
    uint64_t cap = static_cast<uint64_t>(G.sms);
    if (G.cfg.max_ctas > 0) cap = std::min<uint64_t>(cap, static_cast<uint64_t>(G.cfg.max_ctas));
    const unsigned g = static_cast<unsigned>(std::max<uint64_t>(1, std::min<uint64_t>(tiles, cap)));
#if RATEL_TMA_DYNAMIC
    const int slot = ctr_slot(st);
    Q.u.tile_ctr = G.d_ctr + slot;
    Q.u.tile_base = G.ctr_base[slot];
    G.ctr_base[slot] += tiles + g;
#endif
    adam_update_rs_tma_kernel<MODE, CLIP><<<g, kRsTmaThreads, rs_tma_smem_bytes(nmax), st>>>(Q);
    return;
  }
#endif
  uint64_t tiles = 0;
  for (int r = 0; r < Q.u.nr; ++r) tiles += ((Q.u.r[r].n & ~7ull) + kRsTile - 1) / kRsTile;
  const unsigned g = static_cast<unsigned>(
      std::max<uint64_t>(1, std::min<uint64_t>(tiles, static_cast<uint64_t>(G.rs_grid))));
#if RATEL_TMA_DYNAMIC
  const int slot = ctr_slot(st);
  Q.u.tile_ctr = G.d_ctr + slot;
  Q.u.tile_base = G.ctr_base[slot];
  G.ctr_base[slot] += tiles + g;
#endif
  adam_update_rs_kernel<MODE, CLIP><<<g, kThreads, 0, st>>>(Q);
}

// gp != nullptr: the fused-reduction kernel (gp[i] = the rank grads of rd[i]).
// kernel: ratel_k1_kernel to use, -1 = cfg.k1_kernel.
int launch_update(const RangeDesc* rd, int nr, cudaStream_t st, const PeerDesc* pd = nullptr,
                  const GradPeers* gp = nullptr, int kernel = -1) {
  if (kernel < 0) kernel = G.cfg.k1_kernel;
  if (nr == 0) return RATEL_OK;
  std::lock_guard<std::mutex> lk(g_launch_mu);
  UpdateParams P{};
  uint64_t max8 = 0;
  for (int i = 0; i < nr; ++i) {
    P.r[i] = rd[i];
    if (pd != nullptr) {
      P.peers[i] = pd[i];
      if (pd[i].n > 0) P.any_peers = 1;
    }
    max8 = std::max<uint64_t>(max8, (rd[i].n + 7) / 8);
  }
  P.nr = nr;
  P.s = G.scal;
  const bool clip = G.cfg.max_grad_norm > 0.0;
  P.sumsq = G.comm != nullptr ? G.d_sumsq + 1 : G.d_sumsq;
  P.max_norm = G.cfg.max_grad_norm;
  P.nonfinite_flag = G.d_flag;
  const uint64_t want = std::max<uint64_t>(1, (max8 + kThreads - 1) / kThreads);
  const unsigned grid = static_cast<unsigned>(
      std::min<uint64_t>(want, static_cast<uint64_t>(gp != nullptr ? G.rs_grid : G.k1_grid)));
  TimingPair* tp = nullptr;
  if (G.cfg.timing) {
    if (G.tused == G.tpool.size()) {
      TimingPair t;
      CK(cudaEventCreate(&t.a));
      CK(cudaEventCreate(&t.b));
      G.tpool.push_back(t);
    }
    tp = &G.tpool[G.tused++];
    CK(cudaEventRecord(tp->a, st));
  }
  if (gp != nullptr) {
    static RsUpdateParams Q;  // 6.5 KB: static, not on the host stack (the API is not reentrant)
    Q = RsUpdateParams{};
    Q.u = P;
    for (int i = 0; i < nr; ++i) Q.gp[i] = gp[i];
    if (G.cfg.mode == RATEL_ADAMW)
      clip ? launch_k1_rs<RATEL_ADAMW, true>(Q, grid, st) : launch_k1_rs<RATEL_ADAMW, false>(Q, grid, st);
    else
      clip ? launch_k1_rs<RATEL_ADAM_L2, true>(Q, grid, st) : launch_k1_rs<RATEL_ADAM_L2, false>(Q, grid, st);
  } else if (G.cfg.mode == RATEL_ADAMW) {
    clip ? launch_k1<RATEL_ADAMW, true>(P, grid, st, kernel) : launch_k1<RATEL_ADAMW, false>(P, grid, st, kernel);
  } else {
    clip ? launch_k1<RATEL_ADAM_L2, true>(P, grid, st, kernel) : launch_k1<RATEL_ADAM_L2, false>(P, grid, st, kernel);
  }
  CK(cudaGetLastError());
  ++G.launches;
  if (tp) CK(cudaEventRecord(tp->b, st));
  return RATEL_OK;
}

// Rank grads of range i of B at element `off` of this rank's slice: every
// rank's G16 for a range with peer grads, else this rank's own (n = 1,
// scale = 1, which the fused kernels reduce to the plain gradient bit for bit).
GradPeers grad_peers(const Block& B, size_t i, uint64_t off) {
  GradPeers d{};
  const Slice& s = B.slices[i];
  if (i < B.rgrads.size() && !B.rgrads[i].empty()) {
    for (int q = 0; q < G.world; ++q) {
      const uint16_t* base = q == G.rank ? static_cast<const uint16_t*>(B.ranges[i].grad_bf16) : B.rgrads[i][q];
      d.g[q] = base + s.begin + off;
    }
    d.n = G.world;
    d.scale = B.rscale[i];
  } else {
    d.g[0] = grad_ptr(B.ranges[i], s) + off;
    d.n = 1;
    d.scale = 1.0;
  }
  return d;
}

int launch_sumsq(const Block& B) {
  if (B.rs) {
    static RsSumsqParams S;
    S = RsSumsqParams{};
    int nr = 0;
    for (size_t i = 0; i < B.ranges.size(); ++i) {
      const Slice& s = B.slices[i];
      if (s.end == s.begin) continue;
      S.gp[nr] = grad_peers(B, i, 0);
      S.n[nr] = s.end - s.begin;
      ++nr;
    }
    S.nr = nr;
    S.partials = G.d_partials + static_cast<size_t>(B.order) * G.k2_grid;
    grad_sumsq_rs_kernel<<<G.k2_grid, kThreads, 0, G.s_opt>>>(S);
    CK(cudaGetLastError());
    ++G.launches;
    return RATEL_OK;
  }
  SumsqParams S{};
  int nr = 0;
  for (size_t i = 0; i < B.ranges.size(); ++i) {
    const Slice& s = B.slices[i];
    if (s.end == s.begin) continue;
    S.g[nr] = grad_ptr(B.ranges[i], s);
    S.n[nr] = s.end - s.begin;
    ++nr;
  }
  S.nr = nr;
  S.partials = G.d_partials + static_cast<size_t>(B.order) * G.k2_grid;
  grad_sumsq_kernel<<<G.k2_grid, kThreads, 0, G.s_opt>>>(S);
  CK(cudaGetLastError());
  ++G.launches;
  return RATEL_OK;
}

// Peer P16 pointers of range i of B, offset to element `off` of this rank's
// slice (empty when the range uses the NCCL all-gather).
PeerDesc peer_desc(const Block& B, size_t i, uint64_t off) {
  PeerDesc d{};
  if (i < B.peers.size() && !B.peers[i].empty()) {
    for (int q = 0; q < G.world; ++q) {
      if (q == G.rank || B.peers[i][q] == nullptr) continue;
      d.p[d.n++] = B.peers[i][q] + B.slices[i].begin + off;
    }
  }
  return d;
}

bool has_peers(const Block& B, size_t i) { return i < B.peers.size() && !B.peers[i].empty(); }

// One staged tile of a pinned-host range: H2D(theta, m, v) -> K1 -> D2H.
// RATEL_STAGING_ZERO_COPY: the register-staged update kernel reads and
// writes the range's page-locked host states in place (unified addressing:
// the host pointer is a valid device address), so theta/m/v cross the host
// link exactly once each way with no device tiles, copy engines or extra HBM
// traffic; the grid is cfg.max_ctas (default all SMs x the lite kernel's
// occupancy) of no-shared-memory CTAs.
int update_in_place_over_link(const Block& B, size_t ri) {
  const ratel_range& r = B.ranges[ri];
  const Slice& s = B.slices[ri];
  const uint64_t n = s.end - s.begin;
  if (n == 0) return RATEL_OK;
  RangeDesc rd{};
  rd.g = grad_ptr(r, s);
  rd.th = r.master;
  rd.m = r.exp_avg;
  rd.v = r.exp_avg_sq;
  rd.p = static_cast<uint16_t*>(r.param_bf16) + s.begin;
  rd.n = n;
  rd.wd_on = r.apply_weight_decay != 0;
  GradPeers gp{};
  if (B.rs) gp = grad_peers(B, ri, 0);
  const PeerDesc pd = peer_desc(B, ri, 0);
  return launch_update(&rd, 1, G.s_tile, &pd, B.rs ? &gp : nullptr, RATEL_UPDATE_LDG_LITE);
}

int stage_tile(const Block& B, size_t ri, uint64_t off, uint64_t len) {
  Nvtx nv("ratel tile %llu", static_cast<unsigned long long>(G.ring_k));
  const ratel_range& r = B.ranges[ri];
  const Slice& s = B.slices[ri];
  const int k = static_cast<int>(G.ring_k % static_cast<uint64_t>(G.cfg.pipeline_depth));
  const uint64_t T = G.cfg.tile_elems;
  float* th = G.d_tiles + (3ull * k + 0) * T;
  float* m = G.d_tiles + (3ull * k + 1) * T;
  float* v = G.d_tiles + (3ull * k + 2) * T;
  const size_t bytes = len * sizeof(float);
  RangeDesc rd{};
  rd.g = grad_ptr(r, s) + off;
  rd.th = th;
  rd.m = m;
  rd.v = v;
  rd.p = static_cast<uint16_t*>(r.param_bf16) + s.begin + off;
  rd.n = len;
  rd.wd_on = r.apply_weight_decay != 0;
  GradPeers gp{};
  if (B.rs) gp = grad_peers(B, ri, off);
  const bool serial = G.cfg.staging == RATEL_STAGING_SERIALIZED;
  cudaStream_t in = serial ? G.s_tile : G.s_h2d;
  cudaStream_t out = serial ? G.s_tile : G.s_d2h;
  if (!serial && G.ring_k >= static_cast<uint64_t>(G.cfg.pipeline_depth))
    CK(cudaStreamWaitEvent(in, G.ev_d2h[k], 0));  // slot free: its previous write-back done
  CK(cudaMemcpyAsync(th, r.master + off, bytes, cudaMemcpyHostToDevice, in));
  CK(cudaMemcpyAsync(m, r.exp_avg + off, bytes, cudaMemcpyHostToDevice, in));
  CK(cudaMemcpyAsync(v, r.exp_avg_sq + off, bytes, cudaMemcpyHostToDevice, in));
  if (!serial) {
    CK(cudaEventRecord(G.ev_h2d[k], in));
    CK(cudaStreamWaitEvent(G.s_tile, G.ev_h2d[k], 0));
  }
  const PeerDesc pd = peer_desc(B, ri, off);
  RK(launch_update(&rd, 1, G.s_tile, &pd, B.rs ? &gp : nullptr));
  if (!serial) {
    CK(cudaEventRecord(G.ev_k1[k], G.s_tile));
    CK(cudaStreamWaitEvent(out, G.ev_k1[k], 0));
  }
  CK(cudaMemcpyAsync(r.master + off, th, bytes, cudaMemcpyDeviceToHost, out));
  CK(cudaMemcpyAsync(r.exp_avg + off, m, bytes, cudaMemcpyDeviceToHost, out));
  CK(cudaMemcpyAsync(r.exp_avg_sq + off, v, bytes, cudaMemcpyDeviceToHost, out));
  if (!serial) CK(cudaEventRecord(G.ev_d2h[k], out));
  ++G.ring_k;
  return RATEL_OK;
}

int allgather_block(const Block& B) {
  bool any = false;
  for (size_t i = 0; i < B.ranges.size(); ++i) any = any || !has_peers(B, i);
  if (!any) return RATEL_OK;  // every range is gathered by the update kernel's peer stores
  CK(cudaStreamWaitEvent(G.s_comm, B.ev_done, 0));
  NK(g_nccl.GroupStart());
  for (size_t i = 0; i < B.ranges.size(); ++i) {
    if (has_peers(B, i)) continue;
    const ratel_range& r = B.ranges[i];
    const uint64_t s = padded(r.numel, G.world) / G.world;
    uint16_t* p = static_cast<uint16_t*>(r.param_bf16);
    NK(g_nccl.AllGather(p + s * G.rank, p, s, ncclBfloat16, G.comm, G.s_comm));
  }
  NK(g_nccl.GroupEnd());
  return RATEL_OK;
}

void CUDART_CB host_adam_cb(void* arg) {
  HostTask* t = static_cast<HostTask*>(arg);
  Nvtx nv("ratel host handler (%zu ranges)", t->ranges.size());
  double coef = 1.0;
  if (t->sumsq != nullptr) {  // torch clip_grad_norm_: min(1, max/(||g||+1e-6)), NaN propagates
    const double c = t->max_norm / (std::sqrt(*t->sumsq) + 1e-6);
    coef = (c < 1.0 || std::isnan(c)) ? c : 1.0;
    if (!std::isfinite(*t->sumsq)) *G.h_flag = 1;  // reported by a blocking ratel_sync (no kernel may see it)
  }
  for (HostAdamArgs& a : t->ranges) {
    a.coef = coef;
    host_adam_range(a, t->threads);
  }
  delete t;
}

// The paper-literal handler: G16 device->host, CPU AdamW on the host states,
// P16 host->device -- all stream-ordered (cudaLaunchHostFunc), no host blocking.
int enqueue_host_compute(Block& B) {
  CK(cudaStreamWaitEvent(G.s_hc_d2h, B.ev_grad, 0));
  HostTask* task = new HostTask();
  task->threads = G.cfg.host_threads;
  if (G.cfg.max_grad_norm > 0.0) {
    task->sumsq = G.h_sumsq;
    task->max_norm = G.cfg.max_grad_norm;
  }
  for (size_t i = 0; i < B.ranges.size(); ++i) {
    const ratel_range& r = B.ranges[i];
    const Slice& s = B.slices[i];
    const uint64_t n = s.end - s.begin;
    if (n == 0) continue;
    if (cudaMemcpyAsync(B.h_g[i], grad_ptr(r, s), n * 2, cudaMemcpyDeviceToHost, G.s_hc_d2h) != cudaSuccess) {
      delete task;
      return sticky_fail(RATEL_ECUDA, "G16 D2H failed: %s", cudaGetErrorString(cudaGetLastError()));
    }
    HostAdamArgs a{};
    a.g = B.h_g[i];
    a.th = r.master;
    a.m = r.exp_avg;
    a.v = r.exp_avg_sq;
    a.p = B.h_p[i];
    a.n = n;
    a.wd_on = r.apply_weight_decay != 0;
    a.mode = G.cfg.mode;
    a.lr = G.hp_lr;
    a.beta1 = G.hp_b1;
    a.beta2 = G.hp_b2;
    a.eps = G.hp_eps;
    a.wd = G.hp_wd;
    a.bc1 = G.hp_bc1;
    a.bc2 = G.hp_bc2;
    a.coef = 1.0;
    task->ranges.push_back(a);
  }
  cudaError_t e = cudaEventRecord(B.ev_gh, G.s_hc_d2h);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(G.s_host, B.ev_gh, 0);
  if (e == cudaSuccess) e = cudaLaunchHostFunc(G.s_host, host_adam_cb, task);
  if (e != cudaSuccess) {
    delete task;
    return sticky_fail(RATEL_ECUDA, "host handler enqueue failed: %s", cudaGetErrorString(e));
  }
  // P16 host->device on its own copy stream, so the host stream goes straight
  // on to the next block's CPU update while this block's P16 crosses the link.
  CK(cudaEventRecord(B.ev_hc, G.s_host));
  CK(cudaStreamWaitEvent(G.s_hc_h2d, B.ev_hc, 0));
  for (size_t i = 0; i < B.ranges.size(); ++i) {
    const Slice& s = B.slices[i];
    const uint64_t n = s.end - s.begin;
    if (n == 0) continue;
    CK(cudaMemcpyAsync(static_cast<uint16_t*>(B.ranges[i].param_bf16) + s.begin, B.h_p[i], n * 2,
                       cudaMemcpyHostToDevice, G.s_hc_h2d));
  }
  CK(cudaEventRecord(B.ev_done, G.s_hc_h2d));
  return RATEL_OK;
}

// ---------------------------------------------------------------- SSD tier
// The paper's storage pipeline (Fig. 3b): per tile, read
// theta/m/v from the state file (reader thread, pread), H2D, the update
// kernel, D2H, write back (writer thread, pwrite).  The reader runs ahead by
// up to pipeline_depth tiles, so the read of tile k+1, the GPU work of tile k
// and the write-back of tile k-1 overlap; the file sees reads and writes
// concurrently (its queue decides the mix -- the paper's SSD is simplex and
// orders write-back of i after read of i-1).
constexpr uint64_t kSsdAlign = 4096;
uint64_t ssd_stride(uint64_t len) { return (len * 4 + kSsdAlign - 1) / kSsdAlign * kSsdAlign; }

double now_s() {
  timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return ts.tv_sec + 1e-9 * ts.tv_nsec;
}

bool ssd_simplex() { return G.cfg.ssd_schedule == RATEL_SSD_SIMPLEX; }

// Simplex schedule: take / release the one-transfer-at-a-time disk token.
void disk_acquire(SsdEngine& E) {
  if (!ssd_simplex()) return;
  std::unique_lock<std::mutex> lk(E.mu);
  E.cv.wait(lk, [&] { return !E.disk_busy; });
  E.disk_busy = true;
}
void disk_release(SsdEngine& E, bool read_done) {
  {
    std::lock_guard<std::mutex> lk(E.mu);
    if (ssd_simplex()) E.disk_busy = false;
    if (read_done) ++E.tiles_read;
  }
  E.cv.notify_all();
}

int io_full(bool rd, int fd, void* buf, uint64_t bytes, uint64_t off, std::string& msg) {
  uint8_t* p = static_cast<uint8_t*>(buf);
  while (bytes > 0) {
    const ssize_t r = rd ? pread(fd, p, bytes, static_cast<off_t>(off)) : pwrite(fd, p, bytes, static_cast<off_t>(off));
    if (r < 0 && errno == EINTR) continue;
    if (r <= 0) {
      msg = std::string(rd ? "pread" : "pwrite") + " of the SSD state file failed at offset " + std::to_string(off) +
            ": " + (r < 0 ? strerror(errno) : "unexpected end of file");
      return RATEL_EIO;
    }
    p += r;
    bytes -= static_cast<uint64_t>(r);
    off += static_cast<uint64_t>(r);
  }
  return RATEL_OK;
}

// The three arrays (theta, m, v) of one staged tile: file <-> pinned staging,
// by pread/pwrite one request at a time or through the thread's io_uring.
int io_tile(SsdEngine& E, IoRing& ring, bool rd, int fd, float* h, uint64_t T, uint64_t bytes, uint64_t foff,
            uint64_t stride, std::string& msg) {
  if (G.cfg.ssd_io == RATEL_SSD_IO_URING) {
    std::vector<IoRing::Req> reqs;
    for (int a = 0; a < 3; ++a) reqs.push_back({h + a * T, bytes, foff + a * stride});
    return ring.transfer(rd, fd, reqs, msg) == 0 ? RATEL_OK : RATEL_EIO;
  }
  (void)E;
  for (int a = 0; a < 3; ++a) {
    const int rc = io_full(rd, fd, h + a * T, bytes, foff + a * stride, msg);
    if (rc != RATEL_OK) return rc;
  }
  return RATEL_OK;
}

#define SK(call)                                                                                         \
  do {                                                                                                   \
    cudaError_t e_ = (call);                                                                             \
    if (e_ != cudaSuccess) {                                                                             \
      msg = std::string(#call) + " failed: " + cudaGetErrorString(e_);                                   \
      return RATEL_ECUDA;                                                                                \
    }                                                                                                    \
  } while (0)

// One block: every tile of every range of this rank's slices.
// RATEL_SSD_HOST_COMPUTE: the paper's own pipeline -- G16 to host, per tile
// file -> pinned staging, the CPU handler updates it there, the writer puts it
// back; P16 to the device at the end.  Runs on the reader thread (the CPU
// update of a tile is an order of magnitude shorter than reading it).
int ssd_run_job_cpu(SsdEngine& E, Block& B, std::string& msg) {
  const uint64_t T = G.cfg.tile_elems;
  const int D = G.cfg.pipeline_depth;
  for (size_t i = 0; i < B.ranges.size(); ++i) {
    const Slice& s = B.slices[i];
    const uint64_t n = s.end - s.begin;
    if (n) SK(cudaMemcpyAsync(B.h_g[i], grad_ptr(B.ranges[i], s), n * 2, cudaMemcpyDeviceToHost, E.s_in));
  }
  double coef = 1.0;
  if (G.cfg.max_grad_norm > 0.0) {  // torch clip_grad_norm_: min(1, max/(||g||+1e-6)), NaN propagates
    double S = 0.0;
    SK(cudaStreamWaitEvent(E.s_in, G.ev_norm, 0));
    SK(cudaMemcpyAsync(&S, G.comm != nullptr ? G.d_sumsq + 1 : G.d_sumsq, sizeof S, cudaMemcpyDeviceToHost, E.s_in));
    SK(cudaStreamSynchronize(E.s_in));
    const double c = G.cfg.max_grad_norm / (std::sqrt(S) + 1e-6);
    coef = (c < 1.0 || std::isnan(c)) ? c : 1.0;
    if (!std::isfinite(S)) *G.h_flag = 1;  // reported by a blocking ratel_sync
  }
  SK(cudaStreamSynchronize(E.s_in));  // G16 in host staging
  for (size_t i = 0; i < B.ranges.size(); ++i) {
    const ratel_range& r = B.ranges[i];
    const Slice& s = B.slices[i];
    const Block::SsdRange& f = B.ssd[i];
    const uint64_t n = s.end - s.begin;
    for (uint64_t off = 0; off < n; off += T) {
      const uint64_t len = std::min<uint64_t>(T, n - off);
      const int slot = static_cast<int>(E.ring_k % static_cast<uint64_t>(D));
      {
        std::unique_lock<std::mutex> lk(E.mu);
        E.cv.wait(lk, [&] { return !E.slot_busy[slot] || E.err != 0; });
        if (E.err) return E.err;
      }
      float* h = E.h_ring + 3ull * slot * T;
      const uint64_t bytes = (len * 4 + kSsdAlign - 1) / kSsdAlign * kSsdAlign;
      disk_acquire(E);
      const double t0 = now_s();
      {
        const int rc = io_tile(E, E.rd_ring, true, f.fd, h, T, bytes, f.off + off * 4, f.stride, msg);
        if (rc != RATEL_OK) {
          disk_release(E, false);
          return rc;
        }
      }
      E.read_s += now_s() - t0;
      disk_release(E, true);
      E.read_bytes += 3 * bytes;
      HostAdamArgs a{};
      a.g = B.h_g[i] + off;
      a.th = h;
      a.m = h + T;
      a.v = h + 2 * T;
      a.p = B.h_p[i] + off;
      a.n = len;
      a.wd_on = r.apply_weight_decay != 0;
      a.mode = G.cfg.mode;
      a.lr = G.hp_lr;
      a.beta1 = G.hp_b1;
      a.beta2 = G.hp_b2;
      a.eps = G.hp_eps;
      a.wd = G.hp_wd;
      a.bc1 = G.hp_bc1;
      a.bc2 = G.hp_bc2;
      a.coef = coef;
      host_adam_range(a, G.cfg.host_threads);
      {
        std::lock_guard<std::mutex> lk(E.mu);
        E.slot_busy[slot] = 1;
        SsdTile t;
        t.seq = E.ring_k;
        t.slot = slot;
        t.fd = f.fd;
        t.foff = f.off + off * 4;
        t.stride = f.stride;
        t.bytes = bytes;
        t.host = true;
        E.wq.push_back(t);
        ++E.tiles_in;
      }
      E.cv.notify_all();
      ++E.ring_k;
    }
  }
  for (size_t i = 0; i < B.ranges.size(); ++i) {
    const Slice& s = B.slices[i];
    const uint64_t n = s.end - s.begin;
    if (n)
      SK(cudaMemcpyAsync(static_cast<uint16_t*>(B.ranges[i].param_bf16) + s.begin, B.h_p[i], n * 2,
                         cudaMemcpyHostToDevice, E.s_in));
  }
  SK(cudaEventRecord(B.ev_done, E.s_in));
  return RATEL_OK;
}

int ssd_run_job(SsdEngine& E, const SsdJob& job, std::string& msg) {
  for (cudaEvent_t ev : job.wait) SK(cudaEventSynchronize(ev));  // the active message: the gradient exists
  Block& B = G.blocks[job.block];
  if (B.ssd_cpu) return ssd_run_job_cpu(E, B, msg);
  const uint64_t T = G.cfg.tile_elems;
  const int D = G.cfg.pipeline_depth;
  bool first = true;
  for (size_t i = 0; i < B.ranges.size(); ++i) {
    const ratel_range& r = B.ranges[i];
    const Slice& s = B.slices[i];
    const Block::SsdRange& f = B.ssd[i];
    const uint64_t n = s.end - s.begin;
    for (uint64_t off = 0; off < n; off += T) {
      const uint64_t len = std::min<uint64_t>(T, n - off);
      const int slot = static_cast<int>(E.ring_k % static_cast<uint64_t>(D));
      {
        std::unique_lock<std::mutex> lk(E.mu);
        E.cv.wait(lk, [&] { return !E.slot_busy[slot] || E.err != 0; });
        if (E.err) return E.err;
      }
      float* h = E.h_ring + 3ull * slot * T;
      float* d = E.d_ring + 3ull * slot * T;
      const uint64_t bytes = (len * 4 + kSsdAlign - 1) / kSsdAlign * kSsdAlign;
      disk_acquire(E);
      const double t0 = now_s();
      {
        const int rc = io_tile(E, E.rd_ring, true, f.fd, h, T, bytes, f.off + off * 4, f.stride, msg);
        if (rc != RATEL_OK) {
          disk_release(E, false);
          return rc;
        }
      }
      E.read_s += now_s() - t0;
      disk_release(E, true);
      E.read_bytes += 3 * bytes;
      for (int a = 0; a < 3; ++a) SK(cudaMemcpyAsync(d + a * T, h + a * T, len * 4, cudaMemcpyHostToDevice, E.s_in));
      SK(cudaEventRecord(E.ev_h2d[slot], E.s_in));
      SK(cudaStreamWaitEvent(E.s_k, E.ev_h2d[slot], 0));
      if (first) {
        SK(cudaStreamWaitEvent(E.s_k, B.ev_grad, 0));
        if (G.cfg.max_grad_norm > 0.0) SK(cudaStreamWaitEvent(E.s_k, G.ev_norm, 0));
        first = false;
      }
      RangeDesc rd{};
      rd.g = grad_ptr(r, s) + off;
      rd.th = d;
      rd.m = d + T;
      rd.v = d + 2 * T;
      rd.p = static_cast<uint16_t*>(r.param_bf16) + s.begin + off;
      rd.n = len;
      rd.wd_on = r.apply_weight_decay != 0;
      if (launch_update(&rd, 1, E.s_k) != RATEL_OK) {
        msg = t_err;
        return RATEL_ECUDA;
      }
      SK(cudaEventRecord(E.ev_k1[slot], E.s_k));
      SK(cudaStreamWaitEvent(E.s_out, E.ev_k1[slot], 0));
      for (int a = 0; a < 3; ++a) SK(cudaMemcpyAsync(h + a * T, d + a * T, len * 4, cudaMemcpyDeviceToHost, E.s_out));
      SK(cudaEventRecord(E.ev_d2h[slot], E.s_out));
      {
        std::lock_guard<std::mutex> lk(E.mu);
        E.slot_busy[slot] = 1;
        SsdTile t;
        t.seq = E.ring_k;
        t.slot = slot;
        t.fd = f.fd;
        t.foff = f.off + off * 4;
        t.stride = f.stride;
        t.bytes = bytes;
        E.wq.push_back(t);
        ++E.tiles_in;
      }
      E.cv.notify_all();
      ++E.ring_k;
    }
  }
  if (first) {  // no tile on this rank: still order ev_done after the gradient
    SK(cudaStreamWaitEvent(E.s_k, B.ev_grad, 0));
  }
  SK(cudaEventRecord(B.ev_done, E.s_k));
  return RATEL_OK;
}

void ssd_fail(SsdEngine& E, int rc, const std::string& m) {
  std::lock_guard<std::mutex> lk(E.mu);
  if (!E.err) {
    E.err = rc;
    E.msg = m;
  }
}

void ssd_reader_main(SsdEngine* E) {
  cudaSetDevice(G.device);
  for (;;) {
    SsdJob job;
    {
      std::unique_lock<std::mutex> lk(E->mu);
      E->reader_idle = true;
      E->cv.notify_all();  // a simplex write-back may be waiting for "no read pending"
      E->cv.wait(lk, [&] { return E->stop || !E->jobs.empty(); });
      if (E->jobs.empty()) {  // stop
        E->reader_done = true;
        lk.unlock();
        E->cv.notify_all();
        return;
      }
      job = E->jobs.front();
      E->jobs.pop_front();
      E->reader_idle = false;
    }
    bool failed;
    {
      std::lock_guard<std::mutex> lk(E->mu);
      failed = E->err != 0;
    }
    if (!failed) {
      std::string m;
      const int rc = ssd_run_job(*E, job, m);
      if (rc != RATEL_OK) ssd_fail(*E, rc, "SSD reader: " + m);
    }
    {
      std::lock_guard<std::mutex> lk(E->mu);
      ++E->jobs_out;
    }
    E->cv.notify_all();
  }
}

void ssd_writer_main(SsdEngine* E) {
  cudaSetDevice(G.device);
  const uint64_t T = G.cfg.tile_elems;
  for (;;) {
    SsdTile t;
    bool failed;
    {
      std::unique_lock<std::mutex> lk(E->mu);
      // exit only once the reader has stopped: a job still in flight may be
      // waiting for a ring slot that only this thread's write-back frees
      E->cv.wait(lk, [&] { return (E->stop && E->reader_done) || !E->wq.empty(); });
      if (E->wq.empty()) return;  // stop
      t = E->wq.front();
      E->wq.pop_front();
      failed = E->err != 0;
    }
    if (!failed && ssd_simplex()) {
      // the paper's simplex order: write tile k back only after tile k+1 was
      // read (or no read is pending), and never during another transfer
      std::unique_lock<std::mutex> lk(E->mu);
      E->cv.wait(lk, [&] {
        const bool next_read = E->tiles_read > t.seq + 1 ||
                               (E->reader_idle && E->jobs.empty()) || E->err != 0;
        return next_read && !E->disk_busy;
      });
      E->disk_busy = true;
    }
    if (!failed) {
      std::string m;
      int rc = RATEL_OK;
      const cudaError_t e = t.host ? cudaSuccess : cudaEventSynchronize(E->ev_d2h[t.slot]);  // states back in the slot
      if (e != cudaSuccess) {
        rc = RATEL_ECUDA;
        m = std::string("cudaEventSynchronize(d2h) failed: ") + cudaGetErrorString(e);
      }
      const float* h = E->h_ring + 3ull * t.slot * T;
      const double t0 = now_s();
      if (rc == RATEL_OK)
        rc = io_tile(*E, E->wr_ring, false, t.fd, const_cast<float*>(h), T, t.bytes, t.foff, t.stride, m);
      E->write_s += now_s() - t0;
      E->write_bytes += 3 * t.bytes;
      if (ssd_simplex()) disk_release(*E, false);
      if (rc != RATEL_OK) ssd_fail(*E, rc, "SSD writer: " + m);
    }
    {
      std::lock_guard<std::mutex> lk(E->mu);
      E->slot_busy[t.slot] = 0;
      ++E->tiles_out;
    }
    E->cv.notify_all();
  }
}

int ssd_create() {
  SsdEngine* E = new SsdEngine();
  G.ssd = E;  // destroy_all() tears down whatever was created
  if (G.cfg.ssd_io == RATEL_SSD_IO_URING) {
    for (IoRing* r : {&E->rd_ring, &E->wr_ring}) {
      const int e = r->open_ring(32);
      if (e != 0)
        return set_error(RATEL_EIO, "ratel_register_block: cfg.ssd_io = RATEL_SSD_IO_URING but io_uring_setup "
                                    "failed: %s", strerror(-e));
    }
  }
  const size_t n = static_cast<size_t>(G.cfg.pipeline_depth) * 3 * G.cfg.tile_elems;
  CK(cudaHostAlloc(&E->h_ring, n * sizeof(float), cudaHostAllocDefault));
  CK(cudaMalloc(&E->d_ring, n * sizeof(float)));
  int least = 0, greatest = 0;
  CK(cudaDeviceGetStreamPriorityRange(&least, &greatest));
  CK(cudaStreamCreateWithPriority(&E->s_in, cudaStreamNonBlocking, greatest));
  CK(cudaStreamCreateWithPriority(&E->s_k, cudaStreamNonBlocking, greatest));
  CK(cudaStreamCreateWithPriority(&E->s_out, cudaStreamNonBlocking, greatest));
  for (int k = 0; k < kMaxDepth; ++k) {
    CK(cudaEventCreateWithFlags(&E->ev_h2d[k], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&E->ev_k1[k], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&E->ev_d2h[k], cudaEventDisableTiming | cudaEventBlockingSync));
  }
  E->reader = std::thread(ssd_reader_main, E);
  E->writer = std::thread(ssd_writer_main, E);
  return RATEL_OK;
}

void ssd_destroy() {
  SsdEngine* E = G.ssd;
  if (E == nullptr) return;
  {
    std::lock_guard<std::mutex> lk(E->mu);
    E->stop = true;
  }
  E->cv.notify_all();
  if (E->reader.joinable()) E->reader.join();
  if (E->writer.joinable()) E->writer.join();
  for (cudaStream_t s : {E->s_in, E->s_k, E->s_out})
    if (s) cudaStreamSynchronize(s);
  for (int k = 0; k < kMaxDepth; ++k) {
    if (E->ev_h2d[k]) cudaEventDestroy(E->ev_h2d[k]);
    if (E->ev_k1[k]) cudaEventDestroy(E->ev_k1[k]);
    if (E->ev_d2h[k]) cudaEventDestroy(E->ev_d2h[k]);
  }
  for (cudaStream_t s : {E->s_in, E->s_k, E->s_out})
    if (s) cudaStreamDestroy(s);
  if (E->h_ring) cudaFreeHost(E->h_ring);
  if (E->d_ring) cudaFree(E->d_ring);
  delete E;
  G.ssd = nullptr;
}

// Hand block B to the reader (hand-off / arm time).  `wait`: events the
// reader host-waits before touching B's states.
int ssd_submit(Block& B, int id, std::vector<cudaEvent_t> wait) {
  SsdEngine& E = *G.ssd;
  {
    std::lock_guard<std::mutex> lk(E.mu);
    SsdJob j;
    j.block = id;
    j.wait = std::move(wait);
    E.jobs.push_back(std::move(j));
    B.ssd_seq = ++E.jobs_in;
  }
  E.cv.notify_all();
  return RATEL_OK;
}

// Wait until the reader issued every submitted job (and, if `writes`, the
// writer finished every write-back); report an engine failure as sticky.
int ssd_drain(bool writes, uint64_t upto_job = 0) {
  if (G.ssd == nullptr) return RATEL_OK;
  SsdEngine& E = *G.ssd;
  std::unique_lock<std::mutex> lk(E.mu);
  const uint64_t want = upto_job ? upto_job : E.jobs_in;
  E.cv.wait(lk, [&] { return E.err != 0 || (E.jobs_out >= want && (!writes || E.tiles_out == E.tiles_in)); });
  if (E.err) {
    // let the threads finish draining their queues before reporting
    E.cv.wait(lk, [&] { return E.jobs_out == E.jobs_in && E.tiles_out == E.tiles_in; });
    const std::string m = E.msg;
    const int rc = E.err;
    lk.unlock();
    return sticky_fail(rc, "%s", m.c_str());
  }
  return RATEL_OK;
}

// Enqueue the handler of block B (its s_opt wait on ev_grad was issued at
// hand-off).  Device residency: one K1 launch over the rank's slices of all
// ranges.  Pinned-host: the tile ring.
int enqueue_block(Block& B, const std::vector<cudaEvent_t>* ssd_wait = nullptr) {
  if (B.residency == RATEL_SSD) {
    const int id = static_cast<int>(&B - G.blocks.data());
    RK(ssd_submit(B, id, ssd_wait ? *ssd_wait : std::vector<cudaEvent_t>{B.ev_grad}));
    B.enqueued = true;
    return RATEL_OK;
  }
  cudaStream_t ks = G.s_opt;
  if (B.residency == RATEL_DEVICE) {
    // Alternate update streams: this block's kernel can take the SMs the
    // previous block's tail leaves idle (one CTA per SM does not co-reside).
    if (G.cfg.update_streams > 1) {
      ks = G.s_k[G.k_next++ & 1u];
      CK(cudaStreamWaitEvent(ks, B.ev_grad, 0));
      if ((B.rs || B.pp) && G.comm != nullptr) CK(cudaStreamWaitEvent(ks, B.ev_ready, 0));
      if (G.cfg.max_grad_norm > 0.0) CK(cudaStreamWaitEvent(ks, G.ev_norm, 0));
    }
    RangeDesc rd[kMaxRanges];
    PeerDesc pd[kMaxRanges];
    GradPeers gp[kMaxRanges];
    int nr = 0;
    for (size_t i = 0; i < B.ranges.size(); ++i) {
      const ratel_range& r = B.ranges[i];
      const Slice& s = B.slices[i];
      if (s.end == s.begin) continue;
      if (B.rs) gp[nr] = grad_peers(B, i, 0);
      pd[nr] = peer_desc(B, i, 0);
      RangeDesc& d = rd[nr++];
      d.g = grad_ptr(r, s);
      d.th = r.master;
      d.m = r.exp_avg;
      d.v = r.exp_avg_sq;
      d.p = static_cast<uint16_t*>(r.param_bf16) + s.begin;
      d.n = s.end - s.begin;
      d.wd_on = r.apply_weight_decay != 0;
      d.pad_ = 0;
    }
    RK(launch_update(rd, nr, ks, pd, B.rs ? gp : nullptr));
  } else if (B.residency == RATEL_PINNED_HOST) {
    // Tile updates run on a HIGH-priority stream: each is short and gates the
    // copy pipeline, so when a backward GEMM frees SMs they must go first.
    CK(cudaStreamWaitEvent(G.s_tile, B.ev_grad, 0));
    if ((B.rs || B.pp) && G.comm != nullptr) CK(cudaStreamWaitEvent(G.s_tile, B.ev_ready, 0));
    if (G.cfg.max_grad_norm > 0.0) CK(cudaStreamWaitEvent(G.s_tile, G.ev_norm, 0));
    for (size_t i = 0; i < B.ranges.size(); ++i) {
      const Slice& s = B.slices[i];
      const uint64_t n = s.end - s.begin;
      if (G.cfg.staging == RATEL_STAGING_ZERO_COPY) {
        RK(update_in_place_over_link(B, i));
        continue;
      }
      for (uint64_t off = 0; off < n; off += G.cfg.tile_elems)
        RK(stage_tile(B, i, off, std::min<uint64_t>(G.cfg.tile_elems, n - off)));
    }
  }
  if (B.residency == RATEL_HOST_COMPUTE)
    RK(enqueue_host_compute(B));
  else
    CK(cudaEventRecord(B.ev_done, B.residency == RATEL_PINNED_HOST ? G.s_tile : ks));
  if (ks != G.s_opt) CK(cudaStreamWaitEvent(G.s_opt, B.ev_done, 0));
  // Keep ratel_optimizer_stream() ordered after every read of this block's
  // grad (so grad.record_stream(ratel_optimizer_stream()) stays sufficient).
  if (B.residency == RATEL_PINNED_HOST) CK(cudaStreamWaitEvent(G.s_opt, B.ev_done, 0));
  if (B.residency == RATEL_HOST_COMPUTE) CK(cudaStreamWaitEvent(G.s_opt, B.ev_gh, 0));
  if (G.comm != nullptr) RK(allgather_block(B));
  B.enqueued = true;
  return RATEL_OK;
}

// Clip mode: every hand-off has run K2; reduce, allreduce, then update all.
int finalize_clip() {
  sumsq_finalize_kernel<<<1, kThreads, 0, G.s_opt>>>(G.d_partials,
                                                     static_cast<uint64_t>(G.reg.size()) * G.k2_grid,
                                                     G.d_sumsq);
  CK(cudaGetLastError());
  ++G.launches;
  if (G.comm != nullptr)
    NK(g_nccl.AllReduce(G.d_sumsq, G.d_sumsq + 1, 1, ncclFloat64, ncclSum, G.comm, G.s_opt));
  CK(cudaEventRecord(G.ev_norm, G.s_opt));  // the tile stream and the host handler wait on it
  if (G.h_sumsq != nullptr) {  // some block runs the host handler: it needs the norm on the host
    CK(cudaStreamWaitEvent(G.s_host, G.ev_norm, 0));
    CK(cudaMemcpyAsync(G.h_sumsq, G.comm != nullptr ? G.d_sumsq + 1 : G.d_sumsq, sizeof(double),
                       cudaMemcpyDeviceToHost, G.s_host));
  }
  for (int id : G.reg) RK(enqueue_block(G.blocks[id]));
  G.pending.clear();
  return RATEL_OK;
}

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

int check_ptr(const void* p, bool want_device, const char* what, int idx) {
  cudaPointerAttributes a{};
  const cudaError_t e = cudaPointerGetAttributes(&a, p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return set_error(RATEL_EINVAL, "range %d: %s is not a CUDA-visible pointer (%s)", idx, what,
                     cudaGetErrorString(e));
  }
  if (want_device) {
    if (a.type != cudaMemoryTypeDevice || a.device != G.device)
      return set_error(RATEL_EINVAL, "range %d: %s must be device memory on device %d", idx, what, G.device);
  } else if (a.type != cudaMemoryTypeHost) {
    return set_error(RATEL_EINVAL, "range %d: %s must be page-locked host memory (cudaHostAlloc/Register)",
                     idx, what);
  }
  return RATEL_OK;
}

int validate_config(const ratel_config& c) {
  if (c.mode != RATEL_ADAMW && c.mode != RATEL_ADAM_L2) return set_error(RATEL_EINVAL, "cfg.mode");
  if (!(c.max_grad_norm >= 0.0) || !std::isfinite(c.max_grad_norm))
    return set_error(RATEL_EINVAL, "cfg.max_grad_norm must be finite and >= 0");
  if (c.pipeline_depth < 2 || c.pipeline_depth > kMaxDepth)
    return set_error(RATEL_EINVAL, "cfg.pipeline_depth must be in [2, %d]", kMaxDepth);
  if (c.staging != RATEL_STAGING_PIPELINED && c.staging != RATEL_STAGING_SERIALIZED &&
      c.staging != RATEL_STAGING_ZERO_COPY)
    return set_error(RATEL_EINVAL, "cfg.staging");
  if (c.tile_elems == 0 || (c.tile_elems & 7u)) return set_error(RATEL_EINVAL, "cfg.tile_elems must be a positive multiple of 8");
  if (c.max_ctas < 0) return set_error(RATEL_EINVAL, "cfg.max_ctas must be >= 0");
  if (c.comm != RATEL_COMM_AUTO && c.comm != RATEL_COMM_NONE && c.comm != RATEL_COMM_NCCL)
    return set_error(RATEL_EINVAL, "cfg.comm");
  if (c.host_threads < 0) return set_error(RATEL_EINVAL, "cfg.host_threads must be >= 0");
  if (c.update_streams < 1 || c.update_streams > 2) return set_error(RATEL_EINVAL, "cfg.update_streams must be 1 or 2");
  if (c.cta_tiles < 0) return set_error(RATEL_EINVAL, "cfg.cta_tiles must be >= 0");
  if (c.k1_kernel != RATEL_UPDATE_TMA && c.k1_kernel != RATEL_UPDATE_LDG && c.k1_kernel != RATEL_UPDATE_LDG_LITE)
    return set_error(RATEL_EINVAL, "cfg.k1_kernel");
  if (c.ssd_schedule != RATEL_SSD_DUPLEX && c.ssd_schedule != RATEL_SSD_SIMPLEX)
    return set_error(RATEL_EINVAL, "cfg.ssd_schedule");
  if (c.ssd_io != RATEL_SSD_IO_PREAD && c.ssd_io != RATEL_SSD_IO_URING) return set_error(RATEL_EINVAL, "cfg.ssd_io");
  return RATEL_OK;
}

void reset_step_state() {
  for (int id : G.reg) {
    G.blocks[id].handed_off = false;
    G.blocks[id].enqueued = false;
  }
  G.pending.clear();
  G.n_handed = 0;
  G.armed = false;
}

void destroy_all() {
  ssd_destroy();  // joins the SSD threads before their streams and buffers go
  for (int id : G.reg) {
    Block& B = G.blocks[id];
    if (B.ev_grad) cudaEventDestroy(B.ev_grad);
    if (B.ev_done) cudaEventDestroy(B.ev_done);
    if (B.ev_gh) cudaEventDestroy(B.ev_gh);
    if (B.ev_hc) cudaEventDestroy(B.ev_hc);
    if (B.ev_ready) cudaEventDestroy(B.ev_ready);
    if (B.ev_rel) cudaEventDestroy(B.ev_rel);
    for (uint16_t* p : B.h_g) cudaFreeHost(p);
    for (uint16_t* p : B.h_p) cudaFreeHost(p);
  }
  for (TimingPair& t : G.tpool) {
    cudaEventDestroy(t.a);
    cudaEventDestroy(t.b);
  }
  for (int k = 0; k < kMaxDepth; ++k) {
    if (G.ev_h2d[k]) cudaEventDestroy(G.ev_h2d[k]);
    if (G.ev_k1[k]) cudaEventDestroy(G.ev_k1[k]);
    if (G.ev_d2h[k]) cudaEventDestroy(G.ev_d2h[k]);
  }
  for (cudaEvent_t e : G.ev_end)
    if (e) cudaEventDestroy(e);
  if (G.d_tiles) cudaFree(G.d_tiles);
  if (G.d_partials) cudaFree(G.d_partials);
  if (G.d_sumsq) cudaFree(G.d_sumsq);
  if (G.d_ctr) cudaFree(G.d_ctr);
  if (G.h_flag) cudaFreeHost(G.h_flag);
  if (G.h_sumsq) cudaFreeHost(G.h_sumsq);
  if (G.ev_norm) cudaEventDestroy(G.ev_norm);
  if (G.comm) g_nccl.CommDestroy(G.comm);
  for (cudaStream_t s : {G.s_opt, G.s_h2d, G.s_d2h, G.s_comm, G.s_host, G.s_tile, G.s_k[0], G.s_k[1],
                         G.s_hc_d2h, G.s_hc_h2d})
    if (s) cudaStreamDestroy(s);
  G.~Ctx();
  new (&G) Ctx();
}

int init_body(int device, int rank, int world_size, const void* nccl_unique_id, const ratel_config& c) {
  G.device = device;
  G.rank = rank;
  G.world = world_size;
  G.cfg = c;
  CK(cudaSetDevice(device));
  cudaDeviceProp prop{};
  CK(cudaGetDeviceProperties(&prop, device));
  if (prop.major < 10)
    return set_error(RATEL_ECUDA, "ratel_init: device %d is sm_%d%d; this library is built for sm_100a",
                     device, prop.major, prop.minor);
  G.sms = prop.multiProcessorCount;
  int least = 0, greatest = 0;
  CK(cudaDeviceGetStreamPriorityRange(&least, &greatest));
  CK(cudaStreamCreateWithPriority(&G.s_opt, cudaStreamNonBlocking, least));  // lowest priority
  CK(cudaStreamCreateWithPriority(&G.s_k[0], cudaStreamNonBlocking, least));
  CK(cudaStreamCreateWithPriority(&G.s_k[1], cudaStreamNonBlocking, least));
  CK(cudaStreamCreateWithPriority(&G.s_h2d, cudaStreamNonBlocking, greatest));
  CK(cudaStreamCreateWithPriority(&G.s_d2h, cudaStreamNonBlocking, greatest));
  CK(cudaStreamCreateWithPriority(&G.s_comm, cudaStreamNonBlocking, greatest));
  CK(cudaStreamCreateWithPriority(&G.s_host, cudaStreamNonBlocking, greatest));
  CK(cudaStreamCreateWithPriority(&G.s_tile, cudaStreamNonBlocking, greatest));
  CK(cudaStreamCreateWithPriority(&G.s_hc_d2h, cudaStreamNonBlocking, greatest));
  CK(cudaStreamCreateWithPriority(&G.s_hc_h2d, cudaStreamNonBlocking, greatest));
  CK(cudaEventCreateWithFlags(&G.ev_norm, cudaEventDisableTiming));
  for (cudaEvent_t& ev : G.ev_end) CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  for (int k = 0; k < kMaxDepth; ++k) {
    CK(cudaEventCreateWithFlags(&G.ev_h2d[k], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&G.ev_k1[k], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&G.ev_d2h[k], cudaEventDisableTiming));
  }
  int occ = 0;
  if (c.mode == RATEL_ADAMW)
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, adam_update_kernel<RATEL_ADAMW, false>, kThreads, 0));
  else
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, adam_update_kernel<RATEL_ADAM_L2, false>, kThreads, 0));
  G.k1_grid = G.sms * std::max(occ, 1);
  int occ_rs = 0;
  if (c.mode == RATEL_ADAMW)
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_rs, adam_update_rs_kernel<RATEL_ADAMW, false>, kThreads, 0));
  else
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_rs, adam_update_rs_kernel<RATEL_ADAM_L2, false>, kThreads, 0));
  G.rs_grid = G.sms * std::max(occ_rs, 1);
  if (c.max_ctas > 0) G.rs_grid = std::min(G.rs_grid, c.max_ctas);
  CK((prepare_k1<RATEL_ADAMW, false>()));
  CK((prepare_k1<RATEL_ADAMW, true>()));
  CK((prepare_k1<RATEL_ADAM_L2, false>()));
  CK((prepare_k1<RATEL_ADAM_L2, true>()));
  if (c.max_ctas > 0) G.k1_grid = std::min(G.k1_grid, c.max_ctas);
  int occ_lite = 0;
  if (c.mode == RATEL_ADAMW)
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_lite, adam_update_kernel<RATEL_ADAMW, false, 1, 4>, kThreads, 0));
  else
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_lite, adam_update_kernel<RATEL_ADAM_L2, false, 1, 4>, kThreads, 0));
  G.lite_grid = G.sms * std::max(occ_lite, 1);
  if (c.max_ctas > 0) G.lite_grid = std::min(G.lite_grid, c.max_ctas);
  G.k2_grid = G.sms * 4;
  CK(cudaMalloc(&G.d_ctr, 5 * sizeof(unsigned long long)));
  CK(cudaMemset(G.d_ctr, 0, 5 * sizeof(unsigned long long)));
  CK(cudaMalloc(&G.d_sumsq, 3 * sizeof(double)));
  CK(cudaMemset(G.d_sumsq, 0, 3 * sizeof(double)));
  G.d_barrier = G.d_sumsq + 2;
  CK(cudaHostAlloc(&G.h_flag, sizeof(int), cudaHostAllocMapped));
  *G.h_flag = 0;
  CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&G.d_flag), G.h_flag, 0));
  G.blocks.assign(RATEL_MAX_BLOCKS, Block());
  const bool want_comm = c.comm == RATEL_COMM_NCCL || (c.comm == RATEL_COMM_AUTO && world_size > 1);
  if (want_comm) {
    if (const char* m = g_nccl.load()) return set_error(RATEL_ENCCL, "ratel_init: cannot load NCCL: %s", m);
    ncclUniqueId id;
    if (nccl_unique_id != nullptr) {
      memcpy(&id, nccl_unique_id, sizeof id);
    } else {  // world_size == 1 with a forced communicator: make our own id
      NK(g_nccl.GetUniqueId(&id));
    }
    ncclComm_t comm = nullptr;
    NK(g_nccl.CommInitRank(&comm, world_size, id, rank));
    G.comm = comm;
  }
  return RATEL_OK;
}

}  // namespace

// Host-only parts of the library (the swap planner) report through the same
// thread-local message as the runtime.
int ratel::report_error(int code, const char* msg) { return set_error(code, "%s", msg); }

extern "C" {

void ratel_default_config(ratel_config* cfg) {
  if (cfg == nullptr) return;
  cfg->mode = RATEL_ADAMW;
  cfg->max_grad_norm = 0.0;
  cfg->pipeline_depth = 4;
  cfg->staging = RATEL_STAGING_PIPELINED;
  cfg->tile_elems = 1ull << 24;
  cfg->max_ctas = 0;
  cfg->timing = 0;
  cfg->comm = RATEL_COMM_AUTO;
  cfg->host_threads = 0;
  cfg->update_streams = 2;
  cfg->cta_tiles = 0;
  cfg->k1_kernel = RATEL_UPDATE_TMA;
  cfg->ssd_schedule = RATEL_SSD_DUPLEX;
  cfg->ssd_io = RATEL_SSD_IO_PREAD;
}

uint64_t ratel_padded_numel(uint64_t numel, int world_size) {
  if (world_size < 1) return 0;
  return padded(numel, world_size);
}

int ratel_rank_slice(uint64_t numel, int world_size, int rank, uint64_t* begin, uint64_t* end) {
  if (world_size < 1 || rank < 0 || rank >= world_size || begin == nullptr || end == nullptr)
    return set_error(RATEL_EINVAL, "ratel_rank_slice: bad arguments");
  const Slice s = slice_of(numel, world_size, rank);
  *begin = s.begin;
  *end = s.end;
  return RATEL_OK;
}

const char* ratel_last_error(void) { return t_err; }

int ratel_get_nccl_unique_id(void* out128) {
  if (out128 == nullptr) return set_error(RATEL_EINVAL, "ratel_get_nccl_unique_id: NULL");
  if (const char* m = g_nccl.load()) return set_error(RATEL_ENCCL, "cannot load NCCL: %s", m);
  ncclUniqueId id;
  const ncclResult_t r = g_nccl.GetUniqueId(&id);
  if (r != ncclSuccess) return set_error(RATEL_ENCCL, "ncclGetUniqueId: %s", g_nccl.GetErrorString(r));
  memcpy(out128, &id, sizeof id);
  return RATEL_OK;
}

int ratel_init(int device, int rank, int world_size, const void* nccl_unique_id, const ratel_config* cfg) {
  if (G.inited) return set_error(RATEL_ESTATE, "ratel_init: already initialised");
  if (world_size < 1 || rank < 0 || rank >= world_size)
    return set_error(RATEL_EINVAL, "ratel_init: need 0 <= rank < world_size");
  if (world_size > 1 && nccl_unique_id == nullptr && (cfg == nullptr || cfg->comm != RATEL_COMM_NONE))
    return set_error(RATEL_EINVAL, "ratel_init: world_size > 1 needs an NCCL unique id");
  ratel_config c;
  ratel_default_config(&c);
  if (cfg) c = *cfg;
  RK(validate_config(c));
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return set_error(RATEL_ECUDA, "ratel_init: no CUDA device (%s)", cudaGetErrorString(e));
  }
  if (device < 0 || device >= ndev) return set_error(RATEL_EINVAL, "ratel_init: device %d out of range", device);
  const int rc = init_body(device, rank, world_size, nccl_unique_id, c);
  if (rc != RATEL_OK) {
    char msg[1024];
    snprintf(msg, sizeof msg, "%s", t_err);
    destroy_all();  // also clears the sticky state: a failed init leaves nothing behind
    cudaGetLastError();
    return set_error(rc, "%s", msg);
  }
  G.inited = true;
  t_err[0] = '\0';
  return RATEL_OK;
}

int ratel_register_block(int block_id, const ratel_range* ranges, int n_ranges, int residency) {
  RK(entry());
  if (G.armed || G.n_handed > 0) return set_error(RATEL_ESTATE, "ratel_register_block: a step is in flight");
  if (block_id < 0 || block_id >= RATEL_MAX_BLOCKS)
    return set_error(RATEL_EINVAL, "ratel_register_block: block id %d out of range", block_id);
  if (G.blocks[block_id].registered)
    return set_error(RATEL_EINVAL, "ratel_register_block: block %d already registered", block_id);
  if (ranges == nullptr || n_ranges < 1 || n_ranges > RATEL_MAX_RANGES_PER_BLOCK)
    return set_error(RATEL_EINVAL, "ratel_register_block: need 1..%d ranges", RATEL_MAX_RANGES_PER_BLOCK);
  if (residency != RATEL_DEVICE && residency != RATEL_PINNED_HOST && residency != RATEL_HOST_COMPUTE &&
      residency != RATEL_SSD && residency != RATEL_SSD_HOST_COMPUTE)
    return set_error(RATEL_EINVAL, "ratel_register_block: bad residency %d", residency);
  const bool ssd_cpu = residency == RATEL_SSD_HOST_COMPUTE;
  if (ssd_cpu) residency = RATEL_SSD;  // the SSD tier with the CPU handler in place of the tile kernel
  if (residency == RATEL_SSD) {
    if (G.comm != nullptr)
      return set_error(RATEL_EINVAL, "ratel_register_block: RATEL_SSD blocks need a single rank without NCCL");
    if (G.cfg.tile_elems % 1024u)
      return set_error(RATEL_EINVAL, "ratel_register_block: RATEL_SSD needs cfg.tile_elems to be a multiple of 1024");
  }
  std::vector<Slice> slices(n_ranges);
  for (int i = 0; i < n_ranges; ++i) {
    const ratel_range& r = ranges[i];
    if (r.numel == 0) return set_error(RATEL_EINVAL, "range %d: numel must be > 0", i);
    slices[i] = slice_of(r.numel, G.world, G.rank);
    const bool has = slices[i].end > slices[i].begin;
    if (r.param_bf16 == nullptr || r.grad_bf16 == nullptr)
      return set_error(RATEL_EINVAL, "range %d: param/grad pointer is NULL", i);
    const bool states = residency != RATEL_SSD;  // SSD: the states are in the file (ratel_register_ssd)
    if (states && has && (r.master == nullptr || r.exp_avg == nullptr || r.exp_avg_sq == nullptr))
      return set_error(RATEL_EINVAL, "range %d: state pointer is NULL", i);
    const void* ps[5] = {r.param_bf16, r.grad_bf16, r.master, r.exp_avg, r.exp_avg_sq};
    for (const void* p : ps)
      if (p && !aligned16(p)) return set_error(RATEL_EINVAL, "range %d: pointers must be 16-byte aligned", i);
    RK(check_ptr(r.param_bf16, true, "param_bf16", i));
    RK(check_ptr(r.grad_bf16, true, "grad_bf16", i));
    if (states && has) {
      const bool dev = residency == RATEL_DEVICE;  // PINNED_HOST and HOST_COMPUTE: page-locked host
      RK(check_ptr(r.master, dev, "master", i));
      RK(check_ptr(r.exp_avg, dev, "exp_avg", i));
      RK(check_ptr(r.exp_avg_sq, dev, "exp_avg_sq", i));
    }
  }
  if (residency == RATEL_PINNED_HOST && G.d_tiles == nullptr) {
    const size_t bytes = static_cast<size_t>(G.cfg.pipeline_depth) * 3 * G.cfg.tile_elems * sizeof(float);
    CK(cudaMalloc(&G.d_tiles, bytes));
  }
  if (G.cfg.max_grad_norm > 0.0) {
    const size_t need = (G.reg.size() + 1) * static_cast<size_t>(G.k2_grid);
    if (need > G.partial_cap) {
      const size_t cap = std::max(need, 2 * G.partial_cap);
      // Partials are per-step scratch (every K2 writes its block's slots before
      // K3 reads them), so the old contents are not carried over; cudaFree
      // waits for any kernel of the previous step still reading them.
      double* p = nullptr;
      CK(cudaMalloc(&p, cap * sizeof(double)));
      if (G.d_partials) CK(cudaFree(G.d_partials));
      G.d_partials = p;
      G.partial_cap = cap;
    }
  }
  Block& B = G.blocks[block_id];
  if (ssd_cpu) {  // pinned G16 / P16 staging of the rank slices (2 + 2 B/param)
    B.h_g.assign(n_ranges, nullptr);
    B.h_p.assign(n_ranges, nullptr);
    for (int i = 0; i < n_ranges; ++i) {
      const uint64_t n = std::max<uint64_t>(8, slices[i].end - slices[i].begin);
      CK(cudaHostAlloc(&B.h_g[i], n * 2, cudaHostAllocDefault));
      CK(cudaHostAlloc(&B.h_p[i], n * 2, cudaHostAllocDefault));
    }
  }
  B.ssd_cpu = ssd_cpu;
  if (residency == RATEL_HOST_COMPUTE) {
    if (G.h_sumsq == nullptr) {
      CK(cudaHostAlloc(&G.h_sumsq, sizeof(double), cudaHostAllocDefault));
      *G.h_sumsq = 0.0;
    }
    B.h_g.assign(n_ranges, nullptr);
    B.h_p.assign(n_ranges, nullptr);
    for (int i = 0; i < n_ranges; ++i) {
      const uint64_t n = std::max<uint64_t>(8, slices[i].end - slices[i].begin);
      CK(cudaHostAlloc(&B.h_g[i], n * 2, cudaHostAllocDefault));
      CK(cudaHostAlloc(&B.h_p[i], n * 2, cudaHostAllocDefault));
    }
    CK(cudaEventCreateWithFlags(&B.ev_gh, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&B.ev_hc, cudaEventDisableTiming));
  }
  if (residency == RATEL_SSD) {
    if (G.ssd == nullptr) RK(ssd_create());
    B.ssd.assign(n_ranges, Block::SsdRange());
  }
  // (blocking sync: the SSD reader thread sleeps on ev_grad instead of spinning)
  CK(cudaEventCreateWithFlags(&B.ev_grad, cudaEventDisableTiming | cudaEventBlockingSync));
  CK(cudaEventCreateWithFlags(&B.ev_done, cudaEventDisableTiming));
  B.ranges.assign(ranges, ranges + n_ranges);
  B.slices = slices;
  B.residency = residency;
  B.order = static_cast<int>(G.reg.size());
  B.registered = true;
  G.reg.push_back(block_id);
  return RATEL_OK;
}

int ratel_register_peer_params(int block_id, int range_idx, void* const* peer_params, int n) {
  RK(entry());
  if (G.armed || G.n_handed > 0) return set_error(RATEL_ESTATE, "ratel_register_peer_params: a step is in flight");
  if (block_id < 0 || block_id >= RATEL_MAX_BLOCKS || !G.blocks[block_id].registered)
    return set_error(RATEL_EINVAL, "ratel_register_peer_params: block %d is not registered", block_id);
  Block& B = G.blocks[block_id];
  if (range_idx < 0 || range_idx >= static_cast<int>(B.ranges.size()))
    return set_error(RATEL_EINVAL, "ratel_register_peer_params: range %d out of range", range_idx);
  if (B.residency == RATEL_HOST_COMPUTE || B.residency == RATEL_SSD)
    return set_error(RATEL_EINVAL, "ratel_register_peer_params: not for HOST_COMPUTE / SSD blocks");
  if (peer_params == nullptr || n != G.world || G.world - 1 > kMaxPeers)
    return set_error(RATEL_EINVAL, "ratel_register_peer_params: need world_size (%d <= %d) pointers", G.world,
                     kMaxPeers + 1);
  std::vector<uint16_t*> v(n, nullptr);
  for (int q = 0; q < n; ++q) {
    if (q == G.rank || peer_params[q] == nullptr) continue;
    if (!aligned16(peer_params[q]))
      return set_error(RATEL_EINVAL, "ratel_register_peer_params: peer pointers must be 16-byte aligned");
    v[q] = static_cast<uint16_t*>(peer_params[q]);
  }
  if (G.comm != nullptr && B.ev_ready == nullptr) {
    CK(cudaEventCreateWithFlags(&B.ev_ready, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&B.ev_rel, cudaEventDisableTiming));
  }
  if (B.peers.size() != B.ranges.size()) B.peers.resize(B.ranges.size());
  if (B.peers[range_idx].empty()) ++G.n_peer_ranges;
  B.peers[range_idx] = v;
  B.pp = true;
  return RATEL_OK;
}

int ratel_register_peer_grads(int block_id, int range_idx, const void* const* rank_grads, int n,
                              double grad_scale) {
  RK(entry());
  if (G.armed || G.n_handed > 0) return set_error(RATEL_ESTATE, "ratel_register_peer_grads: a step is in flight");
  if (block_id < 0 || block_id >= RATEL_MAX_BLOCKS || !G.blocks[block_id].registered)
    return set_error(RATEL_EINVAL, "ratel_register_peer_grads: block %d is not registered", block_id);
  Block& B = G.blocks[block_id];
  if (range_idx < 0 || range_idx >= static_cast<int>(B.ranges.size()))
    return set_error(RATEL_EINVAL, "ratel_register_peer_grads: range %d out of range", range_idx);
  if (B.residency == RATEL_HOST_COMPUTE || B.residency == RATEL_SSD)
    return set_error(RATEL_EINVAL, "ratel_register_peer_grads: not for HOST_COMPUTE / SSD blocks");
  if (B.ranges[range_idx].grad_is_rank_slice)
    return set_error(RATEL_EINVAL, "ratel_register_peer_grads: the range's grad must be full-range (grad_is_rank_slice = 0)");
  if (rank_grads == nullptr || n != G.world || G.world > kMaxRanks)
    return set_error(RATEL_EINVAL, "ratel_register_peer_grads: need world_size (%d <= %d) pointers", G.world,
                     kMaxRanks);
  if (!(grad_scale > 0.0) || !std::isfinite(grad_scale))
    return set_error(RATEL_EINVAL, "ratel_register_peer_grads: grad_scale must be finite and > 0");
  std::vector<const uint16_t*> v(n, nullptr);
  for (int q = 0; q < n; ++q) {
    if (q == G.rank) continue;  // this rank's own grad_bf16 is used
    if (rank_grads[q] == nullptr || !aligned16(rank_grads[q]))
      return set_error(RATEL_EINVAL, "ratel_register_peer_grads: rank %d's pointer must be non-NULL, 16-byte aligned", q);
    v[q] = static_cast<const uint16_t*>(rank_grads[q]);
  }
  if (G.comm != nullptr && B.ev_ready == nullptr) {
    CK(cudaEventCreateWithFlags(&B.ev_ready, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&B.ev_rel, cudaEventDisableTiming));
  }
  if (B.rgrads.size() != B.ranges.size()) {
    B.rgrads.resize(B.ranges.size());
    B.rscale.assign(B.ranges.size(), 1.0);
  }
  B.rgrads[range_idx] = v;
  B.rscale[range_idx] = grad_scale;
  if (!B.rs) ++G.n_rs_blocks;
  B.rs = true;
  return RATEL_OK;
}

int ratel_register_ssd(int block_id, int range_idx, int fd, uint64_t offset) {
  RK(entry());
  if (G.armed || G.n_handed > 0) return set_error(RATEL_ESTATE, "ratel_register_ssd: a step is in flight");
  if (block_id < 0 || block_id >= RATEL_MAX_BLOCKS || !G.blocks[block_id].registered)
    return set_error(RATEL_EINVAL, "ratel_register_ssd: block %d is not registered", block_id);
  Block& B = G.blocks[block_id];
  if (B.residency != RATEL_SSD) return set_error(RATEL_EINVAL, "ratel_register_ssd: block %d is not RATEL_SSD", block_id);
  if (range_idx < 0 || range_idx >= static_cast<int>(B.ranges.size()))
    return set_error(RATEL_EINVAL, "ratel_register_ssd: range %d out of range", range_idx);
  if (offset % kSsdAlign) return set_error(RATEL_EINVAL, "ratel_register_ssd: offset must be a multiple of 4096");
  struct stat st{};
  if (fd < 0 || fstat(fd, &st) != 0) return set_error(RATEL_EINVAL, "ratel_register_ssd: fd %d is not open", fd);
  const int fl = fcntl(fd, F_GETFL);
  if (fl < 0 || (fl & O_ACCMODE) != O_RDWR) return set_error(RATEL_EINVAL, "ratel_register_ssd: fd must be open O_RDWR");
  const Slice& s = B.slices[range_idx];
  const uint64_t stride = ssd_stride(s.end - s.begin);
  if (static_cast<uint64_t>(st.st_size) < offset + 3 * stride)
    return set_error(RATEL_EINVAL, "ratel_register_ssd: the file holds %lld bytes, needs %llu", (long long)st.st_size,
                     static_cast<unsigned long long>(offset + 3 * stride));
  B.ssd[range_idx].fd = fd;
  B.ssd[range_idx].off = offset;
  B.ssd[range_idx].stride = stride;
  return RATEL_OK;
}

uint64_t ratel_ssd_range_bytes(uint64_t numel, int world_size, int rank) {
  if (world_size < 1 || rank < 0 || rank >= world_size) return 0;
  const Slice s = slice_of(numel, world_size, rank);
  return 3 * ssd_stride(s.end - s.begin);
}

int ratel_adam_step(double lr, double beta1, double beta2, double eps, double weight_decay, int64_t step) {
  Nvtx nv("ratel_adam_step %lld", static_cast<long long>(step));
  RK(entry());
  if (G.armed) return set_error(RATEL_ESTATE, "ratel_adam_step: step %lld already armed", (long long)G.last_step);
  if (step <= G.last_step)
    return set_error(RATEL_ESTATE, "ratel_adam_step: step %lld <= previous %lld", (long long)step,
                     (long long)G.last_step);
  const double vals[5] = {lr, beta1, beta2, eps, weight_decay};
  for (double x : vals)
    if (!std::isfinite(x) || x < 0.0) return set_error(RATEL_EINVAL, "ratel_adam_step: hyperparameters must be finite, >= 0");
  if (beta1 >= 1.0 || beta2 >= 1.0) return set_error(RATEL_EINVAL, "ratel_adam_step: betas must be < 1");
  const double t = static_cast<double>(step);
  const double bc1 = 1.0 - std::pow(beta1, t);
  const double bc2 = 1.0 - std::pow(beta2, t);
  AdamScalars& s = G.scal;
  s.beta1 = static_cast<float>(beta1);
  s.one_minus_beta1 = static_cast<float>(1.0 - beta1);
  s.beta2 = static_cast<float>(beta2);
  s.one_minus_beta2 = static_cast<float>(1.0 - beta2);
  s.neg_step_size = static_cast<float>(-lr / bc1);
  s.inv_sqrt_bc2 = static_cast<float>(1.0 / std::sqrt(bc2));
  s.eps = static_cast<float>(eps);
  s.decay = static_cast<float>(1.0 - lr * weight_decay);
  s.wd = static_cast<float>(weight_decay);
  s.wd_d = weight_decay;
  G.hp_lr = lr;
  G.hp_b1 = beta1;
  G.hp_b2 = beta2;
  G.hp_eps = eps;
  G.hp_wd = weight_decay;
  G.hp_bc1 = bc1;
  G.hp_bc2 = bc2;
  G.armed = true;
  G.last_step = step;
  if (G.cfg.max_grad_norm > 0.0) {
    if (!G.reg.empty() && G.n_handed == static_cast<int>(G.reg.size())) RK(finalize_clip());
    return RATEL_OK;
  }
  // Deferred ("Ratel+ZeRO"): the optimizer stage starts after
  // the whole backward -- every handler stream waits for every gradient
  // handed off so far before any state moves (s_opt already waited on each).
  if (!G.pending.empty())
    for (cudaStream_t st : {G.s_h2d, G.s_d2h, G.s_host, G.s_tile, G.s_k[0], G.s_k[1], G.s_hc_d2h, G.s_hc_h2d})
      for (int id : G.pending) CK(cudaStreamWaitEvent(st, G.blocks[id].ev_grad, 0));
  std::vector<cudaEvent_t> all_grads;  // SSD: no state is read before the whole backward
  for (int id : G.pending) all_grads.push_back(G.blocks[id].ev_grad);
  for (int id : G.pending) RK(enqueue_block(G.blocks[id], &all_grads));
  G.pending.clear();
  return RATEL_OK;
}

// The step is not graph-capturable: the tile scheduler's counters, the arming
// state and the NCCL/host work are tracked per call on the host, so a replayed
// capture would run stale launches.  A caller stream under capture is refused
// before anything is enqueued (RATEL_EINVAL, no side effects).
static int check_not_capturing(void* stream, const char* fn) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  const cudaError_t e = cudaStreamIsCapturing(static_cast<cudaStream_t>(stream), &st);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return set_error(RATEL_EINVAL, "%s: cannot use the stream (%s)", fn, cudaGetErrorString(e));
  }
  if (st != cudaStreamCaptureStatusNone)
    return set_error(RATEL_EINVAL, "%s: the stream is being captured into a CUDA graph; the AGO step is not "
                                   "graph-capturable", fn);
  return RATEL_OK;
}

int ratel_offload_grad_chunk(int block_id, void* stream) {
  Nvtx nv("ratel_offload_grad_chunk %d", block_id);
  RK(entry());
  RK(check_not_capturing(stream, "ratel_offload_grad_chunk"));
  if (block_id < 0 || block_id >= RATEL_MAX_BLOCKS || !G.blocks[block_id].registered)
    return set_error(RATEL_ESTATE, "ratel_offload_grad_chunk: block %d is not registered", block_id);
  Block& B = G.blocks[block_id];
  if (B.handed_off)
    return set_error(RATEL_ESTATE, "ratel_offload_grad_chunk: block %d already handed off this step", block_id);
  if (B.residency == RATEL_SSD)
    for (size_t i = 0; i < B.ssd.size(); ++i)
      if (B.ssd[i].fd < 0 && B.slices[i].end > B.slices[i].begin)
        return set_error(RATEL_ESTATE, "ratel_offload_grad_chunk: block %d range %zu has no SSD file", block_id, i);
  CK(cudaEventRecord(B.ev_grad, static_cast<cudaStream_t>(stream)));
  CK(cudaStreamWaitEvent(G.s_opt, B.ev_grad, 0));
  if ((B.rs || B.pp) && G.comm != nullptr) {
    // Fused reduction: this rank is about to read every rank's G16 of the
    // block; fused all-gather: it is about to store its P16 slice into every
    // rank's buffer, which a slower rank's backward may still be reading.  An
    // 8-byte allreduce after the local hand-off is the barrier -- once it
    // completes, every rank's backward has produced the block (and enqueued
    // every GEMM that reads its P16 before the hand-off's event).
    CK(cudaStreamWaitEvent(G.s_comm, B.ev_grad, 0));
    NK(g_nccl.AllReduce(G.d_barrier, G.d_barrier, 1, ncclFloat64, ncclSum, G.comm, G.s_comm));
    CK(cudaEventRecord(B.ev_ready, G.s_comm));
    CK(cudaStreamWaitEvent(G.s_opt, B.ev_ready, 0));
  }
  B.handed_off = true;
  ++G.n_handed;
  if (G.cfg.max_grad_norm > 0.0) {
    RK(launch_sumsq(B));
    if (G.armed && G.n_handed == static_cast<int>(G.reg.size())) RK(finalize_clip());
    return RATEL_OK;
  }
  if (G.armed)
    RK(enqueue_block(B));  // active message: handler runs now, overlapping backward
  else
    G.pending.push_back(block_id);
  return RATEL_OK;
}

int ratel_block_wait(int block_id, void* stream) {
  RK(entry());
  RK(check_not_capturing(stream, "ratel_block_wait"));
  if (block_id < 0 || block_id >= RATEL_MAX_BLOCKS || !G.blocks[block_id].registered)
    return set_error(RATEL_ESTATE, "ratel_block_wait: block %d is not registered", block_id);
  const Block& B = G.blocks[block_id];
  if (B.handed_off && !B.enqueued)
    return set_error(RATEL_ESTATE, "ratel_block_wait: block %d's update is not enqueued yet", block_id);
  if (B.residency == RATEL_SSD && B.enqueued) {
    RK(ssd_drain(false, B.ssd_seq));  // its ev_done is recorded
    // the reader's G16 reads ran on its own streams: keep ratel_optimizer_stream()
    // ordered after them (grad.record_stream(ratel_optimizer_stream()) contract)
    CK(cudaStreamWaitEvent(G.s_opt, B.ev_done, 0));
  }
  if (B.rs && G.comm != nullptr && B.enqueued) {
    // Peers read this rank's G16 too: release it only after every rank's
    // update of the block (collective: every rank calls block_wait alike).
    CK(cudaStreamWaitEvent(G.s_comm, B.ev_done, 0));
    NK(g_nccl.AllReduce(G.d_barrier, G.d_barrier, 1, ncclFloat64, ncclSum, G.comm, G.s_comm));
    CK(cudaEventRecord(B.ev_rel, G.s_comm));
    CK(cudaStreamWaitEvent(static_cast<cudaStream_t>(stream), B.ev_rel, 0));
    return RATEL_OK;
  }
  CK(cudaStreamWaitEvent(static_cast<cudaStream_t>(stream), B.ev_done, 0));
  return RATEL_OK;
}

int ratel_sync(void* stream) {
  Nvtx nv("ratel_sync");
  RK(entry());
  if (stream != nullptr) RK(check_not_capturing(stream, "ratel_sync"));
  if (G.armed || G.n_handed > 0) {
    if (!G.armed) return set_error(RATEL_ESTATE, "ratel_sync: blocks handed off but no ratel_adam_step");
    if (G.n_handed != static_cast<int>(G.reg.size()))
      return set_error(RATEL_ESTATE, "ratel_sync: %d of %zu blocks handed off", G.n_handed, G.reg.size());
  }
  if (G.comm != nullptr && (G.n_peer_ranges > 0 || G.n_rs_blocks > 0)) {
    // Fused all-gather: ranks wrote into each other's P16; fused reduction:
    // ranks read each other's G16.  One 8-byte allreduce after every local
    // update is the cross-rank barrier: once it completes here, every rank's
    // update kernels (their peer stores fenced system-wide, their peer loads
    // done) have finished.
    CK(cudaEventRecord(G.ev_end[0], G.s_opt));
    CK(cudaEventRecord(G.ev_end[5], G.s_tile));
    CK(cudaStreamWaitEvent(G.s_comm, G.ev_end[0], 0));
    CK(cudaStreamWaitEvent(G.s_comm, G.ev_end[5], 0));
    NK(g_nccl.AllReduce(G.d_barrier, G.d_barrier, 1, ncclFloat64, ncclSum, G.comm, G.s_comm));
  }
  // SSD: every job issued to the GPU and every state write-back in the file
  RK(ssd_drain(true));
  const int NS = G.ssd != nullptr ? Ctx::kNS : Ctx::kNS - 3;
  cudaStream_t ss[Ctx::kNS] = {G.s_opt, G.s_h2d, G.s_d2h, G.s_comm, G.s_host, G.s_tile, G.s_k[0], G.s_k[1],
                               G.s_hc_d2h, G.s_hc_h2d,
                               G.ssd ? G.ssd->s_in : nullptr, G.ssd ? G.ssd->s_k : nullptr,
                               G.ssd ? G.ssd->s_out : nullptr};
  for (int i = 0; i < NS; ++i) CK(cudaEventRecord(G.ev_end[i], ss[i]));
  // Order the internal streams too: the next step's stage-in must not read
  // host states still being written back, and its K1 must not overwrite a
  // P16 slice the all-gather is still sending.
  for (int i = 0; i < NS; ++i)
    for (int j = 0; j < NS; ++j)
      if (i != j) CK(cudaStreamWaitEvent(ss[i], G.ev_end[j], 0));
  reset_step_state();
  if (stream != nullptr) {
    for (int i = 0; i < NS; ++i) CK(cudaStreamWaitEvent(static_cast<cudaStream_t>(stream), G.ev_end[i], 0));
    CK(cudaGetLastError());
  } else {
    for (int i = 0; i < NS; ++i) CK(cudaEventSynchronize(G.ev_end[i]));
  }
  if (G.comm) {
    ncclResult_t ar = ncclSuccess;
    NK(g_nccl.CommGetAsyncError(G.comm, &ar));
    if (ar != ncclSuccess && ar != ncclInProgress)
      return sticky_fail(RATEL_ENCCL, "NCCL async error: %s", g_nccl.GetErrorString(ar));
  }
  if (stream == nullptr && G.cfg.max_grad_norm > 0.0 && *G.h_flag) {
    *G.h_flag = 0;
    return set_error(RATEL_ENONFINITE, "ratel_sync: global grad norm was not finite (update applied)");
  }
  return RATEL_OK;
}

int ratel_finalize(void) {
  if (!G.inited) return set_error(RATEL_ESTATE, "ratel_finalize: not initialised");
  cudaSetDevice(G.device);
  for (cudaStream_t s : {G.s_opt, G.s_h2d, G.s_d2h, G.s_comm, G.s_host, G.s_tile, G.s_k[0], G.s_k[1],
                         G.s_hc_d2h, G.s_hc_h2d})
    if (s) cudaStreamSynchronize(s);
  destroy_all();
  cudaGetLastError();
  return RATEL_OK;
}

int ratel_refresh_params(int block_id, void* stream) {
  Nvtx nv("ratel_refresh_params %d", block_id);
  RK(entry());
  if (stream != nullptr) RK(check_not_capturing(stream, "ratel_refresh_params"));
  if (G.armed || G.n_handed > 0) return set_error(RATEL_ESTATE, "ratel_refresh_params: a step is in flight");
  if (block_id < 0 || block_id >= RATEL_MAX_BLOCKS || !G.blocks[block_id].registered)
    return set_error(RATEL_ESTATE, "ratel_refresh_params: block %d is not registered", block_id);
  Block& B = G.blocks[block_id];
  if (B.residency == RATEL_SSD)  // every non-empty slice needs its state file (no side effects on ESTATE)
    for (size_t i = 0; i < B.ranges.size(); ++i)
      if (B.ssd[i].fd < 0 && B.slices[i].end > B.slices[i].begin)
        return set_error(RATEL_ESTATE, "ratel_refresh_params: block %d range %zu has no SSD file", block_id, i);
  const cudaStream_t cs = static_cast<cudaStream_t>(stream);
  // after whatever the caller enqueued (e.g. restored states), and after every
  // earlier update (s_opt is ordered after all of them by ratel_sync)
  CK(cudaEventRecord(B.ev_grad, cs));
  CK(cudaStreamWaitEvent(G.s_opt, B.ev_grad, 0));
  const unsigned grid_max = static_cast<unsigned>(G.sms) * 4u;
  auto launch = [&](const float* th, uint16_t* p, uint64_t n, const PeerDesc& pd) -> int {
    const uint64_t want = std::max<uint64_t>(1, (n / 8 + kThreads - 1) / kThreads);
    const unsigned g = static_cast<unsigned>(std::min<uint64_t>(want, grid_max));
    refresh_p16_kernel<<<g, kThreads, 0, G.s_opt>>>(th, p, n, pd);
    CK(cudaGetLastError());
    ++G.launches;
    return RATEL_OK;
  };
  float* stage = nullptr;  // SSD: the master is in the state file, read tile by tile
  int rc = RATEL_OK;
  for (size_t i = 0; i < B.ranges.size() && rc == RATEL_OK; ++i) {
    const ratel_range& r = B.ranges[i];
    const Slice& s = B.slices[i];
    const uint64_t n = s.end - s.begin;
    if (n == 0) continue;
    uint16_t* p = static_cast<uint16_t*>(r.param_bf16) + s.begin;
    if (B.residency != RATEL_SSD) {  // device or page-locked host master (read in place)
      rc = launch(r.master, p, n, peer_desc(B, i, 0));
      continue;
    }
    const uint64_t T = G.cfg.tile_elems;
    if (stage == nullptr && cudaHostAlloc(&stage, T * sizeof(float), cudaHostAllocDefault) != cudaSuccess) {
      stage = nullptr;
      return sticky_fail(RATEL_ENOMEM, "ratel_refresh_params: staging cudaHostAlloc failed");
    }
    const Block::SsdRange& f = B.ssd[i];
    for (uint64_t off = 0; off < n && rc == RATEL_OK; off += T) {
      const uint64_t len = std::min<uint64_t>(T, n - off);
      const uint64_t bytes = (len * 4 + kSsdAlign - 1) / kSsdAlign * kSsdAlign;
      if (cudaStreamSynchronize(G.s_opt) != cudaSuccess) {  // the previous tile's kernel read the stage
        rc = sticky_fail(RATEL_ECUDA, "ratel_refresh_params: %s", cudaGetErrorString(cudaGetLastError()));
        break;
      }
      std::string msg;
      rc = io_full(true, f.fd, stage, bytes, f.off + off * 4, msg);
      if (rc != RATEL_OK) {
        rc = sticky_fail(rc, "ratel_refresh_params: %s", msg.c_str());
        break;
      }
      rc = launch(stage, p + off, len, peer_desc(B, i, off));
    }
  }
  if (stage != nullptr) {
    cudaStreamSynchronize(G.s_opt);
    cudaFreeHost(stage);
  }
  if (rc != RATEL_OK) return rc;
  CK(cudaEventRecord(B.ev_done, G.s_opt));
  cudaEvent_t last = B.ev_done;
  if (G.comm != nullptr) {
    RK(allgather_block(B));  // NCCL ranges: in-place bf16 all-gather on the comm stream
    CK(cudaStreamWaitEvent(G.s_comm, B.ev_done, 0));
    if (B.pp)  // peer stores: every rank's refresh kernel done (collective)
      NK(g_nccl.AllReduce(G.d_barrier, G.d_barrier, 1, ncclFloat64, ncclSum, G.comm, G.s_comm));
    CK(cudaEventRecord(G.ev_end[3], G.s_comm));
    last = G.ev_end[3];
  }
  if (stream != nullptr) {
    CK(cudaStreamWaitEvent(cs, last, 0));
  } else {
    CK(cudaEventSynchronize(last));
  }
  return RATEL_OK;
}

void* ratel_optimizer_stream(void) { return G.inited ? static_cast<void*>(G.s_opt) : nullptr; }

int ratel_get_grad_sumsq(double* out) {
  RK(entry());
  if (out == nullptr) return set_error(RATEL_EINVAL, "ratel_get_grad_sumsq: NULL");
  if (!(G.cfg.max_grad_norm > 0.0)) return set_error(RATEL_ESTATE, "ratel_get_grad_sumsq: clipping is off");
  CK(cudaStreamSynchronize(G.s_opt));
  CK(cudaMemcpy(out, G.comm != nullptr ? G.d_sumsq + 1 : G.d_sumsq, sizeof(double), cudaMemcpyDeviceToHost));
  return RATEL_OK;
}

int ratel_kernel_timing(double* total_ms, int64_t* launches, int reset) {
  RK(entry());
  if (total_ms == nullptr || launches == nullptr) return set_error(RATEL_EINVAL, "ratel_kernel_timing: NULL");
  // Union of the launch intervals, all measured from the first launch's start
  // event (earlier events give negative offsets).
  std::vector<std::pair<double, double>> iv;
  iv.reserve(G.tused);
  for (size_t i = 0; i < G.tused; ++i) {
    CK(cudaEventSynchronize(G.tpool[i].b));
    float s = 0.f, e = 0.f;
    CK(cudaEventElapsedTime(&s, G.tpool[0].a, G.tpool[i].a));
    CK(cudaEventElapsedTime(&e, G.tpool[0].a, G.tpool[i].b));
    iv.emplace_back(s, e);
  }
  std::sort(iv.begin(), iv.end());
  double tot = 0.0, cs = 0.0, ce = -1e300;
  for (const auto& x : iv) {
    if (x.first > ce) {
      if (ce > cs) tot += ce - cs;
      cs = x.first;
      ce = x.second;
    } else {
      ce = std::max(ce, x.second);
    }
  }
  if (!iv.empty() && ce > cs) tot += ce - cs;
  *total_ms = tot;
  *launches = static_cast<int64_t>(G.tused);
  if (reset) G.tused = 0;
  return RATEL_OK;
}

int64_t ratel_launch_count(void) { return G.launches; }

int ratel_alloc_pinned(uint64_t bytes, void** out) {
  if (out == nullptr) return set_error(RATEL_EINVAL, "ratel_alloc_pinned: NULL");
  *out = nullptr;
  if (bytes == 0) return set_error(RATEL_EINVAL, "ratel_alloc_pinned: 0 bytes");
  const cudaError_t e = cudaHostAlloc(out, bytes, cudaHostAllocPortable);
  if (e != cudaSuccess) {
    cudaGetLastError();
    *out = nullptr;
    return set_error(RATEL_ENOMEM, "cudaHostAlloc(%llu) failed: %s", static_cast<unsigned long long>(bytes),
                     cudaGetErrorString(e));
  }
  return RATEL_OK;
}

int ratel_free_pinned(void* p) {
  if (p == nullptr) return RATEL_OK;
  const cudaError_t e = cudaFreeHost(p);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return set_error(RATEL_EINVAL, "cudaFreeHost failed: %s", cudaGetErrorString(e));
  }
  return RATEL_OK;
}

}  // extern "C"
