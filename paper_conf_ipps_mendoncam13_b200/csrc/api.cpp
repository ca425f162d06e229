// api.cpp — libsw's C-ABI (include/sw.h): database creation, the search driver
// (master + one worker thread per GPU, PSS/WA over the task table of sched.cpp), the
// per-device runtime (streams, profiles, border slots, abort flags), result merge and
// top-k.  Multi-process (torchrun) mode reaches a master in rank 0 over TCP (net.cpp).
//
// The paper's flow (P16 §IV, Fig. 4): register slaves -> acquire sequences -> convert
// format -> allocate tasks (policy) -> execute tasks -> send results -> merge.
#include <algorithm>
#include <atomic>
#include <chrono>
#include <climits>
#include <cmath>
#include <condition_variable>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <memory>
#include <mutex>
#include <numeric>
#include <sstream>
#include <stdexcept>
#include <string>
#include <thread>
#include <type_traits>
#include <vector>
#include <cuda.h>
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>   // header-only NVTX3: ranges per unit launch, marks per grant
#include "sw_internal.h"
#include "net.h"
#include "../../include/sw.h"
#include "../../include/sw_sched.h"

namespace sw {

// ---------------------------------------------------------------- errors
static thread_local std::string g_err;
void set_last_error(const std::string &m) { g_err = m; }
#define CK(call)                                                                      \
  do {                                                                                \
    cudaError_t e_ = (call);                                                          \
    if (e_ != cudaSuccess)                                                            \
      throw Error(SW_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_));      \
  } while (0)

template <class F>
static int guarded(F &&f) {
  try {
    g_err.clear();
    f();
    return SW_OK;
  } catch (const Error &e) {
    g_err = e.what();
    return e.code;
  } catch (const std::bad_alloc &) {
    g_err = "out of host memory";
    return SW_ENOMEM;
  } catch (const std::exception &e) {
    g_err = e.what();
    return SW_EINVAL;
  }
}

// Each worker keeps up to 64 streams in flight, plus its cancellation and local-load
// streams; with several workers on one GPU these exceed the default 8 hardware work queues
// and unrelated streams would serialize (a fast worker's unit waiting behind a straggler's
// kernel).  Raise the limit before the first CUDA context is created (no effect after).
__attribute__((constructor)) static void sw_raise_connections() {
  setenv("CUDA_DEVICE_MAX_CONNECTIONS", "32", 0);
}

static double now_s() {
  using namespace std::chrono;
  return duration<double>(steady_clock::now().time_since_epoch()).count();
}

// ---------------------------------------------------------------- device buffers
template <class T>
struct DBuf {
  T *p = nullptr;
  size_t n = 0;
  int dev = -1;
  void alloc(int d, size_t count) {
    free();
    dev = d;
    n = count;
    if (count == 0) return;
    cudaError_t e = cudaMalloc((void **)&p, sizeof(T) * count);
    if (e != cudaSuccess) {
      p = nullptr;
      throw Error(SW_ENOMEM, std::string("cudaMalloc: ") + cudaGetErrorString(e));
    }
  }
  void free() {
    if (p) { cudaSetDevice(dev); cudaFree(p); }
    p = nullptr; n = 0;
  }
  // grow-only: keep the allocation across searches when it is large enough
  void ensure(int d, size_t count) {
    if (p && dev == d && count <= n) return;
    alloc(d, std::max<size_t>(count, 1));
  }
  ~DBuf() { free(); }
  DBuf() = default;
  DBuf(const DBuf &) = delete;
  DBuf &operator=(const DBuf &) = delete;
};

struct Device;
// per-device search resources, cached in the sw_db across searches (grow-only buffers,
// events and the cancellation stream are created once)
struct DevSearch {
  Device *D = nullptr;
  DBuf<uint8_t> qcodes;
  DBuf<int64_t> qoff;
  DBuf<QueryPair> pairs;
  DBuf<SliceInfo> slices;
  DBuf<int8_t> matrix;
  DBuf<int32_t> prof;
  DBuf<int32_t> scores_own;
  int32_t *scores = nullptr;
  DBuf<int2> ovf;              // [streams][kOvfCap] saturated pairs, one list per stream
  DBuf<int32_t> ovf_count;     // [streams]
  DBuf<int32_t> ovf_cursor;    // [streams][2] entries taken by the int32 re-run (small / big pairs)
  DBuf<uint32_t> ovf_bits;     // [nq*ndb] bits: pair already listed
  int32_t ovf_cap = 0;         // entries per stream list
  DBuf<uint2> k3_border;   // [streams][k3_rows][max_len]
  int64_t k3_rows = 0;
  DBuf<int32_t> k3_prog;   // [streams][k3 slots x warps]: clustered K3 progress counters
  DBuf<int32_t> k2_border;
  DBuf<K2Ctl> k2_ctl;        // [streams]: big-pair tickets, slots and progress counters (K2)
  int32_t k2_blocks = kK2Blocks;   // K2 blocks per launch this search
  DBuf<int32_t> abort_dev;      // per-unit WA cancellation flags (device memory)
  DBuf<int32_t> progress;       // per-unit progress counters (K1 groups / K3 sequence-chunks)
  DBuf<int32_t> gclaim;         // per-unit K1 group claim counters
  int32_t *abort_d = nullptr;
  int32_t *one_h = nullptr;      // pinned constant 1, source of the cancellation copies
  int32_t *ovf_seen_h = nullptr; // pinned [kMaxStreams]: ovf_count copied after each unit
  int32_t *ovf_early_h = nullptr;// pinned, mapped [kMaxStreams]: entries listed, written by the
                                 // DP kernels as they list them (early int32 re-run launch)
  int32_t *ovf_early_d = nullptr;// its device address
  int32_t *prog_h = nullptr;     // pinned [kMaxStreams]: the unit's progress after it ran
  cudaStream_t cancel_st = nullptr;
  cudaStream_t noise_st = nullptr;   // high priority: the local-load kernel (straggler mode 2)
  std::vector<cudaStream_t> epi;     // [1] high priority: the units' K2 + K5u epilogues
  DBuf<int32_t> noise_flag;
  DBuf<uint32_t> noise_sink;
  std::vector<char> cancelled;
  // data plane: per-unit top-k of committed units, merged per worker
  DBuf<int32_t> pack_q;          // queries of each pack (flattened, Plan::pack_q_off)
  DBuf<int2> unit_hits;          // [units][max_unit_q][k]
  DBuf<int2> worker_hits;        // [nq][k] top-k over this worker's committed units
  DBuf<int2> all_hits;           // device 0: [workers][nq][k]
  DBuf<int32_t> list_tab;        // merge tables: list_off[nq+1] then list_idx
  DBuf<SegInfo> segs;            // committed-unit segments (scores data plane)
  DBuf<int32_t> compact;         // this worker's committed scores, dense
  DBuf<int32_t> out_stage;       // multi-process: committed-only score matrix
  std::vector<int32_t> committed;   // units this worker committed
  cudaEvent_t ev_start = nullptr, ev_end = nullptr, ev_data = nullptr;
  std::vector<cudaEvent_t> u_start, u_end;  // per stream
  int launches = 0;
  double k1_sec = 0, k3_sec = 0, k2_sec = 0;
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> k2_ev;   // per K2 launch (rare), this search
  int64_t k1_cells = 0, k3_cells = 0;
  int64_t dup_cells = 0;
  int32_t n_cancelled = 0;
  double finish_wall = 0;
  double last_dev = 0;           // device time of this worker's last unit completion (s)
  int32_t n_ovf = 0;
  void reset_counters() {
    for (auto &e : k2_ev) { cudaEventDestroy(e.first); cudaEventDestroy(e.second); }
    k2_ev.clear();
    launches = 0; k1_sec = k3_sec = k2_sec = 0; k1_cells = k3_cells = 0; dup_cells = 0; n_cancelled = 0;
    finish_wall = 0; last_dev = 0; n_ovf = 0; scores = nullptr; committed.clear();
  }
  ~DevSearch();
};

// ---------------------------------------------------------------- green contexts
// Emulated GPUs (sw_opts.worker_sms, experiments): the workers sharing one B200 each get a
// disjoint SM partition through a green context (driver API, reached through the runtime's
// entry-point table: no link-time libcuda), and their streams are created in it, so a
// worker's kernels run on its SMs only.  Partitions are multiples of 8 SMs on sm_100.
struct GreenApi {
  CUresult (*get_res)(CUdevice, CUdevResource *, CUdevResourceType) = nullptr;
  CUresult (*split)(CUdevResource *, unsigned *, const CUdevResource *, CUdevResource *, unsigned, unsigned) = nullptr;
  CUresult (*gen_desc)(CUdevResourceDesc *, CUdevResource *, unsigned) = nullptr;
  CUresult (*create)(CUgreenCtx *, CUdevResourceDesc, CUdevice, unsigned) = nullptr;
  CUresult (*destroy)(CUgreenCtx) = nullptr;
  CUresult (*stream)(CUstream *, CUgreenCtx, unsigned, int) = nullptr;
  bool ok = false;
};
static const GreenApi &green_api() {
  static GreenApi g;
  static std::once_flag once;
  std::call_once(once, [] {
    auto get = [](const char *name, auto &fn) {
      void *p = nullptr;
      cudaDriverEntryPointQueryResult q;
      if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) == cudaSuccess && q == cudaDriverEntryPointSuccess)
        fn = reinterpret_cast<std::remove_reference_t<decltype(fn)>>(p);
      return fn != nullptr;
    };
    g.ok = get("cuDeviceGetDevResource", g.get_res) && get("cuDevSmResourceSplitByCount", g.split) &&
           get("cuDevResourceGenerateDesc", g.gen_desc) && get("cuGreenCtxCreate", g.create) &&
           get("cuGreenCtxDestroy", g.destroy) && get("cuGreenCtxStreamCreate", g.stream);
  });
  return g;
}
struct GreenSet {   // one device split into n partitions of sms SMs (asked for: req)
  int dev = -1, req = 0, sms = 0, n = 0;
  std::vector<CUgreenCtx> ctx;
  ~GreenSet() {
    for (CUgreenCtx c : ctx)
      if (c) green_api().destroy(c);
  }
};
// a stream in green context g (nullptr: the device's primary context)
static cudaStream_t make_stream(CUgreenCtx g, int prio) {
  cudaStream_t st;
  if (g) {
    CUstream cs;
    if (green_api().stream(&cs, g, CU_STREAM_NON_BLOCKING, prio) != CUDA_SUCCESS)
      throw Error(SW_ECUDA, "cuGreenCtxStreamCreate failed");
    return (cudaStream_t)cs;
  }
  CK(cudaStreamCreateWithPriority(&st, cudaStreamNonBlocking, prio));
  return st;
}

struct Device {
  int id = 0;
  int n_sm = 0;
  int n_eff = 0;                // SMs its kernels are sized for: n_sm, or its green partition's
  CUgreenCtx gctx = nullptr;    // the green context its streams belong to (emulated GPUs)
  DBuf<uint4> packed;
  DBuf<GroupInfo> groups;
  DBuf<int32_t> perm, sorted_len;
  DBuf<uint2> k1_border;   // per-SM slots
  DBuf<int32_t> slot_busy;
  int32_t slots_per_sm = 0, slot_cols = 0, sm_slots = 0;
  std::vector<cudaStream_t> streams;
  std::unique_ptr<DevSearch> ws;   // cached search resources
  ~Device() {
    cudaSetDevice(id);
    ws.reset();
    for (auto s : streams) cudaStreamDestroy(s);
  }
};
inline DevSearch::~DevSearch() {
  if (one_h) cudaFreeHost(one_h);
  if (ovf_seen_h) cudaFreeHost(ovf_seen_h);
  if (ovf_early_h) cudaFreeHost(ovf_early_h);
  if (prog_h) cudaFreeHost(prog_h);
  if (cancel_st) cudaStreamDestroy(cancel_st);
  if (noise_st) cudaStreamDestroy(noise_st);
  for (auto e : epi) cudaStreamDestroy(e);
  if (ev_start) cudaEventDestroy(ev_start);
  if (ev_end) cudaEventDestroy(ev_end);
  for (auto &e : k2_ev) { cudaEventDestroy(e.first); cudaEventDestroy(e.second); }
  if (ev_data) cudaEventDestroy(ev_data);
  for (auto e : u_start) cudaEventDestroy(e);
  for (auto e : u_end) cudaEventDestroy(e);
}


}  // namespace sw

struct sw_db {
  sw::PackedDB host;
  std::vector<std::unique_ptr<sw::GreenSet>> green;   // emulated GPUs (destroyed after devs)
  std::vector<std::unique_ptr<sw::Device>> devs;
  std::vector<char> peer_ok;     // [i * n + j]: device of worker i can read worker j's memory
  std::atomic<int> busy{0};
  std::string unit_log;
  std::string sched_log;
};

namespace sw {

// ---------------------------------------------------------------- search plan
struct Plan {
  std::vector<QueryPair> pairs;       // query packs
  std::vector<SliceInfo> slices;      // all packs' slice tables
  std::vector<int64_t> real_rows;     // per pack: sum of its query lengths
  std::vector<uint8_t> qcodes;
  std::vector<int64_t> qoff;
  std::vector<Unit> units;
  int64_t prof_total = 0;
  int64_t cells = 0;
  int32_t n_long_seqs = 0;   // sequences [0, n_long_seqs) in sorted order go to K3
  int32_t first_short_group = 0;
  int32_t max_k3_seqs = 0;   // largest K3 unit (sequences)
  int32_t max_len = 0;
  std::vector<uint8_t> pack_may_ovf;   // per pack: a query whose score bound reaches the s16 flag
  std::vector<int32_t> pack_q;         // queries of each pack, flattened (ascending ids)
  std::vector<int32_t> pack_q_off;     // [packs + 1]
  int32_t max_pack_q = 1;              // most queries in one pack
  int32_t max_unit_q = 1;              // most queries in one unit (a unit spans npk packs)
  uint64_t hash = 0;                   // FNV-1a of the unit table (multi-process handshake)
};
// sorted-sequence range [s0, s1) of a unit's pairs (K1: whole groups; K3: long sequences)
static inline void unit_seq_range(const Unit &U, int32_t n, int32_t &s0, int32_t &s1) {
  if (U.kind == kUnitInter) { s0 = U.b0 * kGroup; s1 = std::min(n, U.b1 * kGroup); }
  else { s0 = U.b0; s1 = U.b1; }
}

static void validate_seqset(const sw_seqset *s, const char *what) {
  if (!s) throw Error(SW_EINVAL, std::string(what) + " is NULL");
  if (s->n < 0) throw Error(SW_EINVAL, std::string(what) + ": n < 0");
  if (s->n > 0 && !s->offsets) throw Error(SW_EINVAL, std::string(what) + ": offsets is NULL");
  if (s->n > 0 && s->offsets[0] != 0) throw Error(SW_EINVAL, std::string(what) + ": offsets[0] != 0");
  for (int32_t k = 0; k < s->n; k++)
    if (s->offsets[k + 1] < s->offsets[k])
      throw Error(SW_EINVAL, std::string(what) + ": offsets not monotone at " + std::to_string(k));
  if (s->n > 0 && s->offsets[s->n] > 0 && !s->residues)
    throw Error(SW_EINVAL, std::string(what) + ": residues is NULL");
}

static Plan make_plan(const sw_seqset *q, const PackedDB &db, const sw_opts &o, int n_workers,
                      const int8_t *M, int32_t thresh, int32_t k1_wave, int32_t k3_slots) {
  Plan P;
  const int32_t nq = q->n;
  P.qoff.resize(nq + 1);
  P.qoff[0] = 0;
  for (int32_t k = 0; k < nq; k++) {
    const int64_t l = q->offsets[k + 1] - q->offsets[k];
    if (l > SW_MAX_QUERY_LEN)
      throw Error(SW_EINVAL, "query " + std::to_string(k) + " longer than 65535 residues (SW_MAX_QUERY_LEN)");
    P.qoff[k + 1] = P.qoff[k] + l;
  }
  P.qcodes.resize(P.qoff[nq]);
  for (int32_t k = 0; k < nq; k++)
    for (int64_t p = 0; p < P.qoff[k + 1] - P.qoff[k]; p++) {
      const int c = encode_residue((unsigned char)q->residues[q->offsets[k] + p]);
      if (c < 0)
        throw Error(SW_ERESIDUE, "query " + std::to_string(k) + ": invalid residue '" +
                                     std::string(1, q->residues[q->offsets[k] + p]) +
                                     "' at position " + std::to_string(p));
      P.qcodes[P.qoff[k] + p] = (uint8_t)c;
    }
  // query packs (sw_internal.h): 2*NP half-streams of queries, each query starting on a
  // 16-row slice; queries (longest first) go to the least loaded half (LPT), halves are
  // paired by load.  NP ~ total rows / (2 x longest query), so a half is about as long as
  // the longest query and the halves of a pack differ by little.
  std::vector<int32_t> qo(nq);
  std::iota(qo.begin(), qo.end(), 0);
  std::stable_sort(qo.begin(), qo.end(), [&](int32_t a, int32_t b) {
    return P.qoff[a + 1] - P.qoff[a] > P.qoff[b + 1] - P.qoff[b];
  });
  auto c16 = [](int64_t x) { return (x + 15) / 16 * 16; };
  int64_t tot16 = 0, max16 = 16;
  for (int32_t k = 0; k < nq; k++) {
    const int64_t l = P.qoff[k + 1] - P.qoff[k];
    tot16 += c16(std::max<int64_t>(l, 1));
    max16 = std::max(max16, c16(l));
  }
  int32_t np = nq == 0 ? 0 : (int32_t)std::max<int64_t>(1, (tot16 + max16) / (2 * max16));
  np = std::min(np, std::max(1, (nq + 1) / 2));
  struct Half { int64_t load = 0; std::vector<int32_t> q; };
  std::vector<Half> halves(2 * np);
  for (int32_t k = 0; k < nq; k++) {   // LPT into 2*np halves (first least-loaded wins)
    const int32_t q = qo[k];
    int32_t h = 0;
    for (int32_t j = 1; j < 2 * np; j++)
      if (halves[j].load < halves[h].load) h = j;
    halves[h].q.push_back(q);
    halves[h].load += c16(std::max<int64_t>(P.qoff[q + 1] - P.qoff[q], 1));
  }
  std::stable_sort(halves.begin(), halves.end(),
                   [](const Half &a, const Half &b) { return a.load > b.load; });
  int64_t prof = 0;
  P.real_rows.clear();
  for (int32_t k = 0; k < np; k++) {
    const Half &lo = halves[2 * k], &hi = halves[2 * k + 1];
    QueryPair qp;
    qp.rows = (int32_t)std::max<int64_t>(std::max(lo.load, hi.load), 16);
    qp.rows_padded = (qp.rows + kProfileRowAlign - 1) / kProfileRowAlign * kProfileRowAlign;
    qp.prof_off = prof;
    qp.slice_off = (int32_t)P.slices.size();
    qp.pad_ = 0;
    prof += (int64_t)kNCodes * qp.rows_padded;
    const int32_t ns = qp.rows_padded / 16;
    std::vector<SliceInfo> sl(ns, SliceInfo{-1, 0, -1, 0});
    int64_t real = 0;
    for (int half = 0; half < 2; half++) {
      int64_t row = 0;
      for (int32_t q : (half == 0 ? lo : hi).q) {
        const int64_t l = P.qoff[q + 1] - P.qoff[q];
        real += l;
        const int64_t span = c16(std::max<int64_t>(l, 1));
        for (int64_t r = 0; r < span; r += 16) {
          SliceInfo &x = sl[(row + r) / 16];
          if (half == 0) { x.q_lo = q; x.off_lo = (int32_t)r; }
          else { x.q_hi = q; x.off_hi = (int32_t)r; }
        }
        row += span;
      }
    }
    P.slices.insert(P.slices.end(), sl.begin(), sl.end());
    P.real_rows.push_back(real);
    P.pairs.push_back(qp);
  }
  P.prof_total = prof;
  P.max_len = db.max_len;
  // packs that can saturate int16: a query's score is at most the sum over its residues of
  // their best substitution score; units of such packs go first, so the int32 re-run of
  // what they saturate overlaps the rest of the step instead of ending it (C5's planted
  // W/C/Y-rich query)
  {
    int row_best[24];
    for (int a = 0; a < 24; a++) {
      row_best[a] = kPadScore;
      for (int c = 0; c < 24; c++) row_best[a] = std::max(row_best[a], (int)M[a * 24 + c]);
    }
    std::vector<uint8_t> q_may(nq, 0);
    for (int32_t k = 0; k < nq; k++) {
      int64_t bound = 0;
      for (int64_t p = P.qoff[k]; p < P.qoff[k + 1]; p++) bound += std::max(0, row_best[P.qcodes[p]]);
      q_may[k] = bound + kOff >= (int64_t)thresh;
    }
    P.pack_may_ovf.assign(P.pairs.size(), 0);
    for (size_t p = 0; p < P.pairs.size(); p++) {
      const QueryPair &qp = P.pairs[p];
      for (int32_t sidx = 0; sidx < qp.rows_padded / 16; sidx++) {
        const SliceInfo &x = P.slices[qp.slice_off + sidx];
        if ((x.q_lo >= 0 && q_may[x.q_lo]) || (x.q_hi >= 0 && q_may[x.q_hi])) { P.pack_may_ovf[p] = 1; break; }
      }
    }
  }
  // long sequences -> K3: whole groups whose longest member exceeds the threshold
  int32_t thr = o.long_threshold == 0 ? 3072 : o.long_threshold;
  const int32_t ng = (int32_t)db.groups.size();
  int32_t gl = 0;
  if (thr > 0)
    while (gl < ng && db.sorted_len[db.groups[gl].first] > thr) gl++;
  P.first_short_group = gl;
  P.n_long_seqs = gl > 0 ? std::min(db.n, gl * kGroup) : 0;

  // cells per pair and unit target
  std::vector<int64_t> grp_res(ng, 0);
  for (int32_t g = 0; g < ng; g++)
    for (int32_t k = 0; k < db.groups[g].count; k++) grp_res[g] += db.sorted_len[db.groups[g].first + k];
  int64_t total_cells = 0;
  for (int64_t r : P.real_rows) total_cells += r * db.residues;
  P.cells = total_cells;
  // K3 cluster size (auto sizing): when long sequences carry most of the work and one
  // worker's share of (pack, long-sequence block) tasks fills too few of the GPU's resident
  // K3 CTAs -- C5 at 8 GPUs: 256 blocks for 592 slots -- each pair's chunks are split over a
  // cluster of 4 (fill < 1/2) or 2 CTAs.  SW_K3_CLUSTER forces a size (tuning, tests).
  // chunk balance: a cluster of C CTAs runs a pair's nch chunks in ceil(nch / C) rounds, and
  // the CTAs idle at the cluster barrier for the rest of the last round; among C - 1, C, C + 1
  // (instantiated sizes 2..5) take the best-balanced size over the packs [p0, p1), ties to
  // the larger (fewer rounds).  C5's 5,000-row packs (10 chunks): 4 -> 5 CTAs, C5 at 1/8 of
  // its database 4.30 -> 4.58 TCUPS, C4 at 1/8 6.16 -> 6.28
  auto balance_cluster = [&](int base, int32_t p0, int32_t p1) {
    int best = base;
    double best_eff = -1.0;
    for (int c = std::max(2, base - 1); c <= std::min(5, base + 1); c++) {
      int64_t used = 0, slots = 0;
      for (int32_t p = p0; p < p1; p++) {
        const int64_t nch = (P.pairs[p].rows + kK3Chunk - 1) / kK3Chunk;
        used += nch;
        slots += (nch + c - 1) / c * c;
      }
      const double eff = slots > 0 ? (double)used / slots : 0.0;
      if (eff > best_eff + 1e-9 || (eff > best_eff - 1e-9 && c > best)) { best = c; best_eff = eff; }
    }
    return best;
  };
  int32_t k3_cluster = 1;
  {
    int64_t long_res = 0;
    for (int32_t s = 0; s < P.n_long_seqs; s++) long_res += db.sorted_len[s];
    int64_t rows_all = 0;
    for (int64_t r : P.real_rows) rows_all += r;
    const int64_t c3 = rows_all * long_res, c1 = total_cells - c3;
    const double sb_per_worker = (double)P.pairs.size() * ((P.n_long_seqs + kK3Warps - 1) / kK3Warps) /
                                 std::max(1, n_workers);
    static const int forced = [] { const char *e = getenv("SW_K3_CLUSTER"); return e ? atoi(e) : 0; }();
    if (forced >= 1 && forced <= 8 && forced != 6 && forced != 7) k3_cluster = forced;
    else if (o.target_unit_cells <= 0 && P.n_long_seqs > 0 && c3 >= c1 && k3_slots > 0) {
      const double fill = sb_per_worker / k3_slots;
      k3_cluster = fill < 0.5 ? 4 : fill < 1.0 ? 2 : 1;
      if (k3_cluster > 1) k3_cluster = balance_cluster(k3_cluster, 0, (int32_t)P.pairs.size());
    }
  }
  int64_t target = o.target_unit_cells;
  const int depth = std::max(1, o.streams_per_device);
  if (target <= 0) {
    target = total_cells / std::max(1, n_workers * depth * 8);
    target = std::max<int64_t>(target, 1000000000LL);
    target = std::min<int64_t>(target, 50000000000LL);
  }
  for (int32_t p = 0; p < (int32_t)P.pairs.size(); p++) {
    const QueryPair &qp = P.pairs[p];
    const int64_t rows_eff = P.real_rows[p];
    // K3 units over the long sequences (multiples of kK3Warps), cut greedily at k3_target
    // cells (the last unit of a pack is the remainder: a short unit that fills the tail).
    // A K3 launch runs one warp per sequence, so a unit needs many sequences to cover the
    // SMs: k3_target is at least 4x the unit target and at least the cells of kK3UnitSeqs
    // average sequences (one block per B200 SM); with several workers it is capped so that
    // every stream of every worker gets a unit of each pack's long work.  (An explicit
    // target_unit_cells is taken as given: 4x it per K3 unit.)
    int64_t long_cells = 0;
    for (int32_t s = 0; s < P.n_long_seqs; s++) long_cells += rows_eff * db.sorted_len[s];
    const int64_t n_packs = (int64_t)P.pairs.size();
    const int64_t t4 = target > INT64_MAX / 4 ? INT64_MAX : 4 * target;   // INT64_MAX: very coarse
    int64_t k3_target = t4;
    if (P.n_long_seqs > 0 && o.target_unit_cells <= 0) {   // auto sizing only
      k3_target = std::max<int64_t>(t4, long_cells / P.n_long_seqs * kK3UnitSeqs);
      const int64_t per_pack = ((int64_t)n_workers * depth + n_packs - 1) / n_packs;
      if (per_pack > 1) k3_target = std::max<int64_t>(1, std::min<int64_t>(k3_target, (long_cells + per_pack - 1) / per_pack));
    }
    // (clustered plans: K3 units span every pack, built after this loop)
    for (int32_t s = 0; s < P.n_long_seqs && k3_cluster == 1;) {
      int32_t e = s;
      int64_t cells = 0, work = 0;
      while (e < P.n_long_seqs && (cells < k3_target || e == s || (e - s) % kK3Warps)) {
        cells += rows_eff * db.sorted_len[e];
        work += (int64_t)qp.rows_padded * db.sorted_len[e];
        e++;
      }
      P.units.push_back({kUnitIntra, p, s, e, cells, work, 1, 1});
      P.max_k3_seqs = std::max(P.max_k3_seqs, e - s);
      s = e;
    }
    // K1 units over the short groups
    const int64_t band = k1_band_rows();
    const int64_t rows_k1 = (int64_t)(qp.rows + band - 1) / band * band;
    // Auto sizing cuts a unit at whole waves of groups (k1_wave = resident K1 blocks of the
    // GPU, each block streams through its groups): 1.5 waves would leave half the SMs idle
    // for the last third of the launch.  The groups of a unit have nearly equal widths (length
    // sort), so k waves take ~k group times on every block.  The remainder of a segment
    // (< k waves) is its own, short unit, scheduled late by the LPT order below.
    for (int32_t g = gl; g < ng;) {
      // (units do not straddle the kWideCols boundary: each launch uses one K1 instance)
      const bool wide = db.groups[g].ncols >= kWideCols;
      int32_t seg_end = g;
      int64_t seg_cells = 0;
      while (seg_end < ng && (db.groups[seg_end].ncols >= kWideCols) == wide) seg_cells += rows_eff * grp_res[seg_end++];
      int32_t per_unit = 0;   // groups per unit, 0 = cut by cells
      if (o.target_unit_cells <= 0 && k1_wave > 0) {
        const double n_u = std::max(1.0, std::floor((double)seg_cells / (double)target + 0.5));
        const int32_t gpu = (int32_t)std::ceil((seg_end - g) / n_u);
        // k = ceil(groups / wave) waves; a unit under half a wave keeps its cell-based cut
        // (several streams' small units fill the GPU together; rounding them up to a wave
        // would coarsen small databases for no gain).  SW_K1_WAVES forces k (tuning).
        static const int forced = [] { const char *e = getenv("SW_K1_WAVES"); return e ? atoi(e) : 0; }();
        if (forced > 0) per_unit = forced * k1_wave;
        else if (2 * gpu >= k1_wave) per_unit = (gpu + k1_wave - 1) / k1_wave * k1_wave;
      }
      static const double crit = [] { const char *e = getenv("SW_K1_CRIT"); return e ? atof(e) : 1.5; }();
      while (g < seg_end) {
        int32_t e = g;
        int64_t cells = 0, work = 0;
        while (e < seg_end && (per_unit > 0 ? e - g < per_unit : (cells < target || e == g))) {
          cells += rows_eff * grp_res[e];
          work += rows_k1 * db.groups[e].ncols * kGroup;
          e++;
        }
        // a block runs a whole group: a unit whose per-block share (work / wave) is not well
        // above its widest group's work ends on that group's block alone (the widest C4 unit
        // of a pack: groups of 872-3,048 columns, 2 waves -> 5.2 TCUPS alone vs 6.3 typical);
        // such a unit takes more whole waves until the share is >= crit x the widest group
        // (SW_K1_CRIT, tuning: 0 / 1.5 / 2.5 -> K1 alone 6,102 / 6,177 / 6,002 GCUPS on C4)
        const int64_t w_first = rows_k1 * (int64_t)db.groups[g].ncols * kGroup;
        while (per_unit > 0 && crit > 0 && e < seg_end && (double)work / k1_wave < crit * (double)w_first) {
          for (int32_t k = 0; k < k1_wave && e < seg_end; k++, e++) {
            cells += rows_eff * grp_res[e];
            work += rows_k1 * db.groups[e].ncols * kGroup;
          }
        }
        P.units.push_back({kUnitInter, p, g, e, cells, work, 1, 1});
        g = e;
      }
    }
  }
  // clustered plans (long sequences carry the work, one worker's share is small): a K3 unit is
  // every pack x a contiguous range of sequence blocks, cut at equal cells (units = workers x
  // streams, or 4x an explicit target).  Its clusters claim (pack, block) tasks longest first,
  // so every pack's longest pairs start at once and the streams' units take about as long --
  // per-pack units finished in launch order (C5 at 1/8: 27 / 34 / 46 / 52 ms)
  if (k3_cluster > 1 && P.n_long_seqs > 0 && !P.pairs.empty()) {
    int64_t rows_all = 0, rows_pad = 0, long_res = 0;
    for (size_t p = 0; p < P.pairs.size(); p++) { rows_all += P.real_rows[p]; rows_pad += P.pairs[p].rows_padded; }
    for (int32_t s = 0; s < P.n_long_seqs; s++) long_res += db.sorted_len[s];
    const int64_t k3_cells = rows_all * long_res;
    const int64_t t4 = target > INT64_MAX / 4 ? INT64_MAX : 4 * target;
    const int64_t unit_target = o.target_unit_cells > 0
        ? t4 : std::max<int64_t>(1, k3_cells / std::max(1, n_workers * std::max(1, o.streams_per_device)));
    for (int32_t s = 0; s < P.n_long_seqs;) {
      int32_t e = s;
      int64_t cells = 0, work = 0;
      while (e < P.n_long_seqs && (cells < unit_target || e == s || (e - s) % kK3Warps)) {
        cells += rows_all * db.sorted_len[e];
        work += rows_pad * db.sorted_len[e];
        e++;
      }
      P.units.push_back({kUnitIntra, 0, s, e, cells, work, k3_cluster, (int32_t)P.pairs.size()});
      P.max_k3_seqs = std::max(P.max_k3_seqs, e - s);
      s = e;
    }
  }
  // drop empty units (e.g. all-empty queries still produce valid zero scores: keep them
  // so that every pair gets written, but they must have cells > 0 for the scheduler)
  for (auto &u : P.units) u.cells = std::max<int64_t>(u.cells, 1);
  // mixed regime (K1 carries most cells; K3 units overlap K1 units): a K3 unit too small for
  // its stream's share of the resident K3 CTAs holds a stream for its longest pair's whole
  // critical path; split its chunks over clusters of 4 (C4 at 1/8 of its database, 64
  // sequence blocks per unit: 5.82 -> 6.17 TCUPS; at full size, 148 blocks per unit, C = 4
  // costs 2 %)
  {
    static const int forced = [] { const char *e = getenv("SW_K3_CLUSTER"); return e ? atoi(e) : 0; }();
    static const int mixc = [] { const char *e = getenv("SW_K3_MIXC"); return e && atoi(e) > 1 ? atoi(e) : 4; }();
    if (forced == 0 && k3_cluster == 1 && o.target_unit_cells <= 0 && k3_slots > 0)
      for (Unit &u : P.units)
        if (u.kind == kUnitIntra) {
          const double ratio = (double)((u.b1 - u.b0 + kK3Warps - 1) / kK3Warps) * depth / k3_slots;
          if (ratio < 0.75) u.cluster = getenv("SW_K3_MIXC") ? mixc : balance_cluster(4, u.pair, u.pair + u.npk);
        }
  }
  // LPT by expected duration: intra-task (long-sequence) units first -- each warp walks a
  // whole long pair, so they have the longest latency -- then inter-task units by work.
  // A small K3 unit (fewer sequences than one block per SM) is interleaved with the largest
  // K1 units instead (K3, K1, K3, K1, ...): small K3 units alone on every stream would
  // leave SMs idle at the start of the step (C4 at 1/8 of its database: 140 ms of 447)
  static const bool interleave = [] { const char *e = getenv("SW_UNIT_INTERLEAVE"); return !(e && atoi(e) == 0); }();
  auto small3 = [](const Unit &u) {
    return interleave && u.kind == kUnitIntra && u.cluster == 1 && u.b1 - u.b0 < kK3UnitSeqs;
  };
  auto may_ovf = [&](const Unit &u) {
    for (int32_t p = u.pair; p < u.pair + u.npk; p++)
      if (P.pack_may_ovf[p]) return 1;
    return 0;
  };
  std::stable_sort(P.units.begin(), P.units.end(), [&](const Unit &a, const Unit &b) {
    const int ra = a.kind == kUnitIntra ? (small3(a) ? 1 : 0) : 2;
    const int rb = b.kind == kUnitIntra ? (small3(b) ? 1 : 0) : 2;
    if (ra != rb) return ra < rb;
    if (may_ovf(a) != may_ovf(b)) return may_ovf(a) > may_ovf(b);
    // clustered K3 units have about equal cells: the one holding the longest sequences (the
    // critical path) goes first -- units launched earlier progress faster when several share
    // the SMs (measured: finishing in launch order even with every CTA resident)
    if (a.kind == kUnitIntra && b.kind == kUnitIntra && a.cluster > 1 && b.cluster > 1 && a.npk > 1 && b.npk > 1)
      return a.b0 < b.b0;
    return a.work > b.work;
  });
  {
    size_t nb = 0, ns = 0;
    while (nb < P.units.size() && P.units[nb].kind == kUnitIntra && !small3(P.units[nb])) nb++;
    ns = nb;
    while (ns < P.units.size() && small3(P.units[ns])) ns++;
    std::vector<Unit> order(P.units.begin(), P.units.begin() + nb);
    size_t i3 = nb, i1 = ns;
    while (i3 < ns || i1 < P.units.size()) {
      if (i3 < ns) order.push_back(P.units[i3++]);
      if (i1 < P.units.size()) order.push_back(P.units[i1++]);
    }
    P.units.swap(order);
  }
  // the queries of each pack (a query lives in one half-run of one pack)
  P.pack_q_off.assign(P.pairs.size() + 1, 0);
  for (size_t p = 0; p < P.pairs.size(); p++) {
    std::vector<int32_t> qs;
    const QueryPair &qp = P.pairs[p];
    for (int32_t sidx = 0; sidx < qp.rows_padded / 16; sidx++) {
      const SliceInfo &x = P.slices[qp.slice_off + sidx];
      if (x.q_lo >= 0) qs.push_back(x.q_lo);
      if (x.q_hi >= 0) qs.push_back(x.q_hi);
    }
    std::sort(qs.begin(), qs.end());
    qs.erase(std::unique(qs.begin(), qs.end()), qs.end());
    P.pack_q.insert(P.pack_q.end(), qs.begin(), qs.end());
    P.pack_q_off[p + 1] = (int32_t)P.pack_q.size();
    P.max_pack_q = std::max<int32_t>(P.max_pack_q, (int32_t)qs.size());
  }
  for (const Unit &u : P.units)
    P.max_unit_q = std::max(P.max_unit_q, P.pack_q_off[u.pair + u.npk] - P.pack_q_off[u.pair]);
  // unit-table hash: ranks of one multi-process search must agree on it (net.cpp handshake)
  uint64_t h = 1469598103934665603ull;
  auto mix = [&](int64_t v) {
    for (int b = 0; b < 8; b++) { h ^= (uint64_t)((v >> (8 * b)) & 0xff); h *= 1099511628211ull; }
  };
  mix(nq); mix(db.n); mix(db.residues); mix((int64_t)P.units.size());
  for (const Unit &u : P.units) {
    mix(u.kind); mix(u.pair); mix(u.npk); mix(u.b0); mix(u.b1); mix(u.cells); mix(u.cluster);
  }
  for (int32_t q : P.pack_q) mix(q);
  P.hash = h;
  return P;
}

// ---------------------------------------------------------------- per-search device state
struct UnitLog {
  int32_t unit, worker, stream;
  double t_grant, t_start, t_end;   // host clock (s since the search start)
  int64_t cells;                    // the unit's cells
  int64_t cells_done;               // cells this replica computed (< cells when cancelled)
  int committed;                    // 1 = this replica committed the unit
  int cancelled;                    // 1 = cut short by WA cancellation (the unit finished elsewhere)
  int slowed;                       // 1 = ran under the straggler emulation
  float device_ms;                  // CUDA events around the unit's kernels on its stream
  float dev_t0, dev_t1;             // device ms of its start / end since the worker's start event
};

static const int kOvfCap = 1 << 20;


// K2 border row stride (columns): whole 4-column tiles, 32-byte aligned rows (cp.async)
static int64_t k2_stride(const Plan &P) { return (std::max<int64_t>(P.max_len, 1) + 3) / 4 * 4; }

// K2 arguments for the saturated-pair list of one stream
static K2Args k2_args(const Plan &P, const PackedDB &db, DevSearch &S, int stream_idx, int32_t alpha,
                      int32_t beta) {
  Device &D = *S.D;
  K2Args a;
  a.qcodes = S.qcodes.p; a.qoff = S.qoff.p;
  a.packed = D.packed.p; a.groups = D.groups.p; a.sorted_len = D.sorted_len.p; a.perm = D.perm.p;
  a.matrix = S.matrix.p;
  a.ovf = S.ovf.p + (size_t)stream_idx * S.ovf_cap; a.ovf_count = S.ovf_count.p + stream_idx;
  a.ovf_cap = S.ovf_cap; a.ovf_cursor = S.ovf_cursor.p + 2 * stream_idx;
  // a pair of at least big_cells (SW_K2_BIG: tuning, tests) is split over a K2 cluster:
  // 2^24 cells take ~1 ms on one SM
  // (a search routed to int32 lists every pair: many blocks, one pair each -- throughput,
  // not one pair's latency -- unless SW_K2_BIG says otherwise)
  static const int64_t big = [] { const char *e = getenv("SW_K2_BIG"); return e && atoll(e) > 0 ? atoll(e) : 0LL; }();
  a.big_cells = big > 0 ? big : S.k2_blocks > kK2Blocks ? INT64_MAX : (1LL << 24);
  a.ctl = S.k2_ctl.p + stream_idx;
  a.scores = S.scores; a.ndb = db.n; a.alpha = alpha; a.beta = beta; a.one = 1;
  const int64_t stride = k2_stride(P);
  a.border = S.k2_border.p + (size_t)stream_idx * k2_rows(S.k2_blocks) * stride * 2;
  a.border_stride = stride;
  return a;
}

// resident K3 CTAs a clustered launch may use: its stream's share (SW_K3_SHARE: percent of
// that share, tuning)
static int k3_share(int slots, int streams) {
  static const int pct = [] { const char *e = getenv("SW_K3_SHARE"); return e && atoi(e) > 0 ? atoi(e) : 100; }();
  return (int)((int64_t)slots * pct / 100 / std::max(1, streams));
}
// sm_cap > 0: the unit's kernels get at most sm_cap SMs' worth of blocks (a slower PE,
// straggler mode 1)
static void launch_unit(const Plan &P, const PackedDB &db, DevSearch &S, const Unit &U, int uidx,
                        int stream_idx, int32_t alpha, int32_t beta, int32_t thresh, int sm_cap) {
  Device &D = *S.D;
  cudaStream_t st = D.streams[stream_idx];
  const uint32_t na = ((uint32_t)(-alpha) & 0xffffu) * 0x10001u;
  const uint32_t nbm = ((uint32_t)(-beta) & 0xffffu) * 0x10001u;
  if (U.kind == kUnitInter) {
    K1Args a;
    a.packed = D.packed.p; a.groups = D.groups.p; a.perm = D.perm.p;
    a.prof = S.prof.p; a.pairs = S.pairs.p; a.slices = S.slices.p;
    a.pair = U.pair; a.g0 = U.b0;
    a.scores = S.scores; a.ndb = db.n;
    a.thresh = thresh;
    a.ovf = S.ovf.p + (size_t)stream_idx * S.ovf_cap; a.ovf_count = S.ovf_count.p + stream_idx;
    a.ovf_cap = S.ovf_cap; a.ovf_bits = S.ovf_bits.p;
    a.ovf_early = S.ovf_early_d + stream_idx;
    a.border = D.k1_border.p; a.border_slot_cols = D.slot_cols; a.slots_per_sm = D.slots_per_sm;
    a.slot_busy = D.slot_busy.p;
    a.abort_flag = S.abort_d + uidx;
    a.progress = S.progress.p + uidx;
    a.gclaim = S.gclaim.p + uidx;
    a.na = na; a.nb = nbm;
    launch_k1(a, U.b1 - U.b0, db.groups[U.b1 - 1].ncols, P.pairs[U.pair].rows_padded, st,
              sm_cap > 0 ? std::min(sm_cap, D.n_eff) : D.n_eff);
  } else {
    K3Args a;
    a.packed = D.packed.p; a.groups = D.groups.p; a.perm = D.perm.p; a.sorted_len = D.sorted_len.p;
    a.prof = S.prof.p; a.pairs = S.pairs.p; a.slices = S.slices.p;
    a.pair = U.pair; a.npk = U.npk; a.l0 = U.b0; a.l1 = U.b1;
    a.scores = S.scores; a.ndb = db.n;
    a.thresh = thresh;
    a.ovf = S.ovf.p + (size_t)stream_idx * S.ovf_cap; a.ovf_count = S.ovf_count.p + stream_idx;
    a.ovf_cap = S.ovf_cap; a.ovf_bits = S.ovf_bits.p;
    a.ovf_early = S.ovf_early_d + stream_idx;
    const int64_t stride = (std::max<int64_t>(P.max_len, 1) + 15) / 16 * 16;  // >= tiles * T
    a.border = S.k3_border.p + (size_t)stream_idx * S.k3_rows * stride;
    a.border_stride = stride;
    a.border_rows = S.k3_rows;
    a.kprog = nullptr;
    a.claim = nullptr;
    // tiles between a clustered chunk's progress publications (SW_K3_PUB: tuning)
    static const int pub = [] { const char *e = getenv("SW_K3_PUB"); return e && atoi(e) > 0 ? atoi(e) : 8; }();
    a.pub_every = pub;
    const int slots = D.n_eff * k3_blocks_per_sm();
    if (U.cluster > 1) {   // counters + the launch's claim counter, zeroed on its stream
      a.kprog = S.k3_prog.p + (size_t)stream_idx * (slots * kK3Warps + 1);
      a.claim = a.kprog + slots * kK3Warps;
      CK(cudaMemsetAsync(a.kprog, 0, sizeof(int32_t) * (slots * kK3Warps + 1), st));
    }
    a.abort_flag = S.abort_d + uidx;
    a.progress = S.progress.p + uidx;
    a.na = na; a.nb = nbm;
    // grid: cluster 1 -> a block per kK3Warps sequences; a slower PE -> its SM budget;
    // clustered units spanning every pack (long sequences carry the work) -> up to the whole
    // GPU (a later launch's queued clusters take the SMs an earlier unit frees: C5 at 1/4 of
    // its database 5.02 -> 5.37 TCUPS over per-pack units with equal shares); a clustered
    // per-pack unit beside K1 units (C4 at 1/8) -> its stream's share of the resident CTAs
    const int maxb = sm_cap > 0 ? std::min(D.n_eff, sm_cap) * k3_blocks_per_sm()
                   : U.cluster > 1 ? (U.npk > 1 ? slots : std::max(U.cluster, k3_share(slots, (int)D.streams.size())))
                                   : INT32_MAX;
    launch_k3(a, U.cluster, maxb, st);
  }
  S.launches++;
  // saturated pairs listed so far on this stream -> host (4 bytes): the worker launches
  // the int32 re-run (K2) on this stream when the unit completes and the list grew.  K2's
  // blocks need a whole SM's worth of shared memory, so an empty K2 launched after every
  // unit would wait for a K1 block to leave and stall the stream.
  CK(cudaMemcpyAsync(S.ovf_seen_h + stream_idx, S.ovf_count.p + stream_idx, sizeof(int32_t),
                     cudaMemcpyDeviceToHost, st));
  // and the unit's progress counter (the cells a cancelled replica really computed)
  CK(cudaMemcpyAsync(S.prog_h + stream_idx, S.progress.p + uidx, sizeof(int32_t),
                     cudaMemcpyDeviceToHost, st));
}
// progress units of a whole unit: K1 groups, K3 (sequence, chunk) pairs
static int64_t unit_progress_total(const Plan &P, const Unit &U) {
  if (U.kind == kUnitInter) return U.b1 - U.b0;
  int64_t nch = 0;
  for (int32_t p = U.pair; p < U.pair + U.npk; p++) nch += (P.pairs[p].rows + kK3Chunk - 1) / kK3Chunk;
  return (int64_t)(U.b1 - U.b0) * nch;
}

}  // namespace sw

using namespace sw;

extern "C" {

const char *sw_last_error(void) { return g_err.c_str(); }
const char *sw_version(void) { return "libsw 0.1 (sm_100a)"; }

void sw_opts_default(sw_opts *o) {
  if (!o) return;
  std::memset(o, 0, sizeof(*o));
  o->policy = SW_POLICY_PSS;
  o->workload_adjust = 1;
  o->omega = 4;
  o->streams_per_device = 4;
  o->target_unit_cells = 0;
  o->long_threshold = 0;
  o->straggler_slowdown = 6;
  o->straggler_mode = SW_STRAGGLER_SM_CAP;
}

int sw_db_create(const sw_seqset *dbs, const int *devices, int n_devices, sw_db **out) {
  return guarded([&] {
    if (!out) throw Error(SW_EINVAL, "out is NULL");
    *out = nullptr;
    validate_seqset(dbs, "db");
    int ndev_avail = 0;
    if (cudaGetDeviceCount(&ndev_avail) != cudaSuccess || ndev_avail <= 0)
      throw Error(SW_ECUDA, "no CUDA device available (libsw has no CPU fallback)");
    std::vector<int> devs;
    if (!devices || n_devices <= 0) devs.push_back(0);
    else devs.assign(devices, devices + n_devices);
    for (int d : devs)
      if (d < 0 || d >= ndev_avail) throw Error(SW_EINVAL, "device " + std::to_string(d) + " not present");
    auto db = std::make_unique<sw_db>();
    std::string err;
    int rc = pack_database(dbs->offsets, dbs->residues, dbs->n, db->host, err);
    if (rc != SW_OK) throw Error(rc, err);
    const PackedDB &H = db->host;
    for (int d : devs) {
      auto D = std::make_unique<Device>();
      D->id = d;
      CK(cudaSetDevice(d));
      CK(cudaDeviceGetAttribute(&D->n_sm, cudaDevAttrMultiProcessorCount, d));
      D->n_eff = D->n_sm;
      D->packed.alloc(d, std::max<size_t>(H.packed.size(), 1));
      D->groups.alloc(d, std::max<size_t>(H.groups.size(), 1));
      D->perm.alloc(d, std::max<size_t>(H.perm.size(), 1));
      D->sorted_len.alloc(d, std::max<size_t>(H.sorted_len.size(), 1));
      if (!H.packed.empty()) CK(cudaMemcpy(D->packed.p, H.packed.data(), sizeof(uint4) * H.packed.size(), cudaMemcpyHostToDevice));
      if (!H.groups.empty()) CK(cudaMemcpy(D->groups.p, H.groups.data(), sizeof(GroupInfo) * H.groups.size(), cudaMemcpyHostToDevice));
      if (!H.perm.empty()) CK(cudaMemcpy(D->perm.p, H.perm.data(), sizeof(int32_t) * H.perm.size(), cudaMemcpyHostToDevice));
      if (!H.sorted_len.empty()) CK(cudaMemcpy(D->sorted_len.p, H.sorted_len.data(), sizeof(int32_t) * H.sorted_len.size(), cudaMemcpyHostToDevice));
      db->devs.push_back(std::move(D));
    }
    // the merge reads the other GPUs' committed scores directly over NVLink (peer access)
    const size_t nd_ = devs.size();
    db->peer_ok.assign(nd_ * nd_, 0);
    for (size_t i = 0; i < nd_; i++)
      for (size_t j = 0; j < nd_; j++) {
        const int a = devs[i], b = devs[j];
        if (a == b) { db->peer_ok[i * nd_ + j] = 1; continue; }
        int ok = 0;
        if (cudaDeviceCanAccessPeer(&ok, a, b) == cudaSuccess && ok) {
          CK(cudaSetDevice(a));
          const cudaError_t e = cudaDeviceEnablePeerAccess(b, 0);
          if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
          else CK(e);
          db->peer_ok[i * nd_ + j] = 1;
        }
      }
    *out = db.release();
  });
}

void sw_db_destroy(sw_db *db) { delete db; }
int64_t sw_db_residues(const sw_db *db) { return db ? db->host.residues : 0; }
int32_t sw_db_size(const sw_db *db) { return db ? db->host.n : 0; }
int32_t sw_db_devices(const sw_db *db) { return db ? (int32_t)db->devs.size() : 0; }

int sw_topk_device(sw_db *db, const int32_t *scores_dev, int32_t nq, int32_t ndb, int32_t k,
                   sw_hit *hits_dev) {
  return guarded([&] {
    if (!db || db->devs.empty()) throw Error(SW_EINVAL, "db is NULL");
    if (k < 0 || k > SW_MAX_TOP_K) throw Error(SW_EINVAL, "top_k must be in [0, 64]");
    if (nq <= 0 || k == 0) return;
    CK(cudaSetDevice(db->devs[0]->id));
    launch_topk(scores_dev, nq, ndb, k, reinterpret_cast<int2 *>(hits_dev), 0);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
  });
}

int sw_search(const sw_seqset *queries, sw_db *db, const int8_t *matrix, int32_t gap_open,
              int32_t gap_extend, int32_t top_k, int32_t *scores, sw_hit *hits,
              const sw_opts *opts_in, sw_stats *stats) {
  if (db && db->busy.exchange(1)) {
    g_err = "a search is already running on this sw_db";
    return SW_EBUSY;
  }
  int rc = guarded([&] {
    if (!db) throw Error(SW_EINVAL, "db is NULL");
    validate_seqset(queries, "queries");
    if (gap_open < 0 || gap_extend < 0) throw Error(SW_EINVAL, "gap penalties must be >= 0");
    if ((int64_t)gap_open + 2 * (int64_t)gap_extend > (1 << 20))
      throw Error(SW_EINVAL, "gap_open + 2*gap_extend must be <= 2^20");
    if (top_k < 0 || top_k > SW_MAX_TOP_K) throw Error(SW_EINVAL, "top_k must be in [0, 64]");
    sw_opts o;
    sw_opts_default(&o);
    if (opts_in) o = *opts_in;
    if (o.omega < 1) o.omega = 4;
    if (o.streams_per_device <= 0) o.streams_per_device = 4;
    if (o.streams_per_device > kMaxStreams) throw Error(SW_EINVAL, "streams_per_device must be <= 64");
    if (o.policy != SW_POLICY_SS && o.policy != SW_POLICY_PSS) throw Error(SW_EINVAL, "bad policy");
    if (o.straggler_mode < 0 || o.straggler_mode > 2) throw Error(SW_EINVAL, "bad straggler_mode");
    const bool dist = o.dist_world > 1;
    if (dist && (o.dist_rank < 0 || o.dist_rank >= o.dist_world || !o.dist_host || o.dist_port <= 0))
      throw Error(SW_EINVAL, "bad multi-process options");
    if (dist && db->devs.size() != 1) throw Error(SW_EINVAL, "multi-process mode needs one device per rank");
    const int8_t *M = matrix ? matrix : blosum62();
    int max_s = INT_MIN, min_s = INT_MAX;
    for (int k = 0; k < 24 * 24; k++) { max_s = std::max(max_s, (int)M[k]); min_s = std::min(min_s, (int)M[k]); }
    const int32_t alpha = gap_open + gap_extend, beta = gap_extend;
    // precision routing: s16x2 only while alpha + beta <= 16384
    const bool s16_ok = (int64_t)alpha + beta <= 16384;
    // flag a lane half iff best~ + max(S) > 32767; if s16 is not usable
    // every pair is flagged (thresh = INT_MIN) and re-scored by the int32 kernel
    const int32_t thresh = s16_ok ? (max_s > 0 ? 32768 - max_s : 32768) : INT_MIN;

    const PackedDB &H = db->host;
    const int32_t nq = queries->n, nd = H.n;
    const int nW = dist ? 1 : (int)db->devs.size();
    // emulated GPUs (worker_sms > 0, in-process): every worker on a device gets a green SM
    // partition of worker_sms SMs rounded down to a multiple of 8 when the device splits
    // into enough of them, otherwise (or without green contexts) its DP grids are capped
    // to worker_sms SMs' worth of blocks (CTA caps: blocks of several workers share SMs)
    int32_t partition_mode = 0, partition_sms = 0;
    if (!dist && !db->devs.empty()) {
      std::vector<int> want_n;   // workers per device id
      for (auto &d : db->devs) {
        if ((int)want_n.size() <= d->id) want_n.resize(d->id + 1, 0);
        want_n[d->id]++;
      }
      const int sms8 = o.worker_sms / 8 * 8;
      bool green_ok = o.worker_sms > 0 && sms8 >= 8 && green_api().ok;
      auto reset_streams = [&](int dev_id) {   // the streams of every worker on dev_id
        for (auto &d : db->devs) {
          if (d->id != dev_id) continue;
          CK(cudaSetDevice(d->id));
          CK(cudaDeviceSynchronize());
          for (auto st : d->streams) cudaStreamDestroy(st);
          d->streams.clear();
          if (d->ws) {
            DevSearch &X = *d->ws;
            for (auto e : X.epi) cudaStreamDestroy(e);
            X.epi.clear();
            if (X.cancel_st) cudaStreamDestroy(X.cancel_st);
            if (X.noise_st) cudaStreamDestroy(X.noise_st);
            X.cancel_st = X.noise_st = nullptr;
          }
          d->gctx = nullptr;
        }
      };
      for (int dev = 0; green_ok && dev < (int)want_n.size(); dev++) {
        if (want_n[dev] == 0) continue;
        GreenSet *gs = nullptr;
        for (auto &g : db->green)
          if (g->dev == dev) gs = g.get();
        if (gs && gs->req == sms8 && gs->n >= want_n[dev]) continue;
        reset_streams(dev);   // before the old contexts go
        db->green.erase(std::remove_if(db->green.begin(), db->green.end(),
                                       [&](const std::unique_ptr<GreenSet> &g) { return g->dev == dev; }),
                        db->green.end());
        const GreenApi &ga = green_api();
        CK(cudaSetDevice(dev));
        CK(cudaFree(nullptr));   // the primary context exists
        CUdevResource all, rem;
        unsigned n = 0;
        if (ga.get_res(dev, &all, CU_DEV_RESOURCE_TYPE_SM) != CUDA_SUCCESS ||
            ga.split(nullptr, &n, &all, nullptr, 0, sms8) != CUDA_SUCCESS || (int)n < want_n[dev]) {
          green_ok = false;
          break;
        }
        std::vector<CUdevResource> parts(n);
        auto ng = std::make_unique<GreenSet>();
        ng->dev = dev;
        ng->req = sms8;
        if (ga.split(parts.data(), &n, &all, &rem, 0, sms8) != CUDA_SUCCESS || (int)n < want_n[dev]) {
          green_ok = false;
          break;
        }
        ng->sms = (int)parts[0].sm.smCount;
        for (int i = 0; i < want_n[dev]; i++) {
          CUdevResourceDesc desc;
          CUgreenCtx gc = nullptr;
          if (ga.gen_desc(&desc, &parts[i], 1) != CUDA_SUCCESS ||
              ga.create(&gc, desc, dev, CU_GREEN_CTX_DEFAULT_STREAM) != CUDA_SUCCESS) {
            green_ok = false;
            break;
          }
          ng->ctx.push_back(gc);
        }
        ng->n = (int)ng->ctx.size();
        db->green.push_back(std::move(ng));
      }
      // each worker's context (in order on its device) and SM count; a device whose workers
      // change context gets all its streams rebuilt (lazily, in the setup below)
      std::vector<int> used(want_n.size(), 0);
      std::vector<CUgreenCtx> want(db->devs.size(), nullptr);
      std::vector<int> neff(db->devs.size(), 0);
      for (size_t w = 0; w < db->devs.size(); w++) {
        Device &d = *db->devs[w];
        neff[w] = d.n_sm;
        if (!green_ok) continue;
        for (auto &g : db->green)
          if (g->dev == d.id && used[d.id] < g->n) {
            want[w] = g->ctx[used[d.id]++];
            neff[w] = g->sms;
          }
      }
      for (size_t w = 0; w < db->devs.size(); w++)
        if (db->devs[w]->gctx != want[w]) reset_streams(db->devs[w]->id);
      for (size_t w = 0; w < db->devs.size(); w++) {
        db->devs[w]->gctx = want[w];
        db->devs[w]->n_eff = neff[w];
      }
      if (o.worker_sms > 0) {
        partition_mode = green_ok ? 2 : 1;
        partition_sms = green_ok ? db->devs[0]->n_eff : o.worker_sms;
      }
    }
    // one wave of K1 blocks on the (first) GPU: SMs x resident K1 blocks per SM
    int32_t k1_wave = 0, k3_slots = 0;
    if (!db->devs.empty()) {
      CK(cudaSetDevice(db->devs[0]->id));
      k1_wave = db->devs[0]->n_eff * k1_blocks_per_sm();
      k3_slots = db->devs[0]->n_eff * k3_blocks_per_sm();
    }
    Plan P = make_plan(queries, H, o, dist ? o.dist_world : nW, M, thresh, k1_wave, k3_slots);
    bool any_cluster = false;
    for (const Unit &u : P.units) any_cluster |= u.cluster > 1;
    // K3 border rows per stream: one per sequence of the largest unit (cluster 1), and
    // (resident clusters x warps x C buffers) = k3_slots x kK3Warps when a unit is clustered
    const int64_t k3_rows = std::max<int64_t>(std::max(P.max_k3_seqs, 1), any_cluster ? (int64_t)k3_slots * kK3Warps : 0);
    const double wall0 = now_s();
    const int K = (hits && top_k > 0 && nq > 0) ? top_k : 0;   // hits wanted
    const int64_t nsc = (int64_t)nq * nd;
    const int32_t nU = (int32_t)P.units.size();

    std::vector<DevSearch *> S(nW);
    // ---------------- per device setup (cached, grow-only resources; not device-timed)
    for (int w = 0; w < nW; w++) {
      Device &D = *db->devs[w];
      CK(cudaSetDevice(D.id));
      if (!D.ws) D.ws = std::make_unique<DevSearch>();
      S[w] = D.ws.get();
      DevSearch &X = *S[w];
      X.D = &D;
      X.reset_counters();
      const int depth = o.streams_per_device;
      while ((int)D.streams.size() < depth) D.streams.push_back(make_stream(D.gctx, 0));
      if (D.slots_per_sm == 0) {
        D.slots_per_sm = k1_blocks_per_sm();
        D.sm_slots = 256;  // %smid < 256
        D.slot_cols = 0;
      }
      int32_t need_cols = 0;
      for (int32_t g = P.first_short_group; g < (int32_t)H.groups.size(); g++)
        need_cols = std::max(need_cols, H.groups[g].ncols);
      need_cols = (need_cols + kWordCols - 1) / kWordCols * kWordCols;   // whole 16-column tiles
      if (need_cols > D.slot_cols) {
        D.k1_border.alloc(D.id, (size_t)D.sm_slots * D.slots_per_sm * need_cols * 32);
        D.slot_busy.alloc(D.id, (size_t)D.sm_slots * D.slots_per_sm);
        CK(cudaMemset(D.slot_busy.p, 0, sizeof(int32_t) * D.slot_busy.n));
        D.slot_cols = need_cols;
      }
      X.qcodes.ensure(D.id, P.qcodes.size());
      X.qoff.ensure(D.id, P.qoff.size());
      X.pairs.ensure(D.id, P.pairs.size());
      X.matrix.ensure(D.id, 24 * 24);
      X.prof.ensure(D.id, (size_t)P.prof_total);
      if (!P.qcodes.empty()) CK(cudaMemcpy(X.qcodes.p, P.qcodes.data(), P.qcodes.size(), cudaMemcpyHostToDevice));
      CK(cudaMemcpy(X.qoff.p, P.qoff.data(), sizeof(int64_t) * P.qoff.size(), cudaMemcpyHostToDevice));
      if (!P.pairs.empty()) CK(cudaMemcpy(X.pairs.p, P.pairs.data(), sizeof(QueryPair) * P.pairs.size(), cudaMemcpyHostToDevice));
      X.slices.ensure(D.id, P.slices.size());
      if (!P.slices.empty()) CK(cudaMemcpy(X.slices.p, P.slices.data(), sizeof(SliceInfo) * P.slices.size(), cudaMemcpyHostToDevice));
      CK(cudaMemcpy(X.matrix.p, M, 24 * 24, cudaMemcpyHostToDevice));
      if (w == 0 && o.outputs_on_device && scores && !dist) X.scores = scores;
      else { X.scores_own.ensure(D.id, nsc); X.scores = X.scores_own.p; }
      // saturated-pair lists: 2^20 per stream, or every pair when the s16x2 path is not
      // usable (alpha + beta > 16384: all pairs are re-scored in int32)
      X.ovf_cap = s16_ok ? kOvfCap : (int32_t)std::min<int64_t>((int64_t)nq * nd + 1, INT32_MAX / 2);
      X.ovf.ensure(D.id, (size_t)depth * X.ovf_cap);
      X.ovf_count.ensure(D.id, depth);
      X.ovf_cursor.ensure(D.id, 2 * depth);
      X.k2_ctl.ensure(D.id, (size_t)depth);
      X.ovf_bits.ensure(D.id, ((size_t)nq * nd + 31) / 32);
      // K2 blocks: a few pairs normally; every pair when the search is routed to int32
      X.k2_blocks = s16_ok ? kK2Blocks : std::max(kK2Blocks, 3 * D.n_eff);
      X.k2_border.ensure(D.id, (size_t)depth * k2_rows(X.k2_blocks) * k2_stride(P) * 2);
      const size_t k3b = (size_t)depth * k3_rows * ((std::max<int64_t>(P.max_len, 1) + 15) / 16 * 16);
      if (P.n_long_seqs > 0) X.k3_border.ensure(D.id, k3b);
      if (any_cluster) X.k3_prog.ensure(D.id, (size_t)depth * (k3_slots * kK3Warps + 1));
      X.k3_rows = k3_rows;
      const size_t nu = std::max<size_t>(P.units.size(), 1);
      X.abort_dev.ensure(D.id, nu);
      CK(cudaMemset(X.abort_dev.p, 0, sizeof(int32_t) * nu));
      X.progress.ensure(D.id, nu);
      CK(cudaMemset(X.progress.p, 0, sizeof(int32_t) * nu));
      X.gclaim.ensure(D.id, nu);
      CK(cudaMemset(X.gclaim.p, 0, sizeof(int32_t) * nu));
      X.abort_d = X.abort_dev.p;
      X.cancelled.assign(nu, 0);
      if (K > 0) {
        X.pack_q.ensure(D.id, std::max<size_t>(P.pack_q.size(), 1));
        if (!P.pack_q.empty()) CK(cudaMemcpy(X.pack_q.p, P.pack_q.data(), sizeof(int32_t) * P.pack_q.size(), cudaMemcpyHostToDevice));
        X.unit_hits.ensure(D.id, nu * P.max_unit_q * K);
        X.worker_hits.ensure(D.id, (size_t)nq * K);
      }
      if (!X.one_h) {
        CK(cudaHostAlloc((void **)&X.one_h, sizeof(int32_t), cudaHostAllocDefault));
        *X.one_h = 1;
        CK(cudaHostAlloc((void **)&X.ovf_seen_h, sizeof(int32_t) * kMaxStreams, cudaHostAllocDefault));
        CK(cudaHostAlloc((void **)&X.prog_h, sizeof(int32_t) * kMaxStreams, cudaHostAllocDefault));
        CK(cudaHostAlloc((void **)&X.ovf_early_h, sizeof(int32_t) * kMaxStreams, cudaHostAllocMapped));
        CK(cudaHostGetDevicePointer((void **)&X.ovf_early_d, X.ovf_early_h, 0));
      }
      for (int k = 0; k < kMaxStreams; k++) ((volatile int32_t *)X.ovf_early_h)[k] = 0;
      if (!X.cancel_st) X.cancel_st = make_stream(D.gctx, 0);
      {
        int lo = 0, hi = 0;
        CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
        // (the local-load stream is created only when a worker emulates one: every stream
        // takes one of the GPU's hardware work queues)
        if (!X.noise_st && o.straggler_mode == SW_STRAGGLER_NOISE && o.straggler_mask)
          X.noise_st = make_stream(D.gctx, hi);
        while (X.epi.empty()) X.epi.push_back(make_stream(D.gctx, hi));   // one per worker
      }
      if (!X.ev_start) CK(cudaEventCreate(&X.ev_start));
      if (!X.ev_end) CK(cudaEventCreate(&X.ev_end));
      if (!X.ev_data) CK(cudaEventCreateWithFlags(&X.ev_data, cudaEventDisableTiming));
      while ((int)X.u_start.size() < depth) {
        cudaEvent_t a, b;
        CK(cudaEventCreate(&a));
        CK(cudaEventCreate(&b));
        X.u_start.push_back(a);
        X.u_end.push_back(b);
      }
      CK(cudaDeviceSynchronize());
    }

    // ---------------- scheduler (in-process master, or TCP client of rank 0's master)
    std::vector<int64_t> ucells(P.units.size());
    for (size_t u = 0; u < P.units.size(); u++) ucells[u] = P.units[u].cells;
    std::unique_ptr<MasterServer> server;
    std::unique_ptr<SchedClient> client;
    sw_sched *sched = nullptr;
    if (dist) {
      if (o.dist_rank == 0) {
        server = std::make_unique<MasterServer>();
        server->start(o.dist_port, o.dist_world, (int32_t)ucells.size(), ucells.data(), o.policy,
                      o.workload_adjust, o.omega, P.hash);
      }
      client = std::make_unique<SchedClient>();
      client->connect(o.dist_host, o.dist_port, o.dist_rank, 30.0, P.hash);
    } else {
      sched = sw_sched_create(nW, (int32_t)ucells.size(), ucells.data(), o.policy, o.workload_adjust, o.omega);
      if (!sched && !ucells.empty()) throw Error(SW_EINVAL, "scheduler creation failed");
    }
    struct SchedGuard { sw_sched *s; ~SchedGuard() { if (s) sw_sched_destroy(s); } } sg{sched};
    const int my_worker_base = dist ? o.dist_rank : 0;
    auto sreq = [&](int w, double t, int32_t *out, int cap) -> int32_t {
      if (client) return client->request(t, out, cap);
      if (!sched) return -1;
      return sw_sched_request(sched, w, t, out, cap);
    };
    // an idle worker's request: one message that waits at the master (long poll)
    auto sreq_wait = [&](int w, double t, int32_t *out, int cap, double timeout) -> int32_t {
      if (client) return client->request_wait(t, out, cap, timeout);
      if (!sched) return -1;
      return sw_sched_request_wait(sched, w, t, out, cap, timeout);
    };
    auto srep = [&](int w, double t, double cells, double sec) {
      if (client) client->report(t, cells, sec);
      else if (sched) sw_sched_report(sched, w, t, cells, sec);
    };
    auto scomp = [&](int w, int u, double t) -> int {
      if (client) return client->complete(u, t);
      return sched ? sw_sched_complete(sched, w, u, t) : 1;
    };
    auto sabandon = [&](int w, int u, double t) {
      if (client) client->abandon(u, t);
      else if (sched) sw_sched_abandon(sched, w, u, t);
    };
    auto sfin = [&](int u) -> int {
      if (client) return client->is_finished(u);
      return sched ? sw_sched_is_finished(sched, u) : 0;
    };
    auto sstart = [&](int w, int u, double t) -> int {
      if (client) return client->start(u, t);
      return sched ? sw_sched_start(sched, w, u, t) : 1;
    };

    // ---------------- workers: one thread per device
    std::vector<UnitLog> ulog;
    std::mutex ulog_mu;
    std::vector<std::vector<SegInfo>> worker_segs_(nW);   // committed segments of workers > 0
    std::atomic<int> ready{0};
    std::atomic<bool> failed{false};   // a worker failed: the others stop (no hang on its units)
    std::vector<std::string> werr(nW);
    std::vector<int> wcode(nW, 0);
    const double t0 = now_s();
    auto worker = [&](int w) {
      DevSearch &X = *S[w];
      Device &D = *X.D;
      const int wid = my_worker_base + w;
      bool noise_on = false;
      auto stop_noise = [&] {
        if (!noise_on) return;
        noise_on = false;
        cudaMemcpyAsync(X.noise_flag.p, X.one_h, sizeof(int32_t), cudaMemcpyHostToDevice, X.cancel_st);
        cudaStreamSynchronize(X.noise_st);
      };
      try {
        CK(cudaSetDevice(D.id));
        const int depth = o.streams_per_device;
        cudaStream_t s0 = D.streams[0];
        // barrier across workers, then the common device start
        ready.fetch_add(1);
        while (ready.load() < nW) std::this_thread::yield();
        CK(cudaEventRecord(X.ev_start, s0));
        launch_fill(X.scores, (int64_t)nq * nd, -1, s0);
        CK(cudaMemsetAsync(X.ovf_count.p, 0, sizeof(int32_t) * depth, s0));
        CK(cudaMemsetAsync(X.ovf_cursor.p, 0, sizeof(int32_t) * 2 * depth, s0));
        // list slots read (-1, -1) until written: a K2 running beside the unit that lists an
        // entry may see it counted before it is stored
        CK(cudaMemsetAsync(X.ovf.p, 0xff, sizeof(int2) * (size_t)depth * X.ovf_cap, s0));
        CK(cudaMemsetAsync(X.ovf_bits.p, 0, sizeof(uint32_t) * (((size_t)nq * nd + 31) / 32), s0));
        launch_profile(X.qcodes.p, X.qoff.p, X.pairs.p, (int)P.pairs.size(), X.slices.p, X.matrix.p,
                       X.prof.p, P.prof_total, s0);
        X.launches += 2 + (P.pairs.empty() ? 0 : 1);
        CK(cudaGetLastError());
        cudaEvent_t setup_done;
        CK(cudaEventCreateWithFlags(&setup_done, cudaEventDisableTiming));
        CK(cudaEventRecord(setup_done, s0));
        for (int k = 1; k < depth; k++) CK(cudaStreamWaitEvent(D.streams[k], setup_done, 0));
        // slower-PE emulation (SURVEY §8(d) WA experiment; P24 §V.C local load from t_after)
        const bool straggler = (o.straggler_mask >> wid) & 1ull;
        const int slow = std::max(1, o.straggler_slowdown);
        // the worker's SM budget: the whole GPU, or its partition (worker_sms, experiments)
        const int budget = D.gctx ? D.n_eff : o.worker_sms > 0 ? std::min(o.worker_sms, D.n_sm) : D.n_sm;
        const int sm_cap = (budget + slow - 1) / slow;     // ceil(budget / slowdown)
        // a budget is split over the worker's streams (up to `depth` units run at once), so
        // the whole worker holds ~budget SMs' worth of blocks
        const int sm_share = std::max(1, (sm_cap + depth - 1) / depth);
        // (a green partition needs no cap: its kernels cannot leave its SMs)
        const int part_share = (o.worker_sms > 0 && !D.gctx) ? std::max(1, (budget + depth - 1) / depth) : 0;
        const double t_after = 1e-3 * std::max(0, o.straggler_after_ms);
        std::deque<int32_t> pending;
        std::vector<int32_t> inflight(depth, -1);
        std::vector<double> t_grant(P.units.size(), 0), t_launch(depth, 0);
        std::vector<double> hold_until(depth, 0);
        std::vector<int> completed_wait(depth, 0), slowed(depth, 0);
        std::vector<int32_t> k2_upto(depth, 0);   // saturated pairs handed to K2 per stream
        // the int32 re-run (K2) of stream k's saturated pairs once `seen` of them are listed,
        // on the epilogue stream
        auto launch_rerun = [&](int k, int32_t seen) {
          if (seen <= k2_upto[k]) return;
          const K2Args k2a = k2_args(P, H, X, k, alpha, beta);
          std::pair<cudaEvent_t, cudaEvent_t> ev;
          CK(cudaEventCreate(&ev.first));
          CK(cudaEventCreate(&ev.second));
          X.k2_ev.push_back(ev);
          CK(cudaMemsetAsync(k2a.ctl, 0, sizeof(K2Ctl), X.epi[0]));
          CK(cudaEventRecord(ev.first, X.epi[0]));
          launch_k2(k2a, X.k2_blocks, X.epi[0]);
          CK(cudaEventRecord(ev.second, X.epi[0]));
          CK(cudaGetLastError());
          X.launches++;
          k2_upto[k] = seen;
        };
        bool done = false, changed = true;
        double last_req = 0, req_gap = 2e-3;
        std::vector<double> stream_rate(depth, 0.0);
        int32_t buf[64];
        while (true) {
          if (failed.load()) throw Error(SW_ECUDA, "another worker failed");
          bool progressed = false;
          const double tn = now_s();
          const bool slow_now = straggler && slow > 1 && tn - t0 >= t_after;
          if (slow_now && o.straggler_mode == SW_STRAGGLER_NOISE && !noise_on) {
            // local load: SM-filling blocks on all but ceil(n_sm / slowdown) SMs
            X.noise_flag.ensure(D.id, 1);
            X.noise_sink.ensure(D.id, D.n_eff);
            CK(cudaMemsetAsync(X.noise_flag.p, 0, sizeof(int32_t), X.noise_st));
            launch_noise(X.noise_flag.p, D.n_eff - sm_cap, 60ull * 1000000000ull, X.noise_sink.p, X.noise_st);
            CK(cudaGetLastError());
            noise_on = true;
          }
          // saturated pairs listed by running units (published by the DP kernels as they list
          // them): their int32 re-run starts now, beside the unit, instead of after it -- a
          // long pair's re-run was the tail of C5 at 1/8 of its database (SW_K2_EARLY=0: after
          // the unit; C5 at 1/8 5.05 vs 4.85 TCUPS, full C5 6.06 vs 6.03)
          static const bool early = [] { const char *e = getenv("SW_K2_EARLY"); return !(e && atoi(e) == 0); }();
          if (early)
            for (int k = 0; k < depth; k++) launch_rerun(k, ((volatile int32_t *)X.ovf_early_h)[k]);
          // completions
          for (int k = 0; k < depth; k++) {
            if (inflight[k] < 0) continue;
            const int u = inflight[k];
            if (!completed_wait[k]) {
              cudaError_t q = cudaEventQuery(X.u_end[k]);
              if (q == cudaErrorNotReady) continue;
              CK(q);
              completed_wait[k] = 1;
              if (slowed[k] && o.straggler_mode == SW_STRAGGLER_HOLD && !X.cancelled[u]) {
                // host-side emulation: hold the completion back (slow-1) x the device time
                float ms = 0;
                cudaEventElapsedTime(&ms, X.u_start[k], X.u_end[k]);
                hold_until[k] = tn + (slow - 1.0) * ms * 1e-3;
              } else {
                hold_until[k] = tn;
              }
            }
            // an emulated slow PE stops holding a replica whose task finished elsewhere
            // (WA: the first result wins and the other replicas are cancelled)
            const bool cut = tn < hold_until[k] && sfin(u);
            if (tn < hold_until[k] && !cut) continue;
            const Unit &U = P.units[u];
            float ms = 0, d0 = 0, d1 = 0;
            cudaEventElapsedTime(&ms, X.u_start[k], X.u_end[k]);
            cudaEventElapsedTime(&d0, X.ev_start, X.u_start[k]);
            cudaEventElapsedTime(&d1, X.ev_start, X.u_end[k]);
            // what the replica really computed: its progress counter (groups / sequence-chunks)
            const int64_t ptot = std::max<int64_t>(1, unit_progress_total(P, U));
            const int64_t pdone = std::min<int64_t>(ptot, ((volatile int32_t *)X.prog_h)[k]);
            const bool was_cancelled = X.cancelled[u] && pdone < ptot;
            const int64_t cells_done = was_cancelled ? (int64_t)((double)U.cells * pdone / ptot) : U.cells;
            int committed = 0;
            if (was_cancelled) {
              // a losing replica stopped early by its abort flag: give it up; its partial
              // cells count as duplicated work and as this PE's progress
              sabandon(wid, u, tn);
              X.n_cancelled++;
            } else {
              committed = scomp(wid, u, tn);
            }
            // progress notification (P18 §IV.A.2): the worker's current rate = the sum over
            // its streams of (cells / duration) of each stream's last unit -- units share the
            // GPU, so each one's rate is its share; a duration is launch -> observed
            // completion, which includes a GPU-side slowdown (SM cap, local load) and the
            // host-side hold
            if (!cut && cells_done > 0) {
              stream_rate[k] = (double)cells_done / std::max(1e-6, tn - t_launch[k]);
              double v = 0;
              for (double r : stream_rate) v += r;
              srep(wid, tn, v, 1.0);
            }
            if (U.kind == kUnitInter) { X.k1_sec += ms * 1e-3; X.k1_cells += cells_done; }
            else { X.k3_sec += ms * 1e-3; X.k3_cells += cells_done; }
            if (!committed) X.dup_cells += cells_done;
            X.last_dev = std::max(X.last_dev, 1e-3 * d1);
            {
              std::lock_guard<std::mutex> g(ulog_mu);
              ulog.push_back({u, wid, k, t_grant[u] - t0, t_launch[k] - t0, tn - t0, U.cells, cells_done,
                              committed, was_cancelled ? 1 : 0, slowed[k], ms, d0, d1});
            }
            inflight[k] = -1;
            completed_wait[k] = 0;
            progressed = changed = true;
            req_gap = 2e-3;
            // epilogue of a completed unit on the worker's high-priority epilogue stream, so
            // the stream goes straight on to its next unit: the int32 re-run of what the
            // stream's units saturated (K2), then (committed) the unit's top-k (K5u).  Both
            // small kernels wait for free SM slots behind persistent K1 blocks; on the unit's
            // own stream they delayed its next unit (C4 at 1/8 of its database: 16 % idle).
            // K2 may see entries a later unit on the stream is appending: it recomputes such
            // a pair exactly, and the later partial maxima of its other slices are smaller.
            launch_rerun(k, ((volatile int32_t *)X.ovf_seen_h)[k]);
            if (committed) {
              X.committed.push_back(u);
              // K5u: this unit's top-k per query of its pack (after its int32 re-run)
              if (K > 0) {
                int32_t s0u, s1u;
                unit_seq_range(U, nd, s0u, s1u);
                const int32_t q0 = P.pack_q_off[U.pair], nqp = P.pack_q_off[U.pair + U.npk] - q0;
                launch_unit_topk(X.scores, nd, D.perm.p, s0u, s1u, X.pack_q.p + q0, nqp, K,
                                 X.unit_hits.p + (size_t)u * P.max_unit_q * K, X.epi[0]);
                CK(cudaGetLastError());
                X.launches++;
              }
            }
          }
          // cancel in-flight replicas whose task finished elsewhere (WA loser)
          for (int k = 0; k < depth; k++)
            if (inflight[k] >= 0 && !X.cancelled[inflight[k]] && sfin(inflight[k])) {
              X.cancelled[inflight[k]] = 1;
              CK(cudaMemcpyAsync(X.abort_d + inflight[k], X.one_h, sizeof(int32_t),
                                 cudaMemcpyHostToDevice, X.cancel_st));
            }
          // launch pending units on free streams
          for (int k = 0; k < depth && !pending.empty(); k++) {
            if (inflight[k] >= 0) continue;
            const int u = pending.front();
            pending.pop_front();
            // finished elsewhere, or moved to an idle worker by WA before it started
            if (!sstart(wid, u, now_s())) { progressed = changed = true; k--; continue; }
            const bool sl = straggler && slow > 1 && now_s() - t0 >= t_after;
            CK(cudaEventRecord(X.u_start[k], D.streams[k]));
            // NVTX range around the unit's launches, e.g. for a profiler:
            //   ncu --nvtx --nvtx-include "regex:K1 unit 19 .*/" ... (push/pop range: trailing /)
            char nv[64];
            snprintf(nv, sizeof(nv), "%s unit %d worker %d", P.units[u].kind == kUnitInter ? "K1" : "K3", u, wid);
            nvtxRangePushA(nv);
            launch_unit(P, H, X, P.units[u], u, k, alpha, beta, thresh,
                        (sl && o.straggler_mode == SW_STRAGGLER_SM_CAP) ? sm_share : part_share);
            nvtxRangePop();
            CK(cudaGetLastError());
            CK(cudaEventRecord(X.u_end[k], D.streams[k]));
            inflight[k] = u;
            slowed[k] = sl ? 1 : 0;
            t_launch[k] = now_s();
            progressed = true;
          }
          // ask the master for more when the local queue is empty and a stream is free:
          // once per change (a completion) or every 2 ms while units run; an idle worker
          // sends one request that waits at the master until the task table changes
          int n_inflight = 0;
          for (int k = 0; k < depth; k++) n_inflight += inflight[k] >= 0;
          if (!done && pending.empty() && n_inflight < depth) {
            int32_t r = 0;
            const double tq = now_s();
            if (n_inflight == 0) {
              // the master answers as soon as its table changes; the timeout only re-tests
              // WA's time-dependent ETA condition (WA off: nothing to re-test)
              r = sreq_wait(wid, tq, buf, 64, o.workload_adjust ? 0.005 : 0.25);
              last_req = tq;
              changed = false;
            } else if (changed || tq - last_req > req_gap) {
              r = sreq(wid, tq, buf, 64);
              last_req = tq;
              changed = false;
              // nothing granted while units still run here: ask again later and later
              // (2 ms doubling to 64 ms; a completion or a grant resets it)
              req_gap = r == 0 ? std::min(0.064, 2 * req_gap) : 2e-3;
            }
            if (r < 0) done = true;
            else {
              for (int32_t i = 0; i < r; i++) { pending.push_back(buf[i]); t_grant[buf[i]] = now_s(); }
              if (r > 0) {   // one mark per task-allocation interaction (P24 Figs. 7/8)
                char nv[64];
                snprintf(nv, sizeof(nv), "grant %d unit(s) to worker %d", r, wid);
                nvtxMarkA(nv);
              }
              if (r > 0) progressed = changed = true;
            }
          }
          if (done && pending.empty() && n_inflight == 0) break;
          // poll completions every 20 us
          if (!progressed && n_inflight > 0) std::this_thread::sleep_for(std::chrono::microseconds(20));
        }
        stop_noise();
        // the int32 re-runs ran on each stream after the units that saturated; check the lists
        for (int k = 0; k < depth; k++) CK(cudaStreamSynchronize(D.streams[k]));
        CK(cudaStreamSynchronize(X.epi[0]));
        for (auto &e : X.k2_ev) {
          float ms = 0;
          CK(cudaEventElapsedTime(&ms, e.first, e.second));
          X.k2_sec += 1e-3 * ms;
        }
        std::vector<int32_t> novf(depth, 0), ncur(2 * depth, 0);
        CK(cudaMemcpy(novf.data(), X.ovf_count.p, sizeof(int32_t) * depth, cudaMemcpyDeviceToHost));
        CK(cudaMemcpy(ncur.data(), X.ovf_cursor.p, sizeof(int32_t) * 2 * depth, cudaMemcpyDeviceToHost));
        X.n_ovf = 0;
        for (int k = 0; k < depth; k++) {
          if (novf[k] > X.ovf_cap) throw Error(SW_ENOMEM, "overflow list capacity exceeded");
          X.n_ovf += novf[k];
          if (ncur[2 * k] < novf[k] || ncur[2 * k + 1] < novf[k])
            throw Error(SW_ECUDA, "int32 re-run left saturated pairs");
        }
        // ---- data plane, on this device: top-k over the units this worker committed
        // (K5m), and (in-process, device != first) the committed units' scores packed densely
        // for the peer copy; multi-process: the committed-only score matrix
        std::vector<SegInfo> segs;
        int64_t seg_total = 0;
        const bool need_segs = (dist && scores) || (!dist && w > 0 && scores);
        if (need_segs)
          for (int32_t u : X.committed) {
            int32_t s0u, s1u;
            unit_seq_range(P.units[u], nd, s0u, s1u);
            for (int32_t j = P.pack_q_off[P.units[u].pair]; j < P.pack_q_off[P.units[u].pair + P.units[u].npk]; j++) {
              segs.push_back({P.pack_q[j], s0u, s1u, 0, seg_total});
              seg_total += s1u - s0u;
            }
          }
        std::vector<int32_t> tab;   // list_off[nq+1], then list_idx
        if (K > 0) {
          std::vector<std::vector<int32_t>> per_q(nq);
          for (int32_t u : X.committed) {
            const int32_t p = P.units[u].pair, p1 = p + P.units[u].npk;
            for (int32_t j = P.pack_q_off[p]; j < P.pack_q_off[p1]; j++)
              per_q[P.pack_q[j]].push_back(u * P.max_unit_q + (j - P.pack_q_off[p]));
          }
          tab.assign(nq + 1, 0);
          for (int32_t q = 0; q < nq; q++) tab[q + 1] = tab[q] + (int32_t)per_q[q].size();
          for (int32_t q = 0; q < nq; q++) tab.insert(tab.end(), per_q[q].begin(), per_q[q].end());
        }
        if (!tab.empty() || !segs.empty()) {
          X.list_tab.ensure(D.id, std::max<size_t>(tab.size(), 1));
          if (!tab.empty()) CK(cudaMemcpyAsync(X.list_tab.p, tab.data(), sizeof(int32_t) * tab.size(), cudaMemcpyHostToDevice, s0));
          X.segs.ensure(D.id, std::max<size_t>(segs.size(), 1));
          if (!segs.empty()) CK(cudaMemcpyAsync(X.segs.p, segs.data(), sizeof(SegInfo) * segs.size(), cudaMemcpyHostToDevice, s0));
        }
        if (K > 0) {
          launch_merge_topk(X.unit_hits.p, K, X.list_tab.p, X.list_tab.p + nq + 1, nq, K, X.worker_hits.p, s0);
          X.launches++;
        }
        if (dist && scores && nsc > 0) {   // this rank's output: its committed pairs, -1 elsewhere
          X.out_stage.ensure(D.id, o.outputs_on_device ? 1 : nsc);
          int32_t *dst = o.outputs_on_device ? scores : X.out_stage.p;
          launch_fill(dst, nsc, -1, s0);
          launch_seg_copy(X.scores, dst, nd, D.perm.p, X.segs.p, (int)segs.size(), 2, s0);
          X.launches += segs.empty() ? 1 : 2;
        } else if (!segs.empty() && !db->peer_ok[(size_t)w]) {
          // device 0 cannot read this GPU's memory: pack the committed pairs densely for a
          // (host-staged) peer copy
          X.compact.ensure(D.id, std::max<int64_t>(seg_total, 1));
          launch_seg_copy(X.scores, X.compact.p, nd, D.perm.p, X.segs.p, (int)segs.size(), 0, s0);
          X.launches++;
        }
        CK(cudaGetLastError());
        CK(cudaEventRecord(X.ev_data, s0));
        CK(cudaEventRecord(X.ev_end, s0));
        CK(cudaEventSynchronize(X.ev_end));
        CK(cudaEventDestroy(setup_done));
        X.finish_wall = now_s();
        // seg list kept for the merge stage (device 0 needs the offsets)
        if (!dist && w > 0) {
          std::lock_guard<std::mutex> g(ulog_mu);
          worker_segs_[w].swap(segs);
        }
      } catch (const Error &e) {
        stop_noise();
        werr[w] = e.what();
        wcode[w] = e.code;
        failed.store(true);
        ready.fetch_add(1 << 20);  // release the barrier
      } catch (const std::exception &e) {
        stop_noise();
        werr[w] = e.what();
        wcode[w] = SW_ECUDA;
        failed.store(true);
        ready.fetch_add(1 << 20);
      }
    };
    std::vector<std::thread> threads;
    for (int w = 0; w < nW; w++) threads.emplace_back(worker, w);
    for (auto &t : threads) t.join();
    for (int w = 0; w < nW; w++)
      if (wcode[w] && werr[w] != "another worker failed")
        throw Error(wcode[w], "worker " + std::to_string(w) + ": " + werr[w]);
    for (int w = 0; w < nW; w++)
      if (wcode[w]) throw Error(wcode[w], "worker " + std::to_string(w) + ": " + werr[w]);
    int32_t n_req = 0, n_wa = 0, n_grant = 0;
    if (sched) {
      n_wa = (int32_t)sw_sched_counter(sched, 1);
      n_req = (int32_t)sw_sched_counter(sched, 0);
      n_grant = (int32_t)sw_sched_counter(sched, 3);
      db->sched_log = sw_sched_log_json(sched);
    }
    if (client) {
      client->done();
      n_wa = client->wa_grants();
      n_req = client->requests();
      n_grant = client->grant_msgs();
    }
    if (server) {
      server->stop();
      db->sched_log = server->final_log();
    } else if (!sched) {
      db->sched_log = "[]";
    }

    // ---------------- merge (the paper's "the slaves send their results to the master, that
    // merges them", P16 §IV).  In-process with several GPUs: a kernel on the first GPU reads
    // every other GPU's committed units' scores over NVLink (peer access enabled at
    // sw_db_create; without it they are packed densely and copied) and the top-k lists are
    // copied and merged (K5m).
    // Multi-process: each rank keeps its committed pairs and hits; the binding gathers the
    // hits (NCCL) and merges them with sw_merge_hits.
    DevSearch &X0 = *S[0];
    const int dev0 = X0.D->id;
    CK(cudaSetDevice(dev0));
    cudaStream_t s0 = X0.D->streams[0];
    cudaEvent_t m_start, m_end;
    CK(cudaEventCreate(&m_start));
    CK(cudaEventCreate(&m_end));
    CK(cudaEventRecord(m_start, s0));
    int64_t peer_bytes = 0;
    DBuf<int32_t> stage;
    DBuf<SegInfo> segs0;
    DBuf<int32_t> tab0;
    DBuf<int2> hits_tmp;
    const int2 *hits_final = nullptr;
    if (!dist && nW > 1) {
      for (int w = 1; w < nW; w++) {
        const std::vector<SegInfo> &sg_ = worker_segs_[w];
        if (sg_.empty()) continue;
        const int64_t total = sg_.back().off + (sg_.back().s1 - sg_.back().s0);
        CK(cudaStreamWaitEvent(s0, S[w]->ev_data, 0));
        segs0.ensure(dev0, sg_.size());
        CK(cudaMemcpyAsync(segs0.p, sg_.data(), sizeof(SegInfo) * sg_.size(), cudaMemcpyHostToDevice, s0));
        if (db->peer_ok[(size_t)w]) {
          // one kernel on device 0 reads worker w's committed pairs over NVLink (peer loads)
          // and writes them into the result: no staging buffer, no separate copy
          launch_seg_copy(S[w]->scores, X0.scores, nd, X0.D->perm.p, segs0.p, (int)sg_.size(), 2, s0);
        } else {
          stage.ensure(dev0, std::max<int64_t>(total, 1));
          CK(cudaMemcpyPeerAsync(stage.p, dev0, S[w]->compact.p, S[w]->D->id, sizeof(int32_t) * total, s0));
          launch_seg_copy(stage.p, X0.scores, nd, X0.D->perm.p, segs0.p, (int)sg_.size(), 1, s0);
        }
        peer_bytes += sizeof(int32_t) * total;
        X0.launches++;
        // segs0 / the staging buffer are reused by the next worker: ordered on s0
      }
      if (K > 0) {
        X0.all_hits.ensure(dev0, (size_t)nW * nq * K);
        for (int w = 0; w < nW; w++) {
          CK(cudaStreamWaitEvent(s0, S[w]->ev_data, 0));
          CK(cudaMemcpyPeerAsync(X0.all_hits.p + (size_t)w * nq * K, dev0, S[w]->worker_hits.p, S[w]->D->id,
                                 sizeof(int2) * nq * K, s0));
          if (w > 0) peer_bytes += sizeof(int2) * nq * K;
        }
        std::vector<int32_t> tab(nq + 1 + (size_t)nq * nW);
        for (int32_t q = 0; q <= nq; q++) tab[q] = q * nW;
        for (int32_t q = 0; q < nq; q++)
          for (int w = 0; w < nW; w++) tab[nq + 1 + (size_t)q * nW + w] = w * nq + q;
        tab0.ensure(dev0, tab.size());
        CK(cudaMemcpyAsync(tab0.p, tab.data(), sizeof(int32_t) * tab.size(), cudaMemcpyHostToDevice, s0));
        hits_tmp.ensure(dev0, (size_t)nq * K);
        launch_merge_topk(X0.all_hits.p, K, tab0.p, tab0.p + nq + 1, nq, K, hits_tmp.p, s0);
        X0.launches++;
        hits_final = hits_tmp.p;
      }
    } else if (K > 0) {
      hits_final = X0.worker_hits.p;
    }
    if (K > 0 && o.outputs_on_device)
      CK(cudaMemcpyAsync(hits, hits_final, sizeof(int2) * nq * K, cudaMemcpyDeviceToDevice, s0));
    CK(cudaGetLastError());
    CK(cudaEventRecord(m_end, s0));
    CK(cudaEventSynchronize(m_end));
    float merge_ms = 0;
    cudaEventElapsedTime(&merge_ms, m_start, m_end);
    cudaEventDestroy(m_start);
    cudaEventDestroy(m_end);

    // device time: max over devices of (end - start), device 0 extended by the merge
    double dev_sec = 0;
    for (int w = 0; w < nW; w++) {
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, S[w]->ev_start, S[w]->ev_end));
      double sec = ms * 1e-3 + (w == 0 ? merge_ms * 1e-3 : 0);
      dev_sec = std::max(dev_sec, sec);
    }
    // outputs
    if (scores && nsc > 0 && !o.outputs_on_device) {
      const int32_t *src = dist ? X0.out_stage.p : X0.scores;
      CK(cudaMemcpy(scores, src, sizeof(int32_t) * nsc, cudaMemcpyDeviceToHost));
    }
    if (K > 0 && !o.outputs_on_device)
      CK(cudaMemcpy(hits, hits_final, sizeof(int2) * nq * K, cudaMemcpyDeviceToHost));
    const double wall = now_s() - wall0;

    if (stats) {
      std::memset(stats, 0, sizeof(*stats));
      stats->cells = P.cells;
      stats->seconds_device = dev_sec;
      stats->seconds_wall = wall;
      stats->gcups = dev_sec > 0 ? (double)P.cells / dev_sec / 1e9 : 0;
      stats->n_units = (int32_t)P.units.size();
      stats->n_devices = nW;
      std::vector<double> fin;
      for (int w = 0; w < nW; w++) {
        stats->duplicated_cells += S[w]->dup_cells;
        stats->n_overflow_pairs += S[w]->n_ovf;
        stats->kernel_launches += S[w]->launches;
        stats->kernel_seconds_k1 += S[w]->k1_sec;
        stats->kernel_seconds_k3 += S[w]->k3_sec;
        stats->kernel_seconds_k2 += S[w]->k2_sec;
        stats->n_k2_launches += (int32_t)S[w]->k2_ev.size();
        stats->partition_mode = partition_mode;
        stats->partition_sms = partition_sms;
        stats->cells_k1 += S[w]->k1_cells;
        stats->cells_k3 += S[w]->k3_cells;
        stats->n_cancelled += S[w]->n_cancelled;
        fin.push_back(S[w]->last_dev);
      }
      // tail: makespan of the units minus the (lower) median over workers of
      // each worker's last device completion (device clocks from each worker's start event)
      std::sort(fin.begin(), fin.end());
      stats->seconds_last_unit = fin.empty() ? 0 : fin.back();
      stats->tail_seconds = fin.empty() ? 0 : fin.back() - fin[(fin.size() - 1) / 2];
      stats->n_wa_grants = n_wa;
      stats->n_requests = n_req;
      stats->n_grant_messages = n_grant;
      stats->peer_bytes = peer_bytes;
      std::ostringstream js;
      js << "[";
      for (size_t k = 0; k < ulog.size(); k++) {
        const UnitLog &L = ulog[k];
        const Unit &U = P.units[L.unit];
        js << (k ? "," : "") << "{\"unit\":" << L.unit << ",\"kind\":" << U.kind << ",\"pair\":" << U.pair
           << ",\"npk\":" << U.npk
           << ",\"b0\":" << U.b0 << ",\"b1\":" << U.b1 << ",\"cluster\":" << U.cluster
           << ",\"worker\":" << L.worker << ",\"t_grant\":" << L.t_grant << ",\"t_start\":" << L.t_start
           << ",\"t_end\":" << L.t_end << ",\"cells\":" << L.cells << ",\"cells_done\":" << L.cells_done
           << ",\"committed\":" << L.committed << ",\"cancelled\":" << L.cancelled << ",\"slowed\":" << L.slowed
           << ",\"stream\":" << L.stream << ",\"device_ms\":" << L.device_ms << ",\"dev_t0\":" << L.dev_t0
           << ",\"dev_t1\":" << L.dev_t1 << "}";
      }
      js << "]";
      db->unit_log = js.str();
      stats->unit_log_json = db->unit_log.c_str();
      stats->sched_log_json = db->sched_log.c_str();
    }
  });
  if (db) db->busy.store(0);
  return rc;
}

int sw_merge_hits(sw_db *db, const sw_hit *lists_dev, int32_t n_sources, int32_t nq, int32_t k_in,
                  int32_t top_k, sw_hit *hits_dev) {
  return guarded([&] {
    if (!db || db->devs.empty()) throw Error(SW_EINVAL, "db is NULL");
    if (n_sources < 0 || nq < 0 || k_in < 0 || top_k < 0) throw Error(SW_EINVAL, "negative size");
    if (top_k > SW_MAX_TOP_K) throw Error(SW_EINVAL, "top_k must be in [0, 64]");
    if (nq == 0 || top_k == 0) return;
    if (!hits_dev || (n_sources > 0 && k_in > 0 && !lists_dev)) throw Error(SW_EINVAL, "NULL buffer");
    const int dev = db->devs[0]->id;
    CK(cudaSetDevice(dev));
    std::vector<int32_t> tab(nq + 1 + (size_t)nq * n_sources);
    for (int32_t q = 0; q <= nq; q++) tab[q] = q * n_sources;
    for (int32_t q = 0; q < nq; q++)
      for (int32_t r = 0; r < n_sources; r++) tab[nq + 1 + (size_t)q * n_sources + r] = r * nq + q;
    DBuf<int32_t> t;
    t.alloc(dev, tab.size());
    CK(cudaMemcpy(t.p, tab.data(), sizeof(int32_t) * tab.size(), cudaMemcpyHostToDevice));
    launch_merge_topk(reinterpret_cast<const int2 *>(lists_dev), std::max(k_in, 1), t.p, t.p + nq + 1, nq, top_k,
                      reinterpret_cast<int2 *>(hits_dev), 0);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
  });
}

int sw_align(const sw_seqset *queries, sw_db *db, const int8_t *matrix, int32_t gap_open,
             int32_t gap_extend, const int32_t *query_index, const int32_t *db_index, int32_t n_pairs,
             sw_alignment *out, char *ops, int64_t ops_capacity) {
  if (db && db->busy.exchange(1)) {
    g_err = "a search is already running on this sw_db";
    return SW_EBUSY;
  }
  int rc = guarded([&] {
    if (!db || db->devs.empty()) throw Error(SW_EINVAL, "db is NULL");
    validate_seqset(queries, "queries");
    if (gap_open < 0 || gap_extend < 0) throw Error(SW_EINVAL, "gap penalties must be >= 0");
    if ((int64_t)gap_open + 2 * (int64_t)gap_extend > (1 << 20))
      throw Error(SW_EINVAL, "gap_open + 2*gap_extend must be <= 2^20");
    if (n_pairs < 0) throw Error(SW_EINVAL, "n_pairs < 0");
    if (n_pairs == 0) return;
    if (!query_index || !db_index || !out) throw Error(SW_EINVAL, "NULL pair or output array");
    const PackedDB &Hd = db->host;
    const int8_t *M = matrix ? matrix : blosum62();
    // inverse of the length sort: original -> sorted index
    std::vector<int32_t> inv(Hd.n);
    for (int32_t k = 0; k < Hd.n; k++) inv[Hd.perm[k]] = k;
    // encode the queries
    const int32_t nq = queries->n;
    std::vector<int64_t> qoff(nq + 1, 0);
    for (int32_t k = 0; k < nq; k++) qoff[k + 1] = qoff[k] + (queries->offsets[k + 1] - queries->offsets[k]);
    std::vector<uint8_t> qc(std::max<int64_t>(qoff[nq], 1));
    for (int32_t k = 0; k < nq; k++)
      for (int64_t p = 0; p < qoff[k + 1] - qoff[k]; p++) {
        const int c = encode_residue((unsigned char)queries->residues[queries->offsets[k] + p]);
        if (c < 0) throw Error(SW_ERESIDUE, "query " + std::to_string(k) + ": invalid residue at position " + std::to_string(p));
        qc[qoff[k] + p] = (uint8_t)c;
      }
    int64_t need = 0;
    for (int32_t k = 0; k < n_pairs; k++) {
      if (query_index[k] < 0 || query_index[k] >= nq || db_index[k] < 0 || db_index[k] >= Hd.n)
        throw Error(SW_EINVAL, "pair " + std::to_string(k) + ": index out of range");
      need += (qoff[query_index[k] + 1] - qoff[query_index[k]]) + Hd.sorted_len[inv[db_index[k]]];
    }
    if (!ops || ops_capacity < need)
      throw Error(SW_EINVAL, "ops buffer too small: need " + std::to_string(need) + " bytes");
    Device &D = *db->devs[0];
    CK(cudaSetDevice(D.id));
    DBuf<uint8_t> dq; dq.alloc(D.id, qc.size());
    CK(cudaMemcpy(dq.p, qc.data(), qc.size(), cudaMemcpyHostToDevice));
    DBuf<int8_t> dm; dm.alloc(D.id, 24 * 24);
    CK(cudaMemcpy(dm.p, M, 24 * 24, cudaMemcpyHostToDevice));
    // K6 works in linear space: per pair one chunk of direction bytes (256 x n) plus the
    // chunk checkpoints ((nch - 1) x n x 8 B); pairs are batched under 1 GiB of both
    const int64_t kBudget = int64_t(1) << 30;
    int64_t ops_pos = 0;
    for (int32_t p0 = 0; p0 < n_pairs;) {
      std::vector<TbPair> batch;
      int64_t dir_total = 0, ckpt_total = 0, ops_total = 0;
      int32_t p1 = p0;
      while (p1 < n_pairs) {
        TbPair T;
        T.m = (int32_t)(qoff[query_index[p1] + 1] - qoff[query_index[p1]]);
        T.sorted = inv[db_index[p1]];
        T.n = Hd.sorted_len[T.sorted];
        const int64_t nch = (T.m + kTbChunk - 1) / kTbChunk, nblk = (T.n + kTbCols - 1) / kTbCols;
        const int64_t dbytes = (int64_t)kTbChunk * kTbCols;
        const int64_t cbytes = std::max<int64_t>(0, nch - 1) * T.n * 8;
        const int64_t kbytes = std::max<int64_t>(0, nblk - 1) * nch * kTbChunk * 8;
        if (!batch.empty() && dir_total + ckpt_total * 8 + dbytes + cbytes + kbytes > kBudget) break;
        T.q_off = qoff[query_index[p1]];
        T.pad_ = 0;
        T.dir_off = dir_total;
        T.ops_off = ops_total;
        T.ckpt_off = ckpt_total;
        T.colck_off = ckpt_total + cbytes / 8;
        dir_total += dbytes;
        ckpt_total += (cbytes + kbytes) / 8;
        ops_total += T.m + T.n;
        batch.push_back(T);
        p1++;
      }
      const int nb = (int)batch.size();
      DBuf<TbPair> dp; dp.alloc(D.id, nb);
      CK(cudaMemcpy(dp.p, batch.data(), sizeof(TbPair) * nb, cudaMemcpyHostToDevice));
      DBuf<uint8_t> ddir; ddir.alloc(D.id, std::max<int64_t>(dir_total, 1));
      DBuf<char> dops; dops.alloc(D.id, std::max<int64_t>(ops_total, 1));
      // the kernel writes only the last n_ops bytes of each pair's area; the whole area is
      // copied back, so clear it (compute-sanitizer initcheck clean)
      CK(cudaMemset(dops.p, 0, std::max<int64_t>(ops_total, 1)));
      DBuf<TbResult> dres; dres.alloc(D.id, nb);
      DBuf<int2> dckpt; dckpt.alloc(D.id, std::max<int64_t>(ckpt_total, 1));
      TbArgs a;
      a.qcodes = dq.p; a.packed = D.packed.p; a.groups = D.groups.p; a.matrix = dm.p;
      a.pairs = dp.p; a.dir = ddir.p; a.ops = dops.p; a.results = dres.p;
      a.border = reinterpret_cast<int32_t *>(dckpt.p);
      a.alpha = gap_open + gap_extend; a.beta = gap_extend;
      launch_traceback(a, nb, 0);
      CK(cudaGetLastError());
      CK(cudaDeviceSynchronize());
      std::vector<TbResult> res(nb);
      std::vector<char> hops(std::max<int64_t>(ops_total, 1));
      CK(cudaMemcpy(res.data(), dres.p, sizeof(TbResult) * nb, cudaMemcpyDeviceToHost));
      CK(cudaMemcpy(hops.data(), dops.p, ops_total, cudaMemcpyDeviceToHost));
      for (int k = 0; k < nb; k++) {
        const TbPair &T = batch[k];
        const TbResult &R = res[k];
        sw_alignment &A = out[p0 + k];
        A.score = R.score; A.q_begin = R.q_begin; A.q_end = R.q_end;
        A.d_begin = R.d_begin; A.d_end = R.d_end; A.n_ops = R.n_ops;
        A.ops_offset = ops_pos;
        std::memcpy(ops + ops_pos, hops.data() + T.ops_off + (T.m + T.n) - R.n_ops, R.n_ops);
        ops_pos += R.n_ops;
      }
      p0 = p1;
    }
  });
  if (db) db->busy.store(0);
  return rc;
}

}  // extern "C"
