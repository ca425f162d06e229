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
#include <cstring>
#include <deque>
#include <memory>
#include <mutex>
#include <numeric>
#include <sstream>
#include <stdexcept>
#include <string>
#include <thread>
#include <vector>
#include <cuda_runtime.h>
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
  DBuf<int32_t> ovf_cursor;    // [streams] entries taken by the int32 re-run
  DBuf<uint32_t> ovf_bits;     // [nq*ndb] bits: pair already listed
  int32_t ovf_cap = 0;         // entries per stream list
  DBuf<uint2> k3_border;   // [streams][max_k3_seqs][max_len]
  DBuf<int32_t> k2_border;
  DBuf<int32_t> abort_dev;      // per-unit WA cancellation flags (device memory)
  int32_t *abort_d = nullptr;
  int32_t *one_h = nullptr;      // pinned constant 1, source of the cancellation copies
  int32_t *ovf_seen_h = nullptr; // pinned [kMaxStreams]: ovf_count copied after each unit
  cudaStream_t cancel_st = nullptr;
  std::vector<char> cancelled;
  cudaEvent_t ev_start = nullptr, ev_end = nullptr;
  std::vector<cudaEvent_t> u_start, u_end;  // per stream
  int launches = 0;
  double k1_sec = 0, k3_sec = 0;
  int64_t k1_cells = 0, k3_cells = 0;
  int64_t dup_cells = 0;
  double finish_wall = 0;
  int32_t n_ovf = 0;
  void reset_counters() {
    launches = 0; k1_sec = k3_sec = 0; k1_cells = k3_cells = 0; dup_cells = 0;
    finish_wall = 0; n_ovf = 0; scores = nullptr;
  }
  ~DevSearch();
};

struct Device {
  int id = 0;
  int n_sm = 0;
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
  if (cancel_st) cudaStreamDestroy(cancel_st);
  if (ev_start) cudaEventDestroy(ev_start);
  if (ev_end) cudaEventDestroy(ev_end);
  for (auto e : u_start) cudaEventDestroy(e);
  for (auto e : u_end) cudaEventDestroy(e);
}


}  // namespace sw

struct sw_db {
  sw::PackedDB host;
  std::vector<std::unique_ptr<sw::Device>> devs;
  std::atomic<int> busy{0};
  std::string unit_log;
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
};

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
                      const int8_t *M, int32_t thresh) {
  Plan P;
  const int32_t nq = q->n;
  P.qoff.resize(nq + 1);
  P.qoff[0] = 0;
  for (int32_t k = 0; k < nq; k++) {
    const int64_t l = q->offsets[k + 1] - q->offsets[k];
    if (l > 65535) throw Error(SW_EINVAL, "query " + std::to_string(k) + " longer than 65535");
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
    for (int32_t s = 0; s < P.n_long_seqs;) {
      int32_t e = s;
      int64_t cells = 0, work = 0;
      while (e < P.n_long_seqs && (cells < k3_target || e == s || (e - s) % kK3Warps)) {
        cells += rows_eff * db.sorted_len[e];
        work += (int64_t)qp.rows_padded * db.sorted_len[e];
        e++;
      }
      P.units.push_back({kUnitIntra, p, s, e, cells, work});
      P.max_k3_seqs = std::max(P.max_k3_seqs, e - s);
      s = e;
    }
    // K1 units over the short groups
    const int64_t band = k1_band_rows();
    const int64_t rows_k1 = (int64_t)(qp.rows + band - 1) / band * band;
    for (int32_t g = gl; g < ng;) {
      int32_t e = g;
      int64_t cells = 0, work = 0;
      // (units do not straddle the kWideCols boundary: each launch uses one K1 instance)
      const bool wide = db.groups[g].ncols >= kWideCols;
      while (e < ng && (cells < target || e == g) && (db.groups[e].ncols >= kWideCols) == wide) {
        cells += rows_eff * grp_res[e];
        work += rows_k1 * db.groups[e].ncols * kGroup;
        e++;
      }
      P.units.push_back({kUnitInter, p, g, e, cells, work});
      g = e;
    }
  }
  // drop empty units (e.g. all-empty queries still produce valid zero scores: keep them
  // so that every pair gets written, but they must have cells > 0 for the scheduler)
  for (auto &u : P.units) u.cells = std::max<int64_t>(u.cells, 1);
  // LPT by expected duration: intra-task (long-sequence) units first -- each warp walks a
  // whole long pair, so they have the longest latency -- then inter-task units by work.
  // A small K3 unit (fewer sequences than one block per SM) is interleaved with the largest
  // K1 units instead (K3, K1, K3, K1, ...): small K3 units alone on every stream would
  // leave SMs idle at the start of the step (C4 at 1/8 of its database: 140 ms of 447)
  static const bool interleave = [] { const char *e = getenv("SW_UNIT_INTERLEAVE"); return !(e && atoi(e) == 0); }();
  auto small3 = [](const Unit &u) { return interleave && u.kind == kUnitIntra && u.b1 - u.b0 < kK3UnitSeqs; };
  std::stable_sort(P.units.begin(), P.units.end(), [&](const Unit &a, const Unit &b) {
    const int ra = a.kind == kUnitIntra ? (small3(a) ? 1 : 0) : 2;
    const int rb = b.kind == kUnitIntra ? (small3(b) ? 1 : 0) : 2;
    if (ra != rb) return ra < rb;
    if (P.pack_may_ovf[a.pair] != P.pack_may_ovf[b.pair]) return P.pack_may_ovf[a.pair] > P.pack_may_ovf[b.pair];
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
  return P;
}

// ---------------------------------------------------------------- per-search device state
struct UnitLog {
  int32_t unit, worker, stream;
  double t_grant, t_start, t_end;   // host clock (s since the search start)
  int64_t cells;
  int committed;
  float device_ms;                  // CUDA events around the unit's kernels on its stream
};

static const int kOvfCap = 1 << 20;


// K2 arguments for the saturated-pair list of one stream
static K2Args k2_args(const Plan &P, const PackedDB &db, DevSearch &S, int stream_idx, int32_t alpha,
                      int32_t beta) {
  Device &D = *S.D;
  K2Args a;
  a.qcodes = S.qcodes.p; a.qoff = S.qoff.p;
  a.packed = D.packed.p; a.groups = D.groups.p; a.sorted_len = D.sorted_len.p; a.perm = D.perm.p;
  a.matrix = S.matrix.p;
  a.ovf = S.ovf.p + (size_t)stream_idx * S.ovf_cap; a.ovf_count = S.ovf_count.p + stream_idx;
  a.ovf_cap = S.ovf_cap; a.ovf_cursor = S.ovf_cursor.p + stream_idx;
  a.scores = S.scores; a.ndb = db.n; a.alpha = alpha; a.beta = beta; a.one = 1;
  const int64_t stride = std::max<int64_t>(P.max_len, 1);
  a.border = S.k2_border.p + (size_t)stream_idx * kK2Blocks * stride * 2;
  a.border_stride = stride;
  return a;
}

static void launch_unit(const Plan &P, const PackedDB &db, DevSearch &S, const Unit &U, int uidx,
                        int stream_idx, int32_t alpha, int32_t beta, int32_t thresh) {
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
    a.border = D.k1_border.p; a.border_slot_cols = D.slot_cols; a.slots_per_sm = D.slots_per_sm;
    a.slot_busy = D.slot_busy.p;
    a.abort_flag = S.abort_d + uidx;
    a.na = na; a.nb = nbm;
    launch_k1(a, U.b1 - U.b0, db.groups[U.b1 - 1].ncols, P.pairs[U.pair].rows_padded, st, D.n_sm);
  } else {
    K3Args a;
    a.packed = D.packed.p; a.groups = D.groups.p; a.perm = D.perm.p; a.sorted_len = D.sorted_len.p;
    a.prof = S.prof.p; a.pairs = S.pairs.p; a.slices = S.slices.p;
    a.pair = U.pair; a.l0 = U.b0; a.l1 = U.b1;
    a.scores = S.scores; a.ndb = db.n;
    a.thresh = thresh;
    a.ovf = S.ovf.p + (size_t)stream_idx * S.ovf_cap; a.ovf_count = S.ovf_count.p + stream_idx;
    a.ovf_cap = S.ovf_cap; a.ovf_bits = S.ovf_bits.p;
    const int64_t stride = (std::max<int64_t>(P.max_len, 1) + 15) / 16 * 16;  // >= tiles * T
    a.border = S.k3_border.p + (size_t)stream_idx * P.max_k3_seqs * k3_phases() * stride;
    a.border_stride = stride;
    a.abort_flag = S.abort_d + uidx;
    a.na = na; a.nb = nbm;
    launch_k3(a, P.pairs[U.pair].rows_padded, st);
  }
  S.launches++;
  // saturated pairs listed so far on this stream -> host (4 bytes): the worker launches
  // the int32 re-run (K2) on this stream when the unit completes and the list grew.  K2's
  // blocks need a whole SM's worth of shared memory, so an empty K2 launched after every
  // unit would wait for a K1 block to leave and stall the stream.
  CK(cudaMemcpyAsync(S.ovf_seen_h + stream_idx, S.ovf_count.p + stream_idx, sizeof(int32_t),
                     cudaMemcpyDeviceToHost, st));
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
    if (k < 0 || k > 64) throw Error(SW_EINVAL, "top_k must be in [0, 64]");
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
    if (top_k < 0 || top_k > 64) throw Error(SW_EINVAL, "top_k must be in [0, 64]");
    sw_opts o;
    sw_opts_default(&o);
    if (opts_in) o = *opts_in;
    if (o.omega < 1) o.omega = 4;
    if (o.streams_per_device <= 0) o.streams_per_device = 4;
    if (o.streams_per_device > kMaxStreams) throw Error(SW_EINVAL, "streams_per_device must be <= 64");
    if (o.policy != SW_POLICY_SS && o.policy != SW_POLICY_PSS) throw Error(SW_EINVAL, "bad policy");
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
    Plan P = make_plan(queries, H, o, dist ? o.dist_world : nW, M, thresh);
    const double wall0 = now_s();

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
      while ((int)D.streams.size() < depth) {
        cudaStream_t st;
        CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
        D.streams.push_back(st);
      }
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
      const size_t nsc = (size_t)nq * nd;
      if (w == 0 && o.outputs_on_device && scores && !dist) X.scores = scores;
      else { X.scores_own.ensure(D.id, nsc); X.scores = X.scores_own.p; }
      // saturated-pair lists: 2^20 per stream, or every pair when the s16x2 path is not
      // usable (alpha + beta > 16384: all pairs are re-scored in int32)
      X.ovf_cap = s16_ok ? kOvfCap : (int32_t)std::min<int64_t>((int64_t)nq * nd + 1, INT32_MAX / 2);
      X.ovf.ensure(D.id, (size_t)depth * X.ovf_cap);
      X.ovf_count.ensure(D.id, depth);
      X.ovf_cursor.ensure(D.id, depth);
      X.ovf_bits.ensure(D.id, ((size_t)nq * nd + 31) / 32);
      X.k2_border.ensure(D.id, (size_t)depth * kK2Blocks * std::max<int64_t>(P.max_len, 1) * 2);
      const size_t k3b = (size_t)depth * std::max(P.max_k3_seqs, 1) * k3_phases() *
                         ((std::max<int64_t>(P.max_len, 1) + 15) / 16 * 16);
      if (P.n_long_seqs > 0) X.k3_border.ensure(D.id, k3b);
      const size_t nu = std::max<size_t>(P.units.size(), 1);
      X.abort_dev.ensure(D.id, nu);
      CK(cudaMemset(X.abort_dev.p, 0, sizeof(int32_t) * nu));
      X.abort_d = X.abort_dev.p;
      X.cancelled.assign(nu, 0);
      if (!X.one_h) {
        CK(cudaHostAlloc((void **)&X.one_h, sizeof(int32_t), cudaHostAllocDefault));
        *X.one_h = 1;
        CK(cudaHostAlloc((void **)&X.ovf_seen_h, sizeof(int32_t) * kMaxStreams, cudaHostAllocDefault));
      }
      if (!X.cancel_st) CK(cudaStreamCreateWithFlags(&X.cancel_st, cudaStreamNonBlocking));
      if (!X.ev_start) CK(cudaEventCreate(&X.ev_start));
      if (!X.ev_end) CK(cudaEventCreate(&X.ev_end));
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
                      o.workload_adjust, o.omega);
      }
      client = std::make_unique<SchedClient>();
      client->connect(o.dist_host, o.dist_port, o.dist_rank, 30.0);
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
    auto srep = [&](int w, double t, double cells, double sec) {
      if (client) client->report(t, cells, sec);
      else if (sched) sw_sched_report(sched, w, t, cells, sec);
    };
    auto scomp = [&](int w, int u, double t) -> int {
      if (client) return client->complete(u, t);
      return sched ? sw_sched_complete(sched, w, u, t) : 1;
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
    std::atomic<int> ready{0};
    std::atomic<bool> failed{false};   // a worker failed: the others stop (no hang on its units)
    std::vector<std::string> werr(nW);
    std::vector<int> wcode(nW, 0);
    const double t0 = now_s();
    auto worker = [&](int w) {
      DevSearch &X = *S[w];
      Device &D = *X.D;
      const int wid = my_worker_base + w;
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
        CK(cudaMemsetAsync(X.ovf_cursor.p, 0, sizeof(int32_t) * depth, s0));
        CK(cudaMemsetAsync(X.ovf_bits.p, 0, sizeof(uint32_t) * (((size_t)nq * nd + 31) / 32), s0));
        launch_profile(X.qcodes.p, X.qoff.p, X.pairs.p, (int)P.pairs.size(), X.slices.p, X.matrix.p,
                       X.prof.p, P.prof_total, s0);
        X.launches += 2 + (P.pairs.empty() ? 0 : 1);
        CK(cudaGetLastError());
        cudaEvent_t setup_done;
        CK(cudaEventCreateWithFlags(&setup_done, cudaEventDisableTiming));
        CK(cudaEventRecord(setup_done, s0));
        for (int k = 1; k < depth; k++) CK(cudaStreamWaitEvent(D.streams[k], setup_done, 0));
        const bool straggler = (o.straggler_mask >> wid) & 1ull;
        const double slow = std::max(1, o.straggler_slowdown);
        std::deque<int32_t> pending;
        std::vector<int32_t> inflight(depth, -1);
        std::vector<double> t_grant(P.units.size(), 0), t_launch(depth, 0);
        std::vector<double> hold_until(depth, 0);
        std::vector<int> completed_wait(depth, 0);
        std::vector<int32_t> k2_upto(depth, 0);   // saturated pairs handed to K2 per stream
        bool done = false;
        double last_report = now_s();
        int32_t buf[64];
        while (true) {
          if (failed.load()) throw Error(SW_ECUDA, "another worker failed");
          bool progressed = false;
          const double tn = now_s();
          // completions
          for (int k = 0; k < depth; k++) {
            if (inflight[k] < 0) continue;
            if (!completed_wait[k]) {
              cudaError_t q = cudaEventQuery(X.u_end[k]);
              if (q == cudaErrorNotReady) continue;
              CK(q);
              completed_wait[k] = 1;
              if (straggler && tn - t0 >= 1e-3 * o.straggler_after_ms) {
                // emulate a PE `slow` times slower (SURVEY §8(d) WA experiment; P24 §V.C)
                float ms = 0;
                cudaEventElapsedTime(&ms, X.u_start[k], X.u_end[k]);
                hold_until[k] = tn + (slow - 1.0) * ms * 1e-3;
              } else {
                hold_until[k] = tn;
              }
            }
            // an emulated slow PE stops working on a replica whose task finished elsewhere
            // (WA: the first result wins and the other replicas are cancelled)
            if (tn < hold_until[k] && !sfin(inflight[k])) continue;
            const int u = inflight[k];
            const Unit &U = P.units[u];
            float ms = 0;
            cudaEventElapsedTime(&ms, X.u_start[k], X.u_end[k]);
            const int committed = scomp(wid, u, tn);
            srep(wid, tn, (double)U.cells, std::max(1e-6, tn - last_report));
            last_report = tn;
            if (U.kind == kUnitInter) { X.k1_sec += ms * 1e-3; X.k1_cells += U.cells; }
            else { X.k3_sec += ms * 1e-3; X.k3_cells += U.cells; }
            if (!committed) X.dup_cells += U.cells;
            {
              std::lock_guard<std::mutex> g(ulog_mu);
              ulog.push_back({u, wid, k, t_grant[u] - t0, t_launch[k] - t0, tn - t0, U.cells, committed, ms});
            }
            inflight[k] = -1;
            completed_wait[k] = 0;
            progressed = true;
            // int32 re-run of what this unit saturated, on its stream before the next unit
            // (overlaps the units in flight on the other streams)
            const int32_t seen = ((volatile int32_t *)X.ovf_seen_h)[k];
            if (seen > k2_upto[k]) {
              launch_k2(k2_args(P, H, X, k, alpha, beta), kK2Blocks, D.streams[k]);
              CK(cudaGetLastError());
              X.launches++;
              k2_upto[k] = seen;
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
            if (!sstart(wid, u, now_s())) { progressed = true; k--; continue; }
            CK(cudaEventRecord(X.u_start[k], D.streams[k]));
            launch_unit(P, H, X, P.units[u], u, k, alpha, beta, thresh);
            CK(cudaGetLastError());
            CK(cudaEventRecord(X.u_end[k], D.streams[k]));
            inflight[k] = u;
            t_launch[k] = now_s();
            progressed = true;
          }
          // ask the master for more when the local queue is empty and a stream is free
          int n_inflight = 0;
          for (int k = 0; k < depth; k++) n_inflight += inflight[k] >= 0;
          if (!done && pending.empty() && n_inflight < depth) {
            const int32_t r = sreq(wid, now_s(), buf, 64);
            if (r < 0) done = true;
            else {
              for (int32_t i = 0; i < r; i++) { pending.push_back(buf[i]); t_grant[buf[i]] = now_s(); }
              if (r > 0) progressed = true;
            }
          }
          if (done && pending.empty() && n_inflight == 0) break;
          // poll completions every 20 us; an idle worker (nothing in flight, nothing granted)
          // asks the master again every 100 us
          if (!progressed)
            std::this_thread::sleep_for(std::chrono::microseconds(n_inflight > 0 ? 20 : 100));
        }
        // the int32 re-runs ran on each stream after the units that saturated; check the lists
        for (int k = 0; k < depth; k++) CK(cudaStreamSynchronize(D.streams[k]));
        std::vector<int32_t> novf(depth, 0), ncur(depth, 0);
        CK(cudaMemcpy(novf.data(), X.ovf_count.p, sizeof(int32_t) * depth, cudaMemcpyDeviceToHost));
        CK(cudaMemcpy(ncur.data(), X.ovf_cursor.p, sizeof(int32_t) * depth, cudaMemcpyDeviceToHost));
        X.n_ovf = 0;
        for (int k = 0; k < depth; k++) {
          if (novf[k] > X.ovf_cap) throw Error(SW_ENOMEM, "overflow list capacity exceeded");
          X.n_ovf += novf[k];
          if (ncur[k] < novf[k]) throw Error(SW_ECUDA, "int32 re-run left saturated pairs");
        }
        CK(cudaEventRecord(X.ev_end, s0));
        CK(cudaEventSynchronize(X.ev_end));
        CK(cudaEventDestroy(setup_done));
        X.finish_wall = now_s();
      } catch (const Error &e) {
        werr[w] = e.what();
        wcode[w] = e.code;
        failed.store(true);
        ready.fetch_add(1 << 20);  // release the barrier
      } catch (const std::exception &e) {
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
    if (client) client->done();
    if (server) server->stop();

    // ---------------- merge (in-process multi-device: device 0 pulls the others over
    // NVLink and takes the element-wise max; every pair was written by >= 1 device with
    // identical values, the rest are -1), then top-k on device 0
    DevSearch &X0 = *S[0];
    CK(cudaSetDevice(X0.D->id));
    cudaStream_t s0 = X0.D->streams[0];
    cudaEvent_t m_start, m_end;
    CK(cudaEventCreate(&m_start));
    CK(cudaEventCreate(&m_end));
    CK(cudaEventRecord(m_start, s0));
    const int64_t nsc = (int64_t)nq * nd;
    DBuf<int32_t> tmp;
    if (nW > 1 && nsc > 0) {
      tmp.alloc(X0.D->id, nsc);
      for (int w = 1; w < nW; w++) {
        CK(cudaMemcpyPeerAsync(tmp.p, X0.D->id, S[w]->scores, S[w]->D->id, sizeof(int32_t) * nsc, s0));
        launch_max_merge(X0.scores, tmp.p, nsc, s0);
        X0.launches++;
      }
    }
    DBuf<int2> hits_dev;
    int2 *hits_out = nullptr;
    if (hits && top_k > 0 && nq > 0) {
      if (o.outputs_on_device) hits_out = reinterpret_cast<int2 *>(hits);
      else { hits_dev.alloc(X0.D->id, (size_t)nq * top_k); hits_out = hits_dev.p; }
      launch_topk(X0.scores, nq, nd, top_k, hits_out, s0);
      X0.launches++;
    }
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
    if (scores && nsc > 0) {
      if (o.outputs_on_device) {
        if (X0.scores != scores) CK(cudaMemcpy(scores, X0.scores, sizeof(int32_t) * nsc, cudaMemcpyDeviceToDevice));
      } else {
        CK(cudaMemcpy(scores, X0.scores, sizeof(int32_t) * nsc, cudaMemcpyDeviceToHost));
      }
    }
    if (hits && top_k > 0 && nq > 0 && !o.outputs_on_device)
      CK(cudaMemcpy(hits, hits_dev.p, sizeof(int2) * nq * top_k, cudaMemcpyDeviceToHost));
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
        stats->cells_k1 += S[w]->k1_cells;
        stats->cells_k3 += S[w]->k3_cells;
        fin.push_back(S[w]->finish_wall - t0);
      }
      std::sort(fin.begin(), fin.end());
      stats->tail_seconds = fin.empty() ? 0 : fin.back() - fin[fin.size() / 2];
      if (sched) {
        stats->n_wa_grants = (int32_t)sw_sched_counter(sched, 1);
        stats->n_requests = (int32_t)sw_sched_counter(sched, 0);
      } else if (client) {
        stats->n_wa_grants = client->wa_grants();
        stats->n_requests = client->requests();
      }
      std::ostringstream js;
      js << "[";
      for (size_t k = 0; k < ulog.size(); k++) {
        const UnitLog &L = ulog[k];
        const Unit &U = P.units[L.unit];
        js << (k ? "," : "") << "{\"unit\":" << L.unit << ",\"kind\":" << U.kind << ",\"pair\":" << U.pair
           << ",\"worker\":" << L.worker << ",\"t_grant\":" << L.t_grant << ",\"t_start\":" << L.t_start
           << ",\"t_end\":" << L.t_end << ",\"cells\":" << L.cells << ",\"committed\":" << L.committed
           << ",\"stream\":" << L.stream << ",\"device_ms\":" << L.device_ms << "}";
      }
      js << "]";
      db->unit_log = js.str();
      stats->unit_log_json = db->unit_log.c_str();
    }
  });
  if (db) db->busy.store(0);
  return rc;
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
    const int64_t kBudget = int64_t(2) << 30;   // direction bytes per batch
    int64_t ops_pos = 0;
    for (int32_t p0 = 0; p0 < n_pairs;) {
      std::vector<TbPair> batch;
      int64_t dir_total = 0, ops_total = 0;
      int32_t max_n = 1;
      int32_t p1 = p0;
      while (p1 < n_pairs) {
        TbPair T;
        T.m = (int32_t)(qoff[query_index[p1] + 1] - qoff[query_index[p1]]);
        T.sorted = inv[db_index[p1]];
        T.n = Hd.sorted_len[T.sorted];
        const int64_t cells = (int64_t)T.m * T.n;
        if (!batch.empty() && dir_total + cells > kBudget) break;
        T.q_off = qoff[query_index[p1]];
        T.pad_ = 0;
        T.dir_off = dir_total;
        T.ops_off = ops_total;
        dir_total += cells;
        ops_total += T.m + T.n;
        max_n = std::max(max_n, T.n);
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
      DBuf<int32_t> dborder; dborder.alloc(D.id, (size_t)nb * max_n * 2);
      TbArgs a;
      a.qcodes = dq.p; a.packed = D.packed.p; a.groups = D.groups.p; a.matrix = dm.p;
      a.pairs = dp.p; a.dir = ddir.p; a.ops = dops.p; a.results = dres.p;
      a.border = dborder.p; a.border_stride = max_n;
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
