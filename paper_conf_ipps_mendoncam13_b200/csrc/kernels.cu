// kernels.cu — the sm_100a kernels of the hot path.
//
// All DP kernels compute the Gotoh/Smith-Waterman recurrence of PAPER.md P12 §II.A
// (Eq. 1 with zero first row/column; affine gaps via "3 DP matrices: H, E and F"):
//   E(i,j) = max(E(i,j-1) - beta, H(i,j-1) - alpha)
//   F(i,j) = max(F(i-1,j) - beta, H(i-1,j) - alpha)
//   H(i,j) = max(0, H(i-1,j-1) + S[q_i][d_j], E(i,j), F(i,j));   score = max H
// with alpha = open + extend, beta = extend (gap of length L costs open + L*extend).
//
// s16x2 kernels (K1, K3) keep two queries per 32-bit lane word (query pair qa = low
// half, qb = high half) and use the "offset representation" of DESIGN.md §6:
//   every H, E, F is stored as value + kOff, E and F floored at 0 (exact for H, proof
//   in DESIGN.md §6: flooring E/F at 0 never changes max(0, ., E, F));
//   x  = Hdiag~ + V         one 32-bit IADD; V = S_b*65536 + S_a is the "signed-packed"
//                           profile entry, exact because Hdiag~ >= kOff >= -min(S)
//   h  = vimax3(x, E, F)    VIMNMX3.S16x2 (E, F >= kOff, so h >= kOff = H floor 0)
//   t  = max(h - alpha, kOff)                 VIADDMNMX.S16x2
//   E' = max(E - beta, t),  F' = max(F - beta, t)   VIADDMNMX.S16x2 (x2)
// Saturation: no half can wrap while best~ + max(S) <= 32767;
// a lane half whose best~ reaches 32768 - max(S) is flagged and re-scored in int32 (K2).
#include <cuda_runtime.h>
#include <cooperative_groups.h>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <algorithm>
#include <mutex>
#include "sw_internal.h"
#include "../../include/sw.h"

// Checked build (SW_CHECKED=1 at build / load time: libsw_checked.so): bounds of the border
// rows, ring slots, profile codes and list entries are asserted in the kernels; a violation
// prints where and traps.  compute-sanitizer is closed on this GPU pool, so the GPU tests run
// the split paths on this build too (tests/test_gpu_parity.py::test_checked_build).
#ifdef SW_CHECKED
#define SW_CHECK(c)                                                                          \
  do {                                                                                       \
    if (!(c)) {                                                                              \
      printf("SW_CHECK failed %s:%d: %s (block %d thread %d)\n", __FILE__, __LINE__, #c,      \
             (int)blockIdx.x, (int)threadIdx.x);                                             \
      __trap();                                                                              \
    }                                                                                        \
  } while (0)
#else
#define SW_CHECK(c) do { } while (0)
#endif

namespace sw {

constexpr bool kK1PairLoads = true;   // K1 reads two profile rows per LDS.64
__constant__ uint8_t c_code_of_slot[kNCodes] = SW_CODE_OF_SLOT_INIT;   // database slot -> code
__device__ __forceinline__ uint32_t pk2(int v) { return ((uint32_t)(v & 0xffff)) * 0x10001u; }
__device__ __forceinline__ void cp_async8(void *smem_dst, const void *gsrc) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async16(void *smem_dst, const void *gsrc) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" ::"r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit_wait1() {   // <= 1 group still in flight
  asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 1;" ::: "memory");
}
__device__ __forceinline__ void cp_async_commit_wait() {
  asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
}
// WA cancellation flag (device memory, set by the host with an async copy): read once by
// thread 0 and broadcast, so a block start costs one L2 read
__device__ __forceinline__ bool block_aborted(const volatile int32_t *flag) {
  __shared__ int ab;
  if (threadIdx.x == 0) ab = flag ? *flag : 0;
  __syncthreads();
  return ab != 0;
}
constexpr int kAbortPoll = 32;   // K1 pipeline steps between WA cancellation polls
__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ uint32_t smid() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

// ------------------------------------------------------------------------------------
// K4: query-pair profiles.  prof[pair][c][row] = S_b*65536 + S_a (signed-packed int32), c = database slot,
// S_a = S[qa_row][code of slot c] (kPadScore past the end of qa or for the pad code), same for qb.
// ------------------------------------------------------------------------------------
__global__ void profile_kernel(const uint8_t *__restrict__ qcodes, const int64_t *__restrict__ qoff,
                               const QueryPair *__restrict__ pairs, const SliceInfo *__restrict__ slices,
                               const int8_t *__restrict__ M, int32_t *__restrict__ prof) {
  const QueryPair P = pairs[blockIdx.y];
  const int64_t n = (int64_t)kNCodes * P.rows_padded;
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n;
       k += (int64_t)gridDim.x * blockDim.x) {
    const int c = (int)(k / P.rows_padded), row = (int)(k % P.rows_padded);
    const SliceInfo si = slices[P.slice_off + row / 16];
    int sa = kPadScore, sb = kPadScore;
    if (c < 24) {   // c = database slot
      const int dc = c_code_of_slot[c];
      if (si.q_lo >= 0) {
        const int64_t r = si.off_lo + row % 16;
        if (r < qoff[si.q_lo + 1] - qoff[si.q_lo]) sa = M[qcodes[qoff[si.q_lo] + r] * 24 + dc];
      }
      if (si.q_hi >= 0) {
        const int64_t r = si.off_hi + row % 16;
        if (r < qoff[si.q_hi + 1] - qoff[si.q_hi]) sb = M[qcodes[qoff[si.q_hi] + r] * 24 + dc];
      }
    }
    prof[P.prof_off + k] = sb * 65536 + sa;
  }
}

void launch_profile(const uint8_t *qcodes, const int64_t *qoff, const QueryPair *pairs, int npairs,
                    const SliceInfo *slices, const int8_t *matrix, int32_t *prof, int64_t,
                    cudaStream_t st) {
  if (npairs == 0) return;
  dim3 grid(64, npairs);
  profile_kernel<<<grid, 256, 0, st>>>(qcodes, qoff, pairs, slices, matrix, prof);
}

// ------------------------------------------------------------------------------------
// Shared per-cell update of the s16x2 kernels (one query row, one DB column).
// ------------------------------------------------------------------------------------
struct Cell {
  static __device__ __forceinline__ void row(uint32_t v, uint32_t &hd, uint32_t &Hi, uint32_t &Ei,
                                             uint32_t &f, uint32_t &best, uint32_t na, uint32_t nb,
                                             uint32_t koff) {
    const uint32_t x = hd + v;                        // Hdiag~ + S  (exact 32-bit add)
    const uint32_t h = __vimax3_s16x2(x, Ei, f);      // H~(i,j) (>= kOff)
    const uint32_t t = __viaddmax_s16x2(h, na, koff); // max(H - alpha, 0) + kOff
    Ei = __viaddmax_s16x2(Ei, nb, t);                 // E(i, j+1)
    f = __viaddmax_s16x2(f, nb, t);                   // F(i+1, j)
    hd = Hi;                                          // H(i, j-1): diagonal of row i+1
    Hi = h;
    best = __vmaxs2(best, h);
  }
};

// One half of a lane's running maximum (offset representation) for query q: saturated
// halves go to the int32 re-run list, the others raise the score with atomicMax (a query
// spans several warps / lanes / bands, each contributes the maximum over its rows).  A
// listed entry is published to the host (ovf_early, host-mapped) so that the worker can
// start the int32 re-run while the unit still runs; list slots hold (-1, -1) until written.
__device__ __forceinline__ void flush_half(int q, int v, int ss, int orig, int32_t *scores,
                                           int64_t ndb, int thresh, int2 *ovf, int32_t *ovf_count,
                                           int ovf_cap, uint32_t *ovf_bits, int32_t *ovf_early) {
  if (q < 0) return;
  if (v >= thresh) {   // several warps / lanes may saturate on one pair: list it once
    const int64_t bit = (int64_t)q * ndb + orig;
    const uint32_t m = 1u << (bit & 31);
    if (!(atomicOr(ovf_bits + (bit >> 5), m) & m)) {
      const int k = atomicAdd(ovf_count, 1);
      if (k < ovf_cap) {
        ovf[k] = make_int2(q, ss);
        // a hint: two writers may land out of order (the worker also reads the device count
        // after every unit), so a plain store, no host atomics; only at counts 1, 2, 4, 8, ...
        // (a search routed to int32 lists every pair: no system fence per pair)
        if (ovf_early && ((k + 1) & k) == 0) {
          __threadfence_system();   // the entry before the host sees its count
          *(volatile int32_t *)ovf_early = k + 1;
        }
      }
    }
  } else {
    atomicMax(scores + (int64_t)q * ndb + orig, v - kOff);
  }
}
__device__ __forceinline__ int lo16(uint32_t v) { return (int)(int16_t)(v & 0xffff); }
__device__ __forceinline__ int hi16(uint32_t v) { return (int)(int16_t)(v >> 16); }
// half masks of a slice that starts a query (its input row above is reset to H = F = 0)
__device__ __forceinline__ uint32_t start_mask(const SliceInfo &n) {
  return (n.q_lo >= 0 && n.off_lo == 0 ? 0x0000ffffu : 0u) | (n.q_hi >= 0 && n.off_hi == 0 ? 0xffff0000u : 0u);
}

// G consecutive columns of one lane's K rows, skewed by one row per column so the G
// dependency chains (row i of column g needs row i of column g-1 and row i-1 of column g)
// are interleaved explicitly: at step k column g updates row k - g.  Column g starts with
// diagonal hdc[g] and top F fc[g]; on return out_h[g] / fc[g] hold its bottom-row H and
// the F passed down.  PS = profile stride between consecutive rows.
// PAIR: the profile of rows i, i+1 (i even) is one 8-byte word at prc + (i/2)*PPS, read
// with one LDS.64 (K1: consecutive rows, PPS = 2; K3: row pairs interleaved per lane, PPS = 64).
template <int K, int G, int PS, bool PAIR = false, int PPS = 2>
__device__ __forceinline__ void dp_tile(const uint32_t *const (&prc)[G], uint32_t (&H)[K],
                                        uint32_t (&E)[K], uint32_t (&hdc)[G], uint32_t (&fc)[G],
                                        uint32_t (&out_h)[G], uint32_t &best, uint32_t na, uint32_t nb,
                                        uint32_t koff) {
  static_assert(!PAIR || K % 2 == 0, "pair loads need an even row count");
  uint2 pv[G];
#pragma unroll
  for (int k = 0; k < K + G - 1; k++) {
#pragma unroll
    for (int g = 0; g < G; g++) {
      const int i = k - g;
      if (i >= 0 && i < K) {
        uint32_t v;
        if (PAIR) {
          if ((i & 1) == 0) pv[g] = *reinterpret_cast<const uint2 *>(prc[g] + (i / 2) * PPS);
          v = (i & 1) ? pv[g].y : pv[g].x;
        } else {
          v = prc[g][i * PS];
        }
        Cell::row(v, hdc[g], H[i], E[i], fc[g], best, na, nb, koff);
        if (i == K - 1) out_h[g] = H[K - 1];
      }
    }
  }
}

// ------------------------------------------------------------------------------------
// K1: inter-task kernel.  Block = one packing group of 32 DB sequences (lane = sequence)
// x W warps; warp w owns rows [w*K, (w+1)*K) of each band of W*K query rows.  Warps form
// a pipeline over (band, column tile): at step s warp w works on element e = s - w; the
// bottom row (H, F) of a tile goes to warp w+1 through shared memory (double-buffered)
// and, for the last warp, to warp 0 of the next band through a global border row held
// in a per-SM slot.  One __syncthreads per step.
// ------------------------------------------------------------------------------------
// UQ: 8 = one skewed tile over all 8 columns of a step, otherwise tiles of 4 columns
template <int K, int W, int T, int MINB, int UQ>
__global__ void __launch_bounds__(W * 32, MINB) k1_kernel(const K1Args a) {
  static_assert(T == 4 || T == 8 || T == 16, "tile = 1, 2 or 4 32-bit words of residues");
  constexpr int BAND = W * K;
  // profile stride: odd (lanes reading one row with different codes hit different banks),
  // or even with pair loads (rows i, i+1 of one code in one LDS.64)
  constexpr int S = kK1PairLoads ? BAND + 2 : BAND + 1;
  constexpr int TPW = kWordCols / T;   // tiles per 16-column residue word
  extern __shared__ __align__(16) uint32_t smem[];
  uint32_t *prof_s = smem;                                            // [2][kNCodes][S]
  uint2 *hand = reinterpret_cast<uint2 *>(smem + 2 * kNCodes * S);    // [W][2][T][32]
  uint32_t *red = reinterpret_cast<uint32_t *>(hand + W * 2 * T * 32);  // [2][W][32]
  uint2 *bsm = reinterpret_cast<uint2 *>(red + 2 * W * 32);           // [2][T][32]
  uint2 *kin = bsm + 2 * T * 32;                                      // [T][32] = (kOff, kOff)
  __shared__ int slot_s;

  if (block_aborted(a.abort_flag)) return;  // WA: this replica lost the race
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const QueryPair P = a.pairs[a.pair];
  const int rows = P.rows;   // 16-aligned, >= 16
  const int nb = (rows + BAND - 1) / BAND;
  const uint32_t koff = pk2(kOff), na = a.na, nbeta = a.nb;
  const int32_t *gprof = a.prof + P.prof_off;
  // this block streams through the unit's groups without draining the warp pipeline between
  // them, claiming them dynamically from the unit's counter: the groups are sorted by
  // decreasing width, so claims go widest first and a block that took a wide group takes
  // fewer (list scheduling; a static stride left the widest unit of each pack at 0.77 of
  // the others).  The block's r-th group is gring[r & 3].  The next group is claimed late,
  // when warp 0 enters the current group's second-to-last band (at the group's start when
  // it has <= 2 bands), so a block claims only when it is about to need it, and every warp
  // (lagging warp 0 by < one band) reads a slot written at least one band earlier.
  const int gend = a.g0 + a.n_groups;
  __shared__ int gring[4];
  auto claim = [&]() -> int {
    const int i = atomicAdd(a.gclaim, 1);
    return i < a.n_groups ? a.g0 + i : gend;
  };

  uint2 *border = nullptr;
  if (threadIdx.x == 0) {
    gring[0] = claim();
    gring[1] = (nb <= 2 && gring[0] < gend) ? claim() : gend;   // nb > 2: claimed at band nb-2
    if (nb > 1 && gring[0] < gend) {   // a border-row slot of this SM (released at exit)
      const int base = (int)smid() * a.slots_per_sm;
      int k = 0;
      for (;; k = (k + 1) % a.slots_per_sm)
        if (atomicCAS(&a.slot_busy[base + k], 0, 1) == 0) break;
      slot_s = base + k;
    }
  }
  auto load_band = [&](int b, int slot) {
    uint32_t *dst = prof_s + slot * kNCodes * S;
    for (int idx = threadIdx.x; idx < kNCodes * BAND; idx += W * 32) {
      const int c = idx / BAND, r = idx - c * BAND;
      dst[c * S + r] = (uint32_t)__ldg(gprof + (int64_t)c * P.rows_padded + b * BAND + r);
    }
  };
  load_band(0, 0);
  if (nb > 1) load_band(1, 1);
  for (int k = threadIdx.x; k < T * 32; k += W * 32) kin[k] = make_uint2(koff, koff);
  __syncthreads();
  const int gfirst = gring[0];
  if (gfirst >= gend) return;   // nothing left for this block (uniform: read after the barrier)
  if (nb > 1) border = a.border + (size_t)slot_s * a.border_slot_cols * 32;

  // block-uniform tracker of warp 0's band starts: the profile of global band B+1 is
  // loaded into slot (B+1)&1 when warp W-1 leaves band B-1, i.e. W-1 steps after warp 0
  // starts band B (every band has nt >= W+1 steps, so warp 0 needs it later)
  int t_r = 0, t_g = gfirst, t_band = 0, t_nt = (a.groups[gfirst].ncols + T - 1) / T, t_start = 0, t_B = 0;
  int end_step = INT32_MAX;   // set when warp 0 runs out of groups: + W - 1 drains the pipeline
  int rl_step = -1, rl_band = 0, rl_slot = 0;

  // per-warp iterator over (group, band, tile); the queries of this warp's current slice
  // (per half) and the start mask of the slice below it
  int g = gfirst, gr = 0, gk = 0, band = 0, tile = 0, gband = 0;
  int cq_lo = -1, cq_hi = -1;
  uint32_t omask = 0;
  const int nslices = P.rows_padded / 16;
  GroupInfo G = a.groups[g];
  int nt = (G.ncols + T - 1) / T, nwords = (G.ncols + kWordCols - 1) / kWordCols, wnext = nwords > 1 ? 1 : 0;
  const uint4 *wp = a.packed + G.word_off + lane;
  uint4 r4 = wp[0], r4n = wp[(size_t)wnext * 32];
  uint32_t H[K], E[K];
  uint32_t best = koff, hprev_top = koff;

  for (int s = 0; s < end_step; s++) {
    if (s == t_start + t_nt) {   // warp 0 enters its next band at this step
      t_start += t_nt;
      t_B++;
      if (++t_band == nb) {
        t_band = 0;
        t_g = gring[(++t_r) & 3];   // claimed at least one band ago
        if (t_g < gend) t_nt = (a.groups[t_g].ncols + T - 1) / T;
        else end_step = s + W - 1;
      }
      // claim the group after this one (only thread 0 writes; read no earlier than the
      // next band transition)
      if (threadIdx.x == 0 && t_g < gend && t_band == (nb > 2 ? nb - 2 : 0) && (nb > 2 || t_r > 0))
        gring[(t_r + 1) & 3] = claim();
      // the band after this one: rows (t_band+1) mod nb, slot (t_B+1)&1 (nb > 2: the
      // group's bands rotate through two profile slots)
      if (nb > 2 && t_B + 1 >= 2) {
        const bool last_overall = t_g >= gend || (t_band == nb - 1 && gring[(t_r + 1) & 3] >= gend);
        if (!last_overall) {
          rl_step = t_start + W - 1;
          rl_band = t_band + 1 == nb ? 0 : t_band + 1;
          rl_slot = (t_B + 1) & 1;
        }
      }
    }
    if (nb > 2 && s == rl_step) {
      load_band(rl_band, rl_slot);
      __syncthreads();
    }
    const int e = s - warp;
    if (e >= 0 && g < gend) {
      if (tile == 0) {
#pragma unroll
        for (int i = 0; i < K; i++) { H[i] = koff; E[i] = koff; }
        hprev_top = koff;
        // this warp's slice in this band: flush a half whose query changed
        const int sidx = band * W + warp;
        const SliceInfo si = a.slices[P.slice_off + sidx];
        if (si.q_lo != cq_lo || si.q_hi != cq_hi) {
          if (lane < G.count) {
            const int ss = G.first + lane, orig = a.perm[ss];
            if (si.q_lo != cq_lo)
              flush_half(cq_lo, lo16(best), ss, orig, a.scores, a.ndb, a.thresh, a.ovf, a.ovf_count, a.ovf_cap, a.ovf_bits, a.ovf_early);
            if (si.q_hi != cq_hi)
              flush_half(cq_hi, hi16(best), ss, orig, a.scores, a.ndb, a.thresh, a.ovf, a.ovf_count, a.ovf_cap, a.ovf_bits, a.ovf_early);
          }
          if (si.q_lo != cq_lo) best = (best & 0xffff0000u) | (koff & 0xffffu);
          if (si.q_hi != cq_hi) best = (best & 0x0000ffffu) | (koff & 0xffff0000u);
          cq_lo = si.q_lo;
          cq_hi = si.q_hi;
        }
        omask = sidx + 1 < nslices ? start_mask(a.slices[P.slice_off + sidx + 1]) : 0u;
        if (band > 0) {   // new band of the same group: restart at word 0 (prefetched)
          r4 = r4n;
          wnext = nwords > 1 ? 1 : 0;
          r4n = wp[(size_t)wnext * 32];
        }
      } else if ((tile % TPW) == 0) {
        r4 = r4n;
        wnext = (wnext + 1 == nwords) ? 0 : wnext + 1;
        r4n = wp[(size_t)wnext * 32];
      }
      // warp 0: copy the border row of its next element into shared memory with cp.async,
      // one step ahead (warp W-1 wrote it >= 1 step earlier: nt >= W+1)
      if (warp == 0) {
        const bool wrap = tile + 1 == nt;
        const int band2 = wrap ? band + 1 : band, tile2 = wrap ? 0 : tile + 1;
        if (band2 >= 1 && band2 < nb) {
#pragma unroll
          for (int jj = 0; jj < T; jj++)
            cp_async8(&bsm[(((s + 1) & 1) * T + jj) * 32 + lane], &border[(size_t)(tile2 * T + jj) * 32 + lane]);
        }
      }
      // top input of this tile (shared memory, so the column loop is branch-free):
      // warp 0 <- constant row (band 0) or the cp.async'd border; warp w <- warp w-1
      const uint2 *inp = warp == 0 ? (band == 0 ? kin : bsm + (s & 1) * T * 32)
                                   : hand + ((warp - 1) * 2 + ((s - 1) & 1)) * T * 32;
      uint2 *outp = hand + (warp * 2 + (s & 1)) * T * 32;
      const int slot = nb <= 2 ? band : (gband & 1);
      const uint32_t *pr_base = prof_s + slot * kNCodes * S + warp * K;
      const int wq = (tile % TPW) * (T / 4);   // first 32-bit word of r4 used by this tile
      uint32_t wds[T / 4];
#pragma unroll
      for (int q = 0; q < T / 4; q++) {
        const int k = wq + q;
        wds[q] = k == 0 ? r4.x : k == 1 ? r4.y : k == 2 ? r4.z : r4.w;
      }
      // rows of the last band past the longer query are padding: skip them (nobody reads
      // their output; the last band writes no border)
      const bool live = band < nb - 1 || warp * K < rows - (nb - 1) * BAND;
      // UQ: 8 = skewed tiles of 8 columns, 4 = of 4 columns, 81 = tiles of 8 columns with the
      // tile loop kept rolled (half the code of T = 16: the step fits the instruction cache)
      constexpr int GS = (UQ == 8 || UQ == 81) ? 8 : 4;
      // group columns are a multiple of 8: with 16-column tiles the last tile of a band
      // may hold 8 real columns; its second half (pad codes) is skipped (outputs unused)
      const int nq_tile = (T == 16 && tile == nt - 1 && (G.ncols & 15)) ? T / GS / 2 : T / GS;
#pragma unroll(UQ == 81 ? 1 : T / GS)
      for (int q = 0; q < T / GS && live; q++) {
        if (q >= nq_tile) break;
        const uint32_t *prc[GS];
        uint32_t hdc[GS], fc[GS], oh[GS];
#pragma unroll
        for (int j = 0; j < GS; j++) {
          const int jj = q * GS + j;
          const uint32_t word = wds[jj / 4];
          const int c = (word >> (8 * (jj % 4))) & 0xff;
          const uint2 v = inp[jj * 32 + lane];
          prc[j] = pr_base + c * S;
          hdc[j] = hprev_top;   // H(row above, previous column)
          fc[j] = v.y;
          hprev_top = v.x;
        }
        dp_tile<K, GS, 1, kK1PairLoads>(prc, H, E, hdc, fc, oh, best, na, nbeta, koff);
        if (omask) {   // the slice below starts a query: it sees H = F = 0 above
#pragma unroll
          for (int j = 0; j < GS; j++) {
            oh[j] = (oh[j] & ~omask) | (koff & omask);
            fc[j] = (fc[j] & ~omask) | (koff & omask);
          }
        }
#pragma unroll
        for (int j = 0; j < GS; j++) outp[(q * GS + j) * 32 + lane] = make_uint2(oh[j], fc[j]);
      }
      if (warp == W - 1 && band < nb - 1) {
        SW_CHECK(tile * T + T <= a.border_slot_cols);
#pragma unroll
        for (int jj = 0; jj < T; jj++) border[(size_t)(tile * T + jj) * 32 + lane] = outp[jj * 32 + lane];
      }
      // advance; at the end of a group publish this warp's best and move on
      if (++tile == nt) {
        tile = 0;
        gband++;
        if (++band == nb) {
          band = 0;
          if (lane < G.count) {   // end of the group: flush both halves
            const int ss = G.first + lane, orig = a.perm[ss];
            flush_half(cq_lo, lo16(best), ss, orig, a.scores, a.ndb, a.thresh, a.ovf, a.ovf_count, a.ovf_cap, a.ovf_bits, a.ovf_early);
            flush_half(cq_hi, hi16(best), ss, orig, a.scores, a.ndb, a.thresh, a.ovf, a.ovf_count, a.ovf_cap, a.ovf_bits, a.ovf_early);
          }
          best = koff;
          cq_lo = cq_hi = -1;
          gk++;
          g = gring[(++gr) & 3];
          if (g < gend) {
            G = a.groups[g];
            nt = (G.ncols + T - 1) / T;
            nwords = (G.ncols + kWordCols - 1) / kWordCols;
            wnext = nwords > 1 ? 1 : 0;
            wp = a.packed + G.word_off + lane;
            r4 = wp[0];
            r4n = wp[(size_t)wnext * 32];
          }
        }
      }
      if (warp == 0) cp_async_commit_wait();
    }
    // WA cancellation (P18 §IV.A.3: the first replica to finish wins): every kAbortPoll
    // steps thread 0 reads the unit's flag and the step's barrier ORs it over the block,
    // so a losing replica stops within kAbortPoll steps (~0.1 ms), not at the end of its
    // groups.  Partial maxima already flushed are <= the true scores (atomicMax-safe).
    if ((s % kAbortPoll) == kAbortPoll - 1 && a.abort_flag) {
      if (__syncthreads_or(threadIdx.x == 0 && *a.abort_flag != 0)) break;
    } else {
      __syncthreads();
    }
  }
  // groups this block finished (warp W-1 is the last to leave a group): the host turns
  // the unit's count into the cells a cancelled replica really computed
  if (a.progress && warp == W - 1 && lane == 0 && gk > 0) atomicAdd(a.progress, gk);
  if (nb > 1 && threadIdx.x == 0) atomicExch(&a.slot_busy[slot_s], 0);
}

template <int W, int T>
static size_t k1_smem() {
  constexpr int S = kK1PairLoads ? kK1Rows * W + 2 : kK1Rows * W + 1;
  return sizeof(uint32_t) * 2 * kNCodes * S + sizeof(uint2) * W * 2 * T * 32 +
         sizeof(uint32_t) * 2 * W * 32 + sizeof(uint2) * 3 * T * 32;
}

// K1 variants (tuning; SW_K1_VARIANT), (warps per block W, tile T, min blocks/SM, skew G):
// 0 = (8, 8, 2, 4), 1 = (8, 4, 3, 4), 2 = (8, 8, 3, 4), 3 = (8, 8, 2, 8) (default),
// 4 = (4, 8, 4, 8).  Groups of >= kWideCols columns use (8, 16, 2, 8) unless SW_K1_WIDE=0
// (half the pipeline steps and barriers; needs nt >= W+1 tiles of 16 columns).
static int k1_variant() {
  static const int v = [] {
    const char *e = getenv("SW_K1_VARIANT");
    const int x = e ? atoi(e) : 3;
    return (x < 0 || x > 4) ? 3 : x;
  }();
  return v;
}
template <int W, int T, int MINB, int UQ>
static int k1_occ() {
  auto fn = k1_kernel<kK1Rows, W, T, MINB, UQ>;
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)k1_smem<W, T>());
  cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
  int n = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, fn, W * 32, k1_smem<W, T>()) != cudaSuccess) n = 8;
  return n > 0 ? n : 1;
}
int k1_blocks_per_sm() {
  static std::once_flag once;
  static int v = 1;
  std::call_once(once, [] {
    switch (k1_variant()) {
      case 0: v = k1_occ<8, 8, 2, 4>(); break;
      case 1: v = k1_occ<8, 4, 3, 4>(); break;
      case 2: v = k1_occ<8, 8, 3, 4>(); break;
      case 4: v = k1_occ<4, 8, 4, 8>(); break;
      default: v = k1_occ<8, 8, 2, 8>(); break;
    }
  });
  return v;
}
int k1_band_rows() { return k1_variant() == 4 ? kK1Rows * 4 : kK1Rows * 8; }
static bool k1_wide_rolled() {   // SW_K1_WIDE_ROLLED=1: 16-column steps with a rolled tile loop
  static const bool v = [] { const char *e = getenv("SW_K1_WIDE_ROLLED"); return e && atoi(e) == 1; }();
  return v;
}
static bool k1_wide_enabled() {
  static const bool v = [] { const char *e = getenv("SW_K1_WIDE"); return !(e && atoi(e) == 0); }();
  return v;
}

// dynamic shared memory above 48 KB needs the function attribute on the launching device;
// it is set before every launch (cheap, and correct with several devices and threads)
template <int W, int T, int MINB, int UQ>
static void k1_go(const K1Args &a, dim3 g, cudaStream_t st) {
  auto fn = k1_kernel<kK1Rows, W, T, MINB, UQ>;
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)k1_smem<W, T>());
  cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
  fn<<<g, W * 32, k1_smem<W, T>(), st>>>(a);
}

void launch_k1(const K1Args &a_in, int n_groups, int min_cols, int, cudaStream_t st, int n_sm) {
  if (n_groups <= 0) return;
  K1Args a = a_in;
  a.n_groups = n_groups;
  // one wave of blocks (each streams through n_groups / grid groups)
  const int cap = std::max(1, n_sm) * k1_blocks_per_sm();
  const dim3 g(std::min(n_groups, cap));
  if (min_cols >= kWideCols && k1_variant() == 3 && k1_wide_enabled()) {
    if (k1_wide_rolled()) k1_go<8, 16, 2, 81>(a, g, st);
    else k1_go<8, 16, 2, 8>(a, g, st);
    return;
  }
  switch (k1_variant()) {
    case 0: k1_go<8, 8, 2, 4>(a, g, st); break;
    case 1: k1_go<8, 4, 3, 4>(a, g, st); break;
    case 2: k1_go<8, 8, 3, 4>(a, g, st); break;
    case 4: k1_go<4, 8, 4, 8>(a, g, st); break;
    default: k1_go<8, 8, 2, 8>(a, g, st); break;
  }
}

// ------------------------------------------------------------------------------------
// K3: intra-task kernel for long DB sequences (P14 §II.B fine-grained approach, Fig. 3a:
// "the calculations that can be done in parallel evolve as waves on diagonals").  A warp
// works on one (query pack, long sequence) pair; lane l owns rows [l*K, (l+1)*K) of each
// chunk of 32*K query rows.  At step t lane l updates the T-column tile t - l (T columns
// give the lane T independent dependency chains); it receives the bottom row (H, F) of
// that tile and its residue codes from lane l-1 by __shfl_up_sync, lane 0 takes them from
// the previous chunk's border row and the packed database (streamed by cp.async through a
// 3-deep shared-memory ring, two tiles ahead), and lane 31 writes the chunk's bottom row
// to the border.
// Block = kK3Warps sequences sharing the chunk profile in shared memory, laid out
// [slot][row pair][lane][2] (8-byte bank pair = lane mod 16: conflict-free although every
// lane reads a different code).  The unit's WA cancellation flag is polled at every chunk
// start (__syncthreads_or), and each warp counts the (sequence, chunk) pairs it completed
// into the unit's progress counter.
//
// Chunk split over a thread-block cluster (C = 2 or 4, for units with too few long pairs to
// fill the GPU -- one GPU's share of C5 at 8 GPUs): the C CTAs of a cluster take the same
// kK3Warps sequences, CTA r the chunks r, r+C, r+2C, ... (the wavefront of Fig. 3a once more,
// across CTAs: "it sends its border column to P1", P14).  Chunk ch writes its bottom row to
// border buffer ch % C and publishes its progress every kK3Pub tiles (st.release, a
// per-(warp slot, buffer) counter counting tiles since the launch); the CTA running chunk
// ch+1 acquires that counter before prefetching a tile (cp.async.cg: L2, never a stale L1
// line).  A buffer is rewritten by chunk ch+C only after chunk ch+1 consumed it: chunk ch+C
// tile t needs chunk ch+C-1 tile t, ..., which needs chunk ch+1 past tile t.  The cluster
// guarantees producer and consumer are co-resident, so the waits cannot deadlock.  Border
// rows go through L2 rather than DSMEM: a DSMEM ring must hold the producer's 32-tile lane
// skew (>= 40 tiles x 64 B x 4 warps), which would drop K3 from 4 to 3 CTAs per SM.
// A persistent loop walks sequence blocks (grid capped to the resident clusters for C > 1,
// or to an SM budget when emulating a slower PE).
// ------------------------------------------------------------------------------------
__device__ __forceinline__ void cp_async16_cg(void *smem_dst, const void *gsrc) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(smem_dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ int ld_acquire(const int *p) {
  int v;
  asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(int *p, int v) {
  asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

template <int K, int T, int C>
__global__ void __launch_bounds__(kK3Warps * 32, 4) k3_kernel(const K3Args a) {
  static_assert(T == 4 || T == 8, "tile = one or two 32-bit words of packed residues");
  constexpr int NW = T / 4;          // 32-bit residue words per tile
  constexpr int TPU = 4 / NW;        // tiles per 128-bit word
  constexpr int CH = 32 * K;
  extern __shared__ __align__(16) uint32_t smem[];  // [kNCodes][K/2][32][2], then the rings
  uint4 *ring4 = reinterpret_cast<uint4 *>(smem + kNCodes * K * 32);   // [warps][3]
  uint2 *ring2 = reinterpret_cast<uint2 *>(ring4 + kK3Warps * 3);     // [warps][3][T]
  if (block_aborted(a.abort_flag)) return;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t koff = pk2(kOff), na = a.na, nbeta = a.nb;
  const uint32_t padw = 0x01010101u * kPadCode;
  uint32_t *prof_s = smem;
  // tasks = (pack, sequence block of kK3Warps sequences); a unit spans packs [pair, pair + npk)
  // (clustered units only), task t = pack pair + t % npk of block t / npk: longest blocks first,
  // every pack's at once
  const int nsb = (a.l1 - a.l0 + kK3Warps - 1) / kK3Warps;
  const int ntask = nsb * a.npk;
  const int crank = C > 1 ? (int)(blockIdx.x % C) : 0;     // CTA rank in the cluster
  const int cid = blockIdx.x / C, ncl = gridDim.x / C;
  // C > 1: this warp's (slot, buffer) border rows and progress counters are per grid slot
  // (reused across the sequence blocks of the persistent loop); cum[b] = tiles of buffer b
  // published in earlier sequence blocks, identical in the producer and consumer CTAs
  const int gslot = cid * kK3Warps + warp;
  int cum[C];
#pragma unroll
  for (int b = 0; b < C; b++) cum[b] = 0;
  int done = 0;          // (sequence, chunk) pairs this warp completed
  bool aborted = false;
  // C > 1: the clusters of a launch claim tasks dynamically (longest blocks first, the
  // sorted order) from a per-launch counter; rank 0 claims and broadcasts over DSMEM
  __shared__ int sb_claim;
  auto next_task = [&](int prev) -> int {
    if (C == 1) return prev < 0 ? cid : prev + ncl;
    namespace cg = cooperative_groups;
    cg::cluster_group cl = cg::this_cluster();
    if (crank == 0 && threadIdx.x == 0)
      sb_claim = (aborted || (a.abort_flag && *a.abort_flag != 0)) ? ntask : atomicAdd(a.claim, 1);
    cl.sync();
    const int v = *cl.map_shared_rank(&sb_claim, 0);
    cl.sync();   // rank 0 may overwrite sb_claim only after every CTA read it
    return v;
  };

  for (int task = next_task(-1); task < ntask; task = next_task(task)) {
    if (aborted) continue;   // C > 1: go straight to the next claim (it returns the end)
    const int sb = task / a.npk;
    const QueryPair P = a.pairs[a.pair + task % a.npk];
    const int rows = P.rows;
    const int nch = (rows + CH - 1) / CH;
    const int nslices = P.rows_padded / 16;
    const int32_t *gprof = a.prof + P.prof_off;
    const int s = a.l0 + sb * kK3Warps + warp;
    const bool valid = s < a.l1;
    const int len = valid ? a.sorted_len[s] : 0;
    const GroupInfo G = a.groups[valid ? s / kGroup : 0];
    const int gl = s % kGroup;
    const uint4 *wp = a.packed + G.word_off + gl;
    const int ntile = (len + T - 1) / T;   // columns up to ntile*T <= G.ncols carry pad codes
    const int orig = valid ? a.perm[s] : 0;
    uint32_t best = koff;
    int cq_lo = -1, cq_hi = -1;   // queries of this lane's slice (per half)

    for (int ch = crank; ch < nch; ch += C) {
      // every warp is done with the previous chunk profile; WA cancellation poll
      if (__syncthreads_or(threadIdx.x == 0 && a.abort_flag && *a.abort_flag != 0)) {
        aborted = true;
        break;
      }
      for (int idx = threadIdx.x; idx < kNCodes * CH; idx += kK3Warps * 32) {
        const int c = idx / CH, r = idx - c * CH;     // r = l*K + i
        const int l = r / K, i = r - l * K;
        prof_s[((c * (K / 2) + i / 2) * 32 + l) * 2 + (i & 1)] =
            (uint32_t)__ldg(gprof + (int64_t)c * P.rows_padded + ch * CH + r);
      }
      __syncthreads();
      if (!valid) continue;
      // lane l's rows of this chunk are slice ch*32 + l: flush a half whose query changed;
      // the start mask of the slice below applies to what this lane hands down
      uint32_t omask = 0;
      {
        const int sidx = ch * 32 + lane;
        const SliceInfo si = a.slices[P.slice_off + sidx];
        if (si.q_lo != cq_lo) {
          flush_half(cq_lo, lo16(best), s, orig, a.scores, a.ndb, a.thresh, a.ovf, a.ovf_count, a.ovf_cap, a.ovf_bits, a.ovf_early);
          best = (best & 0xffff0000u) | (koff & 0xffffu);
          cq_lo = si.q_lo;
        }
        if (si.q_hi != cq_hi) {
          flush_half(cq_hi, hi16(best), s, orig, a.scores, a.ndb, a.thresh, a.ovf, a.ovf_count, a.ovf_cap, a.ovf_bits, a.ovf_early);
          best = (best & 0x0000ffffu) | (koff & 0xffff0000u);
          cq_hi = si.q_hi;
        }
        if (sidx + 1 < nslices) omask = start_mask(a.slices[P.slice_off + sidx + 1]);
      }
      done++;
      if (len == 0) continue;
      // border rows: C == 1: one row per sequence (slot sb*kK3Warps + warp of the unit);
      // C > 1: buffer ch % C of this grid slot
      const int bin = (ch + C - 1) % C, bout = ch % C;
      const uint2 *border_in = C == 1 ? a.border + (size_t)(sb * kK3Warps + warp) * a.border_stride
                                      : a.border + (size_t)(gslot * C + bin) * a.border_stride;
      uint2 *border_out = C == 1 ? a.border + (size_t)(sb * kK3Warps + warp) * a.border_stride
                                 : a.border + (size_t)(gslot * C + bout) * a.border_stride;
      SW_CHECK(C > 1 ? (int64_t)gslot * C + C <= a.border_rows : (int64_t)sb * kK3Warps + warp < a.border_rows);
      const int *prog_in = a.kprog + gslot * C + bin;
      int *prog_out = a.kprog + gslot * C + bout;
      // counters count tiles written into a buffer since the launch: earlier sequence blocks
      // (cum[]) plus this sequence's earlier chunks of the same residue class mod C
      const int need0 = C > 1 && ch > 0 ? cum[bin] + ((ch - 1) / C) * ntile : 0;
      const int pub0 = C > 1 ? cum[bout] + (ch / C) * ntile : 0;
      int seen = 0;                 // (lane 0) last acquired value of prog_in
      const bool any_mask = __any_sync(0xffffffffu, omask != 0);   // warp-uniform
      uint32_t H[K], E[K];
#pragma unroll
      for (int i = 0; i < K; i++) { H[i] = koff; E[i] = koff; }
      uint32_t hprev_top = koff;
      uint32_t out_h[T], out_f[T], out_c[NW];
#pragma unroll
      for (int jj = 0; jj < T; jj++) { out_h[jj] = koff; out_f[jj] = koff; }
#pragma unroll
      for (int q = 0; q < NW; q++) out_c[q] = padw;
      // lane 0 streams the tile inputs (border row of the previous chunk, residue words)
      // into a 3-deep per-warp shared-memory ring with cp.async, two tiles ahead
      uint2 *bring = ring2 + warp * 3 * T;   // [3][T]
      uint4 *wring = ring4 + warp * 3;       // [3] words of 16 residues
      auto fetch = [&](int tt) {             // lane 0: inputs of tile tt into slot tt % 3
        if (tt < ntile) {
          const int sl = tt % 3;
          if (ch > 0) {
            if (C > 1) {   // wait until the chunk above has published tile tt
              const int want = need0 + tt + 1;
              if (seen < want) {
                seen = ld_acquire(prog_in);
                if (seen < want) {
                  // really waiting.  (%globaltimer is slow to read: an earlier version that
                  // read it on every entry here ran the first consumer chunks ~3x slower.)
                  const long long t_wait = clock64();
                  while ((seen = ld_acquire(prog_in)) < want) {
                    if (a.abort_flag && *a.abort_flag != 0) break;   // the producer stops too
                    if (clock64() - t_wait > (1ll << 36)) __trap();   // ~35 s: never hang the GPU
                  }
                }
              }
              SW_CHECK((int64_t)tt * T + T <= a.border_stride);
#pragma unroll
              for (int jj = 0; jj < T; jj += 2) cp_async16_cg(&bring[sl * T + jj], &border_in[tt * T + jj]);
            } else {
#pragma unroll
              for (int jj = 0; jj < T; jj += 2) cp_async16(&bring[sl * T + jj], &border_in[tt * T + jj]);
            }
          }
          if (tt % TPU == 0) cp_async16(&wring[(tt / TPU) % 3], &wp[(size_t)(tt / TPU) * kGroup]);
        }
      };
      if (lane == 0) {
        fetch(0);
        asm volatile("cp.async.commit_group;" ::: "memory");
        fetch(1);
        cp_async_commit_wait1();   // tile 0 has landed
      }
      __syncwarp();
      const int steps = ntile + 31;
      for (int t = 0; t < steps; t++) {
        uint32_t in_h[T], in_f[T], in_c[NW];
#pragma unroll
        for (int jj = 0; jj < T; jj++) {
          in_h[jj] = __shfl_up_sync(0xffffffffu, out_h[jj], 1);
          in_f[jj] = __shfl_up_sync(0xffffffffu, out_f[jj], 1);
        }
#pragma unroll
        for (int q = 0; q < NW; q++) in_c[q] = __shfl_up_sync(0xffffffffu, out_c[q], 1);
        if (lane == 0 && t < ntile) {
          const uint4 wv = wring[(t / TPU) % 3];
          const int q0 = (t % TPU) * NW;
#pragma unroll
          for (int q = 0; q < NW; q++) {
            const int k = q0 + q;
            in_c[q] = k == 0 ? wv.x : k == 1 ? wv.y : k == 2 ? wv.z : wv.w;
          }
          const int sl = t % 3;
#pragma unroll
          for (int jj = 0; jj < T; jj++) {
            const uint2 v = ch > 0 ? bring[sl * T + jj] : make_uint2(koff, koff);
            in_h[jj] = v.x;
            in_f[jj] = v.y;
          }
          fetch(t + 2);              // slot (t+2)%3 == (t-1)%3, consumed last step
          cp_async_commit_wait1();   // tile t+1 has landed
        }
        const int tile = t - lane;
        if (tile >= 0 && tile < ntile) {
          const uint32_t *prc[T];
          uint32_t hdc[T];
#pragma unroll
          for (int jj = 0; jj < T; jj++) {
            const uint32_t c = (in_c[jj / 4] >> (8 * (jj % 4))) & 0xffu;
            prc[jj] = prof_s + (c * (K / 2) * 32 + lane) * 2;
            hdc[jj] = hprev_top;
            out_f[jj] = in_f[jj];
            hprev_top = in_h[jj];
          }
          dp_tile<K, T, 32, true, 64>(prc, H, E, hdc, out_f, out_h, best, na, nbeta, koff);
          if (any_mask) {   // bit-select: omask is 0 except in a lane above a query start
#pragma unroll
            for (int jj = 0; jj < T; jj++) {
              out_h[jj] = (out_h[jj] & ~omask) | (koff & omask);
              out_f[jj] = (out_f[jj] & ~omask) | (koff & omask);
            }
          }
#pragma unroll
          for (int q = 0; q < NW; q++) out_c[q] = in_c[q];
          if (lane == 31 && ch < nch - 1) {
            SW_CHECK((int64_t)tile * T + T <= a.border_stride);
#pragma unroll
            for (int jj = 0; jj < T; jj++) border_out[tile * T + jj] = make_uint2(out_h[jj], out_f[jj]);
            if (C > 1 && ((tile + 1) % a.pub_every == 0 || tile + 1 == ntile))
              st_release(prog_out, pub0 + tile + 1);   // orders this lane's border stores
          }
        }
      }
      if (lane == 0) asm volatile("cp.async.wait_all;" ::: "memory");
    }
    // every CTA of the cluster advances the same cum[]: buffer b received ntile tiles from
    // each chunk ch < nch - 1 with ch % C == b
#pragma unroll
    for (int b = 0; b < C; b++)
      if (C > 1 && nch - 1 > b) cum[b] += ((nch - 1 - b + C - 1) / C) * ntile;
    if (valid && !aborted) {   // every lane flushes what it holds
      flush_half(cq_lo, lo16(best), s, orig, a.scores, a.ndb, a.thresh, a.ovf, a.ovf_count, a.ovf_cap, a.ovf_bits, a.ovf_early);
      flush_half(cq_hi, hi16(best), s, orig, a.scores, a.ndb, a.thresh, a.ovf, a.ovf_count, a.ovf_cap, a.ovf_bits, a.ovf_early);
    }
    if (C == 1 && aborted) break;   // (C > 1: every CTA of the cluster reaches the claim, which ends)
  }
  if (a.progress && lane == 0 && done > 0) atomicAdd(a.progress, done);
}
// K3 tile width (tuning; SW_K3_T): 8 columns per lane step (default) or 4.
static int k3_tile() {
  static const int v = [] { const char *e = getenv("SW_K3_T"); return (e && atoi(e) == 4) ? 4 : 8; }();
  return v;
}
template <int T>
static size_t k3_smem() {
  return sizeof(uint32_t) * kNCodes * kK3Rows * 32 + sizeof(uint4) * kK3Warps * 3 +
         sizeof(uint2) * kK3Warps * 3 * T;
}
template <int T, int C>
static void k3_go(const K3Args &a, int n, int max_blocks, cudaStream_t st) {
  const size_t smem = k3_smem<T>();
  const int nsb = (n + kK3Warps - 1) / kK3Warps * std::max(1, a.npk);   // tasks
  auto fn = k3_kernel<kK3Rows, T, C>;
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
  const int clusters = std::max(1, std::min(nsb, std::max(1, max_blocks / C)));
  if (C == 1) {
    fn<<<clusters, kK3Warps * 32, smem, st>>>(a);
    return;
  }
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(clusters * C);
  cfg.blockDim = dim3(kK3Warps * 32);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = C;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cudaLaunchKernelEx(&cfg, fn, a);
}
int k3_blocks_per_sm() {
  static std::once_flag once;
  static int v = 4;
  std::call_once(once, [] {
    int n = 0;
    const size_t smem = k3_tile() == 4 ? k3_smem<4>() : k3_smem<8>();
    auto fn = k3_tile() == 4 ? k3_kernel<kK3Rows, 4, 1> : k3_kernel<kK3Rows, 8, 1>;
    cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, fn, kK3Warps * 32, smem) == cudaSuccess && n > 0) v = n;
  });
  return v;
}
// cluster size 1, 2, 3, 4, 5 or 8 (3, 5, 8: 8-column tiles only; a.kprog: [grid slots][C] zeroed progress counters when C > 1).
// max_blocks caps the grid (resident CTAs; an SM budget when emulating a slower PE);
// C > 1 needs at most the resident clusters (persistent loop, sequence blocks claimed
// through a.claim, zeroed), C == 1 one block per kK3Warps sequences
void launch_k3(const K3Args &a, int cluster, int max_blocks, cudaStream_t st) {
  const int n = a.l1 - a.l0;
  if (n <= 0) return;
  const bool t4 = k3_tile() == 4;
  switch (cluster) {
    case 2: if (t4) k3_go<4, 2>(a, n, max_blocks, st); else k3_go<8, 2>(a, n, max_blocks, st); break;
    case 4: if (t4) k3_go<4, 4>(a, n, max_blocks, st); else k3_go<8, 4>(a, n, max_blocks, st); break;
    case 3: k3_go<8, 3>(a, n, max_blocks, st); break;
    case 5: k3_go<8, 5>(a, n, max_blocks, st); break;
    case 8: k3_go<8, 8>(a, n, max_blocks, st); break;
    default: if (t4) k3_go<4, 1>(a, n, max_blocks, st); else k3_go<8, 1>(a, n, max_blocks, st); break;
  }
}

// ------------------------------------------------------------------------------------
// Local load (P24 §V.C "introduced local load ... after 60 seconds", the superpi analogue
// on a GPU): one block per SM holding all of its shared memory, so no DP block can share
// the SM, spinning on integer work until the host raises *stop (or max_ns elapses: the
// kernel can never outlive a lost host).  Launched on its own high-priority stream.
// ------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) noise_kernel(const volatile int32_t *stop, uint64_t max_ns,
                                                    uint32_t *sink) {
  extern __shared__ uint32_t noise_s[];
  const uint64_t t0 = globaltimer();
  uint32_t x = threadIdx.x * 2654435761u + blockIdx.x;
  while (true) {
#pragma unroll 8
    for (int k = 0; k < 4096; k++) x = __vimax3_s16x2(x * 1664525u + 1013904223u, x, k);
    if (*stop != 0 || globaltimer() - t0 > max_ns) break;
  }
  noise_s[threadIdx.x] = x;
  if (x == 0x9e3779b9u) sink[blockIdx.x] = noise_s[(threadIdx.x + 1) & 255];
}
size_t noise_smem() {
  int dev = 0, v = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  return v > 0 ? (size_t)v : 227 * 1024;
}
void launch_noise(const int32_t *stop, int n_blocks, uint64_t max_ns, uint32_t *sink, cudaStream_t st) {
  if (n_blocks <= 0) return;
  const size_t smem = noise_smem();
  cudaFuncSetAttribute(noise_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  noise_kernel<<<n_blocks, 256, smem, st>>>(stop, max_ns, sink);
}

// ------------------------------------------------------------------------------------
// K2: int32 re-run of saturated (query, sequence) pairs.  Same recurrence as K1/K3 in
// plain int32 (E and F floored at 0, exact for H: DESIGN.md §6), run by a BLOCK of
// kK2Threads: thread L owns rows [L*R, (L+1)*R) of a chunk of 128*R query rows and runs
// the wavefront of P14 §II.B (Fig. 3a) across the block -- at step t thread L updates the
// K2C-column tile t - L and hands its bottom row (H, F) and the tile's residue codes to
// thread L+1 through a double-buffered shared-memory slot (one __syncthreads per step);
// thread 0 streams the codes and the border row of the chunk above through a cp.async ring.
// Scores come from a per-chunk int8 profile [code][thread][R] in shared memory: one LDS of
// R bytes per column and thread, bank = thread (no conflicts).
// A block is the size of a K3 block (128 threads, <= 128 registers, ~60 KB of shared
// memory), so it starts in the SM slot that one K3 block leaves: a 512-thread block that
// needed a whole SM waited behind the persistent K3 blocks until the step's end.
// Two kinds of pairs:
//  * big pairs (m*n >= big_cells; C5: a 5,000-aa query inside a 35k-residue sequence) are
//    split into chunks run by as many blocks at once: chunk r+1 follows chunk r tile by
//    tile through a border row in L2 (a progress counter tagged with the pair's number,
//    released every kK2Pub tiles and acquired before each prefetch).  Blocks take chunk
//    tickets in order, so a chunk only waits for chunks whose blocks already run (no
//    co-scheduling needed).  One block per pair ran C5's planted pair in 12.3 ms;
//  * the other pairs are taken by single blocks, chunks of 128*kK2RSmall rows in order.
// Each list has its own cursor (small: ovf_cursor[0], big: ovf_cursor[1]); a cursor
// skips the other kind's entries and never passes the count this launch saw.
// ------------------------------------------------------------------------------------
constexpr int K2C = 4;           // columns per tile (one aligned 32-bit word of codes)
constexpr int kK2RSmall = 16;    // rows per thread of a single-block pair (2,048-row chunks)
constexpr int kK2MaxR = 16;
constexpr int kK2Pub = 8;        // tiles between a big pair's progress publications
constexpr int kK2Ring = 8;       // tiles in flight (thread 0's cp.async ring)
constexpr size_t kK2Smem = (size_t)kNCodes * kK2Threads * kK2MaxR + sizeof(int2) * 2 * kK2Threads * K2C +
                           sizeof(uint32_t) * 2 * kK2Threads;
static_assert(kK2Span * kK2Threads * kK2MaxR > SW_MAX_QUERY_LEN, "a big pair is at most kK2Span chunks");

__device__ __forceinline__ long long ld_acquire64(const long long *p) {
  long long v;
  asm volatile("ld.acquire.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release64(long long *p, long long v) {
  asm volatile("st.release.gpu.global.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// claim the next entry of one kind from cursor `cur` (thread 0); returns count when none.
// An entry counted but not yet written (its writer is between the atomicAdd and the store:
// K2 can run beside the unit that lists it) still holds (-1, -1): wait for it
__device__ __forceinline__ int k2_claim(const K2Args &a, int *cur_p, int count, bool big, int2 &entry) {
  int cur = *(volatile int32_t *)cur_p;
  while (cur < count) {
    int2 e;
    const long long t_wait = clock64();
    while (true) {
      const long long v = *(const volatile long long *)(a.ovf + cur);   // one 8-byte load
      e = make_int2((int)(v & 0xffffffffll), (int)(v >> 32));
      if (e.x >= 0) break;
      if (clock64() - t_wait > (1ll << 36)) __trap();
    }
    const int64_t cells = (a.qoff[e.x + 1] - a.qoff[e.x]) * (int64_t)a.sorted_len[e.y];
    const int seen = atomicCAS(cur_p, cur, cur + 1);
    if (seen != cur) { cur = seen; continue; }          // someone else moved it: retry there
    if ((cells >= a.big_cells) == big) { entry = e; return cur; }   // ours
    cur++;                                              // skipped (the other kind's)
  }
  return count;
}

template <int R> struct K2Word;
template <> struct K2Word<4> { typedef uint32_t T; };
template <> struct K2Word<8> { typedef uint2 T; };
template <> struct K2Word<16> { typedef uint4 T; };
template <int R>
__device__ __forceinline__ int k2_score(const typename K2Word<R>::T &w, int i) {   // signed byte i
  uint32_t v;
  if constexpr (R == 4) v = w;
  else if constexpr (R == 8) v = (i < 4) ? w.x : w.y;
  else v = (i < 4) ? w.x : (i < 8) ? w.y : (i < 12) ? w.z : w.w;
  return (int)(int8_t)(v >> (8 * (i & 3)));
}

// One chunk [r0, r0 + nact*R) of pair (qc, m) x (sequence of group G, lane gl) on this
// block; returns this thread's maximum H.  bin / bout: border rows in / out (nullptr: the
// first / last chunk); prog_in / prog_out: (big pairs) the producer's / this chunk's
// progress counter, values (epoch << 32) + tiles.  bin == bout is allowed when the chunks
// of a pair run in order on one block (the writer trails the reader by nact tiles).
template <int R>
__device__ __forceinline__ int k2_chunk(const K2Args &a, const int8_t *Ms, int8_t *prof, int2 *hand,
                                        uint32_t *handc, int2 *ring, uint32_t *cring, const uint8_t *qc,
                                        int m, int r0, int nact, const GroupInfo &G, int gl, int ntile,
                                        const int2 *bin, int2 *bout, const long long *prog_in,
                                        long long *prog_out, long long epoch) {
  typedef typename K2Word<R>::T W;
  const int L = threadIdx.x;
  const uint32_t *words = reinterpret_cast<const uint32_t *>(a.packed);
  const int na = -a.alpha, nb = -a.beta;
  // this chunk's profile: byte i of prof[c][L] = S[q(r0 + L*R + i)][code of slot c]
  __syncthreads();   // the previous chunk's profile is no longer read
  {
    uint32_t pw[R / 4];
    for (int c = 0; c < kNCodes; c++) {
#pragma unroll
      for (int k = 0; k < R / 4; k++) {
        uint32_t v = 0;
#pragma unroll
        for (int b = 0; b < 4; b++) {
          const int row = r0 + L * R + k * 4 + b;
          const int sc = (row < m && c < 24) ? (int)Ms[qc[row] * 24 + c_code_of_slot[c]] : kPadScore;
          v |= (uint32_t)(uint8_t)(int8_t)sc << (8 * b);
        }
        pw[k] = v;
      }
      uint32_t *dst = reinterpret_cast<uint32_t *>(prof + ((size_t)c * kK2Threads + L) * R);
#pragma unroll
      for (int k = 0; k < R / 4; k++) dst[k] = pw[k];
    }
  }
  __syncthreads();
  auto codes_at = [&](int tt) -> const uint32_t * {   // codes of columns tt*4 .. tt*4+3
    const int col = tt * K2C;
    return words + ((G.word_off + (int64_t)(col >> 4) * kGroup + gl) * 4 + ((col & 15) >> 2));
  };
  // big pairs: wait until the chunk above has published tile tt (thread 0 only)
  long long seen = 0;
  auto wait_tile = [&](int tt) {
    if (!prog_in) return;
    const long long want = (epoch << 32) + tt + 1;
    if (seen >= want) return;
    const long long t_wait = clock64();
    while ((seen = ld_acquire64(prog_in)) < want)
      if (clock64() - t_wait > (1ll << 36)) __trap();   // ~35 s: never hang the GPU
  };
  // thread 0 streams the tile inputs -- the residue codes and the border row of the chunk
  // above (cp.async.cg: L2, never a stale L1 line) -- into a kK2Ring-tile shared-memory ring,
  // kK2Ring - 1 tiles ahead: an L2 round trip is longer than a step
  auto fetch = [&](int tt) {
    if (tt < ntile) {
      const unsigned d = (unsigned)__cvta_generic_to_shared(&cring[tt % kK2Ring]);
      asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(d), "l"(codes_at(tt)) : "memory");
      if (bin) {
        SW_CHECK((int64_t)tt * K2C + K2C <= a.border_stride);
        wait_tile(tt);
        cp_async16_cg(&ring[(tt % kK2Ring) * K2C], bin + tt * K2C);
        cp_async16_cg(&ring[(tt % kK2Ring) * K2C + 2], bin + tt * K2C + 2);
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  const bool active = L < nact;
  int H[R], E[R];
#pragma unroll
  for (int i = 0; i < R; i++) { H[i] = 0; E[i] = 0; }
  int hprev_top = 0, best = 0;
  const int steps = ntile + nact - 1;
  if (L == 0)
    for (int tt = 0; tt < kK2Ring - 1; tt++) fetch(tt);
  const W *pbase = reinterpret_cast<const W *>(prof) + L;   // + c * kK2Threads
  for (int t = 0; t < steps; t++) {
    const int tile = t - L;
    if (active && tile >= 0 && tile < ntile) {
      uint32_t cw;
      int2 in[K2C];
      if (L == 0) {
        fetch(tile + kK2Ring - 1);   // into the slot of tile - 1, consumed last step
        asm volatile("cp.async.wait_group %0;" ::"n"(kK2Ring - 1) : "memory");   // tile landed
        cw = cring[tile % kK2Ring];
#pragma unroll
        for (int g = 0; g < K2C; g++) in[g] = bin ? ring[(tile % kK2Ring) * K2C + g] : make_int2(0, 0);
      } else {
        cw = handc[((t - 1) & 1) * kK2Threads + L - 1];
#pragma unroll
        for (int g = 0; g < K2C; g++) in[g] = hand[(((t - 1) & 1) * K2C + g) * kK2Threads + L - 1];
      }
      W sw[K2C];
      int hd[K2C], f[K2C], oh[K2C];
#pragma unroll
      for (int g = 0; g < K2C; g++) {
        SW_CHECK(((cw >> (8 * g)) & 0xffu) < (uint32_t)kNCodes);
        sw[g] = pbase[((cw >> (8 * g)) & 0xffu) * kK2Threads];
        hd[g] = hprev_top;
        f[g] = in[g].y;
        hprev_top = in[g].x;
      }
      // skewed tile: at sub-step k column g updates row k - g (K2C independent chains)
#pragma unroll
      for (int k = 0; k < R + K2C - 1; k++) {
#pragma unroll
        for (int g = 0; g < K2C; g++) {
          const int i = k - g;
          if (i >= 0 && i < R) {
            const int x = k2_score<R>(sw[g], i) + hd[g];
            const int h = __vimax3_s32(x, E[i], f[g]);      // >= 0: E, F floored at 0
            const int tt = __viaddmax_s32(h, na, 0);        // max(H - alpha, 0)
            E[i] = __viaddmax_s32(E[i], nb, tt);            // E(i, j+1)
            f[g] = __viaddmax_s32(f[g], nb, tt);            // F(i+1, j)
            hd[g] = H[i];
            H[i] = h;
            best = max(best, h);
            if (i == R - 1) oh[g] = h;
          }
        }
      }
#pragma unroll
      for (int g = 0; g < K2C; g++) hand[((t & 1) * K2C + g) * kK2Threads + L] = make_int2(oh[g], f[g]);
      handc[(t & 1) * kK2Threads + L] = cw;
      if (L == nact - 1 && bout) {
        SW_CHECK((int64_t)tile * K2C + K2C <= a.border_stride);
#pragma unroll
        for (int g = 0; g < K2C; g++) bout[tile * K2C + g] = make_int2(oh[g], f[g]);
        if (prog_out && ((tile + 1) % kK2Pub == 0 || tile + 1 == ntile))
          st_release64(prog_out, (epoch << 32) + tile + 1);   // orders this thread's border stores
      }
    }
    __syncthreads();
  }
  if (L == 0) asm volatile("cp.async.wait_all;" ::: "memory");
  return best;
}

__global__ void __launch_bounds__(kK2Threads) k2_kernel(const K2Args a) {
  extern __shared__ __align__(16) int32_t k2s[];
  int2 *hand = reinterpret_cast<int2 *>(k2s);                                // [2][K2C][threads]
  uint32_t *handc = reinterpret_cast<uint32_t *>(hand + 2 * K2C * kK2Threads);   // [2][threads]
  int8_t *prof = reinterpret_cast<int8_t *>(handc + 2 * kK2Threads);          // [codes][threads][R]
  __shared__ __align__(16) uint32_t cring[kK2Ring];
  __shared__ __align__(16) int2 ring[kK2Ring * K2C];
  __shared__ int8_t Ms[24 * 24];
  __shared__ int claim_s;
  __shared__ int2 claim_e;
  __shared__ int red_s[kK2Threads / 32];
  const int count = min(*a.ovf_count, a.ovf_cap);
  if (*(volatile int32_t *)a.ovf_cursor >= count && *(volatile int32_t *)(a.ovf_cursor + 1) >= count)
    return;   // nothing saturated (the usual case)
  for (int k = threadIdx.x; k < 24 * 24; k += kK2Threads) Ms[k] = a.matrix[k];
  const int L = threadIdx.x, lane = L & 31;
  auto block_max = [&](int best) {   // -> thread 0
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) best = max(best, __shfl_xor_sync(0xffffffffu, best, o));
    if (lane == 0) red_s[L >> 5] = best;
    __syncthreads();
    int b = 0;
    if (L == 0)
      for (int w = 0; w < kK2Threads / 32; w++) b = max(b, red_s[w]);
    return b;
  };
  auto spin_until = [](const volatile int32_t *p, int want) {   // acquire
    const long long t_wait = clock64();
    while (true) {
      int v;
      asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
      if (v >= want) break;
      if (clock64() - t_wait > (1ll << 36)) __trap();   // ~35 s: never hang the GPU
    }
  };
  // ---- big pairs: blocks take chunk tickets in order (ticket t = chunk t % kK2Span of big
  // pair t / kK2Span), so a chunk only ever waits for chunks with earlier tickets, whose
  // blocks are already running.  Ticket 0 of a pair finds it in the list and publishes it;
  // pairs alternate between two slots of border rows and progress counters, and a pair
  // starts only when the pair two before it (same slot) has finished every ticket.
  K2Ctl *ctl = a.ctl;
  int2 *bbase = reinterpret_cast<int2 *>(a.border) + (size_t)gridDim.x * a.border_stride;
  while (true) {
    if (L == 0) claim_s = atomicAdd(&ctl->tickets, 1);
    __syncthreads();
    const int t = claim_s;
    const int j = t / kK2Span, c = t % kK2Span, sl = j & 1;
    K2Pair *pp = &ctl->pairs[j & 7];
    if (L == 0) {
      if (c == 0) {
        spin_until(&ctl->slot_done[sl], j / 2);   // the pair two before has finished
        int2 e = make_int2(-1, -1);
        if (k2_claim(a, a.ovf_cursor + 1, count, true, e) >= count) e = make_int2(-1, -1);
        pp->q = e.x;
        pp->s = e.y;
        asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(&pp->tag), "r"(j + 1) : "memory");
        claim_e = e;
      } else {
        spin_until(&pp->tag, j + 1);
        claim_e = make_int2(*(volatile int32_t *)&pp->q, *(volatile int32_t *)&pp->s);
      }
    }
    __syncthreads();
    const int q = claim_e.x, s = claim_e.y;
    SW_CHECK(q < 0 || (s >= 0 && (int64_t)s < a.ndb));
    auto finish_ticket = [&]() {   // thread 0: this ticket is done with pair j's slot
      if (atomicAdd(&ctl->chunks_done[sl], 1) == kK2Span - 1) {
        ctl->chunks_done[sl] = 0;
        __threadfence();
        atomicAdd(&ctl->slot_done[sl], 1);
      }
    };
    if (q < 0) {   // no big pair left (every later ticket finds none too)
      if (L == 0) finish_ticket();
      break;
    }
    const int m = (int)(a.qoff[q + 1] - a.qoff[q]);
    const int len = a.sorted_len[s];
    const int ntile = (len + K2C - 1) / K2C;   // columns up to ntile*4 <= G.ncols are pad codes
    // rows per thread: fewer rows shorten a step's dependency chain (a block is
    // latency-bound), more rows mean fewer chunks, each adding a pipeline lag of ~nact steps
    const int R = m <= kK2Threads * 4 * 12 ? 4 : m <= kK2Threads * 8 * 16 ? 8 : 16;
    const int rc = kK2Threads * R;   // rows per chunk
    const int nch = (m + rc - 1) / rc;
    int best = 0;
    if (c < nch && len > 0) {
      const int r0 = c * rc;
      const int nact = (min(rc, m - r0) + R - 1) / R;
      const uint8_t *qc = a.qcodes + a.qoff[q];
      const GroupInfo G = a.groups[s / kGroup];
      SW_CHECK(nch <= kK2Span && R * kK2Threads >= (m + kK2Span - 1) / kK2Span);
      int2 *bi = c > 0 ? bbase + (size_t)(sl * kK2Span + c - 1) * a.border_stride : nullptr;
      int2 *bo = c < nch - 1 ? bbase + (size_t)(sl * kK2Span + c) * a.border_stride : nullptr;
      const long long *pi = c > 0 ? &ctl->prog[sl][c - 1] : nullptr;
      long long *po = c < nch - 1 ? &ctl->prog[sl][c] : nullptr;
      const long long ep = j + 1;
      if (R == 4)
        best = k2_chunk<4>(a, Ms, prof, hand, handc, ring, cring, qc, m, r0, nact, G, s % kGroup, ntile, bi, bo, pi, po, ep);
      else if (R == 8)
        best = k2_chunk<8>(a, Ms, prof, hand, handc, ring, cring, qc, m, r0, nact, G, s % kGroup, ntile, bi, bo, pi, po, ep);
      else
        best = k2_chunk<16>(a, Ms, prof, hand, handc, ring, cring, qc, m, r0, nact, G, s % kGroup, ntile, bi, bo, pi, po, ep);
    }
    const int b = block_max(best);
    if (L == 0) {
      if (c < nch) atomicMax(a.scores + (int64_t)q * a.ndb + a.perm[s], b);   // max over chunks
      finish_ticket();
    }
    __syncthreads();   // claim_s / claim_e / red_s reused
  }
  // ---- the other pairs: one block per pair, chunks in order
  int2 *border = reinterpret_cast<int2 *>(a.border) + (size_t)blockIdx.x * a.border_stride;
  constexpr int CH = kK2Threads * kK2RSmall;
  while (true) {
    if (L == 0) claim_s = k2_claim(a, a.ovf_cursor, count, false, claim_e);
    __syncthreads();
    const int p = claim_s;
    if (p >= count) break;
    const int q = claim_e.x, s = claim_e.y;
    const int m = (int)(a.qoff[q + 1] - a.qoff[q]);
    const int len = a.sorted_len[s];
    const int ntile = (len + K2C - 1) / K2C;
    const int nch = (m + CH - 1) / CH;
    int best = 0;
    for (int ch = 0; ch < nch && len > 0; ch++) {
      const int r0 = ch * CH;
      const int nact = min(kK2Threads, (m - r0 + kK2RSmall - 1) / kK2RSmall);   // threads with real rows
      best = max(best, k2_chunk<kK2RSmall>(a, Ms, prof, hand, handc, ring, cring, a.qcodes + a.qoff[q], m, r0, nact,
                                           a.groups[s / kGroup], s % kGroup, ntile, ch > 0 ? border : nullptr,
                                           ch < nch - 1 ? border : nullptr, nullptr, nullptr, 0));
    }
    const int b = block_max(best);
    if (L == 0) a.scores[(int64_t)q * a.ndb + a.perm[s]] = b;
    __syncthreads();   // claim_s / red_s reused by the next pair
  }
}

// a.ctl zeroed before the launch on its stream; a.border: k2_rows(blocks) rows
void launch_k2(const K2Args &a, int blocks, cudaStream_t st) {
  cudaFuncSetAttribute(k2_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kK2Smem);
  k2_kernel<<<blocks, kK2Threads, kK2Smem, st>>>(a);
}

// ------------------------------------------------------------------------------------
// K6: Phase 2 (P12 §II.A.2, NEXT-3): the optimal local alignment of selected pairs, in
// linear space.  One warp per pair, int32 DPX, the wavefront of K2/K3 (lane l owns rows
// [l*R, (l+1)*R) of each chunk of 32*R = 256 rows).
//   forward:   every chunk in order, score only; the bottom row (H, F) of each chunk is kept
//              as a checkpoint (nch * n * 8 bytes) and the highest cell is found (ties:
//              smallest row, then smallest column);
//   backtrack: the chunk holding the current cell is recomputed from the checkpoint above
//              it, for columns [0, j) only, storing one direction byte per cell (256 * n
//              bytes, reused): bits 0-1 = H source (0 zero, 1 diagonal, 2 E, 3 F), bit 2 = E
//              extends E(i,j-1), bit 3 = F extends F(i-1,j); lane 0 follows the arrows until
//              they leave the chunk (upwards: the chunk above is recomputed, the H/E/F state
//              carries over) or reach a zero, writing ops ('M', 'I', 'D') backwards.
// Work: <= 2x the cells (each chunk is recomputed at most once, and only left of j);
// memory: (nch * 8 + 256) bytes per database column instead of m bytes per column.
// ------------------------------------------------------------------------------------
constexpr int K6R = 8;
constexpr int K6CH = 32 * K6R;   // rows per chunk
static_assert(K6CH == kTbChunk, "host and kernel chunk heights");
constexpr int K6C = 4;   // columns per lane step: 4 independent skewed chains (a lane is latency-bound)
static_assert(kTbCols % K6C == 0 && kTbCols == 256, "column checkpoints at tile ends");
// One 256-row chunk of a pair, columns [cs, ce): forward (cs = 0, ce = n: score only; the
// chunk's bottom row as a checkpoint, every row's (H, E) after columns 255, 511, ... as column
// checkpoints, the highest cell) or backtrack recompute of one 256 x 256 tile (cs = a multiple
// of 256, ce <= cs + 256: state at cs - 1 from the column checkpoints; one direction byte per
// cell, [column - cs][256 rows]: a lane's 8 bytes of a column are one 8-byte store).  At step t
// lane l updates the K6C-column tile t - l, skewed like K2 (at sub-step k column g updates row
// k - g), and hands each column's bottom (H, F) and residue code to lane l+1 by shuffles.
// prog_in / prog_out (forward, several warps): shared-memory counters of the checkpoint
// columns the chunk above has written / this chunk has written (nullptr: in order on one warp)
__device__ __forceinline__ void tb_chunk(const TbArgs &a, const TbPair &T, const int32_t *Ms, const uint8_t *qc,
                                         const uint8_t *bytes, const GroupInfo &G, int gl, int ch, int cs, int ce,
                                         bool fwd, int &bv, int &bi, int &bj,
                                         const volatile int *prog_in = nullptr, volatile int *prog_out = nullptr) {
  constexpr int NEG = -(1 << 29);
  const int lane = threadIdx.x & 31;
  const int m = T.m, n = T.n;
  const int nch = (m + K6CH - 1) / K6CH;
  int2 *ckpt = reinterpret_cast<int2 *>(a.border) + T.ckpt_off;     // [nch - 1][n]
  int2 *colck = reinterpret_cast<int2 *>(a.border) + T.colck_off;   // [nblk - 1][nch * 256]
  const int rows_all = nch * K6CH;
  const int2 *top = ch > 0 ? ckpt + (size_t)(ch - 1) * n : nullptr;
  int2 *bottom = (fwd && ch < nch - 1) ? ckpt + (size_t)ch * n : nullptr;
  uint8_t *dir = a.dir + T.dir_off;   // [kTbCols][K6CH] (backtrack only)
  const int r_first = ch * K6CH + lane * K6R;   // this lane's first row (0-based)
  int qr[K6R];
#pragma unroll
  for (int i = 0; i < K6R; i++) {
    const int row = r_first + i;
    qr[i] = (row < m ? qc[row] : kPadCode) * 32;
  }
  int H[K6R], E[K6R];
  int hprev_top = 0;   // H(row above this lane's first row, cs - 1)
  if (cs == 0) {
#pragma unroll
    for (int i = 0; i < K6R; i++) { H[i] = 0; E[i] = NEG; }
  } else {
    const int2 *ck = colck + (size_t)(cs / kTbCols - 1) * rows_all;
#pragma unroll
    for (int i = 0; i < K6R; i++) { const int2 v = ck[r_first + i]; H[i] = v.x; E[i] = v.y; }
    hprev_top = lane > 0 ? ck[r_first - 1].x : (top ? __ldcg(top + cs - 1).x : 0);
  }
  int out_h[K6C], out_f[K6C], out_c[K6C];
#pragma unroll
  for (int g = 0; g < K6C; g++) { out_h[g] = 0; out_f[g] = NEG; out_c[g] = kPadCode; }
  // forward: per row the maximum and the first column reaching it (a row's columns come in
  // order), folded into (bv, bi, bj) at the end: the same (value desc, row asc, column asc)
  // rule as a per-cell comparison, in 3 instructions per cell instead of ~8
  int rmax[K6R], rcol[K6R];
#pragma unroll
  for (int i = 0; i < K6R; i++) { rmax[i] = 0; rcol[i] = 0; }
  const int ncols = ce - cs;
  const int ntile = (ncols + K6C - 1) / K6C;
  for (int t = 0; t < ntile + 31; t++) {
    int in_h[K6C], in_f[K6C], in_c[K6C];
#pragma unroll
    for (int g = 0; g < K6C; g++) {
      in_h[g] = __shfl_up_sync(0xffffffffu, out_h[g], 1);
      in_f[g] = __shfl_up_sync(0xffffffffu, out_f[g], 1);
      in_c[g] = __shfl_up_sync(0xffffffffu, out_c[g], 1);
    }
    if (lane == 0 && t < ntile) {
      if (top && prog_in) {   // the chunk above (another warp) has written these columns
        const int want = min(ce, cs + (t + 1) * K6C);
        const long long t_wait = clock64();
        while (*prog_in < want)
          if (clock64() - t_wait > (1ll << 36)) __trap();
        __threadfence_block();
      }
#pragma unroll
      for (int g = 0; g < K6C; g++) {
        const int col = cs + t * K6C + g;
        if (col < ce) {
          in_c[g] = bytes[(G.word_off + (int64_t)(col >> 4) * kGroup + gl) * 16 + (col & 15)];
          if (top) { const int2 v = __ldcg(top + col); in_h[g] = v.x; in_f[g] = v.y; }
          else { in_h[g] = 0; in_f[g] = NEG; }
        } else {
          in_c[g] = kPadCode; in_h[g] = 0; in_f[g] = NEG;
        }
      }
    }
    const int tile = t - lane;
    if (tile >= 0 && tile < ntile) {
      const int c0 = cs + tile * K6C;
      int hd[K6C], hup[K6C], f[K6C], oh[K6C];
      uint32_t db[K6C][2];
#pragma unroll
      for (int g = 0; g < K6C; g++) {
        hd[g] = g == 0 ? hprev_top : in_h[g - 1];   // H(row above, previous column)
        hup[g] = in_h[g];
        f[g] = in_f[g];
        oh[g] = 0;
        db[g][0] = db[g][1] = 0u;
      }
      hprev_top = in_h[K6C - 1];
#pragma unroll
      for (int k = 0; k < K6R + K6C - 1; k++) {
#pragma unroll
        for (int g = 0; g < K6C; g++) {
          const int i = k - g;
          if (i >= 0 && i < K6R) {
            const int row = r_first + i;   // 0-based query row
            const int col = c0 + g;
            const int eo = H[i] - a.alpha, ee = E[i] - a.beta;
            const int e = max(ee, eo);                     // E(i,j)
            const int fo = hup[g] - a.alpha, fe = f[g] - a.beta;
            f[g] = max(fe, fo);                            // F(i,j)
            const int dg = hd[g] + Ms[qr[i] + in_c[g]];    // diagonal
            const int h = __vimax3_s32(max(dg, 0), e, f[g]);   // H(i,j)
            if (fwd) {
              const bool up = h > rmax[i] && col < ce;   // rows past m are skipped at the end
              rcol[i] = up ? col : rcol[i];
              rmax[i] = up ? h : rmax[i];
            } else if (row < m && col < ce) {
              const int src = h == 0 ? 0 : h == dg ? 1 : h == e ? 2 : 3;
              db[g][i >> 2] |= (uint32_t)(src | ((ee > eo) << 2) | ((fe > fo) << 3)) << (8 * (i & 3));
            }
            hd[g] = H[i]; H[i] = h; E[i] = e; hup[g] = h;
            if (i == K6R - 1) oh[g] = h;
          }
        }
      }
#pragma unroll
      for (int g = 0; g < K6C; g++) {
        const int col = c0 + g;
        out_h[g] = oh[g]; out_f[g] = f[g]; out_c[g] = in_c[g];
        if (col < ce) {
          if (!fwd)
            *reinterpret_cast<uint2 *>(dir + (size_t)(col - cs) * K6CH + lane * K6R) = make_uint2(db[g][0], db[g][1]);
          if (lane == 31 && bottom) bottom[col] = make_int2(oh[g], f[g]);
        }
      }
      // forward: every row's (H, E) after the last column of a 256-column block
      if (fwd && (c0 + K6C) % kTbCols == 0 && c0 + K6C < n) {
        int2 *ck = colck + (size_t)((c0 + K6C) / kTbCols - 1) * rows_all + r_first;
#pragma unroll
        for (int i = 0; i < K6R; i++) ck[i] = make_int2(H[i], E[i]);
      }
      if (lane == 31 && bottom && prog_out) {
        __threadfence_block();   // the checkpoint columns before their count
        *prog_out = min(ce, c0 + K6C);
      }
    }
  }
  if (fwd)
#pragma unroll
    for (int i = 0; i < K6R; i++) {
      const int row = r_first + i;
      if (row < m && rmax[i] > 0 &&
          (rmax[i] > bv || (rmax[i] == bv && (row + 1 < bi || (row + 1 == bi && rcol[i] + 1 < bj))))) {
        bv = rmax[i]; bi = row + 1; bj = rcol[i] + 1;
      }
    }
}

constexpr int kTbWarps = 8;   // warps per pair in the forward pass (chunk ch on warp ch % 8)
__global__ void __launch_bounds__(kTbWarps * 32) traceback_kernel(const TbArgs a) {
  __shared__ int32_t Ms[kNCodes * 32];
  __shared__ int cprog[(SW_MAX_QUERY_LEN + K6CH) / K6CH];   // checkpoint columns written per chunk
  __shared__ int red_v[kTbWarps], red_i[kTbWarps], red_j[kTbWarps];
  for (int k = threadIdx.x; k < kNCodes * 32; k += blockDim.x) {
    const int r = k / 32, c = k % 32;   // query code, database slot
    Ms[k] = (r < 24 && c < 24) ? (int32_t)a.matrix[r * 24 + c_code_of_slot[c]] : kPadScore;
  }
  for (int k = threadIdx.x; k < (SW_MAX_QUERY_LEN + K6CH) / K6CH; k += blockDim.x) cprog[k] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const TbPair T = a.pairs[blockIdx.x];
  const int m = T.m, n = T.n;
  const uint8_t *qc = a.qcodes + T.q_off;
  const GroupInfo G = a.groups[T.sorted / kGroup];
  const int gl = T.sorted % kGroup;
  const uint8_t *bytes = reinterpret_cast<const uint8_t *>(a.packed);
  const int nch = (m + K6CH - 1) / K6CH;
  // forward pass: checkpoints + the highest cell.  Chunk ch runs on warp ch % kTbWarps and
  // follows chunk ch - 1 column by column through its checkpoint row (a wavefront across
  // warps, P14 §II.B); a warp's chunks wait only on earlier chunks, so no deadlock
  int bv = 0, bi = 0, bj = 0;   // best value and its 1-based cell (0,0 = empty alignment)
  for (int ch = warp; ch < nch; ch += kTbWarps)
    tb_chunk(a, T, Ms, qc, bytes, G, gl, ch, 0, n, true, bv, bi, bj, ch > 0 ? &cprog[ch - 1] : nullptr, &cprog[ch]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {   // warp reduction of (value desc, row asc, column asc)
    const int v2 = __shfl_xor_sync(0xffffffffu, bv, o), i2 = __shfl_xor_sync(0xffffffffu, bi, o),
              j2 = __shfl_xor_sync(0xffffffffu, bj, o);
    if (v2 > bv || (v2 == bv && (i2 < bi || (i2 == bi && j2 < bj)))) { bv = v2; bi = i2; bj = j2; }
  }
  if (lane == 0) { red_v[warp] = bv; red_i[warp] = bi; red_j[warp] = bj; }
  __syncthreads();   // also: every checkpoint row written before the backtrack reads it
  if (warp != 0) return;   // the backtrack follows one path: warp 0
  for (int w = 1; w < kTbWarps; w++) {
    const int v2 = red_v[w], i2 = red_i[w], j2 = red_j[w];
    if (v2 > bv || (v2 == bv && (i2 < bi || (i2 == bi && j2 < bj)))) { bv = v2; bi = i2; bj = j2; }
  }
  TbResult R;
  R.score = bv;
  int k = 0;
  char *ops_end = a.ops + T.ops_off + (m + n);   // ops written backwards from here
  int i = bi, j = bj, state = 0;                 // 0 = H, 1 = E, 2 = F
  bool stop = bv <= 0;
  const uint8_t *dir = a.dir + T.dir_off;
  int dummy_v = 0, dummy_i = 0, dummy_j = 0;
  while (!stop) {
    // recompute the 256 x 256 tile holding cell (i-1, j-1) (0-based): rows of its chunk,
    // columns [cs, j) from the column checkpoint at cs - 1 (forward pass)
    const int ch = (i - 1) / K6CH, row0 = ch * K6CH;
    const int cs = (j - 1) / kTbCols * kTbCols;
    __syncwarp();
    tb_chunk(a, T, Ms, qc, bytes, G, gl, ch, cs, j, false, dummy_v, dummy_i, dummy_j);
    __syncwarp();
    __threadfence_block();
    if (lane == 0) {
      while (i > 0 && j > 0 && i - 1 >= row0 && j - 1 >= cs) {
        const uint8_t b = dir[(size_t)(j - 1 - cs) * K6CH + (i - 1 - row0)];
        if (state == 0) {
          const int src = b & 3;
          if (src == 0) { stop = true; break; }
          if (src == 1) { *(--ops_end) = 'M'; k++; i--; j--; }
          else state = src == 2 ? 1 : 2;
        } else if (state == 1) {
          *(--ops_end) = 'D'; k++;
          state = (b >> 2) & 1 ? 1 : 0;
          j--;
        } else {
          *(--ops_end) = 'I'; k++;
          state = (b >> 3) & 1 ? 2 : 0;
          i--;
        }
      }
      if (i == 0 || j == 0) stop = true;
    }
    stop = __shfl_sync(0xffffffffu, (int)stop, 0);
    i = __shfl_sync(0xffffffffu, i, 0);
    j = __shfl_sync(0xffffffffu, j, 0);
    state = __shfl_sync(0xffffffffu, state, 0);
  }
  if (lane != 0) return;
  if (bv > 0) {
    R.q_begin = i; R.q_end = bi; R.d_begin = j; R.d_end = bj;
  } else {
    R.q_begin = R.q_end = R.d_begin = R.d_end = 0;
  }
  R.n_ops = k;
  a.results[blockIdx.x] = R;
}

void launch_traceback(const TbArgs &a, int n_pairs, cudaStream_t st) {
  if (n_pairs > 0) traceback_kernel<<<n_pairs, kTbWarps * 32, 0, st>>>(a);
}

// ------------------------------------------------------------------------------------
// helpers
// ------------------------------------------------------------------------------------
__global__ void fill_kernel(int32_t *p, int64_t n, int32_t v) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x)
    p[k] = v;
}
void launch_fill(int32_t *p, int64_t n, int32_t v, cudaStream_t st) {
  if (n > 0) fill_kernel<<<592, 256, 0, st>>>(p, n, v);
}
// ------------------------------------------------------------------------------------
// Segments of committed units (the cross-GPU data plane): a segment is query
// q x sorted sequences [s0, s1) of one committed unit; its pairs sit at scores[q][perm[s]]
// (original order) and at compact[off + s - s0] in a dense per-worker buffer.
//   mode 0: gather  matrix -> compact      (committing GPU, before the peer copy)
//   mode 1: scatter compact -> matrix      (device 0, after the peer copy)
//   mode 2: copy    matrix -> matrix       (multi-process: this rank's committed pairs only)
// ------------------------------------------------------------------------------------
__global__ void seg_copy_kernel(const int32_t *__restrict__ src, int32_t *__restrict__ dst, int64_t ndb,
                                const int32_t *__restrict__ perm, const SegInfo *__restrict__ segs, int mode) {
  const SegInfo g = segs[blockIdx.x];
  const int64_t row = (int64_t)g.q * ndb;
  for (int s = g.s0 + threadIdx.x; s < g.s1; s += blockDim.x) {
    const int64_t m = row + perm[s];
    const int64_t c = g.off + (s - g.s0);
    if (mode == 0) dst[c] = src[m];
    else if (mode == 1) dst[m] = src[c];
    else dst[m] = src[m];
  }
}
void launch_seg_copy(const int32_t *src, int32_t *dst, int64_t ndb, const int32_t *perm, const SegInfo *segs,
                     int nseg, int mode, cudaStream_t st) {
  if (nseg > 0) seg_copy_kernel<<<nseg, 256, 0, st>>>(src, dst, ndb, perm, segs, mode);
}

// ------------------------------------------------------------------------------------
// K5: top-k under (score desc, db_index asc) -- R13.  Keys are score << 32 | ~index (0 =
// empty), so one unsigned comparison orders both fields.  A block keeps one descending
// list per thread over a strided slice of its candidates (an insertion per candidate
// above the thread's k-th key, equal keys kept once), then warps merge their lanes' lists
// with shuffles and warp 0 merges the warps' lists.
//   K5u  unit_topk_kernel:  one block per query of a committed unit's pack, candidates =
//        that query's pairs in the unit (scores[q][perm[s]], s in [s0, s1)), on the unit's
//        stream right after it (and after the int32 re-run of what it saturated);
//   K5m  merge_topk_kernel: one block per query, candidates = the hits of several lists
//        (a worker's committed units, then the workers / ranks): the paper's "merges" (P16).
// ------------------------------------------------------------------------------------
constexpr int kTopkMax = 64;
__device__ __forceinline__ uint64_t xor64(uint64_t v, int o) {
  uint32_t lo = __shfl_xor_sync(0xffffffffu, (uint32_t)v, o);
  uint32_t hi = __shfl_xor_sync(0xffffffffu, (uint32_t)(v >> 32), o);
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ uint64_t hit_key(int score, int idx) {
  return (idx < 0 || score < 0) ? 0ull : (((uint64_t)(uint32_t)score << 32) | (uint32_t)(~(uint32_t)idx));
}
// warp merge: each lane holds a descending list (len k, 0 = empty); lane 0 gets the merged
// top-k in out[0..k).  A key held by several lanes is emitted once.
__device__ void warp_merge(const uint64_t *list, int k, uint64_t *out) {
  const int lane = threadIdx.x & 31;
  int head = 0;
  for (int r = 0; r < k; r++) {
    uint64_t mine = head < k ? list[head] : 0ull;
    uint64_t m = mine;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) { uint64_t v = xor64(m, o); m = v > m ? v : m; }
    if (m != 0ull && mine == m) head++;
    if (lane == 0) out[r] = m;
  }
}
template <int NT, class KeyOf>
__device__ void block_topk(KeyOf key_of, int64_t n, int k, int2 *out) {
  __shared__ uint64_t wl[NT / 32][kTopkMax];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t list[kTopkMax];
  for (int i = 0; i < k; i++) list[i] = 0ull;
  uint64_t kth = 0ull;
  for (int64_t d = threadIdx.x; d < n; d += NT) {
    const uint64_t key = key_of(d);
    if (key <= kth) continue;
    int pos = k - 1;
    while (pos > 0 && list[pos - 1] < key) pos--;
    if (pos > 0 && list[pos - 1] == key) continue;   // already held
    for (int i = k - 1; i > pos; i--) list[i] = list[i - 1];
    list[pos] = key;
    kth = list[k - 1];
  }
  uint64_t merged[kTopkMax];
  warp_merge(list, k, merged);
  if (lane == 0)
    for (int i = 0; i < k; i++) wl[warp][i] = merged[i];
  __syncthreads();
  if (warp == 0) {
    uint64_t l2[kTopkMax];
    for (int i = 0; i < k; i++) l2[i] = lane < NT / 32 ? wl[lane][i] : 0ull;
    uint64_t fin[kTopkMax];
    warp_merge(l2, k, fin);
    if (lane == 0)
      for (int i = 0; i < k; i++) {
        const uint64_t v = fin[i];
        out[i] = v ? make_int2((int)(v >> 32), (int)(~(uint32_t)v)) : make_int2(0, -1);
      }
  }
}

__global__ void __launch_bounds__(1024) topk_kernel(const int32_t *__restrict__ scores, int64_t ndb,
                                                    int k, int2 *__restrict__ hits) {
  const int32_t *row = scores + (int64_t)blockIdx.x * ndb;
  block_topk<1024>([&](int64_t d) { return hit_key(row[d], (int)d); }, ndb, k, hits + (int64_t)blockIdx.x * k);
}
void launch_topk(const int32_t *scores, int32_t nq, int64_t ndb, int32_t k, int2 *hits, cudaStream_t st) {
  if (nq <= 0 || k <= 0) return;
  topk_kernel<<<nq, 1024, 0, st>>>(scores, ndb, k, hits);
}

__global__ void __launch_bounds__(256) unit_topk_kernel(const int32_t *__restrict__ scores, int64_t ndb,
                                                        const int32_t *__restrict__ perm, int32_t s0, int32_t s1,
                                                        const int32_t *__restrict__ queries, int k,
                                                        int2 *__restrict__ out) {
  const int q = queries[blockIdx.x];
  const int32_t *row = scores + (int64_t)q * ndb;
  block_topk<256>([&](int64_t d) {
        const int o = perm[s0 + (int)d];
        return hit_key(row[o], o);
      }, (int64_t)(s1 - s0), k, out + (int64_t)blockIdx.x * k);
}
void launch_unit_topk(const int32_t *scores, int64_t ndb, const int32_t *perm, int32_t s0, int32_t s1,
                      const int32_t *queries, int nqp, int k, int2 *out, cudaStream_t st) {
  if (nqp <= 0 || k <= 0) return;
  unit_topk_kernel<<<nqp, 256, 0, st>>>(scores, ndb, perm, s0, s1, queries, k, out);
}

__global__ void __launch_bounds__(256) merge_topk_kernel(const int2 *__restrict__ lists, int k_in,
                                                         const int32_t *__restrict__ list_off,
                                                         const int32_t *__restrict__ list_idx, int k,
                                                         int2 *__restrict__ out) {
  const int q = blockIdx.x;
  const int32_t j0 = list_off[q], nl = list_off[q + 1] - j0;
  block_topk<256>([&](int64_t d) {
        const int l = (int)(d / k_in), r = (int)(d - (int64_t)l * k_in);
        const int2 h = lists[(int64_t)list_idx[j0 + l] * k_in + r];
        return hit_key(h.x, h.y);
      }, (int64_t)nl * k_in, k, out + (int64_t)q * k);
}
void launch_merge_topk(const int2 *lists, int k_in, const int32_t *list_off, const int32_t *list_idx, int nq,
                       int k, int2 *out, cudaStream_t st) {
  if (nq <= 0 || k <= 0) return;
  merge_topk_kernel<<<nq, 256, 0, st>>>(lists, k_in, list_off, list_idx, k, out);
}

}  // namespace sw
