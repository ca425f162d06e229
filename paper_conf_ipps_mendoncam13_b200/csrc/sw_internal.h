// sw_internal.h — internal declarations shared by libsw's host runtime and kernels.
// (Nothing here is shared with oracle/: the product path has its own alphabet table,
// BLOSUM62 transcription and arithmetic.)
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include <stdexcept>
#include <string>
#include <vector>

namespace sw {

// internal exception carrying an SW_E* code; converted to a return code at the C-ABI
struct Error : std::runtime_error {
  int code;
  Error(int c, const std::string &m) : std::runtime_error(m), code(c) {}
};

// ---- alphabet / scoring constants -------------------------------------------------
constexpr int kNCodes = 25;        // 24 NCBI letters ARNDCQEGHILKMFPSTWYVBZX* + pad
constexpr int kPadCode = 24;       // packing pad (DB columns beyond a sequence's end)
constexpr int kPadScore = -1;      // S[.][pad] and pad query rows: <= 0 (reading R9)
// Database residues are stored in the packed database as "slots", a permutation of the
// codes: the K1 profile is read two rows per LDS.64 with a row stride of 65 8-byte words,
// so the bank pair a lane hits is slot mod 16.  The 16 most frequent amino acids (Swiss-Prot
// composition) get slots 0..15, one bank pair each; M H C W B Z X * share bank pairs with
// the 8 least frequent of them (slots 16..23); the pad code keeps slot 24.  Profiles, the
// K2/K6 matrices and the K3 profile are indexed by slot; query rows stay codes.
//                                     slot: 0  1  2 3  4  5 6 7  8 9 10 11 12 13 14 15 16 17 18 19 20 21 22 23 24
#define SW_CODE_OF_SLOT_INIT            {18,13,5,2,14,16,3,1,10,0, 7,19, 6,15, 9,11,12, 8, 4,17,20,21,22,23,24}
constexpr int kOff = 128;          // offset representation bias of the s16x2 kernels
                                   // (>= -min int8 score so 32-bit adds never borrow)
constexpr int kWordCols = 16;      // residues per packed 128-bit word
constexpr int kGroup = 32;         // DB sequences per packing group (one per lane)

// K1 (inter-task) geometry: W warps per block split each band of W*K rows
constexpr int kK1Rows = 16;        // K: rows per warp (registers H[K], E[K])
constexpr int kK1Warps = 8;        // W
constexpr int kK1Tile = 8;         // T: columns per pipeline step
constexpr int kK1Band = kK1Rows * kK1Warps;
// K3 (intra-task) geometry: one warp per (query pair, long DB sequence)
constexpr int kK3Rows = 16;        // rows per lane
constexpr int kK3Chunk = 32 * kK3Rows;   // rows per warp chunk
constexpr int kK3Warps = 4;        // long sequences per block (share the chunk profile)
constexpr int kK3UnitSeqs = 148 * kK3Warps;   // long sequences that give each B200 SM one K3 block
constexpr int kProfileRowAlign = 512;    // lcm(kK1Band, kK3Chunk)

// ---- packed database (device) -------------------------------------------------------
struct GroupInfo {       // one packing group of up to 32 length-sorted sequences
  int64_t word_off;      // offset (in uint4 words) of word 0, lane 0
  int32_t ncols;         // padded columns (multiple of kColAlign, >= kMinCols)
  int32_t first;         // index of the group's first sequence in sorted order
  int32_t count;         // real sequences in the group (<= 32)
  int32_t pad_;
};
constexpr int kColAlign = 8;       // group columns rounded to one K1 tile
constexpr int kWideCols = 144;     // groups this wide run the 16-column-step K1 instance
constexpr int kMinCols = 80;       // groups padded to >= (W+1)*T columns (rounded to 16): the K1 pipeline
                                   // prefetches warp 0's border one step ahead

// ---- a unit of work (one task of the paper's scheduler) -----------------------------
enum UnitKind : int32_t { kUnitInter = 0, kUnitIntra = 1 };
struct Unit {
  int32_t kind;
  int32_t pair;          // query pair index
  int32_t b0, b1;        // group range [b0,b1) (inter) or long-seq range (intra)
  int64_t cells;         // real cells (sum |q|*|d|), for GCUPS and PSS rates
  int64_t work;          // padded lane-cells (balancing)
  int32_t cluster = 1;   // K3: CTAs per thread-block cluster splitting each pair's chunks
  int32_t npk = 1;       // packs [pair, pair + npk) (> 1 only for clustered K3 units)
};

// ---- query packs ------------------------------------------------------------------------
// The s16x2 kernels run two query "halves" per 32-bit lane word.  A pack fills each half
// with a run of queries, every query starting on a 16-row slice boundary (16 = the rows of
// one K1 warp / one K3 lane), so a short query does not leave the other half idle.  At a
// slice that starts a query the producer of the row above hands down H = F = 0 for that
// half, and a warp (K1) or lane (K3) flushes its running maximum of a half whenever the
// query of its slice changes (atomicMax into the score matrix).
struct SliceInfo {       // 16 consecutive pack rows
  int32_t q_lo, off_lo;  // query of the low half (-1 none) and the row of that query at the
  int32_t q_hi, off_hi;  // slice's first row (0 = the slice starts the query)
};
struct QueryPair {       // a pack
  int32_t rows;          // rows to compute: the longer half (16-aligned)
  int32_t rows_padded;   // profile rows (multiple of kProfileRowAlign)
  int64_t prof_off;      // offset (in int32) of this pack's profile [kNCodes][rows_padded]
  int32_t slice_off;     // first SliceInfo of the pack (rows_padded / 16 entries)
  int32_t pad_;
};

// ---- kernel launchers (kernels.cu) -------------------------------------------------------
struct K1Args {
  const uint4 *packed; const GroupInfo *groups; const int32_t *perm;
  const int32_t *prof; const QueryPair *pairs; const SliceInfo *slices;
  int32_t pair; int32_t g0;          // unit: pack, first group
  int32_t n_groups;                  // groups [g0, g0 + n_groups) (set by launch_k1)
  int32_t *scores; int64_t ndb;      // [nq][ndb]
  int32_t thresh;                    // overflow threshold on best~ (offset repr)
  int2 *ovf; int32_t *ovf_count; int32_t ovf_cap; uint32_t *ovf_bits;
  int32_t *ovf_early;                // host-mapped: entries listed so far (early K2 launch)
  uint2 *border; int32_t border_slot_cols; int32_t slots_per_sm; int32_t *slot_busy;
  const volatile int32_t *abort_flag; // WA cancellation flag of the unit (polled in the loop)
  int32_t *progress;                 // unit's counter: groups completed (atomicAdd per block)
  int32_t *gclaim;                   // unit's counter: groups claimed by its blocks (zeroed)
  uint32_t na, nb;                   // packed -alpha, -beta
};
struct K3Args {   // sequences [l0,l1) in sorted order (the long groups) x packs [pair, pair + npk)
  const uint4 *packed; const GroupInfo *groups; const int32_t *perm; const int32_t *sorted_len;
  const int32_t *prof; const QueryPair *pairs; const SliceInfo *slices;
  int32_t pair; int32_t npk; int32_t l0, l1;
  int32_t *scores; int64_t ndb;
  int32_t thresh;
  int2 *ovf; int32_t *ovf_count; int32_t ovf_cap; uint32_t *ovf_bits;
  int32_t *ovf_early;                // host-mapped: entries listed so far (early K2 launch)
  uint2 *border; int64_t border_stride;   // border rows (>= max long len): per sequence (C = 1)
                                          // or per (grid slot, buffer) (cluster C > 1)
  int64_t border_rows;                    // rows allocated (checked build)
  int32_t *kprog;                         // C > 1: per (grid slot, buffer) progress counters (zeroed)
  int32_t *claim;                         // C > 1: sequence blocks claimed so far (zeroed)
  int32_t pub_every;                      // C > 1: tiles between progress publications
  const volatile int32_t *abort_flag;     // WA cancellation flag (polled at chunk starts)
  int32_t *progress;                      // unit's counter: (sequence, chunk) pairs completed
  uint32_t na, nb;
};
constexpr int kMaxStreams = 64;    // sw_opts.streams_per_device limit
constexpr int kK2Blocks = 32;      // K2 blocks per launch (a search routed to int32: 3 per SM)
constexpr int kK2Threads = 128;    // K2 block size (the size of a K3 block)
constexpr int kK2Span = 32;        // chunk tickets per big saturated pair (at most kK2Span chunks)
// K2 border rows per stream: one per block (single-block pairs), then 2 x kK2Span (big pairs)
inline int k2_rows(int blocks) { return blocks + 2 * kK2Span; }
struct K2Pair { int32_t tag, q, s, pad; };   // a published big pair (tag = pair number + 1)
struct K2Ctl {                     // per stream, zeroed before each K2 launch
  int32_t tickets;                 // chunk tickets taken: ticket t = chunk t % kK2Span of big pair t / kK2Span
  int32_t chunks_done[2];          // per pair slot (pair % 2): tickets of its current pair finished
  int32_t slot_done[2];            // per pair slot: pairs finished in it
  int32_t pad[3];
  long long prog[2][kK2Span];      // per pair slot and chunk: (pair + 1) << 32 | tiles published
  K2Pair pairs[8];                 // ring of published pairs (pair % 8)
};
struct K2Args {   // int32 re-run of saturated pairs (block per pair)
  const uint8_t *qcodes; const int64_t *qoff;
  const uint4 *packed; const GroupInfo *groups; const int32_t *sorted_len; const int32_t *perm;
  const int8_t *matrix;                   // 24x24 (device)
  const int2 *ovf; const int32_t *ovf_count; int32_t ovf_cap;
  int32_t *ovf_cursor;                    // [2]: small / big pairs, taken with atomicCAS
  int64_t big_cells;                      // m*n at which a pair is split over a cluster
  int32_t *scores; int64_t ndb;
  int32_t alpha, beta;
  int32_t one;                              // = 1 (opaque to the compiler, see k2_kernel)
  int32_t *border; int64_t border_stride;   // border rows (2 x int32 per column): one per block,
                                            // then 2 x kK2Span for the big pairs' pair slots
  struct K2Ctl *ctl;                        // big pairs' tickets and slots, zeroed per launch
};

struct TbPair {     // one pair of a traceback batch
  int32_t m, n;      // query and database lengths
  int64_t q_off;     // query codes offset
  int32_t sorted;    // database sequence (sorted order)
  int32_t pad_;
  int64_t dir_off;   // direction bytes of one 256 x 256 tile offset in the batch buffer
  int64_t ops_off;   // ops area (m+n bytes) offset in the batch buffer
  int64_t ckpt_off;  // chunk checkpoints ((nch - 1) * n int2) offset in the batch buffer
  int64_t colck_off; // column checkpoints ((nblk - 1) * nch * 256 int2, nblk = ceil(n / 256)):
                     // (H, E) of every row after columns 255, 511, ... (same buffer as ckpt)
};
constexpr int kTbCols = 256;    // K6 backtrack tile width (column checkpoint spacing)
struct TbResult { int32_t score, q_begin, q_end, d_begin, d_end, n_ops; };
struct TbArgs {
  const uint8_t *qcodes; const uint4 *packed; const GroupInfo *groups; const int8_t *matrix;
  const TbPair *pairs; uint8_t *dir; char *ops; TbResult *results;
  int32_t *border;   // checkpoint rows (int2 (H, F) per column), per pair at TbPair::ckpt_off
  int32_t alpha, beta;
};
constexpr int kTbChunk = 256;   // K6 rows per chunk (32 lanes x 8)
void launch_traceback(const TbArgs &a, int n_pairs, cudaStream_t st);

void launch_profile(const uint8_t *qcodes, const int64_t *qoff, const QueryPair *pairs, int npairs,
                    const SliceInfo *slices, const int8_t *matrix, int32_t *prof, int64_t prof_total,
                    cudaStream_t st);
void launch_k1(const K1Args &a, int n_groups, int min_cols, int rows_padded, cudaStream_t st,
               int n_sm);
void launch_k3(const K3Args &a, int cluster, int max_blocks, cudaStream_t st);
void launch_k2(const K2Args &a, int blocks, cudaStream_t st);
void launch_fill(int32_t *p, int64_t n, int32_t v, cudaStream_t st);
// committed-unit segments (cross-GPU data plane): query q x sorted sequences [s0, s1)
struct SegInfo { int32_t q, s0, s1, pad_; int64_t off; };
void launch_seg_copy(const int32_t *src, int32_t *dst, int64_t ndb, const int32_t *perm, const SegInfo *segs,
                     int nseg, int mode, cudaStream_t st);   // 0 gather, 1 scatter, 2 copy
void launch_topk(const int32_t *scores, int32_t nq, int64_t ndb, int32_t k, int2 *hits,
                 cudaStream_t st);
// K5u: top-k of one committed unit, per query of its pack -> out[nqp][k]
void launch_unit_topk(const int32_t *scores, int64_t ndb, const int32_t *perm, int32_t s0, int32_t s1,
                      const int32_t *queries, int nqp, int k, int2 *out, cudaStream_t st);
// K5m: per query q, merge lists list_idx[list_off[q] .. list_off[q+1]) (k_in hits each)
void launch_merge_topk(const int2 *lists, int k_in, const int32_t *list_off, const int32_t *list_idx, int nq,
                       int k, int2 *out, cudaStream_t st);
int k1_blocks_per_sm();
int k3_blocks_per_sm();
// local-load kernel: n_blocks SM-filling blocks spinning until *stop != 0 (or max_ns)
void launch_noise(const int32_t *stop, int n_blocks, uint64_t max_ns, uint32_t *sink, cudaStream_t st);
int k1_band_rows();   // rows per K1 band (W*K of the selected variant)

// ---- host packing (pack.cpp) ----------------------------------------------------------------
int encode_residue(int ascii);   // -1 if invalid
const int8_t *blosum62();        // libsw's own transcription (24x24)

struct PackedDB {
  int32_t n = 0;
  int64_t residues = 0;
  std::vector<int32_t> perm;         // sorted order -> original index
  std::vector<int32_t> sorted_len;   // lengths in sorted order (descending)
  std::vector<GroupInfo> groups;     // groups of 32 consecutive sorted sequences
  std::vector<uint4> packed;         // interleaved words
  int32_t max_len = 0;
};
// Encode (strict alphabet), sort by length (descending, stable), group and interleave.
// Returns 0 or an SW_E* code with the message in err.
int pack_database(const int64_t *offsets, const char *residues, int32_t n, PackedDB &out,
                  std::string &err);

}  // namespace sw
