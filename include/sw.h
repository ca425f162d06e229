/*
 * sw.h — C-ABI of libsw: score-only Smith-Waterman/Gotoh protein database search on
 * B200 (sm_100a), scheduled over 1..8 GPUs with the paper's PSS policy and workload
 * adjustment (WA).
 *
 * Paper: Mendonca & Melo, "Biological Sequence Comparison on Hybrid Platforms with
 * Dynamic Workload Adjustment", IPDPSW 2013 (PAPER.md; "P<n>" = line n, one PDF page).
 *
 *   The problem (P14 §II.B): "a set of x query sequences (q 1,q 2,...,q x ) will be
 *   compared to a set of y database sequences (d 1,d 2,...,d y )" (x << y); the user
 *   provides query and database (P16 §IV) and the allocation policy (P18 §IV.A); the
 *   master "merges" the slaves' results (P16 §IV).
 *
 *   Every (query, database sequence) score is the Smith-Waterman local-alignment score
 *   (P12 §II.A.1, Eq. 1, zero first row/column) with Gotoh's affine gaps (P12 §II.A.3,
 *   "3 Dynamic Programming (DP) matrices: H, E and F"), i.e. with alpha = open + extend,
 *   beta = extend:
 *     E(i,j) = max(E(i,j-1) - beta, H(i,j-1) - alpha)
 *     F(i,j) = max(F(i-1,j) - beta, H(i-1,j) - alpha)
 *     H(i,j) = max(0, H(i-1,j-1) + S[q_i][d_j], E(i,j), F(i,j)),   score = max H.
 *   A gap of length L costs gap_open + L*gap_extend (reading R3).
 *
 * Residues: ASCII letters of the NCBI protein alphabet ARNDCQEGHILKMFPSTWYVBZX*
 * (case-insensitive); the substitution matrix is 24x24 int8 in that order with the
 * QUERY residue as the row.  NULL matrix = BLOSUM62 (reading R1), the default gaps
 * are open 10 / extend 2 (reading R2).
 *
 * Errors: every int-returning entry point returns SW_OK (0) or a negative SW_E* code;
 * sw_last_error() then returns a thread-local message valid until the next call on
 * that thread.  No entry point aborts the process.  There is no CPU fallback: without
 * a usable CUDA device the search entry points return SW_ECUDA.
 *
 * Ownership: inputs are borrowed for the duration of a call (sw_db_create copies what
 * it needs); outputs are caller-allocated; a sw_db owns its device memory until
 * sw_db_destroy.  One sw_search per sw_db at a time (SW_EBUSY otherwise).
 */
#ifndef SW_H
#define SW_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum {
  SW_OK = 0,
  SW_EINVAL = -1,   /* bad argument (message says which) */
  SW_ERESIDUE = -2, /* letter outside the alphabet (message names the sequence index) */
  SW_ENOMEM = -3,   /* host or device allocation failed */
  SW_ECUDA = -4,    /* CUDA error or no device */
  SW_ENET = -5,     /* multi-process control-plane error (TCP master/worker) */
  SW_EBUSY = -6     /* a search is already running on this sw_db */
};

/* Limits (checked; SW_EINVAL beyond them).  The s16x2 kernels keep a query row index in 16
 * bits of their slice tables, and K5's per-thread lists hold at most 64 hits. */
#define SW_MAX_QUERY_LEN 65535 /* residues per query */
#define SW_MAX_TOP_K 64        /* hits per query */

/* Slower-PE emulation for the workload-adjustment experiments (P24 §V.C
 * "introduced local load"), applied to the workers in sw_opts.straggler_mask from
 * straggler_after_ms on, with factor straggler_slowdown (s): */
enum {
  SW_STRAGGLER_HOLD = 0,   /* host-side: each completion is held back (s-1) x the unit's device
                              time (the GPU itself runs at full speed) */
  SW_STRAGGLER_SM_CAP = 1, /* GPU-side (default): the worker's DP kernels together get
                              ceil(n_SM / s) SMs' worth of resident blocks (split over its
                              streams; persistent grids), so its GPU really runs ~s x slower */
  SW_STRAGGLER_NOISE = 2   /* GPU-side local load: a high-priority kernel occupies all but
                              ceil(n_SM / s) SMs of the worker's GPU (one SM-filling block each)
                              until the worker's last unit ends */
};

/* Task allocation policies (P18 §IV.A). */
enum {
  SW_POLICY_SS = 0, /* Self-Scheduling: Allocate(N, p_i) = 1 (P18 §IV.A.1) */
  SW_POLICY_PSS = 1 /* Package Weighted Adaptive Self-Scheduling, Eq. 2 (P18 §IV.A.2);
                       the paper's default ("The PSS policy was used in all the tests", P20) */
};

/* The paper's indexed sequence format (P20 §IV.B: "the total number of sequences, the
 * size of the biggest sequence and the offset that marks the beginning of each
 * sequence").  Sequence k is residues[offsets[k] .. offsets[k+1]). */
typedef struct {
  int32_t n;              /* number of sequences, >= 0 */
  const int64_t *offsets; /* n+1 entries, offsets[0] = 0, non-decreasing (host memory) */
  const char *residues;   /* ASCII residues (host memory), offsets[n] bytes */
  int32_t max_len;        /* optional hint ("size of the biggest sequence"); 0 = compute */
} sw_seqset;

/* One top-k hit: score and ORIGINAL database index; {0, -1} marks an empty slot. */
typedef struct {
  int32_t score;
  int32_t db_index;
} sw_hit;

typedef struct {
  int32_t policy;            /* SW_POLICY_SS | SW_POLICY_PSS (default PSS) */
  int32_t workload_adjust;   /* 1 = WA on (default, P20 "always activated"), 0 = off */
  int32_t omega;             /* PSS history length (Omega, P18 §IV.A.2); default 4 (reading R10) */
  int32_t streams_per_device;/* units in flight per GPU (default 4, at most 64) */
  int64_t target_unit_cells; /* cells per work unit; 0 = auto; INT64_MAX = one unit per
                                query pair and kernel kind (the paper's very coarse
                                "comparison of one query sequence to one genomic database",
                                P16 §IV) */
  int32_t long_threshold;    /* DB sequences longer than this go to the intra-task
                                (warp wavefront) kernel; 0 = auto (3072), <0 = never */
  int32_t outputs_on_device; /* 1: `scores` / `hits` are device pointers on the first
                                device of the sw_db (inputs-resident timing mode) */
  uint64_t straggler_mask;   /* experiments: worker w emulates a slower PE if bit w is set
                                (how: straggler_mode; SURVEY §8(d) WA experiment, P24 §V.C) */
  int32_t straggler_slowdown;/* slowdown factor (default 6, Fig. 5's GPU:SSE ratio) */
  /* multi-process mode (one process per GPU, torchrun): world > 1 makes every rank a
     worker of one master, run as a thread of rank 0 and reached over TCP */
  int32_t dist_rank;
  int32_t dist_world;        /* 0/1 = single process (in-process master) */
  int32_t dist_port;         /* TCP port of the master (on dist_host) */
  const char *dist_host;     /* master address, e.g. "127.0.0.1" */
  int32_t straggler_after_ms;/* the straggler slows down only after this many ms (local
                                load introduced mid-run, P24 §V.C); 0 = from the start */
  int32_t straggler_mode;    /* SW_STRAGGLER_* (default SW_STRAGGLER_SM_CAP) */
  int32_t worker_sms;        /* experiments: > 0 makes several workers sharing one GPU behave like
                                separate smaller GPUs.  Each worker gets a green-context SM
                                partition of worker_sms rounded down to a multiple of 8 (its
                                kernels run on those SMs only) when the device splits into
                                enough of them; otherwise its DP kernels are capped to worker_sms
                                SMs' worth of resident blocks (split over its streams).  A
                                straggler (SW_STRAGGLER_SM_CAP) then gets ceil(SMs / s).  See
                                sw_stats.partition_mode.  0 = no partition (default) */
  int32_t reserved[5];
} sw_opts;

typedef struct {
  int64_t cells;            /* sum over (query, db) pairs of |q|*|d| (real residues; each
                               pair once even when WA duplicated it) */
  double seconds_device;    /* whole-box device time: max over GPUs of their last event
                               minus the common start (host barrier, then start events) */
  double seconds_wall;      /* host wall clock of the same span */
  double gcups;             /* cells / seconds_device / 1e9 */
  int64_t duplicated_cells; /* cells of WA replicas that lost the race (wasted work) */
  int32_t n_units;          /* work units in the plan */
  int32_t n_overflow_pairs; /* pairs re-scored by the int32 kernel after saturation */
  int32_t n_wa_grants;      /* duplicates granted by workload adjustment */
  int32_t n_requests;       /* task-request messages to the master (an idle worker's request
                               waits at the master: one message, not a poll loop) */
  int32_t kernel_launches;  /* CUDA kernels launched by this process for the search */
  int32_t n_devices;        /* devices (in-process) or 1 (per rank) */
  double kernel_seconds_k1; /* summed device time of the inter-task kernel launches */
  double kernel_seconds_k3; /* summed device time of the intra-task kernel launches */
  int64_t cells_k1;         /* real cells computed by inter-task launches (incl. duplicates) */
  int64_t cells_k3;         /* real cells computed by intra-task launches (incl. duplicates) */
  double tail_seconds;      /* tail: the last worker's last unit completion minus the (lower)
                               median over workers of their last unit completion (device clocks,
                               each worker's own start event after a common host barrier) */
  const char *unit_log_json;/* per-replica log: unit, kind, pack, worker, stream, host times
                               (t_grant, t_start, t_end), device times (dev_t0, dev_t1 ms since
                               the worker's start; device_ms), cells, cells_done, committed,
                               cancelled, slowed; owned by the sw_db, valid until its next search */
  int32_t n_grant_messages; /* request messages that granted at least one task */
  int32_t n_cancelled;      /* WA replicas stopped early by their abort flag */
  double seconds_last_unit; /* device time of this process's last unit completion (for the
                               cross-rank tail in multi-process mode) */
  int64_t peer_bytes;       /* bytes copied between GPUs by the in-process merge */
  const char *sched_log_json;/* the master's event log with Φ and v̄ per grant (sw_sched.h);
                               in-process, or rank 0 in multi-process mode; owned by the sw_db */
  double kernel_seconds_k2; /* summed device time of the int32 re-run launches (K2), from the
                               launch being enqueued on its stream to its end (includes the
                               wait for free SMs behind the DP kernels) */
  int32_t n_k2_launches;    /* int32 re-run launches */
  int32_t partition_mode;   /* emulated GPUs (sw_opts.worker_sms > 0): 2 = each worker on its own
                               green-context SM partition, 1 = CTA caps (its blocks share SMs
                               with other workers'), 0 = off */
  int32_t partition_sms;    /* SMs per emulated GPU (mode 2: the partition's, a multiple of 8) */
} sw_stats;

typedef struct sw_db sw_db; /* opaque: host index + packed replica on each device */

/* Default options (PSS, WA on, Omega 4, auto unit size, auto long threshold). */
void sw_opts_default(sw_opts *opts);

/* Validate and encode `db`, sort by length, pack into interleaved warp groups and
 * upload one replica to each of devices[0..n_devices) (NULL / 0 devices = device 0).
 * The packed layout is DESIGN.md §5.  Returns SW_OK and *out, or an error. */
int sw_db_create(const sw_seqset *db, const int *devices, int n_devices, sw_db **out);

void sw_db_destroy(sw_db *db);

/* Number of sequences, residues and devices of a database (for the binding). */
int64_t sw_db_residues(const sw_db *db);
int32_t sw_db_size(const sw_db *db);
int32_t sw_db_devices(const sw_db *db);

/* Compare every query with every database sequence.
 *   queries     at most SW_MAX_QUERY_LEN residues each
 *   matrix      24x24 int8, row-major, query residue = row; NULL = BLOSUM62
 *   gap_open, gap_extend  >= 0, gap_open + 2*gap_extend <= 2^20
 *   top_k       0 .. SW_MAX_TOP_K hits per query under (score desc, db_index asc)
 *   scores      [nq][ndb] int32 in the ORIGINAL orders, or NULL
 *   hits        [nq][top_k] sw_hit, or NULL
 *   (host pointers, or device pointers on the sw_db's first device when
 *    opts->outputs_on_device)
 * Data plane (P16 §IV "the slaves send their results to the master, that merges them"):
 * every committed work unit's top-k is computed on its GPU right after it (K5u); each GPU
 * merges the lists of the units it committed (K5m).  In-process with several GPUs, the
 * other GPUs' committed scores (dense, only their units) and top-k lists are copied to the
 * first GPU over NVLink and merged there -- no full-matrix transfer or reduction.
 * In multi-process mode every rank passes the same inputs; each rank's `scores` then
 * holds exactly the pairs of the units it committed (others = -1: the ranks' slices are
 * disjoint) and `hits` the top-k over those; the binding all-gathers the hits (NCCL,
 * nq*top_k*8 bytes per rank) and merges them with sw_merge_hits.
 * Results are bit-identical for every GPU count, policy and WA setting. */
int sw_search(const sw_seqset *queries, sw_db *db, const int8_t *matrix, int32_t gap_open,
              int32_t gap_extend, int32_t top_k, int32_t *scores, sw_hit *hits,
              const sw_opts *opts, sw_stats *stats);

/* Top-k of a device score matrix [nq][ndb] (entries < 0 are ignored) on the sw_db's
 * first device, hits into device memory [nq][top_k].  Used by the binding to finish a
 * cross-rank reduction.  */
int sw_topk_device(sw_db *db, const int32_t *scores_dev, int32_t nq, int32_t ndb, int32_t top_k,
                   sw_hit *hits_dev);

/* Merge per-source top-k lists into the global top-k (the master's merge, P16 §IV).
 *   lists_dev  [n_sources][nq][k_in] sw_hit on the sw_db's first device ({x, -1} = empty)
 *   hits_dev   [nq][top_k] sw_hit, device memory
 * Order (score desc, db_index asc); a db_index appearing in several sources with the same
 * score is kept once (sources are expected to be disjoint, e.g. ranks' committed units).
 * top_k <= SW_MAX_TOP_K.  Synchronous. */
int sw_merge_hits(sw_db *db, const sw_hit *lists_dev, int32_t n_sources, int32_t nq, int32_t k_in,
                  int32_t top_k, sw_hit *hits_dev);

/* ---- Phase 2: the alignments of selected pairs (NEXT-3) ---------------------------------
 * P12 §II.A.2: "In order to obtain the optimal local alignment, the algorithm starts from
 * the cell that has the highest value in H i, j, following the arrows until the value zero
 * is reached."  For each requested (query, database sequence) pair the GPU runs the Gotoh
 * recurrence of sw_search in int32 (a block of 8 warps per pair) in linear space: a forward
 * pass keeps row checkpoints every 256 query rows and column checkpoints every 256 database
 * columns and finds the highest cell (ties: smallest query row, then smallest database
 * column); the backtrack recomputes the 256 x 256 tiles on the path with one direction byte
 * per cell and follows the arrows back to a zero.
 * Ops: 'M' = q_i aligned with d_j (match or mismatch), 'I' = q_i against a gap, 'D' = d_j
 * against a gap; listed from the alignment start.  Coordinates are 0-based, end-exclusive:
 * the alignment covers q[q_begin, q_end) and d[d_begin, d_end) of the ORIGINAL sequences.
 * An empty alignment (score 0) has n_ops = 0 and all coordinates 0. */
typedef struct {
  int32_t score;
  int32_t q_begin, q_end, d_begin, d_end;
  int32_t n_ops;
  int64_t ops_offset;       /* into the caller's ops buffer */
} sw_alignment;

/* query_index[k], db_index[k] (original indices), k < n_pairs.  `ops` is caller-owned with
 * ops_capacity bytes; sum over pairs of (|q| + |d|) always suffices (SW_EINVAL names the
 * size needed otherwise).  Host pointers.  Device memory for the direction bytes is
 * bounded (pairs are processed in batches). */
int sw_align(const sw_seqset *queries, sw_db *db, const int8_t *matrix, int32_t gap_open,
             int32_t gap_extend, const int32_t *query_index, const int32_t *db_index,
             int32_t n_pairs, sw_alignment *out, char *ops, int64_t ops_capacity);

/* Thread-local message of the last error on this thread ("" if none). */
const char *sw_last_error(void);

/* Library version string. */
const char *sw_version(void);

#ifdef __cplusplus
}
#endif
#endif
