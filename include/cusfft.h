/*
 * cusfft.h — C ABI of the B200-native sparse FFT engine (sFFT hot path as
 * parallelised by cusFFT, Wang/Chandrasekaran/Chapman, IPDPS'16).
 *
 * Citations are to the paper text, /root/reference/PAPER.md, as L<line>.
 * The paper has no API; the shapes follow its problem statement (L13, L77:
 * x in C^n, k large Fourier coefficients) and its algorithms:
 *
 *   Step 1  random spectral permutation         Def. 1 (L81), Alg. 1
 *   Step 2  flat-window filter + fold into B    L85, Alg. 1, Fig. 3, Alg. 2
 *   Step 3  batched B-point FFT                  L87, L232
 *   Step 4  cutoff (top-num buckets)             L89, Alg. 3
 *   Step 5  reverse hash + vote                  L91-L93, Alg. 4
 *   Step 6  median estimation                    L95, Alg. 5
 *
 * Conventions:
 *   - Signals are interleaved complex fp64 ("complex double", L196): element t
 *     is {re, im} at byte offset 16 t.  Device pointers must be 16-B aligned and
 *     live on the plan's device.
 *   - Forward DFT x^_f = sum_t x_t e^{-2 pi i f t/n}.  The engine returns
 *     x^_f / n, so a planted x_t = sum_f X_f e^{+2 pi i f t/n} is returned as X.
 *   - Every call is stream-ordered on the plan's stream (cusfft_set_stream) and
 *     asynchronous unless stated; no call except cusfft_status /
 *     cusfft_get_debug / cusfft_execute_host synchronises the host.
 *   - A plan is not thread-safe; distinct plans are independent.
 *   - Errors: every function returns 0 (CUSFFT_SUCCESS) or a negative
 *     cusfft_status_t.  On error nothing is launched and outputs are untouched.
 *     There is no CPU fallback: without a CUDA device cusfft_plan fails with
 *     CUSFFT_CUDA.
 */
#ifndef CUSFFT_H_
#define CUSFFT_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CUSFFT_ABI_VERSION 2

typedef struct cusfft_plan_s* cusfft_plan_t; /* opaque; owns all device workspace */

typedef enum {
  CUSFFT_SUCCESS = 0,
  CUSFFT_INVALID_N = -1,      /* n not a power of two, n < 16 or n > 2^31            */
  CUSFFT_INVALID_B = -2,      /* B not a power of two, B < 2, or B >= n               */
  CUSFFT_INVALID_K = -3,      /* k < 1, k > 8192, num_select < k or num_select > B    */
  CUSFFT_INVALID_LOOPS = -4,  /* L < 1, L > 64, L_loc > 32, T > L_loc, L_loc > L, or world !| L */
  CUSFFT_INVALID_PARAM = -5,  /* filter/tolerance/lobefrac/box/taps out of range (incl. a filter longer than n) */
  CUSFFT_NULL_PTR = -6,       /* a required pointer argument is NULL                  */
  CUSFFT_ALLOC = -7,          /* device allocation failed                             */
  CUSFFT_CUDA = -8,           /* a CUDA runtime call failed (cusfft_last_cuda_error)  */
  CUSFFT_HIT_OVERFLOW = -9,   /* more than max_hits frequencies reached T votes       */
  CUSFFT_INVALID_PLAN = -10,  /* NULL or destroyed plan                               */
  CUSFFT_INTERNAL = -11,      /* a device-side consistency check failed               */
  CUSFFT_NCCL = -12           /* NCCL not loadable, or an NCCL call failed (cusfft_last_nccl_error) */
} cusfft_status_t;

typedef enum {
  CUSFFT_FILTER_DOLPH_CHEBYSHEV = 0, /* L25, L85 */
  CUSFFT_FILTER_GAUSSIAN = 1         /* L25, L85 */
} cusfft_filter_t;

/* Step 4 cutoff (L89).  EXACT: the num buckets of largest |u^|^2 (ties to the
 * smaller bucket) by linear-time selection (default).  SORT: the same set by
 * Alg. 3's sort-and-select (L238-L250), a full per-loop sort kept as an
 * ablation (B <= 16384).  THRESHOLD: Alg. 6 (L361-L390), every bucket with
 * |u^|^2 >= cutoff_threshold, a variable count ("slightly more than k", L390). */
typedef enum {
  CUSFFT_CUTOFF_EXACT = 0,
  CUSFFT_CUTOFF_SORT = 1,
  CUSFFT_CUTOFF_THRESHOLD = 2
} cusfft_cutoff_t;

/* Plan parameters.  Fill with cusfft_params_default, then override.
 *
 * Filters (DESIGN.md §3 [Z1]): the taps are a Dolph-Chebyshev or Gaussian
 * window of w taps, w = floor(acosh(1/delta) / (pi lambda)) (Dolph-Chebyshev)
 * or floor(2 ln(1/delta) / (pi lambda)) (Gaussian), forced odd, times a
 * box of width b, normalised to sum 1 ("nearly flat inside the pass region",
 * L85).  The location loops r < L_loc may use their own (delta, lambda)
 * (loc_tolerance, loc_lobefrac; the paper's location loops, L93,
 * against the loops the estimation runs over, L232 / Alg. 5); every loop
 * still estimates with its own filter's response G^.
 *
 * Persisting L2 (l2_persist = 1, the default): a plan whose fold is staged
 * (cusfft_get_info info[11] = 1) raises the DEVICE-WIDE limit
 * cudaLimitPersistingL2CacheSize to its staging buffer size (at most the
 * device maximum, 82 MB on B200) while it lives; its staging stores are
 * evict_last (persisting) so they survive the x stream.  That set-aside is
 * taken from the L2 every kernel of the process sees (dense cuFFT of n = 2^24
 * slows from 292 to 340 us while a C3 plan lives).  Plans share one
 * reference-counted raise per device; the last one destroyed restores the
 * value found before the first.  l2_persist = 0 leaves the limit alone (the
 * staging then competes with x for the normal L2: C3 ~13 us slower). */
typedef struct {
  int32_t filter;          /* cusfft_filter_t; default DOLPH_CHEBYSHEV (L85)                     */
  double tolerance;        /* delta: filter side-lobe / leakage level; default 1e-8              */
  double lobefrac;         /* lambda: main-lobe half width in cycles/sample; default 0.5/B       */
  int64_t box_width;       /* b: width of the frequency box, odd, default n/B - 1                */
  int32_t loc_loops;       /* L_loc <= L: loops that vote (L93); default min(L, 8)                */
  int32_t vote_threshold;  /* T: hit iff votes >= T; default floor(L_loc/2)+1 ("s_i > L/2", L93)  */
  int32_t num_select;      /* buckets kept per location loop (L89); default k                     */
  int32_t tau_mode;        /* 1: random tau (Def. 1); 0: tau = 0 (Alg. 2 L216 literal)       */
  uint64_t seed;           /* drives (a_r, sigma_r, tau_r) through SplitMix64      */
  int64_t max_hits;        /* hit-buffer capacity; default from the expected false-hit count      */
  int32_t device;          /* CUDA device ordinal; default: the current device                   */
  int32_t debug;           /* 1: keep u and per-loop estimates for cusfft_get_debug; default 0   */
  const double* taps;      /* optional HOST array of num_taps real taps g_i (Alg. 1 filter[]) used
                              by every loop; NULL: build the filters from filter / tolerance /
                              lobefrac / box_width (and loc_*).  Copied at plan time; the caller
                              keeps ownership.                                                    */
  int64_t num_taps;        /* length of taps when taps != NULL (odd not required)                */
  int32_t cutoff_mode;     /* cusfft_cutoff_t; default EXACT                                      */
  int32_t shard_mode;      /* cusfft_plan_dist: 0 = loops, one all-gather (default); 1 = signal range;
                              2 = loops, two all-gathers (candidates, then per-loop estimates)      */
  double cutoff_threshold; /* THRESHOLD mode: absolute |u^|^2 threshold (> 0)                    */
  double loc_tolerance;    /* delta of the location loops' filter; 0 (default): tolerance        */
  double loc_lobefrac;     /* lambda of the location loops' filter; 0 (default): lobefrac        */
  int32_t l2_persist;      /* 1 (default): staged plans raise the device's persisting-L2 set-aside
                              while they live (see above); 0: never touch the device limit       */
  int32_t gather;          /* 0 (default): address-sorted staged gather, in stage
                              groups of consecutive loops when the staging of all loops would not
                              fit L2, direct when one loop's would not; 1: always the direct gather;
                              2: the paper's remap + execute kernels on concurrent streams
                              (an ablation; not with shard_mode 1)           */
} cusfft_params;

/* Fill *p with the defaults for (n, k, B).  Returns CUSFFT_NULL_PTR / INVALID_*.
 * Paper: the parameters of Steps 1-6 (L81-L95); the values the paper leaves
 * open are DESIGN.md §3's readings [Z1, Z6, Z8, Z17]. */
int cusfft_params_default(cusfft_params* p, int64_t n, int64_t k, int64_t B);

/* B = floor_pow2(bcst * sqrt(n k / log2 n)); 0 on bad input.
 * Paper: B = O(sqrt(nk / log n)) (L85), = sqrt(nk / log n) (L196, worked
 * example 3,816 at n = 2^18, k = 1000), a power of 2 (L228). */
int64_t cusfft_default_B(int64_t n, int64_t k, double bcst);

/* Create a plan for length-n signals, k outputs, B buckets and L loops.
 * Paper: the per-loop draws a <- random() mod n with gcd(a, n) = 1 and
 * ai = a^-1 (Alg. 1, Def. 1), the flat-window filter (L25, L85)
 * and its response G^ used by the estimation (Alg. 5).
 * p may be NULL (defaults).  Draws (a_r, sigma_r, tau_r), builds the filter
 * taps, the filter response G^(q) for |q| <= n/(2B) and the B-point twiddles
 * on the device, allocates all workspace.  Synchronous.  *out is written only
 * on success. */
int cusfft_plan(cusfft_plan_t* out, int64_t n, int64_t k, int64_t B, int32_t L,
                const cusfft_params* p);

/* Multi-GPU plan for rank `rank` of `world` processes (one GPU each).
 * Paper: the L loops are independent until the vote (L93) and are batched
 * over one B-point FFT (L232); the paper itself runs on one GPU (L119, L398).
 * shard_mode 0 (loops): world must divide L; loop r is owned by rank r mod
 * world, every rank passes the whole signal; outputs are identical on every
 * rank and bit-identical to a world = 1 plan.  The exchange is an ALL-GATHER
 * of the buffer returned by cusfft_exchange_buffer (rank-major slices).
 * shard_mode 1 (signal): world must divide n; rank g passes only
 * its slice x[g n/world, (g+1) n/world) and folds the samples it owns for all
 * L loops; the exchange is a SUM ALL-REDUCE (fp64) of the whole buffer (the
 * B-point FFT is linear, so partial bucket spectra add); every rank then runs
 * Steps 4-6.  Equal to world = 1 within fp64 rounding (the sum order differs).
 * shard_mode 2 (loops, TWO collectives, the
 * north_star's "candidate-index and per-loop estimate lists combined by
 * all-gather"): loops owned as in mode 0; exchange #1 all-gathers the
 * location loops' candidate records (cutoff bitmap | count | J, no u^);
 * every rank then votes over all location loops (identical hit set, L91-L93),
 * sorts the hits ascending and estimates ITS loops for every hit (Alg. 5
 * L308-L325); exchange #2 all-gathers those per-loop estimates; every rank
 * takes the medians (L95, Alg. 5) and selects the output.  Bit-
 * identical to world = 1.  Needs max_hits <= 32768 (the hits are put in
 * ascending order by counting, quadratic in their number) and L <= 64;
 * exchange #2 moves world x max_hits x L/world x 16 bytes, so set max_hits
 * near the expected hit count.
 *
 * nccl_unique_id: NULL, or 128 bytes from cusfft_nccl_unique_id on one rank,
 * distributed to every rank by the caller (any channel).  With an id the plan
 * owns an NCCL communicator (ncclCommInitRank over the `world` ranks; this
 * call then blocks until every rank has called it) and cusfft_execute runs the
 * whole transform including the collective, stream-ordered and captured in
 * the plan's CUDA graph.  NCCL is loaded at run time (libnccl.so.2: the one
 * already in the process, e.g. PyTorch's, else the system's); CUSFFT_NCCL if
 * it cannot be loaded or initialised.  Without an id the caller runs the
 * exchange between cusfft_execute_local and cusfft_execute_finish
 * (cusfft_exchange_kind) and cusfft_execute returns CUSFFT_INVALID_LOOPS for
 * world > 1. */
int cusfft_plan_dist(cusfft_plan_t* out, int64_t n, int64_t k, int64_t B, int32_t L,
                     const cusfft_params* p, int32_t rank, int32_t world, const void* nccl_unique_id);

/* Write a fresh 128-byte ncclUniqueId to out (ncclGetUniqueId).  CUSFFT_NCCL
 * when NCCL cannot be loaded.  Plumbing for cusfft_plan_dist (no paper passage). */
int cusfft_nccl_unique_id(void* out);

/* Release every device allocation of the plan.  Synchronises the plan's stream.
 * Destroying NULL returns CUSFFT_INVALID_PLAN.  Plumbing (no paper passage). */
int cusfft_destroy(cusfft_plan_t plan);

/* Set the CUDA stream (a cudaStream_t; NULL = legacy default stream).
 * Plumbing (no paper passage); the paper overlaps work on CUDA streams (L345-L351). */
int cusfft_set_stream(cusfft_plan_t plan, void* cuda_stream);

/* The whole transform (world = 1 plans, or multi-GPU plans that own a communicator).
 * Paper: Steps 1-6 (L81-L95; Alg. 1, Alg. 2, Alg. 3
 * L238-L250, Alg. 4, Alg. 5) for the problem of L13/L77.
 *   d_x    : device, read-only, complex fp64 [n]
 *   d_locs : device, int64 [k]      output: recovered frequencies, ascending; -1 pads
 *   d_vals : device, complex fp64 [k] output: x^_f / n at d_locs; 0 pads
 * Runs Steps 1-6 (fold, B-point FFT, cutoff, vote, estimate, output).
 * Asynchronous; hit-buffer overflow is reported by cusfft_status. */
int cusfft_execute(cusfft_plan_t plan, const void* d_x, int64_t* d_locs, void* d_vals);

/* Batched transform of `count` independent signals of length n (the batched
 * configuration of SURVEY.md §8(e); each signal is the problem of L13/L77):
 *   d_x    : device, read-only, complex fp64; signal b at d_x + b * x_stride
 *            elements (x_stride >= n)
 *   d_locs : device, int64 [count][k];  d_vals : device, complex fp64 [count][k]
 * Signal b's outputs equal cusfft_execute on it (same plan draws).  With a
 * pipeline depth D > 1 (cusfft_set_pipeline) signal b runs on internal clone
 * b mod D, each on its own stream forked from and joined back to the plan's
 * stream, so one signal's DRAM-bound gather overlaps another's latency-bound
 * cutoff / vote / estimation.  Asynchronous; count = 0 is a no-op.  Errors:
 * CUSFFT_INVALID_PARAM (count < 0 or x_stride < n), CUSFFT_NULL_PTR. */
int cusfft_execute_batch(cusfft_plan_t plan, const void* d_x, int64_t count, int64_t x_stride, int64_t* d_locs,
                         void* d_vals);

/* Paper: none (engine scheduling); cf. the paper's concurrent streams (L345-L351).
 * Pipeline depth D in [1, 8] of cusfft_execute_batch: creates (or frees) D - 1
 * internal clones of the plan (same parameters and draws, own workspace and
 * stream).  Synchronises the plan's stream.  cusfft_status also reports the
 * clones; cusfft_destroy frees them.  world = 1 plans only. */
int cusfft_set_pipeline(cusfft_plan_t plan, int32_t depth);

/* Paper: the transfer-inclusive timing of the PsFFT comparison (L426).
 * Same transform from HOST buffers.  When h_x is pinned and mapped into the
 * device's address space (cudaHostAlloc / cudaHostRegister with a mapped flag,
 * or any pinned allocation on a UVA system, e.g. torch's pin_memory) the
 * gather reads it in place over PCIe: only the samples the plan's taps touch
 * cross the bus (the sFFT's sublinear sampling; C3: 1.87 M of 16.8 M
 * samples), and h_x must stay valid and unchanged until the call returns.
 * Otherwise h_x [n] is first copied to a plan-owned device buffer.  Then the
 * k locations / values are copied back and the stream synchronised.  Returns
 * the cusfft_status result of the transform. */
int cusfft_execute_host(cusfft_plan_t plan, const void* h_x, int64_t* h_locs, void* h_vals);

/* Loop-sharded execution (any world): Steps 1-4 for this rank's loops, written
 * into this rank's slice of the exchange buffer.  Paper: Steps 1-4 per loop
 * (L81-L89), independent across loops until the vote (L93). */
int cusfft_execute_local(cusfft_plan_t plan, const void* d_x);
/* Steps 5-6 plus output selection, after the exchange buffer holds every
 * rank's slice (shard_mode 2: after the second exchange; the medians and the
 * output only).  Outputs as in cusfft_execute.  Paper: Steps 5-6 (L91-L95,
 * Alg. 4, Alg. 5). */
int cusfft_execute_finish(cusfft_plan_t plan, int64_t* d_locs, void* d_vals);
/* shard_mode 2 only, between the two exchanges: the vote over every location
 * loop from the gathered candidate records (L91-L93, Alg. 4), the
 * hit list sorted ascending, and this rank's per-loop estimates of every hit
 * (Alg. 5) into its slice of exchange buffer 2.  CUSFFT_INVALID_PARAM
 * for other plans. */
int cusfft_execute_mid(cusfft_plan_t plan);
/* Plumbing of the caller-run exchange (no paper passage).
 * The exchange buffer: *d_buf points at world * (*bytes_per_rank) bytes of
 * device memory, rank r's slice at offset r * (*bytes_per_rank) (loop
 * sharding); for signal sharding *bytes_per_rank is the whole buffer. */
int cusfft_exchange_buffer(cusfft_plan_t plan, void** d_buf, int64_t* bytes_per_rank);
/* shard_mode 2: exchange buffer 1 (cusfft_exchange_buffer) holds the candidate
 * records, world slices of ceil(L_loc / world) records; exchange buffer 2 the
 * per-loop estimates, world slices of max_hits x (L / world) complex fp64
 * (rank-major, hit-major).  Both are all-gathered (rank r's slice at offset
 * r * bytes_per_rank).  CUSFFT_INVALID_PARAM for other plans. */
int cusfft_exchange_buffer2(cusfft_plan_t plan, void** d_buf, int64_t* bytes_per_rank);
/* 0: all-gather of the rank slices (loop sharding); 1: element-wise fp64 sum
 * all-reduce of the whole buffer (signal sharding); 2: two all-gathers
 * (shard_mode 2: buffer 1 after cusfft_execute_local, buffer 2 after
 * cusfft_execute_mid); negative: error. */
int32_t cusfft_exchange_kind(cusfft_plan_t plan);

/* Paper: a and ai of Alg. 1 (L146-L153), the offset of Def. 1 (L81), the
 * filter length of Alg. 1's filter[filter_size] (L140).
 * Plan facts (host arrays, caller-owned):
 *   info[0..15] = n, k, B, L, w (taps of the estimation filter), n/B, num_select, loc_loops,
 *                 vote_threshold, max_hits, distinct 32-B sectors of x this rank's gathers
 *                 touch (the fold's DRAM floor), staged (0: direct gather; g >= 1: the
 *                 address-sorted two-phase gather, in g stage groups of
 *                 consecutive slots, each staged and folded in turn when the staging of
 *                 all slots would not fit L2), w of the location filter, number of filters (1 or 2),
 *                 fused tail (1: vote + estimation in one kernel), owns an NCCL
 *                 communicator (1)
 *   a, sigma, tau : int64 [L], in loop order r = 0..L-1 (NULL to skip).  sigma is
 *   the gather stride (Alg. 1's ai), a = sigma^-1 mod n, tau the offset. */
int cusfft_get_info(cusfft_plan_t plan, int64_t* info, int64_t* a, int64_t* sigma, int64_t* tau);

typedef enum {
  CUSFFT_DEBUG_U = 0,        /* complex fp64 [L_local][B]: fold output, this rank's loops;
                                 staged plans write it only with params.debug = 1 (else
                                 CUSFFT_INVALID_PARAM)                                      */
  CUSFFT_DEBUG_UHAT = 1,     /* complex fp64 [L][B]: B-point FFTs, loop order                */
  CUSFFT_DEBUG_WINNERS = 2,  /* int32 [L_loc][cap]: kept buckets, ascending, -1 padded; cap =
                                num_select (B in THRESHOLD mode)                              */
  CUSFFT_DEBUG_HITS = 3,     /* int32 [H]: frequencies with >= T votes (unordered)           */
  CUSFFT_DEBUG_HIT_VALS = 4, /* complex fp64 [H]: median estimates aligned with HITS          */
  CUSFFT_DEBUG_PER_LOOP = 5, /* complex fp64 [H][L]: per-loop estimates (params.debug = 1)    */
  CUSFFT_DEBUG_TAPS = 6,     /* fp64 [w]: filter taps g_i (the estimation loops' filter)     */
  CUSFFT_DEBUG_GHAT = 7,     /* complex fp64 [n/B + 1]: its G^(q), q = -n/(2B) .. n/(2B)      */
  CUSFFT_DEBUG_NUM_HITS = 8, /* int64 [1]: H (may exceed max_hits on overflow)               */
  CUSFFT_DEBUG_LOC_TAPS = 9, /* fp64 [w_loc]: the location loops' filter taps (= TAPS with one filter) */
  CUSFFT_DEBUG_LOC_GHAT = 10 /* complex fp64 [n/B + 1]: its G^                                */
} cusfft_debug_t;

/* Paper: the intermediate arrays of Alg. 1-5 (buckets L164-L168, the FFT
 * output L87, J of Alg. 3, the hit list of Alg. 4, the
 * per-loop estimates of Alg. 5) for parity checks.
 * Copy a debug artefact of the last execution to host memory.  cap is the
 * destination size in bytes; returns the number of bytes the artefact needs
 * (>= 0; nothing copied if cap is smaller) or a negative status.  Synchronises. */
int64_t cusfft_get_debug(cusfft_plan_t plan, int32_t what, void* host_dst, int64_t cap);

/* Synchronise the plan's stream and report device-side status of the last
 * execution: CUSFFT_SUCCESS, CUSFFT_HIT_OVERFLOW (more hits than max_hits;
 * Alg. 4's hit array L279-L281 is unbounded) or CUSFFT_INTERNAL. */
int cusfft_status(cusfft_plan_t plan);

/* Paper: the per-step timing of Fig. 2 (L119) and the average execution
 * times of §VI (L402).
 * Timing (enable): 0 off; 1 direct launches (no graph) with CUDA events
 * between the stages; 2 the normal CUDA graph with event-record nodes before
 * and after phase 1 and at the end (times the gather inside the graph that is
 * otherwise executed).
 * Per-stage device times (ms) of the last execution when timing is enabled:
 * ms[0..5] = fold, B-point FFT, cutoff, vote, estimate, output (with the fused
 * vote + estimation kernel, info[14] = 1, the vote entry holds both and the
 * estimate entry is 0); with cap >= 7,
 * ms[6] = phase 1 of the staged fold alone (the address-ordered permute
 * gather k_stage*), -1 when the plan is not staged.  In mode 2
 * ms[0] is the whole graph and ms[1..5] are -1.  get syncs. */
int cusfft_set_timing(cusfft_plan_t plan, int32_t enable);
int cusfft_get_stage_times(cusfft_plan_t plan, float* ms, int32_t cap);

/* Profiling (no paper passage; the per-step breakdown of Fig. 2):
 * run only the first `stages` stages (1 = fold ... 6 = output,
 * the default) so per-stage times can be taken inside the CUDA graph by
 * differences of whole-execution times.  Outputs are undefined when < 6.
 * Where the location slots' FFT pass 2 runs inside the cutoff kernel
 * (B = 8192, 16384, 32768, exact cutoff), it belongs to stage 3: stage 2 is
 * then the estimation slots' FFT only. */
int cusfft_set_stage_limit(cusfft_plan_t plan, int32_t stages);

/* Number of kernel launches one cusfft_execute issues for this plan (plumbing). */
int32_t cusfft_launches_per_execute(cusfft_plan_t plan);

/* Plumbing: status text, the last CUDA / NCCL error codes, the ABI version. */
const char* cusfft_strerror(int code);
int32_t cusfft_last_cuda_error(void);
int32_t cusfft_last_nccl_error(void);
int32_t cusfft_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CUSFFT_H_ */
