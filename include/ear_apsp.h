/*
 * ear_apsp.h -- C ABI of the B200-native ear-reduced all-pairs-shortest-paths library
 * (libearapsp.so).  Paper: D. Dutta, M. Chaitanya, K. Kothapalli, D. Bera, "Applications of Ear
 * Decomposition to Efficient Heterogeneous Algorithms for Shortest Path/Cycle Problems"
 * (IPDPS-W 2017 / IJNC 8(1) 2018).  "P:NN" = line NN of the paper text.
 *
 * Problem (sec. 1, sec. 2.1.3): an undirected graph G = (V, E) with positive integer edge
 * weights (W: E -> R+; integer reading C1 in DESIGN.md); output S[s,t] = weight of a shortest
 * s-t path for every pair.  The library follows Algorithm 1 APSP(G):
 *   Phase I   ear_decompose   G^r = Reduce(G)                       (Alg. 1 line 2)
 *   Phase II  apsp_reduced    S^r = APSP(G^r), blocked min-plus FW (Alg. 1 lines 4-7; FW
 *                             replaces the per-source Dijkstra -- same unique matrix, reading C10)
 *   Phase III expand_ears     S from S^r by UPDATE_DISTANCE         (Alg. 1 lines 9-11)
 *   apsp_full                 all three phases.
 *
 * Conventions (all functions):
 *   - Plain C types only.  `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *   - Pointers named d_* are DEVICE pointers on the current CUDA device, owned by the caller; h_* are
 *     HOST pointers owned by the caller.  No function allocates or frees caller memory.  Plans and
 *     communicators are owned by the library and released only by *_destroy.
 *   - Vertex ids are 0..n-1 (the caller's order); every output is in the caller's order.
 *   - int32 distances.  EAR_INF marks "unreachable" (reading C11); S[s,s] = 0; S is symmetric.
 *   - Return value: EAR_OK or a negative ear_status_t; nothing throws.  ear_last_error() returns a
 *     thread-local human-readable message for the last failure.
 *   - Asynchronous on `stream` unless stated.  Kernel faults surface as EAR_ECUDA at the next
 *     synchronising call.  A plan is not thread-safe; distinct plans are (every FW call owns its
 *     lookahead side stream, events and tile counters: tests/test_concurrency_gpu.py).
 */
#ifndef EAR_APSP_H
#define EAR_APSP_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define EAR_INF 0x3FFFFFFF   /* unreachable; INF + INF does not overflow int32 */
#define EAR_TILE 128         /* FW tile size B; reduced dimensions are padded to multiples of it */

typedef enum {
  EAR_OK = 0,
  EAR_EINVAL = -1,         /* bad argument: n < 1, m < 0, id out of [0,n), weight < 1, bad range */
  EAR_ENOMEM = -2,         /* device or host allocation failed */
  EAR_ECUDA = -3,          /* CUDA runtime / kernel error */
  EAR_ENCCL = -4,          /* communicator error (the caller's all-gather callback failed) */
  EAR_EOVERFLOW = -5,      /* (n-1) * max weight >= EAR_INF: distances might not fit */
  EAR_EUNSUPPORTED = -6    /* unsupported configuration (e.g. misaligned pointer where required) */
} ear_status_t;

enum {
  EAR_FLAG_NONE = 0,
  EAR_FLAG_NO_CONTRACT = 1, /* every vertex is a terminal: direct blocked FW on G (cfg3 baseline) */
  EAR_FLAG_SSSP = 2,        /* Phase II by per-source SSSP on G^r (the paper's own Phase II, P:101;
                               SURVEY 8.f NEXT 2) instead of blocked FW; same D bit for bit */
  EAR_FLAG_BCC = 4,         /* Phase II by biconnected pieces (paper sec. 2.2; SURVEY 8.f
                               NEXT 3): FW on the largest block of every component and on the pieces
                               hanging off it, joined through the articulation points; same D
                               bit for bit.  With EAR_FLAG_SSSP too, every big piece is reduced again
                                and its reduced graph solved by the per-source SSSP instead of
                               the FW (O(n m) work per piece instead of O(n^3)). */
  EAR_FLAG_PART = 16,       /* Phase II by regions (reading C24): G^r cut into connected
                               regions of <= 256 vertices (Voronoi cells of a multi-source BFS), the
                               distances inside every region by one CTA each, the distances between
                               region boundaries by a blocked FW on the boundary graph, and every row of D
                               by two min-plus products with a region boundary as the inner dimension --
                               sec. 2.2's composition through articulation points with
                               boundary sets as the separators.  Same D bit for bit; applies when the
                               distances fit u16 sums (else the SSSP / FW route of the other flags runs).
                               The bench's route. */
  EAR_FLAG_FW32 = 8         /* single-GPU FW: skip the packed 16-bit attempt and run int32 throughout.
                               By default the FW first runs on a copy of D capped at 0x7FFF with two
                               min-plus per VIADDMNMX.U16x2 (exact for every distance < 0x7FFF, see
                               DESIGN.md sec. 6d) and keeps that result unless a connected pair reached
                               the cap, in which case it re-runs in int32: D is the same bit for bit
                               either way.  The range check synchronises the stream once. */
};

typedef struct ear_plan_s *ear_plan_t; /* Reduce(G) result: descriptors + reduced edge list (device) */
typedef struct ear_comm_s *ear_comm_t; /* peer-memory communicator for row-block sharding; NULL = 1 GPU */

/* Summary of a plan.  n_reduced_padded depends on the number of ranks (padding to EAR_TILE*nranks). */
typedef struct {
  int32_t n;                /* |V| */
  int32_t n_reduced;        /* |V^r| (vertices of degree != 2, plus one anchor per pure cycle) */
  int32_t n_reduced_padded; /* Np: |V^r| rounded up to a multiple of EAR_TILE * nranks */
  int32_t n_chains;         /* number of maximal degree-two chains (ears after reduction) */
  int32_t max_chain_len;    /* most degree-two vertices on one chain */
  int32_t n_promoted;       /* pure-cycle components whose min-id vertex became a terminal (C5) */
  int64_t n_reduced_edges;  /* directed G^r arcs fed to D (both directions; before the P:90 min) */
  int64_t m_simple;         /* undirected edges after dropping self-loops / merging parallels (C3) */
  int32_t rank_rounds;      /* pointer-jumping rounds used by the chain ranking */
  int32_t max_weight;       /* largest input weight */
} ear_plan_info_t;

/* ---------------------------------------------------------------- Phase I: Reduce(G)
 * Alg. 1 line 2 "G^r = Reduce(G)"; the reduced graph of P:88 with the parallel-edge rule of
 * P:90.  Input: m undirected edges (d_src[i], d_dst[i], d_w[i]), caller-owned DEVICE int32 arrays;
 * either or both directions may be given; self-loops are ignored and parallel edges keep the
 * minimum weight (reading C3).  Terminals (V^r) are vertices of degree != 2 (reading C4) plus the
 * minimum-id vertex of every pure-cycle component (C5).  Every maximal chain of degree-two vertices
 * becomes one G^r edge whose weight is the chain's weight sum; each chain vertex records its
 * two chain ends (left/right), its along-chain distance to each (reading C7) and its chain
 * (ear) id.  Terminal ids (tid) are assigned in increasing caller-id order.
 * Synchronises `stream` (N_r is data dependent).  On success *out is a new plan (caller destroys it
 * with ear_plan_destroy).  The library's device scratch comes from the device's default stream-ordered
 * pool (cudaMallocAsync); the first call on a device sets that pool's release threshold to "keep"
 * (EAR_POOL_KEEP=0 in the environment leaves it at the driver default), so freed scratch stays
 * reserved for the next call instead of being mapped again.  Errors: EAR_EINVAL (n < 1, m < 0, ids out of range, weight < 1),
 * EAR_EOVERFLOW ((n-1)*max weight >= EAR_INF), EAR_ENOMEM, EAR_ECUDA. */
ear_status_t ear_decompose(int32_t n, int64_t m, const int32_t *d_src, const int32_t *d_dst,
                           const int32_t *d_w, uint32_t flags, void *stream, ear_plan_t *out);

/* Plan summary for `nranks` ranks (1 for a single GPU).  Host-only, no synchronisation. */
ear_status_t ear_plan_info(ear_plan_t plan, int32_t nranks, ear_plan_info_t *info);

/* Copy the per-vertex descriptors to caller DEVICE arrays of n int32 each (any may be NULL):
 * tid (terminal id or -1), ear (chain id or -1), left/right (tid of the chain ends; a terminal's own
 * tid), off_left/off_right (along-chain distance to those ends; 0 for terminals).  For tests. */
ear_status_t ear_plan_export(ear_plan_t plan, int32_t *d_tid, int32_t *d_ear, int32_t *d_left,
                             int32_t *d_right, int32_t *d_off_left, int32_t *d_off_right, void *stream);

/* Copy the directed G^r arcs (before the P:90 min; both directions) to caller DEVICE arrays of
 * info.n_reduced_edges entries each: (tid u, tid v, weight).  For tests. */
ear_status_t ear_plan_export_reduced_edges(ear_plan_t plan, int32_t *d_u, int32_t *d_v, int32_t *d_w,
                                           void *stream);

/* Release a plan.  Its device arrays come from the device's stream-ordered memory pool and are freed
 * in stream order on the stream given to ear_decompose, which must still be valid. */
void ear_plan_destroy(ear_plan_t plan);

/* ---------------------------------------------------------------- Phase II: APSP(G^r)
 * Alg. 1 lines 4-7: D = S^r, all-pairs shortest paths on G^r, computed by a
 * three-phase blocked min-plus Floyd-Warshall (prior art [23]) over EAR_TILE x EAR_TILE int32
 * tiles; D is initialised here (EAR_INF, 0 diagonal, min over parallel G^r edges).
 * Layout: row-major int32, leading dimension ldd (elements, ldd >= Np and ldd % 4 == 0, d_D 16-byte
 * aligned), Np = info.n_reduced_padded; padded vertices are isolated.
 * With EAR_FLAG_SSSP in the plan's flags, D is computed row by row by per-source label-correcting
 * SSSP on G^r instead (sharded: every rank its own rows, no communication until the gather).
 * With EAR_FLAG_PART (single GPU, comm == NULL), D comes from the region route (regions,
 * region FWs, the boundary graph, two min-plus products through the region boundaries
 * generalised), computed as u16 rows and widened into d_D; when the route declines (distances too
 * large for its u16 sums, or mostly tiny components) the route of the other flags runs.  apsp_full
 * with EAR_FLAG_PART computes D by regions on every rank (no exchange) and expands the rank's rows.
 *   comm == NULL: d_D is the full Np x Np matrix.
 *   comm != NULL (P ranks, even P = 1): d_D holds this rank's OWNED TILE ROWS -- the 128-row blocks
 *                 ti with (ti mod 2P) in {rank, 2P-1-rank} (a zig-zag that balances the upper
 *                 triangle), in ascending order, ear_owned_tile_rows() blocks of 128 rows x ldd.  Each
 *                 round the owner of row k closes the pivot tile and stores it into every peer's window,
 *                 every rank applies phase 2 to the pieces of the pivot row block it holds and stores them
 *                 into every rank's window (the per-round broadcast of the pieces: each rank receives the
 *                 rest of the block once), and every rank updates only its owned UPPER tiles: the
 *                 single-GPU symmetric halving of the work survives the sharding.  Only
 *                 the upper tiles of d_D are meaningful afterwards; ear_gather_reduced assembles the full
 *                 symmetric matrix.  Collective over the communicator's ranks (may call its all-gather
 *                 callback when the exchange window must grow).
 * Asynchronous.  Errors: EAR_EINVAL (ldd too small/misaligned), EAR_ENCCL, EAR_ECUDA. */
ear_status_t apsp_reduced(ear_plan_t plan, int32_t *d_D, int64_t ldd, ear_comm_t comm, void *stream);

/* The sharded schedule of apsp_reduced for `nranks` ranks, emulated in ONE process on the current
 * device: every virtual rank gets its own owned-tile-row storage and runs the same kernels; the
 * all-reduce of the pivot pieces is replaced by a shared pivot-row buffer (the pieces are disjoint)
 * and the final gather by scattering every rank's upper tiles into d_D, the full Np x Np matrix
 * (Np = ear_plan_info(nranks).n_reduced_padded).  Used to test the multi-GPU path on one GPU; the
 * result must equal apsp_reduced bit for bit.  Asynchronous; errors as apsp_reduced. */
ear_status_t apsp_reduced_emulated(ear_plan_t plan, int32_t nranks, int32_t *d_D, int64_t ldd,
                                   void *stream);

/* DIAGNOSTIC, produces no result: the device work of ONE rank `rank` of an `nranks`-rank run of the
 * sharded FW (sec. 7 of DESIGN.md) on the current device -- packed u16x2, or int32 when the plan was made
 * with EAR_FLAG_FW32 -- per round its pivot pieces, phase 1 when it owns the pivot, phase 2 on its pieces
 * and phase 3 on its owned upper tiles, without the other ranks and without the exchange (min-plus work
 * is data-independent, so the time is that rank's compute).  Used to measure per-rank compute scaling on one GPU (tools/rank_timing.py).  Allocates
 * and frees its own scratch; asynchronous.  Errors: EAR_EINVAL (NULL plan, rank out of range),
 * EAR_ENOMEM, EAR_ECUDA. */
ear_status_t apsp_reduced_rank_timing(ear_plan_t plan, int32_t nranks, int32_t rank, void *stream);

/* Number of 128-row tile blocks a rank owns under the sharded layout of apsp_reduced (Np =
 * ear_plan_info(nranks).n_reduced_padded).  Host-only. */
int32_t ear_owned_tile_rows(int32_t n_reduced_padded, int32_t nranks, int32_t rank);

/* Assemble the full Np x Np matrix d_D_full (ldd_full >= Np) from every rank's owned storage written
 * by apsp_reduced with `comm` (the all-gather of D): each rank's owned rows are placed in its exchange
 * window, and every rank reads every tile from the window of the rank that owns it -- the lower
 * triangle as the transpose of the upper tile, so no mirror pass follows -- between two stream-ordered
 * barriers.  d_D_block must not alias d_D_full.  Without comm, a plain copy.  Collective. */
ear_status_t ear_gather_reduced(ear_plan_t plan, const int32_t *d_D_block, int64_t ldd_block,
                                int32_t *d_D_full, int64_t ldd_full, ear_comm_t comm, void *stream);

/* Block structure of G^r used by EAR_FLAG_BCC (paper sec. 2.2).  Blocks are those of the
 * simple reduced graph (parallel G^r edges merged).  A "piece" is the largest block of a
 * connected component (its root piece) or the set of vertices hanging off that block at one
 * articulation point, with that point (reading C22).  Built on first use: synchronises the plan's
 * stream.  Errors: EAR_EINVAL (NULL), EAR_ENOMEM, EAR_ECUDA. */
typedef struct {
  int32_t n_components;   /* connected components of G^r */
  int32_t n_blocks;       /* biconnected components with at least one edge */
  int32_t n_articulation; /* articulation points of G^r */
  int32_t n_pieces;       /* root pieces + hanging pieces, each solved by its own FW */
  int32_t largest_piece;  /* vertices of the largest piece */
  int32_t tree_levels;    /* levels of the BFS spanning forest (latency of the tree sweeps) */
  double sum_cubes;       /* sum over pieces of size^3 (FW work; N_r^3 without EAR_FLAG_BCC) */
  int32_t rereduced_pieces;  /* big pieces that the last solve reduced again (each block is
                                reduced; an articulation point can have degree 2 inside its block) */
  int32_t largest_reduced;   /* size the largest piece's FW ran on in the last solve (0 before one) */
  int32_t rereduce_levels;   /* most nested reductions of one piece in the last solve (a reduced
                                piece is reduced again while that removes >= 1 % of its vertices) */
} ear_bcc_info_t;
ear_status_t ear_bcc_info(ear_plan_t plan, ear_bcc_info_t *info);

/* Region partition used by EAR_FLAG_PART (built on first use; synchronises the plan's stream).
 * Regions are connected, hold <= 256 vertices each, and are numbered by their smallest seed; the
 * boundary of a region is its set of vertices with a neighbour in another region. */
typedef struct {
  int32_t n_regions;
  int32_t n_boundary;           /* |B|: the boundary graph's FW runs on this many vertices */
  int32_t max_region;
  int32_t max_boundary;         /* largest |B_i| (inner dimension of the products) */
  int32_t passes;               /* BFS passes (1 + region splits) */
  int32_t multi_component;      /* G^r has more than one connected component */
  double sum_region_boundary;   /* sum_i |R_i| |B_i|: the products do N_r times this many min-plus */
} ear_part_info_t;
ear_status_t ear_part_info(ear_plan_t plan, ear_part_info_t *info);

/* ---------------------------------------------------------------- Phase III: UPDATE_DISTANCE
 * Alg. 1 lines 9-11 with the rules of sec. 2.1.3: for rows
 * s in [row_begin, row_end) of S and every column t (caller order):
 *   u, v in V^r                : S[u,v] = D[u,v]
 *   x chain vertex, v in V^r   : S[x,v] = min(D[l_x,v] + wt(x,l_x), D[r_x,v] + wt(x,r_x))
 *   x, y chain vertices        : 4-term minimum over {l_x,r_x} x {l_y,r_y}
 *   x, y on the same chain     : also min with the along-chain distance |off_x - off_y|
 *                                (same-ear test by chain id: readings C8, C9)
 * then clamped to EAR_INF.  d_D_full is the FULL Np x Np matrix from apsp_reduced (ldd).  d_out is
 * caller-owned (row_end - row_begin) x n int32, row-major with leading dimension ldo >= n.  The
 * 128-bit store path is used when d_out is 16-byte aligned and ldo % 4 == 0 (otherwise a scalar
 * path).  Asynchronous.  Errors: EAR_EINVAL (range, ldo < n, ldd), EAR_ECUDA. */
ear_status_t expand_ears(ear_plan_t plan, const int32_t *d_D_full, int64_t ldd, int32_t row_begin,
                         int32_t row_end, int32_t *d_out, int64_t ldo, void *stream);

/* Compact / query mode (the paper's storage argument, P:137 and Table 1 "Our's
 * memory"): S[d_s[i], d_t[i]] for npairs arbitrary pairs, evaluated per pair from the full D and the
 * plan's descriptors with the same rules as expand_ears -- O(N_r^2 + N) memory instead of
 * the N^2 matrix.  d_s, d_t: DEVICE int32 vertex ids in [0,n) (not validated: out-of-range ids are
 * undefined behaviour); d_out: DEVICE int32[npairs].  Asynchronous.  Errors: EAR_EINVAL. */
ear_status_t ear_query_pairs(ear_plan_t plan, const int32_t *d_D_full, int64_t ldd, int64_t npairs,
                             const int32_t *d_s, const int32_t *d_t, int32_t *d_out, void *stream);

/* ---------------------------------------------------------------- Everything: Algorithm 1
 * APSP(G): ear_decompose + apsp_reduced (+ all-gather with comm) + expand_ears into rows
 * [row_begin, row_end) of S (d_out as in expand_ears).  Scratch (D) is allocated internally from
 * the device heap and freed before return.  Synchronises `stream` once (inside ear_decompose) and
 * again before freeing scratch.  With comm, each rank passes its own row range (ear_row_block). */
ear_status_t apsp_full(int32_t n, int64_t m, const int32_t *d_src, const int32_t *d_dst,
                       const int32_t *d_w, uint32_t flags, int32_t row_begin, int32_t row_end,
                       int32_t *d_out, int64_t ldo, ear_comm_t comm, void *stream);

/* Same as apsp_full with HOST input and output buffers (h_src/h_dst/h_w: m entries; h_out:
 * (row_end-row_begin) x ldo).  Copies in, computes, copies the rows out (pinned h_out is fastest).
 * Synchronous.  This is the end-to-end entry point bench.py times for its "e2e" figure. */
ear_status_t apsp_full_host(int32_t n, int64_t m, const int32_t *h_src, const int32_t *h_dst,
                            const int32_t *h_w, uint32_t flags, int32_t row_begin, int32_t row_end,
                            int32_t *h_out, int64_t ldo, ear_comm_t comm, void *stream);

/* apsp_full_host split in two, so that consecutive problems pipeline: the call returns once Phases I
 * and II are enqueued on `stream` (it synchronises `stream` once, inside the decomposition), with the
 * expansion on a job-owned stream and the device -> host copies of the rows on the device's host-copy
 * stream (one per device, FIFO: the copies of successive jobs into the same h_out land in order), so
 * that the next job's Phases I-II on `stream` can overlap this job's 4*rows*n bytes of PCIe traffic.
 * The library's own small readbacks (Phase I counts, BCC sizes, the 16-bit range check) are stores
 * into mapped pinned memory and its memsets are kernels, so nothing of the next job waits on the copy
 * engines.  Measured on cfg4 (tools/e2e_pipeline.py, one job in flight ahead): 0.84 s per call vs
 * 1.02 s synchronous -- the 40 GB of D2H copies (~51 GB/s over PCIe) are then the whole cost.  h_out
 * and the input arrays must stay valid, and h_out unread, until ear_job_wait(*job) returns; it waits,
 * frees the job's scratch and returns the job's status.  Errors of the enqueue phase are returned
 * directly (no job).  Library-owned job handle. */
typedef struct ear_job_s *ear_job_t;
ear_status_t apsp_full_host_async(int32_t n, int64_t m, const int32_t *h_src, const int32_t *h_dst,
                                  const int32_t *h_w, uint32_t flags, int32_t row_begin, int32_t row_end,
                                  int32_t *h_out, int64_t ldo, ear_comm_t comm, void *stream, ear_job_t *job);
ear_status_t ear_job_wait(ear_job_t job);

/* ---------------------------------------------------------------- Minimum cycle basis (paper sec. 3)
 * MCB of G (a basis of the cycle space over GF(2) of minimum total weight; dimension
 * f = m - n + k) -- of the canonical simple graph of the input (self-loops dropped, parallel edges ->
 * lightest, reading C3) -- computed on the reduced graph G^r (Lemma 3.1: same weight and
 * dimension; closed ears are self-loops and parallel chains parallel edges of G^r) by de Pina's
 * Algorithm 2 with the paper's processing phase (sec. 3.3.2): shortest-path
 * trees from every vertex of G^r (read off Phase II's APSP matrix), the Mehlhorn-Michail candidate
 * cycles sorted by weight, per phase the labels of Algorithm 3, the first non-orthogonal
 * candidate, and the witness update (the independence test).  The MCB weight is unique; which basis
 * is returned is implementation-defined.  Inputs as ear_decompose (caller-owned DEVICE edge arrays);
 * synchronises `stream` several times.  On success *out is a library-owned result (ear_mcb_destroy).
 * Memory: about 28 * N_r^2 bytes plus 16 bytes per candidate cycle.  Errors: EAR_EINVAL,
 * EAR_EOVERFLOW, EAR_ENOMEM, EAR_ECUDA. */
typedef struct ear_mcb_s *ear_mcb_t;
typedef struct {
  int32_t dim;            /* f = m - n + k basis cycles (counted on G^r; equal for G, Lemma 3.1) */
  int64_t weight;         /* W(MCB): the sum of the basis cycles' weights */
  int32_t n_reduced;      /* vertices of G^r */
  int64_t m_reduced;      /* edges of G^r: one per maximal degree-two chain + the direct edges */
  int32_t components;     /* k */
  int64_t n_candidates;   /* Mehlhorn-Michail candidate cycles */
  int32_t tree_depth;     /* most edges on a shortest-path-tree path (label levels per phase) */
} ear_mcb_info_t;
ear_status_t ear_mcb(int32_t n, int64_t m, const int32_t *d_src, const int32_t *d_dst, const int32_t *d_w,
                     void *stream, ear_mcb_t *out);
ear_status_t ear_mcb_info(ear_mcb_t mcb, ear_mcb_info_t *info);
/* The basis cycles' weights, in phase order, into a caller DEVICE array of info.dim int64. */
ear_status_t ear_mcb_cycle_weights(ear_mcb_t mcb, int64_t *d_weights, void *stream);
/* Post-processing (sec. 3.3.3): basis cycle i as a closed walk of G -- its vertices in caller
 * ids, in order, the first not repeated at the end; every chain edge of G^r replaced by the chain.
 * Writes min(len, cap) ids to d_verts (DEVICE) and the cycle's length to *len (host); cap = 0 queries
 * the length.  Synchronises `stream`.  Errors: EAR_EINVAL (i out of [0, dim)). */
ear_status_t ear_mcb_cycle(ear_mcb_t mcb, int32_t i, int32_t *d_verts, int32_t cap, int32_t *len, void *stream);
void ear_mcb_destroy(ear_mcb_t mcb);

/* ---------------------------------------------------------------- multi-GPU plumbing
 * Contiguous near-equal split of `rows` rows over nranks: rank gets [*begin, *end). */
void ear_row_block(int32_t rows, int32_t nranks, int32_t rank, int32_t *begin, int32_t *end);

/* Host all-gather supplied by the caller (the Python binding uses torch.distributed): every rank passes
 * `bytes` bytes at `send`; on return `recv` holds rank r's bytes at recv + r * bytes.  Collective over
 * all ranks; returns 0 on success.  The library calls it only inside collective calls (ear_comm_init,
 * and apsp_reduced / apsp_full / ear_gather_reduced when a larger exchange window is needed) to trade
 * CUDA IPC handles -- never on the data path. */
typedef int32_t (*ear_allgather_fn)(const void *send, void *recv, int64_t bytes, void *ctx);

/* Create this rank's communicator on the current CUDA device: the peer-memory transport of the
 * row-block-sharded FW.  Every rank owns a device window exported by CUDA IPC and
 * mapped by every other rank (NVLink/NVSwitch peer memory between GPUs; several ranks may share one
 * GPU); each FW round a rank stores its phase-2-updated pieces of the pivot row block straight into
 * every peer's window and raises a flag (the per-round broadcast of the pieces), and the final D is
 * all-gathered by reading the peers' owned tile rows.  Collective over all ranks; nranks <= EAR_MAX_RANKS;
 * `allgather` (with `ctx`) may be NULL only for nranks == 1 and must stay valid until
 * ear_comm_destroy.  Errors: EAR_EINVAL, EAR_ENCCL (the callback failed), EAR_ECUDA. */
#define EAR_MAX_RANKS 16
ear_status_t ear_comm_init(int32_t nranks, int32_t rank, ear_allgather_fn allgather, void *ctx, ear_comm_t *out);
ear_status_t ear_comm_info(ear_comm_t comm, int32_t *nranks, int32_t *rank);
/* Synchronises the device, unmaps the peers' windows and frees this rank's (no other rank may still be
 * using the communicator in a call). */
void ear_comm_destroy(ear_comm_t comm);

/* ---------------------------------------------------------------- profiling (bench.py, tests)
 * When enabled, CUDA events bracket every launch of the library's kernels on the stream they run on
 * (a few microseconds per launch), and per-kernel-class device durations, launch counts and
 * algorithmic work accumulate until ear_profile_reset.  Process-wide, not thread-safe. */
typedef struct {
  int64_t launches;            /* kernels of this library launched (counted whether or not enabled) */
  double decompose_ms;         /* Phase I (ear_decompose), device time including its host syncs */
  double fw_init_ms;           /* D initialisation */
  double fw_phase1_ms, fw_phase2_ms, fw_phase3_ms;
  int64_t fw_phase1_launches, fw_phase2_launches, fw_phase3_launches;
  double fw_phase2_minplus;    /* algorithmic min-plus operations (one VIADDMNMX each) */
  double fw_phase3_minplus;
  double comm_ms;              /* pivot broadcasts + all-gather (multi-GPU) */
  double expand_ms, same_chain_ms;
  int64_t expand_launches;
  double expand_bytes;         /* algorithmic HBM bytes of k_expand: 4*rows*n + 4*Nr^2 + 16*n */
  double sssp_ms;              /* Phase II by per-source SSSP (EAR_FLAG_SSSP) */
  int64_t sssp_launches;
  double sssp_arcs;            /* sources x reduced arcs (one relaxation pass) */
  double bcc_pieces_ms;        /* EAR_FLAG_BCC: piece matrices init + one-CTA FW of the small pieces
                                  (large pieces are counted under fw_phase*) */
  double compose_ms;           /* EAR_FLAG_BCC: S^r rows composed from the pieces */
  double compose_bytes;        /* 4 * rows * Np written by the compose kernel */
  int64_t fw16_used;           /* FW calls whose packed 16-bit result was kept */
  int64_t fw16_fallbacks;      /* FW calls where a connected pair reached the 16-bit cap (int32 re-run) */
  double fw16_conv_ms;         /* 16-bit path: int32 <-> u16 conversions and the range check */
  double fw_phase3_16_ms;      /* the part of fw_phase3_ms spent in the packed 16-bit tile kernel */
  double fw_phase3_16_minplus; /* its algorithmic min-plus (two per VIADDMNMX.U16x2) */
  double fw_side_ms;           /* packed FW lookahead: phases 1-2 of round k+1 on the side stream, timed
                                  there -- they OVERLAP phase 3 of round k, so this is not additive */
  double rereduce_ms;          /* EAR_FLAG_BCC: Phase I + Phase III of re-reduced big pieces */
  double bcc_prepare_ms;       /* EAR_FLAG_BCC: block structure of G^r (first solve of a plan only) */
  int64_t fw16_prechecked;     /* packed FWs abandoned after round 3: the eccentricity of reduced vertex 0
                                  (one SSSP row, overlapped with rounds 0-3) already reached the 16-bit cap;
                                  each is also counted in fw16_fallbacks */
  double expand_d16_ms;        /* pair-major expansion: D narrowed to the u16 rows it stages (with the range
                                  check), before the k_expand_pairs launch timed in expand_ms */
  double part_ms;              /* EAR_FLAG_PART: regions (first solve of a plan), region FWs, boundary FW */
  double part_mp_ms;           /* EAR_FLAG_PART: the two min-plus products (k_region_mp) */
  int64_t part_mp_launches;
  double part_minplus;         /* their algorithmic min-plus: (N_r + |B|) * sum_i |R_i| |B_i| */
} ear_profile_t;

void ear_profile_enable(int32_t on);
void ear_profile_reset(void);
/* Waits for the recorded events, folds them into *out (cumulative since the last reset). */
ear_status_t ear_profile_read(ear_profile_t *out);

/* ---------------------------------------------------------------- diagnostics */
const char *ear_status_string(ear_status_t status);
const char *ear_last_error(void);   /* thread-local; "" if none */
const char *ear_version(void);

#ifdef __cplusplus
}
#endif
#endif /* EAR_APSP_H */
