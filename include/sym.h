/*
 * sym.h -- C-ABI of the B200 symmetry-breaking library (libsym.so, sm_100a).
 *
 * Implements the data-parallel hot path of Nayyaroddeen, Gambhir, Kothapalli,
 * "A Study of Graph Decomposition Algorithms for Parallel Symmetry Breaking"
 * (IPDPS-W 2017).  Citations "P:<line>" refer to that paper's text, and
 * "DESIGN §x" to DESIGN.md, which fixes every reading of a silent or garbled passage.
 *
 *   decomposition  RAND (Alg 2) and DEGk (Alg 3)
 *   MIS            LubyMIS rounds; MIS-Rand; MIS-Deg2
 *   MM             LMAX handshake rounds; MM-Rand (Alg 5);
 *                  MM-Degk (Alg 6)
 *   COLOR          Jones-Plassmann; COLOR-Rand (Alg 8);
 *                  COLOR-Degk (Alg 9)
 *
 * All priorities are a counter-based hash of (vertex or edge, seed) (DESIGN §3 H),
 * so every output is a deterministic function of (graph, params): the
 * lexicographically-first MIS / maximal matching / first-fit colouring of each
 * phase, bit-identical to the CPU oracle and independent of GPU scheduling.
 *
 * Conventions (all functions):
 *  - Pointers inside sym_graph / sym_decomp and the output arrays are DEVICE
 *    pointers; the sym_* structs themselves and sym_stats are HOST memory.
 *  - The caller owns every buffer.  The library allocates no device memory: query
 *    sym_workspace_bytes() first and pass a device workspace of at least that
 *    size (any alignment >= 256 B recommended; the library aligns internally).
 *  - Work is ordered on `stream` (a cudaStream_t; NULL = legacy default stream).
 *    Round loops are host-driven in batches: a call returns after its last host
 *    poll of a device round counter, i.e. with all its kernels complete.
 *  - Arguments are checked on the host before any launch (SYM_EINVAL).  Graph
 *    validity (symmetric, no self-loops, ids in range, rows sorted ascending
 *    without duplicates) is a PRECONDITION, checked only by sym_validate() or
 *    when params->flags has SYM_F_VALIDATE.
 *  - n == 0 is a valid no-op.  Vertex ids must fit in int32 (n < 2^31); arc
 *    offsets are int64 (nnz may exceed 2^31).
 *  - On any error a thread-local message is available from sym_last_error().
 */
#ifndef SYM_H
#define SYM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st *sym_stream_t; /* == cudaStream_t */

/* return codes */
enum {
    SYM_OK = 0,
    SYM_EINVAL = 1,     /* null pointer, n < 0, nnz < 0, RAND p == 0 or p > 65535, bad kind/problem */
    SYM_EWORKSPACE = 2, /* ws_bytes smaller than sym_workspace_bytes() */
    SYM_EGRAPH = 3,     /* sym_validate / SYM_F_VALIDATE found an invalid graph */
    SYM_ECUDA = 4,      /* a CUDA runtime call or kernel launch failed */
    SYM_ENCCL = 5,      /* reserved for the sharded path */
    SYM_EROUNDS = 6     /* params->max_rounds reached before the phase converged */
};

/* decomposition kinds: NONE = no decomposition (the paper's baselines) */
typedef enum { SYM_DECOMP_NONE = 0, SYM_DECOMP_RAND = 1, SYM_DECOMP_DEGK = 2 } sym_decomp_kind;

/* problem ids for sym_workspace_bytes */
typedef enum {
    SYM_PROBLEM_DECOMPOSE = 0,
    SYM_PROBLEM_MIS = 1,
    SYM_PROBLEM_MM = 2,
    SYM_PROBLEM_COLOR = 3,
    SYM_PROBLEM_VALIDATE = 4
} sym_problem;

#define SYM_F_VALIDATE 0x1u /* run sym_validate first; SYM_EGRAPH if invalid */
#define SYM_F_STATS 0x2u    /* fill sym_stats counters that need extra device reads */
#define SYM_F_EXT_DECOMP 0x4u /* a sym_decompose() result will be passed in: the workspace
                                 (query and call) then excludes the internal decomposition,
                                 and sym_mis/mm/color require decomp != NULL */

/* Symmetric simple graph in CSR (directed edges symmetrised, self-loops
   dropped).  row_ptr int64[n+1] with row_ptr[0] = 0 and row_ptr[n] = nnz;
   col_idx int32[nnz] holds neighbour ids; each undirected edge appears as two arcs. */
typedef struct {
    int64_t n, nnz;
    const int64_t *row_ptr;
    const int32_t *col_idx;
} sym_graph;

/* kind: sym_decomp_kind.  param: p = number of parts for RAND (1..65535; the paper's
   "k" of Alg 2, reading G2), k = degree threshold for DEGk (deg <= k -> V_L),
   ignored for NONE.  seed: the 64-bit method seed (priorities and RAND labels).
   max_rounds: cap on rounds per phase (0 = unlimited). */
typedef struct {
    int32_t kind;
    uint32_t param;
    uint64_t seed;
    uint32_t flags;
    uint32_t max_rounds;
} sym_params;

/* Output of sym_decompose (caller-allocated device arrays, filled by the call):
   the induced subgraphs G[V_1..V_p] (RAND) or G_L u G_H (DEGk) as ONE "intra" CSR
   over all n rows, and the cross-edge graph G_{k+1} / G_C as a
   "cross" CSR over all n rows.  Each row's arcs keep their input order.
     row_ptr_in int64[n+1], col_in int32[>= nnz capacity]
     row_ptr_x  int64[n+1], col_x  int32[>= nnz capacity]
     label      uint16[n] optional (may be NULL): RAND part of each vertex, or
                DEGk class (1 = V_H, 0 = V_L).
   nnz_in / nnz_x are written (host) by sym_decompose.  kind/param/seed are
   written too and must match the params of a later sym_mis/mm/color call. */
typedef struct {
    int64_t n;
    int32_t kind;
    uint32_t param;
    uint64_t seed;
    int64_t *row_ptr_in;
    int32_t *col_in;
    int64_t *row_ptr_x;
    int32_t *col_x;
    int64_t nnz_in, nnz_x;
    uint16_t *label;
} sym_decomp;

/* Informational statistics (host struct; not part of the bit-exact result).
   rounds[i] = productive rounds of phase i (phase 0 = the induced/first phase,
   phase 1 = the fix-up phase); phase_vertices[i] = vertices entering phase i;
   result_size = |I|, |M| (edges) or the number of colours; conflicts = COLOR-RAND
   |V'|; max_color = largest colour; ms[0..3] = decompose / phase0 / fix-up /
   phase1 milliseconds (host-measured, includes launch gaps). */
typedef struct {
    uint32_t rounds[3];
    int64_t phase_vertices[3];
    int64_t result_size;
    int64_t conflicts;
    uint32_t max_color;
    float ms[4];
} sym_stats;

/* Bytes of device workspace needed by sym_decompose / sym_mis / sym_mm /
   sym_color / sym_validate (problem = sym_problem) for this graph and params.
   Host only; launches nothing.  The MIS/MM/COLOR sizes include room for an
   internal decomposition (used when their `decomp` argument is NULL).
   Returns 0 on invalid arguments. */
size_t sym_workspace_bytes(const sym_graph *g, const sym_params *p, int problem);

/* RAND (Alg 2): label(v) = floor(pv_RAND(v) * p / 2^32) (DESIGN §3 D1);
   DEGk (Alg 3): class(v) = deg(v) > k (DESIGN §3 D2); NONE: everything
   intra.  Splits every arc (v,w) into intra (same class) or cross, order-preserving.
   Synchronises `stream` once at the end to fill out->nnz_in / out->nnz_x. */
int sym_decompose(const sym_graph *g, const sym_params *p, void *ws, size_t ws_bytes, sym_decomp *out,
                  sym_stream_t stream);

/* Maximal independent set.  in_set uint8[n] (device): 1 iff v in I, else 0.
   NONE: LubyMIS with fixed priorities (= LF-MIS(G)).
   DEGK: MIS-Deg2 (readings G9): I_L = MIS(G_L); remove N[I_L]; I_R = MIS of
         the remaining V_H.
   RAND: MIS-Rand (reading G10): I_A = MIS of the partition interiors;
         remove N[I_A]; I_B = MIS of the remaining graph.
   decomp: a sym_decompose() result for the same graph/params, or NULL to compute
   it inside the workspace.  stats: nullable. */
int sym_mis(const sym_graph *g, const sym_params *p, const sym_decomp *decomp, void *ws, size_t ws_bytes,
            uint8_t *in_set, sym_stats *stats, sym_stream_t stream);

/* Maximal matching.  mate int32[n] (device): partner id, or -1 if unmatched;
   mate[mate[v]] == v.  NONE: LMAX handshake rounds with hash edge
   priorities (= greedy GM order).  RAND: MM-Rand (Alg 5): match inside the
   parts, then on the cross edges among unmatched vertices.  DEGK: MM-Degk (Alg 6):
   match G_H, then G_L u G_C among unmatched vertices. */
int sym_mm(const sym_graph *g, const sym_params *p, const sym_decomp *decomp, void *ws, size_t ws_bytes,
           int32_t *mate, sym_stats *stats, sym_stream_t stream);

/* Vertex colouring.  color uint32[n] (device): colours >= 1, proper on G.
   NONE: Jones-Plassmann = first-fit in priority order.  Computed by
         early-commit rounds (a vertex takes its greedy colour as soon as it is
         determined): same colours, ~10x fewer rounds than JP levels
         on R-MAT; stats->rounds[phase] = those rounds.  Limits: compact ids and
         extra bitmap words < 2^27 (else SYM_EINVAL).
   DEGK: COLOR-Degk (Alg 9): C_H on G_H; G_L coloured with max(C_H)+1 ..
         max(C_H)+k+1 (reading: JP replaces the speculative 3-slot loop).
   RAND: COLOR-Rand (Alg 8): JP on the parts with one palette; the
         endpoints of monochromatic cross edges are re-coloured by JP against G. */
int sym_color(const sym_graph *g, const sym_params *p, const sym_decomp *decomp, void *ws, size_t ws_bytes,
              uint32_t *color, sym_stats *stats, sym_stream_t stream);

/* Checks the CSR precondition on the device: row_ptr[0] = 0, row_ptr monotone,
   row_ptr[n] = nnz; every id in [0,n); no self-loop; each row sorted strictly
   ascending (so no duplicate arcs); symmetry (each arc (v,w) has (w,v), found by
   binary search in row w).  *bad_out (host, nullable) receives the number of
   violating rows/arcs.  Returns SYM_OK, SYM_EGRAPH, or an argument/CUDA error. */
int sym_validate(const sym_graph *g, void *ws, size_t ws_bytes, int64_t *bad_out, sym_stream_t stream);

/* Static description of a return code; and the calling thread's last error text. */
const char *sym_error_string(int code);
const char *sym_last_error(void);

/* Library version string ("symbreak-b200 <semver> sm_100a"). */
const char *sym_version(void);

/* ---- sharded MIS (multi-GPU; one process per GPU) ----
   A rank owns the contiguous vertex range [v_begin, v_end) (v_begin a multiple of
   32) and holds those rows as a local CSR with GLOBAL column ids:
     row_ptr int64[v_end - v_begin + 1] (row_ptr[0] = 0, local arc offsets),
     col_idx int32[nnz] (global ids).
   Every rank keeps a full replica of the MIS status array, uint8[n_global] (0 =
   undecided, 1 = In, 2 = Out), zero-initialised by the caller.  The exchange is the
   caller's (bindings: torch.distributed all_gather over NCCL/NVLink): after each round
   and after the fix-up, the owned segments of the status replicas are all-gathered
   and the next-frontier counts all-reduced; the phase ends when the global count is
   0.  Priorities are the single-GPU ones, so the result equals sym_mis() bit for bit
   (FIXED mode is schedule-independent).  MIS-Deg2: phase L =
   rounds on V_L with cls = 0, sym_shard_mis_kill, phase R = rounds on V_H with
   cls = 1.  MIS-NONE: rounds with cls = -1.  All pointers are device pointers. */
typedef struct {
    int64_t n_global, v_begin, v_end, nnz;
    const int64_t *row_ptr;
    const int32_t *col_idx;
} sym_graph_shard;

/* workspace for sym_shard_mis_round (host only; 0 on invalid arguments) */
size_t sym_shard_workspace_bytes(const sym_graph_shard *g);
/* DEGk class bits (deg > k, Alg 3) of the owned rows into hbits (uint32
   words, n_global bits; words v_begin/32 .. written, the rest untouched) */
int sym_shard_classify(const sym_graph_shard *g, uint32_t k, uint32_t *hbits, sym_stream_t stream);
/* owned undecided vertices of class cls (-1: any) -> list (int32), *count (device u32) */
int sym_shard_frontier(const sym_graph_shard *g, const uint32_t *hbits, int cls, const uint8_t *status,
                       int32_t *list, uint32_t *count, sym_stream_t stream);
/* one Luby round over the owned frontier (list, *count on the device);
   neighbours whose class differs from cls are outside the phase (cls = -1: none);
   still-undecided vertices -> next, *next_count (device u32, set by the call) */
int sym_shard_mis_round(const sym_graph_shard *g, const sym_params *p, const uint32_t *hbits, int cls,
                        uint8_t *status, const int32_t *frontier, const uint32_t *count, int32_t *next,
                        uint32_t *next_count, void *ws, size_t ws_bytes, sym_stream_t stream);
/* MIS-Deg2 fix-up: owned undecided V_H vertices with an In V_L neighbour -> Out */
int sym_shard_mis_kill(const sym_graph_shard *g, const uint32_t *hbits, uint8_t *status, sym_stream_t stream);
/* in_set_owned[v - v_begin] = (status[v] == In) for the owned range */
int sym_shard_mis_finish(const sym_graph_shard *g, const uint8_t *status, uint8_t *in_set_owned,
                         sym_stream_t stream);

/* ---- sharded MM (MM-NONE / MM-Rand, Alg 5; handshake rounds P:152-154) ----
   Same shard layout as above (v_begin need not be 32-aligned here).  Every rank keeps
   full replicas of mate int32[n_global] (caller-initialised to -1) and of two pick
   buffers int32[n_global] (contents arbitrary before round 0).  Round r writes
   pick_cur = picks[r & 1] and reads pick_prev = picks[(r + 1) & 1] (round 0 reads no
   picks).  After each round the caller all-gathers the owned segments of pick_cur
   and mate and all-reduces *next_count; the phase ends when the global count is 0.
   MM-Rand: decompose the owned rows with sym_shard_decompose (labels hash the GLOBAL
   id, so the parts equal the single-GPU ones), phase 1 = rounds on the local intra
   CSR, phase 2 = rounds on the local cross CSR starting from the vertices still
   unmatched.  Priorities are the single-GPU ones, so the result equals sym_mm() bit
   for bit.  All pointers are device pointers. */

/* workspace for sym_shard_decompose (host only; 0 on invalid arguments) */
size_t sym_shard_decompose_workspace_bytes(const sym_graph_shard *g);
/* RAND decomposition (Alg 2) of the owned rows: local intra / cross CSRs
   row_ptr_* int64[v_end - v_begin + 1], col_idx_* int32[nnz] (capacity; global ids),
   the intra arcs first in the same order as sym_decompose.  p->kind RAND or NONE. */
int sym_shard_decompose(const sym_graph_shard *g, const sym_params *p, void *ws, size_t ws_bytes,
                        int64_t *row_ptr_in, int32_t *col_idx_in, int64_t *row_ptr_x, int32_t *col_idx_x,
                        sym_stream_t stream);
/* workspace for sym_shard_mm_round (host only; 0 on invalid arguments) */
size_t sym_shard_mm_workspace_bytes(const sym_graph_shard *g);
/* owned vertices with mate < 0 and at least one arc in g -> list, *count (device u32) */
int sym_shard_mm_frontier(const sym_graph_shard *g, const int32_t *mate, int32_t *list, uint32_t *count,
                          sym_stream_t stream);
/* one handshake round over the owned frontier: resolve round-(r-1) mutual picks
   (r > 0), then pick the heaviest edge to a neighbour with mate < 0; vertices with a
   pick -> next, *next_count (device u32, set by the call) */
int sym_shard_mm_round(const sym_graph_shard *g, const sym_params *p, int round, int32_t *mate,
                       const int32_t *pick_prev, int32_t *pick_cur, const int32_t *frontier, const uint32_t *count,
                       int32_t *next, uint32_t *next_count, void *ws, size_t ws_bytes, sym_stream_t stream);

/* ---- sharded COLOR (COLOR-NONE P:214, COLOR-Rand Alg 8, COLOR-Degk Alg 9
   P:234; Jones-Plassmann rounds [18]) ----
   Same shard layout as sharded MIS (v_begin a multiple of 32).  Every rank keeps a
   full replica of the colour array, uint32[n_global] (0 = uncoloured), zeroed by the
   caller.  p->kind / p->param / p->seed select the class function (NONE: one class;
   RAND: the hash label with p parts, global id; DEGK: the all-gathered V_H bitmap
   hbits of sym_shard_classify) and the vertex priorities (the single-GPU ones).
   admit = 1 restricts every step to arcs whose endpoints share a class (the induced
   subgraphs), admit = 0 uses every arc.  After each round the caller all-gathers the
   owned colour segments and all-reduces *next_count; a phase ends at global count 0.
     COLOR-NONE:  frontier; rounds with admit = 0.
     COLOR-Degk:  frontier; rounds with admit = 1 (G_H and G_L at once); M = the
                  all-reduced max of sym_shard_color_maxh; sym_shard_color_shift(M).
     COLOR-Rand:  frontier; rounds with admit = 1; all-gather; conflicts (V', the
                  owned endpoints of monochromatic cross arcs) -> list; clear;
                  all-gather; rounds on that list with admit = 0.
   The result equals sym_color() bit for bit (any schedule of the rounds gives the
   greedy colouring in priority order).  All pointers are device pointers;
   counts are device uint32. */

/* owned vertices with color == 0 -> list, *count (set by the call) */
int sym_shard_color_frontier(const sym_graph_shard *g, const uint32_t *color, int32_t *list, uint32_t *count,
                             sym_stream_t stream);
/* one JP round over the owned frontier: a vertex whose admitted higher-priority
   neighbours are all coloured takes the smallest colour >= 1 not held by an admitted
   neighbour; the others -> next, *next_count (set by the call) */
int sym_shard_jp_round(const sym_graph_shard *g, const sym_params *p, const uint32_t *hbits, int admit,
                       uint32_t *color, const int32_t *frontier, const uint32_t *count, int32_t *next,
                       uint32_t *next_count, sym_stream_t stream);
/* COLOR-Rand V' (Alg 8): owned v with a cross-class neighbour of the same colour -> list */
int sym_shard_color_conflicts(const sym_graph_shard *g, const sym_params *p, const uint32_t *hbits,
                              const uint32_t *color, int32_t *list, uint32_t *count, sym_stream_t stream);
/* color[list[i]] = 0 for i < *count */
int sym_shard_color_clear(const sym_graph_shard *g, uint32_t *color, const int32_t *list, const uint32_t *count,
                          sym_stream_t stream);
/* *max_out = max colour over owned V_H vertices (0 if none) */
int sym_shard_color_maxh(const sym_graph_shard *g, const uint32_t *hbits, const uint32_t *color, uint32_t *max_out,
                         sym_stream_t stream);
/* color[v] += M for owned V_L vertices (COLOR-Degk's palette shift) */
int sym_shard_color_shift(const sym_graph_shard *g, const uint32_t *hbits, uint32_t *color, uint32_t M,
                          sym_stream_t stream);

/* ---- kernel profiling hook (measurement only; off by default) ----
   sym_profile_enable(1) makes every later call record a CUDA event pair on its
   stream around each hot-kernel launch, grouped by kernel class ("split_degk",
   "split_rand", "mis_round", "mis_huge", "mm_round0", "mm_round", "mm_huge",
   "jp_build", "jp_rounds", ...).  sym_profile_collect() synchronises those
   events and returns, per class: launches, summed device milliseconds and two byte
   counts of those launches (exact: counted by the kernels on device or known on the
   host; -1 if unknown):
     alg_bytes  = SURVEY §8(d)'s algorithmic bytes: a round moves 4 B per scanned arc
                  + 9 B per active vertex (row_ptr pair + status); the split 8 B/arc +
                  24 B per row pointer; JP 8 B/arc + 12 B/vertex of its phase graph
                  (charged to "jp_rounds"; the build reports 0);
     impl_bytes = the words this implementation's kernels load and store (lists,
                  records, counters), i.e. alg plus the implementation's overheads.
   Collect resets the accumulators.  Thread-safe: begin/end pairs nest per stream; the
   state is mutex-guarded. */
typedef struct {
    char name[24];
    int64_t launches;
    double ms;
    double alg_bytes;
    double impl_bytes;
} sym_kernel_profile;

int sym_profile_enable(int on);
int sym_profile_collect(sym_kernel_profile *out, int max_entries, int *count);

#ifdef __cplusplus
}
#endif

#endif /* SYM_H */
