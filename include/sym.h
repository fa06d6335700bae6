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
    SYM_ENCCL = 5,      /* an NCCL call of the sharded path failed */
    SYM_EROUNDS = 6     /* params->max_rounds reached before the phase converged */
};

/* decomposition kinds: NONE = no decomposition (the paper's baselines).
   BRIDGE (Alg 1): the bridges of G (tree edges of a BFS
   forest not covered by any non-tree edge's LCA walk) are the cross edges, the rest
   (the 2-edge-connected components G_1, G_2, ..) the intra edges; MM-Bridge (Alg 4),
   COLOR-Bridge (Alg 7) and MIS-Bridge (Alg 10) then run as the RAND flows.  param is
   ignored; single-GPU; the optional label output is 1 for bridge endpoints. */
typedef enum { SYM_DECOMP_NONE = 0, SYM_DECOMP_RAND = 1, SYM_DECOMP_DEGK = 2, SYM_DECOMP_BRIDGE = 3 } sym_decomp_kind;

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
/* variants: single-GPU calls only (SYM_EINVAL in the
   sharded calls) */
#define SYM_F_PER_ROUND 0x10u     /* sym_mis: classic LubyMIS -- priorities re-drawn
                                     every round from K(seed, VERTEX, round), two-step
                                     synchronous rounds (local maxima join I, then their
                                     neighbours leave); every flow's MIS steps */
#define SYM_F_CONFLICT_DROP 0x20u /* sym_mis RAND: MIS of the parts, the lower In end of every
                                     In-In cross arc dropped, then the MIS of the rest (G10 i) */
#define SYM_F_SPARSER_FIRST 0x40u /* sym_mis RAND: when G_{k+1} has fewer arcs than the parts,
                                     the boundary's MIS first (G10 ii) */
#define SYM_F_LOWER_ONLY 0x80u    /* sym_color RAND: V' = the lower-priority end of each
                                     monochromatic cross edge only (P:232 variant) */
/* the paper's own colouring subroutines, sym_color: speculative
   colouring in synchronous rounds -- every uncoloured vertex takes the smallest colour of
   its window no admitted neighbour holds (else the window moves on, "OFFSET"), then the
   lower-id end of every same-colour edge is reset -- in place of Jones-Plassmann in every
   step of the flow; DEGK colours G_H that way and G_L by Alg 9's literal (k+1)-slot loop
   (all of V_L starts at max(C_H)+1; the lower-id end of a conflict moves to the smallest
   free slot).  Deterministic; NOT the greedy colouring. */
#define SYM_F_COLOR_EB 0x100u     /* edge-based: a 32-colour window */
#define SYM_F_COLOR_VB 0x200u     /* vertex-based: a window of the average degree of
                                     the graph being coloured (FORBIDDEN array) */
/* JP vertex orderings (Hasenplaugh et al. [14]), sym_color
   (JP only): the priority compares the degree in G first -- larger first (LF) or
   smaller first (SF) -- and the FIXED hash second; the colouring is first-fit in that
   order (with SYM_F_LOWER_ONLY, "lower" is in that order too) */
#define SYM_F_ORDER_LF 0x400u
#define SYM_F_ORDER_SF 0x800u

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

/* ---- multi-GPU: sharded MIS / MM / COLOR ----
   One process (or host thread) per rank, each with a communicator.  A rank owns the
   vertex block [v_begin, v_end) = [rank*B, min(n, (rank+1)*B)), B = ceil(n/N) rounded
   up to a multiple of 32 (SYM_EINVAL otherwise), and passes those rows as a local CSR
   with GLOBAL column ids:
     row_ptr int64[v_end - v_begin + 1] (row_ptr[0] = 0, local arc offsets),
     col_idx int32[nnz] (global ids).
   Each call runs the whole flow -- decomposition of the owned rows, every round and
   every fix-up -- inside the library; the only data exchanged are, after each round,
   the state changes of the rank's BOUNDARY vertices (owned vertices with a neighbour
   owned elsewhere): one 8-B all-gather of {delta count, next-frontier count} and one
   all-gather of the delta lists padded to the largest count (4 B per MIS status change,
   8 B per MM pick/match or colour), applied by a scatter kernel.  The result for the
   owned rows equals the single-GPU call (sym_mis / sym_mm / sym_color with the same
   params) bit for bit.  Supported: MIS NONE / DEGK / RAND, MM NONE / RAND, COLOR NONE /
   DEGK / RAND (COLOR runs plain Jones-Plassmann rounds).  n_global < 2^30.
   Calls synchronise the stream once per round (the host reads the gathered counts). */
typedef struct {
    int64_t n_global, v_begin, v_end, nnz;
    const int64_t *row_ptr;
    const int32_t *col_idx;
} sym_graph_shard;

/* communicator: NCCL (one per GPU; rank 0 makes the id with sym_comm_unique_id, the
   caller broadcasts its 128 bytes, every rank calls sym_comm_create on its device), or
   local (N ranks driven by N host threads of one process, any devices; ranks that pass
   the same `group` key join the same group). */
typedef struct sym_comm sym_comm;
#define SYM_COMM_ID_BYTES 128
int sym_comm_unique_id(void *id /* host, SYM_COMM_ID_BYTES */);
int sym_comm_create(sym_comm **out, int nranks, int rank, const void *id);
int sym_comm_create_local(sym_comm **out, int nranks, int rank, uint64_t group);
int sym_comm_destroy(sym_comm *c);
int sym_comm_size(const sym_comm *c, int *nranks, int *rank);

/* per-rank statistics of a sharded call (host struct) */
typedef struct {
    uint32_t rounds[3];         /* rounds of each phase */
    uint32_t exchanges;         /* exchange steps (each: 2 all-gathers) */
    int64_t boundary;           /* owned vertices with a remote neighbour */
    int64_t sent_bytes;         /* delta bytes this rank contributed (sum over exchanges) */
    int64_t gathered_bytes;     /* bytes the padded delta all-gathers delivered to this rank */
    int64_t max_exchange_bytes; /* largest single delta all-gather */
} sym_shard_stats;

/* device workspace of a sharded call (problem = SYM_PROBLEM_MIS / MM / COLOR); host
   only; 0 on invalid arguments */
size_t sym_sharded_workspace_bytes(const sym_graph_shard *g, const sym_params *p, const sym_comm *c, int problem);
/* in_set uint8[v_end - v_begin]: MIS flows as in sym_mis */
int sym_mis_sharded(const sym_graph_shard *g, const sym_params *p, sym_comm *c, void *ws, size_t ws_bytes,
                    uint8_t *in_set, sym_shard_stats *stats, sym_stream_t stream);
/* mate int32[v_end - v_begin] (global partner id or -1): MM flows as in sym_mm
   (Alg 5) */
int sym_mm_sharded(const sym_graph_shard *g, const sym_params *p, sym_comm *c, void *ws, size_t ws_bytes,
                   int32_t *mate, sym_shard_stats *stats, sym_stream_t stream);
/* color uint32[v_end - v_begin] (>= 1): COLOR flows as in sym_color (Alg 8
   P:226/232, Alg 9) */
int sym_color_sharded(const sym_graph_shard *g, const sym_params *p, sym_comm *c, void *ws, size_t ws_bytes,
                      uint32_t *color, sym_shard_stats *stats, sym_stream_t stream);

/* ---- kernel profiling hook (measurement only; off by default) ----
   sym_profile_enable(1) makes every later call record a CUDA event pair on its
   stream around each hot-kernel launch (and count bytes on the device; mode 2 records
   the events only -- the kernels' byte counters cost device time, so timings are taken
   in mode 2 and byte counts in mode 1; 0 turns the hook off), grouped by kernel class ("split_degk",
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
