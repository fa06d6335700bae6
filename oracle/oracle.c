/*
 * oracle/oracle.c -- CPU ORACLE.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference leg may load this library.  It shares no code with the CUDA path
 * (paper_conf_ipps_nayyaroddeengk17_b200/csrc): no headers, no helpers, no
 * constant tables.  The product path never calls it.
 *
 * What it is: plain, slow, single-threaded, obviously-correct definitions of what
 * the hot path computes, each citing the PAPER.md passage it follows
 * ("P:<line>" = /root/reference/PAPER.md line) and, where the paper is silent or
 * garbled, the reading fixed in DESIGN.md §3 (= SURVEY.md §8(c)).
 *
 *   §H   priority / label hash contract          (paper silent, G14; DESIGN §3 H)
 *   §D   RAND / DEGk decomposition               (Alg 2, Alg 3)
 *   §MIS LF-MIS + MIS-NONE/DEGk/RAND
 *   §MM  LF-MM  + MM-NONE/RAND/DEGk              (Alg 5, Alg 6)
 *   §COL LF-COL + COLOR-NONE/DEGk/RAND           (Alg 9, Alg 8)
 *   §RND literal round-based forms (Luby / LMAX / JP rounds) used only to pin the
 *        sequential forms (Blelloch et al. [6])
 *   §CRT O(m) certificates of the lexicographically-first results, used for
 *        parity at sizes where the full sequential run is too slow
 *
 * Conventions: CSR row_ptr int64[n+1], col_idx int32[nnz], symmetric simple graph.
 * MIS status bytes: 0 = undecided, 1 = In, 2 = Out.  Matching: mate[v] = -1 if
 * unmatched.  Colours >= 1, 0 = uncoloured ("C(v) <- 0").
 *
 * Parity pins (tests/test_oracle_*.py): published hash test vectors; brute force on
 * n <= 12; networkx greedy_color / is_maximal_matching; fixed-priority rounds ==
 * sequential greedy (Blelloch [6]); the paper's DEG2 colouring claim;
 * closed forms (K_n, stars, empty graphs); independence / maximality / properness.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_UNDEC 0
#define OR_IN 1
#define OR_OUT 2

enum { OR_NONE = 0, OR_RAND = 1, OR_DEGK = 2, OR_BRIDGE = 3 };
enum { OR_TAG_VERTEX = 1, OR_TAG_EDGE = 2, OR_TAG_RAND = 3 };

/* ------------------------------------------------------------------ §H hash */
/* splitmix64 finaliser; mix64(0x9E3779B97F4A7C15) is splitmix64's first output
   for state 0 (published value 0xE220A8397B1DCDAF). */
uint64_t or_mix64(uint64_t z) {
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ULL;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBULL;
    z ^= z >> 31;
    return z;
}

/* MurmurHash3 fmix32 finaliser; MurmurHash3_x86_32("", seed=1) = fmix32(1) =
   0x514E28B7 (SMHasher test vector). */
uint32_t or_fmix32(uint32_t h) {
    h ^= h >> 16;
    h *= 0x85EBCA6Bu;
    h ^= h >> 13;
    h *= 0xC2B2AE35u;
    h ^= h >> 16;
    return h;
}

/* K(seed, tag, round) = mix64(mix64(seed ^ golden) ^ (tag<<32 | round)) */
uint64_t or_stream_key(uint64_t seed, uint32_t tag, uint32_t round) {
    return or_mix64(or_mix64(seed ^ 0x9E3779B97F4A7C15ULL) ^ (((uint64_t)tag << 32) | (uint64_t)round));
}

/* vertex priority pv(v) = fmix32(v ^ Klo) ^ Khi  ("random priorities") */
uint32_t or_pv(uint64_t key, uint32_t v) {
    return or_fmix32(v ^ (uint32_t)key) ^ (uint32_t)(key >> 32);
}

/* edge key pe(lo,hi) for lo < hi (random edge weights of LMAX/GM) */
uint32_t or_pe(uint64_t key, uint32_t lo, uint32_t hi) {
    return or_fmix32((lo * 0x9E3779B1u) ^ hi ^ (uint32_t)key) ^ (uint32_t)(key >> 32);
}

/* RAND label in [0,p): "choose i uniformly at random" (Alg 2 l.3), integer
   multiply-high of the RAND-stream priority */
uint32_t or_label(uint64_t key_rand, uint32_t v, uint32_t p) {
    return (uint32_t)(((uint64_t)or_pv(key_rand, v) * (uint64_t)p) >> 32);
}

/* total order on vertices: larger (pv, id) first */
static int vgreater(uint64_t key, int32_t a, int32_t b) {
    uint32_t pa = or_pv(key, (uint32_t)a), pb = or_pv(key, (uint32_t)b);
    if (pa != pb) return pa > pb;
    return a > b;
}

/* ------------------------------------------------------------------ §D decomposition */
/* BRIDGE (Alg 1): the bridges are the edges on no cycle ("any bridge in a
   graph can never be a part of a cycle"); G_1, G_2, .. = the connected components
   of G - B.  Bridges by Tarjan's low-link depth-first search (iterative): a tree edge
   (p, v) is a bridge iff no vertex of v's subtree reaches p or above by a non-tree
   edge, low(v) > pre(p).  class(v) = the smallest vertex id of v's component of G - B
   (a bridge's endpoints lie in different components).  Plain, sequential. */
static void bridge_classes(int64_t n, const int64_t *rp, const int32_t *ci, uint32_t *cls) {
    size_t nn = (size_t)(n > 0 ? n : 1);
    int64_t *pre = (int64_t *)malloc(sizeof(int64_t) * nn), *low = (int64_t *)malloc(sizeof(int64_t) * nn);
    int32_t *par = (int32_t *)malloc(sizeof(int32_t) * nn), *stk = (int32_t *)malloc(sizeof(int32_t) * nn);
    int64_t *it = (int64_t *)malloc(sizeof(int64_t) * nn);
    uint8_t *bridge_up = (uint8_t *)calloc(nn, 1); /* the tree edge (v, par v) is a bridge */
    int64_t t = 0;
    for (int64_t v = 0; v < n; v++) pre[v] = -1;
    for (int64_t r = 0; r < n; r++) {
        if (pre[r] >= 0) continue;
        int64_t top = 0;
        stk[top++] = (int32_t)r;
        par[r] = -1;
        pre[r] = low[r] = t++;
        it[r] = rp[r];
        while (top > 0) {
            int32_t v = stk[top - 1];
            if (it[v] < rp[v + 1]) {
                int32_t w = ci[it[v]++];
                if (pre[w] < 0) {                   /* tree edge */
                    par[w] = v;
                    pre[w] = low[w] = t++;
                    it[w] = rp[w];
                    stk[top++] = w;
                } else if (w != par[v] && pre[w] < low[v]) {
                    low[v] = pre[w];                /* back edge (simple graph: one arc to the parent) */
                }
            } else {
                top--;
                int32_t p = par[v];
                if (p >= 0) {
                    if (low[v] < low[p]) low[p] = low[v];
                    if (low[v] > pre[p]) bridge_up[v] = 1;
                }
            }
        }
    }
    /* components of G - B: label = the smallest id, by a BFS over the non-bridge edges */
    for (int64_t v = 0; v < n; v++) cls[v] = 0xFFFFFFFFu;
    for (int64_t r = 0; r < n; r++) {
        if (cls[r] != 0xFFFFFFFFu) continue;
        int64_t head = 0, tail = 0;
        stk[tail++] = (int32_t)r;
        cls[r] = (uint32_t)r;
        while (head < tail) {
            int32_t v = stk[head++];
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                int is_bridge = (par[w] == v && bridge_up[w]) || (par[v] == w && bridge_up[v]);
                if (!is_bridge && cls[w] == 0xFFFFFFFFu) {
                    cls[w] = (uint32_t)r;
                    stk[tail++] = w;
                }
            }
        }
    }
    free(pre);
    free(low);
    free(par);
    free(stk);
    free(it);
    free(bridge_up);
}

/* class(v): RAND -> label(v) (Alg 2); DEGK -> 1 if deg(v) > k else 0 (Alg 3 l.5-8:
   deg <= k goes to V_L); BRIDGE -> v's component of G - B (Alg 1); NONE -> 0. */
void or_classes(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
                uint32_t *cls) {
    if (kind == OR_BRIDGE) {
        bridge_classes(n, rp, ci, cls);
        return;
    }
    uint64_t kr = or_stream_key(seed, OR_TAG_RAND, 0);
    for (int64_t v = 0; v < n; v++) {
        if (kind == OR_RAND) cls[v] = or_label(kr, (uint32_t)v, param);
        else if (kind == OR_DEGK) cls[v] = (rp[v + 1] - rp[v]) > (int64_t)param ? 1u : 0u;
        else cls[v] = 0;
    }
}

/* Split every row's arcs, in input order, into intra arcs (both endpoints in the
   same class: the induced subgraphs G[V_i] / G_L, G_H) and cross arcs
   (G_{k+1} / G_C).  Outputs are CSRs over all n rows. */
void or_decompose(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
                  int64_t *rp_in, int32_t *ci_in, int64_t *rp_x, int32_t *ci_x) {
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(n > 0 ? n : 1));
    or_classes(n, rp, ci, kind, param, seed, cls);
    int64_t a = 0, b = 0;
    rp_in[0] = 0;
    rp_x[0] = 0;
    for (int64_t v = 0; v < n; v++) {
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
            int32_t w = ci[e];
            if (cls[w] == cls[v]) ci_in[a++] = w;
            else ci_x[b++] = w;
        }
        rp_in[v + 1] = a;
        rp_x[v + 1] = b;
    }
    free(cls);
}

/* ------------------------------------------------------------------ sorting helpers */
static uint64_t g_sort_key;
static int cmp_vertex_desc(const void *x, const void *y) {
    int32_t a = *(const int32_t *)x, b = *(const int32_t *)y;
    if (a == b) return 0;
    return vgreater(g_sort_key, a, b) ? -1 : 1;
}
/* vertices of S (mask) sorted by decreasing (pv, id) */
static int32_t *sorted_set(int64_t n, const uint8_t *inS, uint64_t key, int64_t *cnt) {
    int64_t c = 0;
    for (int64_t v = 0; v < n; v++) c += inS[v] ? 1 : 0;
    int32_t *order = (int32_t *)malloc(sizeof(int32_t) * (size_t)(c > 0 ? c : 1));
    c = 0;
    for (int64_t v = 0; v < n; v++)
        if (inS[v]) order[c++] = (int32_t)v;
    g_sort_key = key;
    qsort(order, (size_t)c, sizeof(int32_t), cmp_vertex_desc);
    *cnt = c;
    return order;
}

/* ------------------------------------------------------------------ §MIS */
/* LF-MIS(S, E[S]): the lexicographically-first MIS = sequential greedy in decreasing
   priority (Blelloch et al. [6]).  For v in S (in order): v is In unless a
   neighbour in S is already In.  st[] must be OR_UNDEC on S; vertices outside S are
   ignored as neighbours and left untouched. */
static void lf_mis(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *inS, uint64_t key, uint8_t *st) {
    int64_t c;
    int32_t *order = sorted_set(n, inS, key, &c);
    for (int64_t i = 0; i < c; i++) {
        int32_t v = order[i];
        int in = 1;
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
            int32_t w = ci[e];
            if (inS[w] && st[w] == OR_IN) { in = 0; break; }
        }
        st[v] = in ? OR_IN : OR_OUT;
    }
    free(order);
}

/* MIS flows.  in_set[v] = 1 iff v in I.
   NONE (LubyMIS baseline): I = LF-MIS(V, E).
   DEGK (Algorithm MIS-Deg2; reading G9: the degree<=k part is G_L, which may
        contain paths and cycles; reading "[21] replaced by LF-MIS"):
        I_L = LF-MIS(V_L, E_L); remove from G the vertices in I_L or adjacent to it;
        I_R = LF-MIS of the graph that remains (X = V_H \ N(I_L), E[X]); I = I_L u I_R.
   RAND (Algorithm MIS-Rand; reading G10: H = G_i minus the endpoints of the
        cross edges, by analogy with P:280):
        B = vertices with a cross arc; I_A = LF-MIS(V\B, E[V\B]);
        X = V \ N[I_A]; I_B = LF-MIS(X, E[X]); I = I_A u I_B.                       */
void or_mis(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
            uint8_t *in_set) {
    uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, 0);
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint8_t *st = (uint8_t *)calloc(nn, 1);
    uint8_t *S = (uint8_t *)calloc(nn, 1);
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    or_classes(n, rp, ci, kind, param, seed, cls);
    if (kind == OR_NONE) {
        for (int64_t v = 0; v < n; v++) S[v] = 1;
        lf_mis(n, rp, ci, S, key, st);
    } else if (kind == OR_DEGK) {
        /* I_L = LF-MIS(V_L, E_L) */
        for (int64_t v = 0; v < n; v++) S[v] = (cls[v] == 0);
        lf_mis(n, rp, ci, S, key, st);
        /* X = V_H minus neighbours of I_L */
        for (int64_t v = 0; v < n; v++) {
            S[v] = 0;
            if (cls[v] != 1) continue;
            int hit = 0;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++)
                if (cls[ci[e]] == 0 && st[ci[e]] == OR_IN) { hit = 1; break; }
            if (hit) st[v] = OR_OUT;
            else S[v] = 1;
        }
        /* I_R = LF-MIS(X, E[X]) */
        lf_mis(n, rp, ci, S, key, st);
    } else { /* OR_RAND */
        uint8_t *B = (uint8_t *)calloc(nn, 1);
        for (int64_t v = 0; v < n; v++)
            for (int64_t e = rp[v]; e < rp[v + 1]; e++)
                if (cls[ci[e]] != cls[v]) { B[v] = 1; break; }
        for (int64_t v = 0; v < n; v++) S[v] = !B[v];
        lf_mis(n, rp, ci, S, key, st);                 /* I_A on the interior */
        for (int64_t v = 0; v < n; v++) {              /* X = V \ N[I_A] */
            S[v] = 0;
            if (!B[v]) continue;                       /* interior: already decided */
            int hit = 0;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++)
                if (!B[ci[e]] && st[ci[e]] == OR_IN) { hit = 1; break; }
            if (hit) st[v] = OR_OUT;
            else S[v] = 1;
        }
        lf_mis(n, rp, ci, S, key, st);                 /* I_B on the reduced graph R */
        free(B);
    }
    for (int64_t v = 0; v < n; v++) in_set[v] = (st[v] == OR_IN) ? 1 : 0;
    free(st);
    free(S);
    free(cls);
}

/* ------------------------------------------------------------------ §MM */
typedef struct { uint32_t pe; int32_t lo, hi; } or_edge;
static int cmp_edge_desc(const void *x, const void *y) {
    const or_edge *a = (const or_edge *)x, *b = (const or_edge *)y;
    if (a->pe != b->pe) return a->pe > b->pe ? -1 : 1;
    if (a->lo != b->lo) return a->lo > b->lo ? -1 : 1;
    if (a->hi != b->hi) return a->hi > b->hi ? -1 : 1;
    return 0;
}

/* LF-MM: sequential greedy matching in decreasing (pe, lo, hi) over the edges
   {lo,hi} whose class pair passes `admit` and whose endpoints are both unmatched
   at the start (GM with fixed random edge priorities; LMAX's mutual
   heaviest-edge rule reaches the same matching, P:152-154 / [6]).
   admit: 0 = all edges, 1 = same class, 2 = different class,
          3 = both endpoints class 1 (G_H), 4 = at least one endpoint class 0 (G_L u G_C) */
static int admitted(int admit, uint32_t cu, uint32_t cw) {
    switch (admit) {
    case 0: return 1;
    case 1: return cu == cw;
    case 2: return cu != cw;
    case 3: return cu == 1 && cw == 1;
    case 4: return cu == 0 || cw == 0;
    }
    return 0;
}
static void lf_mm(int64_t n, const int64_t *rp, const int32_t *ci, const uint32_t *cls, int admit, uint64_t key,
                  int32_t *mate) {
    int64_t m = 0;
    for (int64_t v = 0; v < n; v++)
        for (int64_t e = rp[v]; e < rp[v + 1]; e++)
            if (v < ci[e] && mate[v] < 0 && mate[ci[e]] < 0 && admitted(admit, cls[v], cls[ci[e]])) m++;
    or_edge *E = (or_edge *)malloc(sizeof(or_edge) * (size_t)(m > 0 ? m : 1));
    m = 0;
    for (int64_t v = 0; v < n; v++)
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
            int32_t w = ci[e];
            if (v < w && mate[v] < 0 && mate[w] < 0 && admitted(admit, cls[v], cls[w])) {
                E[m].pe = or_pe(key, (uint32_t)v, (uint32_t)w);
                E[m].lo = (int32_t)v;
                E[m].hi = w;
                m++;
            }
        }
    qsort(E, (size_t)m, sizeof(or_edge), cmp_edge_desc);
    for (int64_t i = 0; i < m; i++)
        if (mate[E[i].lo] < 0 && mate[E[i].hi] < 0) {
            mate[E[i].lo] = E[i].hi;
            mate[E[i].hi] = E[i].lo;
        }
    free(E);
}

/* MM flows.
   NONE (GM / LMAX baseline): M = LF-MM(G).
   RAND (Algorithm MM-Rand, Alg 5 l.5-8): M_IS = MM(union of G_i) (intra edges);
        V' = unmatched; M_{k+1} = MM(G_{k+1}[V']) (cross edges); M = M_IS u M_{k+1}.
   DEGK (Algorithm MM-Degk, Alg 6 l.5-8): M_H = MM(G_H); V' = unmatched;
        M_LC = MM((G_L u G_C)[V']); M = M_H u M_LC.                                      */
void or_mm(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
           int32_t *mate) {
    uint64_t key = or_stream_key(seed, OR_TAG_EDGE, 0);
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    or_classes(n, rp, ci, kind, param, seed, cls);
    for (int64_t v = 0; v < n; v++) mate[v] = -1;
    if (kind == OR_NONE) {
        lf_mm(n, rp, ci, cls, 0, key, mate);
    } else if (kind == OR_RAND || kind == OR_BRIDGE) { /* MM-Rand, Alg 5 / MM-Bridge, Alg 4 */
        lf_mm(n, rp, ci, cls, 1, key, mate);   /* phase 1: induced subgraphs */
        lf_mm(n, rp, ci, cls, 2, key, mate);   /* phase 2: cross edges among unmatched */
    } else {
        lf_mm(n, rp, ci, cls, 3, key, mate);   /* phase 1: G_H */
        lf_mm(n, rp, ci, cls, 4, key, mate);   /* phase 2: G_L u G_C among unmatched */
    }
    free(cls);
}

/* ------------------------------------------------------------------ §COL */
/* smallest colour c >= 1 not used by a coloured (C != 0) neighbour over admitted arcs */
static uint32_t mex_colour(const int64_t *rp, const int32_t *ci, int32_t v, const uint32_t *cls, int admit,
                           const uint32_t *C, uint8_t *mark) {
    int64_t d = rp[v + 1] - rp[v];
    memset(mark, 0, (size_t)d + 2);
    for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
        int32_t w = ci[e];
        if (!admitted(admit, cls[v], cls[w])) continue;
        uint32_t c = C[w];
        if (c != 0 && (int64_t)c <= d + 1) mark[c] = 1;
    }
    uint32_t c = 1;
    while (mark[c]) c++;
    return c;
}

/* LF-COL(S, A, C0): greedy (first-fit) colouring of S in decreasing (pv, id): each v
   takes the smallest colour >= 1 not held by an already-coloured neighbour over the
   admitted arcs.  This is the colouring Jones-Plassmann computes with the same
   priorities ([18]).  C holds C0 on entry (0 = uncoloured; must be 0 on S). */
static void lf_col(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *inS, const uint32_t *cls,
                   int admit, uint64_t key, uint32_t *C) {
    int64_t c, maxd = 0;
    for (int64_t v = 0; v < n; v++)
        if (rp[v + 1] - rp[v] > maxd) maxd = rp[v + 1] - rp[v];
    uint8_t *mark = (uint8_t *)malloc((size_t)maxd + 2);
    int32_t *order = sorted_set(n, inS, key, &c);
    for (int64_t i = 0; i < c; i++) C[order[i]] = mex_colour(rp, ci, order[i], cls, admit, C, mark);
    free(order);
    free(mark);
}

/* COLOR flows.  colour[v] >= 1.
   NONE (JP): C = LF-COL(V, E).
   DEGK (Algorithm COLOR-Degk, Alg 9): C_H = LF-COL(V_H, E_H); M = max C_H
        (0 if V_H empty); C_L = LF-COL(V_L, E_L), which uses colours 1..k+1;
        C = C_H on V_H and M + C_L on V_L ("additional k+1 colours max(C_H)+1 ..
        max(C_H)+k+1").  Reading: the speculative FORBIDDEN loop is replaced by
        first-fit in priority order with the same palette.
   RAND (Algorithm COLOR-Rand, Alg 8 (garbled, G7)): C_IS = LF-COL(V,
        E_intra) with one identical palette; V' = both endpoints of every cross edge
        whose endpoints share a colour; C = C_IS with V' uncoloured, then V' is
        re-coloured first-fit in priority order against all its G-neighbours.       */
void or_color(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
              uint32_t *colour) {
    uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, 0);
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    uint8_t *S = (uint8_t *)calloc(nn, 1);
    or_classes(n, rp, ci, kind, param, seed, cls);
    for (int64_t v = 0; v < n; v++) colour[v] = 0;
    if (kind == OR_NONE) {
        for (int64_t v = 0; v < n; v++) S[v] = 1;
        lf_col(n, rp, ci, S, cls, 0, key, colour);
    } else if (kind == OR_DEGK) {
        uint32_t *CL = (uint32_t *)calloc(nn, sizeof(uint32_t));
        for (int64_t v = 0; v < n; v++) S[v] = (cls[v] == 1);
        lf_col(n, rp, ci, S, cls, 1, key, colour);       /* C_H on G_H */
        uint32_t M = 0;
        for (int64_t v = 0; v < n; v++)
            if (cls[v] == 1 && colour[v] > M) M = colour[v];
        for (int64_t v = 0; v < n; v++) S[v] = (cls[v] == 0);
        lf_col(n, rp, ci, S, cls, 1, key, CL);           /* C_L on G_L */
        for (int64_t v = 0; v < n; v++)
            if (cls[v] == 0) colour[v] = M + CL[v];
        free(CL);
    } else { /* OR_RAND */
        for (int64_t v = 0; v < n; v++) S[v] = 1;
        lf_col(n, rp, ci, S, cls, 1, key, colour);       /* C_IS on the induced subgraphs */
        for (int64_t v = 0; v < n; v++) {                /* V' */
            S[v] = 0;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (cls[w] != cls[v] && colour[w] == colour[v]) { S[v] = 1; break; }
            }
        }
        for (int64_t v = 0; v < n; v++)
            if (S[v]) colour[v] = 0;
        lf_col(n, rp, ci, S, cls, 0, key, colour);       /* recolour V' against G */
    }
    free(cls);
    free(S);
}

/* ------------------------------------------------------------------ §RND round forms */
/* Synchronous fixed-priority Luby rounds on S (E[S]): each round, from a snapshot,
   an undecided v with an In neighbour becomes Out, and an undecided v that beats
   every undecided neighbour becomes In.  Returns the number of rounds. */
int or_luby_rounds(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *inS, uint64_t seed,
                   uint8_t *st) {
    uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, 0);
    uint8_t *snap = (uint8_t *)malloc((size_t)(n > 0 ? n : 1));
    int rounds = 0;
    for (;;) {
        int64_t undec = 0;
        for (int64_t v = 0; v < n; v++) undec += (inS[v] && st[v] == OR_UNDEC);
        if (!undec) break;
        memcpy(snap, st, (size_t)n);
        for (int64_t v = 0; v < n; v++) {
            if (!inS[v] || snap[v] != OR_UNDEC) continue;
            int has_in = 0, is_max = 1;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (!inS[w]) continue;
                if (snap[w] == OR_IN) has_in = 1;
                if (snap[w] == OR_UNDEC && vgreater(key, w, (int32_t)v)) is_max = 0;
            }
            if (has_in) st[v] = OR_OUT;
            else if (is_max) st[v] = OR_IN;
        }
        rounds++;
    }
    free(snap);
    return rounds;
}

/* LMAX rounds (Birn et al. [5]): every unmatched vertex with an unmatched
   neighbour picks its heaviest such edge (key (pe, other endpoint)); mutual picks are
   matched; repeat.  Returns rounds. */
int or_lmax_rounds(int64_t n, const int64_t *rp, const int32_t *ci, uint64_t seed, int32_t *mate) {
    uint64_t key = or_stream_key(seed, OR_TAG_EDGE, 0);
    int32_t *pick = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    int rounds = 0;
    for (int64_t v = 0; v < n; v++) mate[v] = -1;
    for (;;) {
        int64_t live = 0;
        for (int64_t v = 0; v < n; v++) {
            pick[v] = -1;
            if (mate[v] >= 0) continue;
            uint64_t best = 0;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (mate[w] >= 0) continue;
                uint32_t lo = v < w ? (uint32_t)v : (uint32_t)w, hi = v < w ? (uint32_t)w : (uint32_t)v;
                uint64_t k = ((uint64_t)or_pe(key, lo, hi) << 32) | (uint32_t)w;
                if (pick[v] < 0 || k > best) { best = k; pick[v] = w; }
            }
            live += pick[v] >= 0;
        }
        if (!live) break;
        for (int64_t v = 0; v < n; v++)
            if (pick[v] >= 0 && pick[pick[v]] == v) mate[v] = pick[v];
        rounds++;
    }
    free(pick);
    return rounds;
}

/* Jones-Plassmann rounds ([18]): each round, every uncoloured vertex whose
   higher-priority neighbours are all coloured takes the smallest colour not used by
   them.  Returns rounds (the dependency depth). */
int or_jp_rounds(int64_t n, const int64_t *rp, const int32_t *ci, uint64_t seed, uint32_t *C) {
    uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, 0);
    int64_t maxd = 0;
    for (int64_t v = 0; v < n; v++)
        if (rp[v + 1] - rp[v] > maxd) maxd = rp[v + 1] - rp[v];
    uint8_t *mark = (uint8_t *)malloc((size_t)maxd + 2);
    uint32_t *snap = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(n > 0 ? n : 1));
    uint32_t *zero = (uint32_t *)calloc((size_t)(n > 0 ? n : 1), sizeof(uint32_t));
    int rounds = 0;
    for (int64_t v = 0; v < n; v++) C[v] = 0;
    for (;;) {
        int64_t left = 0;
        for (int64_t v = 0; v < n; v++) left += C[v] == 0;
        if (!left) break;
        memcpy(snap, C, sizeof(uint32_t) * (size_t)n);
        for (int64_t v = 0; v < n; v++) {
            if (snap[v]) continue;
            int ready = 1;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++)
                if (vgreater(key, ci[e], (int32_t)v) && snap[ci[e]] == 0) { ready = 0; break; }
            if (ready) C[v] = mex_colour(rp, ci, (int32_t)v, zero, 0, snap, mark);
        }
        rounds++;
    }
    free(mark);
    free(snap);
    free(zero);
    return rounds;
}

/* ------------------------------------------------------------------ §CRT certificates */
/* Each returns the number of violated vertices (0 = the given result IS the
   lexicographically-first one).  Proof sketch (induction in priority order): an
   independent set I equals LF-MIS(S) iff every v in S\I has a higher neighbour in I;
   a matching M equals LF-MM iff every admitted edge outside M touches a heavier M
   edge; a colouring equals LF-COL iff every C(v) is the mex of its higher
   neighbours' colours. */

/* I restricted to S vs LF-MIS(S, E[S]); st: 1 In, else not-In. */
int64_t or_cert_mis(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *inS, uint64_t seed,
                    const uint8_t *in_set) {
    uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, 0);
    int64_t bad = 0;
    for (int64_t v = 0; v < n; v++) {
        if (!inS[v]) continue;
        int higher_in = 0, any_in = 0;
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
            int32_t w = ci[e];
            if (!inS[w] || !in_set[w]) continue;
            any_in = 1;
            if (vgreater(key, w, (int32_t)v)) higher_in = 1;
        }
        if (in_set[v] && any_in) bad++;              /* not independent */
        else if (!in_set[v] && !higher_in) bad++;    /* should have been taken */
    }
    return bad;
}

/* matching certificate over admitted edges among vertices with elig[v] = 1 */
int64_t or_cert_mm(int64_t n, const int64_t *rp, const int32_t *ci, const uint32_t *cls, int admit,
                   const uint8_t *elig, uint64_t seed, const int32_t *mate) {
    uint64_t key = or_stream_key(seed, OR_TAG_EDGE, 0);
    int64_t bad = 0;
    for (int64_t v = 0; v < n; v++) {              /* a matching of G's edges */
        if (mate[v] < 0) continue;
        if (mate[v] >= n || mate[mate[v]] != v) { bad++; continue; }
        int adj = 0;
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) adj |= (ci[e] == mate[v]);
        if (!adj) bad++;
    }
    for (int64_t v = 0; v < n; v++) {
        if (!elig[v]) continue;
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
            int32_t w = ci[e];
            if (w <= v || !elig[w] || !admitted(admit, cls[v], cls[w])) continue;
            if (mate[v] == w) continue;
            uint32_t k = or_pe(key, (uint32_t)v, (uint32_t)w);
            /* must touch a heavier matched edge */
            int dom = 0;
            int32_t ends[2] = {(int32_t)v, w};
            for (int t = 0; t < 2 && !dom; t++) {
                int32_t a = ends[t], b = mate[a];
                if (b < 0) continue;
                uint32_t lo = a < b ? (uint32_t)a : (uint32_t)b, hi = a < b ? (uint32_t)b : (uint32_t)a;
                uint32_t kb = or_pe(key, lo, hi);
                if (kb > k || (kb == k && (lo > (uint32_t)v || (lo == (uint32_t)v && hi > (uint32_t)w)))) dom = 1;
            }
            if (!dom) bad++;
        }
    }
    return bad;
}

/* colouring certificate: every v in S has C(v) = mex of colours of its higher admitted
   neighbours that are either in S (processed earlier) or outside S (pre-coloured,
   all count); returns violations. */
int64_t or_cert_col(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *inS, const uint32_t *cls,
                    int admit, uint64_t seed, const uint32_t *C) {
    uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, 0);
    int64_t maxd = 0, bad = 0;
    for (int64_t v = 0; v < n; v++)
        if (rp[v + 1] - rp[v] > maxd) maxd = rp[v + 1] - rp[v];
    uint8_t *mark = (uint8_t *)malloc((size_t)maxd + 2);
    for (int64_t v = 0; v < n; v++) {
        if (!inS[v]) continue;
        int64_t d = rp[v + 1] - rp[v];
        memset(mark, 0, (size_t)d + 2);
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
            int32_t w = ci[e];
            if (!admitted(admit, cls[v], cls[w])) continue;
            if (inS[w] && !vgreater(key, w, (int32_t)v)) continue;
            if (C[w] != 0 && (int64_t)C[w] <= d + 1) mark[C[w]] = 1;
        }
        uint32_t c = 1;
        while (mark[c]) c++;
        if (C[v] != c) bad++;
    }
    free(mark);
    return bad;
}

/* COLOR-Rand certificate (Alg 8; reading C3 of DESIGN §3), O(m + n):
     1. C1 = LF-COL(V, E_intra) computed by a topological sweep of the priority DAG
        over the intra arcs: a vertex is coloured (first fit over its higher intra
        neighbours) once all of them are coloured.  First-fit colour of v depends only
        on the colours of its higher neighbours, so any topological order gives the
        colours of the sorted order -- without the O(n log n) sort.
     2. V' = both endpoints of every cross edge whose endpoints share a C1 colour.
     3. C must equal C1 off V'; on V', C must be LF-COL(V', E, C1 off V'): checked by
        or_cert_col over S = V' with all arcs admitted (non-V' neighbours count as
        pre-coloured with C = C1).
   Returns the number of violated vertices (0 = C is the oracle's COLOR-Rand output);
   *nconf (nullable) receives |V'|. */
static int64_t cert_col_split(int64_t n, const int64_t *rp, const int32_t *ci, const uint32_t *cls, uint64_t seed,
                              const uint32_t *C, int64_t *nconf);

int64_t or_cert_col_rand(int64_t n, const int64_t *rp, const int32_t *ci, uint32_t p, uint64_t seed,
                         const uint32_t *C, int64_t *nconf) {
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(n > 0 ? n : 1));
    or_classes(n, rp, ci, OR_RAND, p, seed, cls);
    int64_t bad = cert_col_split(n, rp, ci, cls, seed, C, nconf);
    free(cls);
    return bad;
}

/* the same certificate for any vertex classes (RAND parts, BRIDGE components) */
static int64_t cert_col_split(int64_t n, const int64_t *rp, const int32_t *ci, const uint32_t *cls, uint64_t seed,
                              const uint32_t *C, int64_t *nconf) {
    uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, 0);
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint32_t *C1 = (uint32_t *)calloc(nn, sizeof(uint32_t));
    int64_t *pend = (int64_t *)malloc(sizeof(int64_t) * nn); /* uncoloured higher intra neighbours */
    int32_t *queue = (int32_t *)malloc(sizeof(int32_t) * nn);
    uint8_t *S = (uint8_t *)calloc(nn, 1);
    int64_t maxd = 0, head = 0, tail = 0, bad = 0, conf = 0;
    for (int64_t v = 0; v < n; v++) {
        if (rp[v + 1] - rp[v] > maxd) maxd = rp[v + 1] - rp[v];
        pend[v] = 0;
        for (int64_t e = rp[v]; e < rp[v + 1]; e++)
            if (cls[ci[e]] == cls[v] && vgreater(key, ci[e], (int32_t)v)) pend[v]++;
        if (pend[v] == 0) queue[tail++] = (int32_t)v;
    }
    uint8_t *mark = (uint8_t *)malloc((size_t)maxd + 2);
    while (head < tail) { /* step 1 */
        int32_t v = queue[head++];
        int64_t d = rp[v + 1] - rp[v];
        memset(mark, 0, (size_t)d + 2);
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
            int32_t w = ci[e];
            if (cls[w] == cls[v] && vgreater(key, w, v) && (int64_t)C1[w] <= d + 1) mark[C1[w]] = 1;
        }
        uint32_t c = 1;
        while (mark[c]) c++;
        C1[v] = c;
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
            int32_t w = ci[e];
            if (cls[w] == cls[v] && vgreater(key, v, w) && --pend[w] == 0) queue[tail++] = w;
        }
    }
    if (tail != n) bad += n - tail; /* unreachable for a DAG; defensive */
    for (int64_t v = 0; v < n; v++) { /* step 2 */
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
            int32_t w = ci[e];
            if (cls[w] != cls[v] && C1[w] == C1[v]) { S[v] = 1; break; }
        }
        conf += S[v];
        if (!S[v] && C[v] != C1[v]) bad++; /* step 3, off V' */
    }
    uint32_t *zero = (uint32_t *)calloc(nn, sizeof(uint32_t));
    bad += or_cert_col(n, rp, ci, S, zero, 0, seed, C); /* step 3, on V' */
    if (nconf) *nconf = conf;
    free(zero);
    free(mark);
    free(S);
    free(queue);
    free(pend);
    free(C1);
    return bad;
}

/* Flow certificates with O(n) extra memory (no arc-sized arrays, so they run at
   R-MAT scale 27 on the host): the result of each problem/decomposition flow is
   checked phase by phase against the definitions in or_mis / or_mm / or_color,
   using the single-phase certificates above.  problem: 1 MIS (uint8 in_set), 2 MM
   (int32 mate), 3 COLOR (uint32 colour).  Returns the number of violations. */
int64_t or_cert_flow(int problem, int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param,
                     uint64_t seed, const void *result) {
    size_t nn = (size_t)(n > 0 ? n : 1);
    int64_t bad = 0;
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    or_classes(n, rp, ci, kind, param, seed, cls);
    if (problem == 3 && (kind == OR_RAND || kind == OR_BRIDGE)) {
        bad = cert_col_split(n, rp, ci, cls, seed, (const uint32_t *)result, 0);
        free(cls);
        return bad;
    }
    uint8_t *S = (uint8_t *)malloc(nn);
    if (problem == 1) { /* MIS: M1 NONE, M2 DEGk, M3 RAND */
        const uint8_t *I = (const uint8_t *)result;
        if (kind == OR_NONE) {
            memset(S, 1, nn);
            bad = or_cert_mis(n, rp, ci, S, seed, I);
        } else {
            /* first set: V_L (DEGk) / interior vertices V \ B (RAND) */
            for (int64_t v = 0; v < n; v++) {
                if (kind == OR_DEGK) {
                    S[v] = cls[v] == 0;
                } else {
                    S[v] = 1;
                    for (int64_t e = rp[v]; e < rp[v + 1]; e++)
                        if (cls[ci[e]] != cls[v]) { S[v] = 0; break; }
                }
            }
            bad = or_cert_mis(n, rp, ci, S, seed, I);
            /* the rest: removed if a first-set neighbour is In, else the second phase */
            uint8_t *X = (uint8_t *)malloc(nn);
            for (int64_t v = 0; v < n; v++) {
                X[v] = 0;
                if (S[v]) continue;
                int killed = 0;
                for (int64_t e = rp[v]; e < rp[v + 1] && !killed; e++) killed = S[ci[e]] && I[ci[e]];
                if (killed) bad += I[v] != 0;
                else X[v] = 1;
            }
            bad += or_cert_mis(n, rp, ci, X, seed, I);
            free(X);
        }
    } else if (problem == 2) { /* MM: MM1 NONE, MM2 RAND (Alg 5), MM3 DEGk (Alg 6) */
        const int32_t *M = (const int32_t *)result;
        if (kind == OR_NONE) {
            memset(S, 1, nn);
            bad = or_cert_mm(n, rp, ci, cls, 0, S, seed, M);
        } else {
            int a1 = kind == OR_DEGK ? 3 : 1, a2 = kind == OR_DEGK ? 4 : 2;
            int32_t *M1 = (int32_t *)malloc(sizeof(int32_t) * nn), *M2 = (int32_t *)malloc(sizeof(int32_t) * nn);
            for (int64_t v = 0; v < n; v++) {
                int32_t w = M[v];
                int in1 = w >= 0 && w < n && admitted(a1, cls[v], cls[w]);
                M1[v] = in1 ? w : -1;
                M2[v] = in1 ? -1 : w;
                S[v] = !in1; /* free after phase 1 */
            }
            uint8_t *all = (uint8_t *)malloc(nn);
            memset(all, 1, nn);
            bad = or_cert_mm(n, rp, ci, cls, a1, all, seed, M1);
            bad += or_cert_mm(n, rp, ci, cls, a2, S, seed, M2);
            free(all);
            free(M1);
            free(M2);
        }
    } else { /* COLOR: C1 NONE, C2 DEGk (Alg 9) */
        const uint32_t *C = (const uint32_t *)result;
        if (kind == OR_NONE) {
            memset(S, 1, nn);
            bad = or_cert_col(n, rp, ci, S, cls, 0, seed, C);
        } else {
            uint32_t M = 0;
            for (int64_t v = 0; v < n; v++) {
                S[v] = cls[v] == 1;
                if (S[v] && C[v] > M) M = C[v];
            }
            bad = or_cert_col(n, rp, ci, S, cls, 1, seed, C); /* C_H on G_H */
            uint32_t *CL = (uint32_t *)malloc(sizeof(uint32_t) * nn);
            for (int64_t v = 0; v < n; v++) {
                S[v] = cls[v] == 0;
                CL[v] = 0;
                if (S[v]) {
                    if (C[v] <= M) bad++; /* L colours start above max C_H */
                    else CL[v] = C[v] - M;
                }
            }
            bad += or_cert_col(n, rp, ci, S, cls, 1, seed, CL); /* C_L on G_L */
            free(CL);
        }
    }
    free(S);
    free(cls);
    return bad;
}

/* ------------------------------------------------------------------ §VAR variants */
/* flag values of the variant contract (the same numbers as SYM_F_* in the C-ABI) */
#define OR_F_PER_ROUND 0x10u      /* MIS: classic Luby -- priorities re-drawn every round */
#define OR_F_CONFLICT_DROP 0x20u  /* MIS-RAND: MIS of the parts, drop the lower In end of In-In cross arcs */
#define OR_F_SPARSER_FIRST 0x40u  /* MIS-RAND: the sparser of E[V\B], E[B] first */
#define OR_F_LOWER_ONLY 0x80u     /* COLOR-RAND: V' = lower-priority endpoints only */

/* LubyMIS as Luby states it ("uses randomization to break symmetry"), the
   two-step synchronous round with FRESH priorities every round: in round r (0, 1, ..
   within the phase) every undecided v of S draws pv_r(v) (stream key K(seed, VERTEX,
   r)); the undecided local maxima of (pv_r, id) over their undecided S-neighbours join
   I; then every undecided vertex with a neighbour that just joined I leaves.  st[]:
   OR_UNDEC on S on entry. */
static void luby_per_round(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *inS, uint64_t seed,
                           uint8_t *st) {
    uint8_t *sel = (uint8_t *)calloc((size_t)(n > 0 ? n : 1), 1);
    for (uint32_t r = 0;; r++) {
        uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, r);
        int64_t undec = 0;
        for (int64_t v = 0; v < n; v++) {        /* step 1: local maxima of the round's draw */
            sel[v] = 0;
            if (!inS[v] || st[v] != OR_UNDEC) continue;
            undec++;
            int best = 1;
            for (int64_t e = rp[v]; e < rp[v + 1] && best; e++) {
                int32_t w = ci[e];
                if (inS[w] && st[w] == OR_UNDEC && vgreater(key, w, (int32_t)v)) best = 0;
            }
            sel[v] = (uint8_t)best;
        }
        if (!undec) break;
        for (int64_t v = 0; v < n; v++)          /* they join I ... */
            if (sel[v]) st[v] = OR_IN;
        for (int64_t v = 0; v < n; v++) {        /* step 2: ... and their neighbours leave */
            if (!inS[v] || st[v] != OR_UNDEC) continue;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++)
                if (inS[ci[e]] && sel[ci[e]]) { st[v] = OR_OUT; break; }
        }
    }
    free(sel);
}

/* the MIS of G[S] a flow step computes: LF-MIS (FIXED priorities) or per-round Luby */
static void mis_step(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *inS, uint64_t seed,
                     uint32_t flags, uint8_t *st) {
    if (flags & OR_F_PER_ROUND) luby_per_round(n, rp, ci, inS, seed, st);
    else lf_mis(n, rp, ci, inS, or_stream_key(seed, OR_TAG_VERTEX, 0), st);
}

/* X = the vertices of `from` none of whose neighbours in `by` is In (the others are
   removed: Out) -- "remove from G vertices that are in I or have a neighbour in I" */
static void reduce(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *from, const uint8_t *by,
                   uint8_t *st, uint8_t *X) {
    for (int64_t v = 0; v < n; v++) {
        X[v] = 0;
        if (!from[v]) continue;
        int hit = 0;
        for (int64_t e = rp[v]; e < rp[v + 1] && !hit; e++) hit = by[ci[e]] && st[ci[e]] == OR_IN;
        if (hit) st[v] = OR_OUT;
        else X[v] = 1;
    }
}

/* MIS flows with the f1 variants (flags 0: exactly or_mis).
   PER_ROUND: every MIS step of the flow (NONE; DEGK's I_L, I_R; RAND's I_A, I_B) is
     per-round Luby instead of LF-MIS; the flow is unchanged.
   RAND + CONFLICT_DROP (reading G10 (i)): I_P = MIS of the induced subgraphs (every
     intra arc, all vertices); D = the In vertices with a higher-priority In cross
     neighbour; I' = I_P \ D (independent in G); X = V \ N[I'] (the vertices not in I'
     without a neighbour in I'); I_B = MIS(X, E[X]); I = I' u I_B.
   RAND + SPARSER_FIRST ("I_A and I_B can be computed in any order. We
     base our decision on which of the two graphs U G_i or G_{k+1} is sparser";
     reading G10 (ii)): B = vertices with a cross arc; if G_{k+1} has fewer arcs than
     U G_i, the boundary goes first -- I_1 = MIS(B, E[B]) (all arcs among B, so that
     I_1 is independent in G), X = interior vertices without a neighbour in I_1,
     I_2 = MIS(X, E[X]), I = I_1 u I_2 -- else the standard order. */
void or_mis_ex(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
               uint32_t flags, uint8_t *in_set) {
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint8_t *st = (uint8_t *)calloc(nn, 1), *S = (uint8_t *)calloc(nn, 1), *X = (uint8_t *)calloc(nn, 1);
    uint8_t *B = (uint8_t *)calloc(nn, 1);
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    or_classes(n, rp, ci, kind, param, seed, cls);
    if (kind == OR_NONE) {
        for (int64_t v = 0; v < n; v++) S[v] = 1;
        mis_step(n, rp, ci, S, seed, flags, st);
    } else if (kind == OR_DEGK) {
        uint8_t *H = (uint8_t *)calloc(nn, 1);
        for (int64_t v = 0; v < n; v++) {
            S[v] = cls[v] == 0;
            H[v] = cls[v] == 1;
        }
        mis_step(n, rp, ci, S, seed, flags, st);  /* I_L */
        reduce(n, rp, ci, H, S, st, X);           /* X = V_H \ N(I_L) */
        mis_step(n, rp, ci, X, seed, flags, st);  /* I_R */
        free(H);
    } else if (flags & OR_F_CONFLICT_DROP) {
        uint8_t *ip = (uint8_t *)calloc(nn, 1);
        /* I_P: the MIS of each part G[V_i] = the MIS of the union of the induced
           subgraphs; computed part by part (every part is an S of its own) */
        for (uint32_t part = 0; part < param; part++) {
            int any = 0;
            for (int64_t v = 0; v < n; v++) any |= (S[v] = cls[v] == part);
            if (any) mis_step(n, rp, ci, S, seed, flags, st);
        }
        for (int64_t v = 0; v < n; v++) {         /* D: lower In end of an In-In cross arc */
            ip[v] = st[v] == OR_IN;
            for (int64_t e = rp[v]; e < rp[v + 1] && ip[v]; e++) {
                int32_t w = ci[e];
                if (cls[w] != cls[v] && st[w] == OR_IN && vgreater(or_stream_key(seed, OR_TAG_VERTEX, 0), w, (int32_t)v))
                    ip[v] = 0;
            }
        }
        for (int64_t v = 0; v < n; v++) {
            st[v] = ip[v] ? OR_IN : OR_UNDEC;
            S[v] = !ip[v];
        }
        reduce(n, rp, ci, S, ip, st, X);          /* X = V \ N[I'] */
        mis_step(n, rp, ci, X, seed, flags, st);  /* I_B */
        free(ip);
    } else {
        for (int64_t v = 0; v < n; v++)
            for (int64_t e = rp[v]; e < rp[v + 1]; e++)
                if (cls[ci[e]] != cls[v]) { B[v] = 1; break; }
        int64_t a_intra = 0, a_cross = 0;  /* arcs of U G_i and of G_{k+1} */
        for (int64_t v = 0; v < n; v++)
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                a_intra += cls[ci[e]] == cls[v];
                a_cross += cls[ci[e]] != cls[v];
            }
        int bfirst = (flags & OR_F_SPARSER_FIRST) && a_cross < a_intra;
        uint8_t *first = (uint8_t *)calloc(nn, 1), *rest = (uint8_t *)calloc(nn, 1);
        for (int64_t v = 0; v < n; v++) {
            first[v] = bfirst ? B[v] : !B[v];
            rest[v] = !first[v];
        }
        mis_step(n, rp, ci, first, seed, flags, st);  /* I_A (or I_1 = MIS(G[B])) */
        reduce(n, rp, ci, rest, first, st, X);
        mis_step(n, rp, ci, X, seed, flags, st);      /* I_B on the reduced graph */
        free(first);
        free(rest);
    }
    for (int64_t v = 0; v < n; v++) in_set[v] = st[v] == OR_IN;
    free(st);
    free(S);
    free(X);
    free(B);
    free(cls);
}

/* COLOR flows with the f1 variant (flags 0: exactly or_color).
   RAND + LOWER_ONLY: V' = the LOWER-priority endpoint of every cross edge whose ends
   share a C_IS colour (instead of both, reading C3); V' is recoloured first-fit in
   priority order against all of G, as in or_color. */
void or_color_ex(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
                 uint32_t flags, uint32_t *colour) {
    if (!(kind == OR_RAND && (flags & OR_F_LOWER_ONLY))) {
        or_color(n, rp, ci, kind, param, seed, colour);
        return;
    }
    uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, 0);
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    uint8_t *S = (uint8_t *)calloc(nn, 1);
    or_classes(n, rp, ci, kind, param, seed, cls);
    for (int64_t v = 0; v < n; v++) {
        colour[v] = 0;
        S[v] = 1;
    }
    lf_col(n, rp, ci, S, cls, 1, key, colour);           /* C_IS on the induced subgraphs */
    for (int64_t v = 0; v < n; v++) {                    /* V' = lower ends of conflicts */
        S[v] = 0;
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
            int32_t w = ci[e];
            if (cls[w] != cls[v] && colour[w] == colour[v] && vgreater(key, w, (int32_t)v)) { S[v] = 1; break; }
        }
    }
    for (int64_t v = 0; v < n; v++)
        if (S[v]) colour[v] = 0;
    lf_col(n, rp, ci, S, cls, 0, key, colour);           /* recolour V' against G */
    free(cls);
    free(S);
}

/* ------------------------------------------------------------------ §SPEC the paper's subroutines */
#define OR_F_COLOR_EB 0x100u  /* colouring subroutine: edge-based speculative colouring */
#define OR_F_COLOR_VB 0x200u  /* colouring subroutine: vertex-based speculative colouring */

/* Speculative colouring rounds as P:216-218 describes Deveci et al. [10], on the
   admitted arcs (admit as in admitted()), with a colour window of W colours (EB: W = 32,
   "a 32 bit integer is used to represent the availability of the colors"; VB: the
   FORBIDDEN array, W = the average degree of the graph being coloured).  C holds
   the colours (0 = uncoloured; every vertex with C = 0 takes part, the others are
   fixed until reset); base[v] = the first colour of v's window (1 on entry).  A round,
   synchronous (every step reads the state the previous step left):
     1. every uncoloured v takes the smallest colour in [base_v, base_v + W) that no
        admitted neighbour holds; if there is none, base_v += W ("OFFSET") and v waits;
     2. every admitted edge whose endpoints share a colour resets its LOWER-id endpoint
        ("the color of the endpoint with the lowest id is reset"; VB's choice is
        not stated -- reading: the same rule);
   until every vertex is coloured.  Returns the rounds. */
static int spec_col(int64_t n, const int64_t *rp, const int32_t *ci, const uint32_t *cls, int admit, uint32_t W,
                    uint32_t *C, uint32_t *base) {
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint32_t *T = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    uint8_t *R = (uint8_t *)calloc(nn, 1);
    uint8_t *mark = (uint8_t *)malloc((size_t)W + 1);
    int rounds = 0;
    for (;;) {
        int64_t left = 0;
        for (int64_t v = 0; v < n; v++) left += C[v] == 0;
        if (!left) break;
        rounds++;
        for (int64_t v = 0; v < n; v++) {         /* step 1 (from the snapshot C) */
            T[v] = C[v];
            if (C[v] != 0) continue;
            memset(mark, 0, (size_t)W);
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (!admitted(admit, cls[v], cls[w])) continue;
                if (C[w] >= base[v] && C[w] - base[v] < W) mark[C[w] - base[v]] = 1;
            }
            uint32_t i = 0;
            while (i < W && mark[i]) i++;
            if (i < W) T[v] = base[v] + i;
            else base[v] += W;
        }
        memcpy(C, T, sizeof(uint32_t) * (size_t)n);
        for (int64_t v = 0; v < n; v++) {         /* step 2 (from the new snapshot) */
            if (C[v] == 0) continue;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (w > v && C[w] == C[v] && admitted(admit, cls[v], cls[w])) { R[v] = 1; break; }
            }
        }
        for (int64_t v = 0; v < n; v++)
            if (R[v]) { C[v] = 0; R[v] = 0; }
    }
    free(T);
    free(R);
    free(mark);
    return rounds;
}

/* COLOR-Degk's literal G_L step (Alg 9 l.6): every V_L vertex starts with colour
   M+1; then, in synchronous rounds, the lower-id endpoint of every G_L edge whose ends
   share a colour takes the smallest colour of the (k+1)-slot FORBIDDEN palette
   M+1 .. M+k+1 not held by a G_L neighbour ("vertices that have a color conflict use the
   FORBIDDEN array to obtain a new color ... this process repeats in iteration until all
   vertices in G_L are validly colored"; which endpoint moves is not stated -- reading:
   the lower id, as in EB).  A free slot always exists (deg <= k).  Returns the rounds. */
static int gl_loop(int64_t n, const int64_t *rp, const int32_t *ci, const uint32_t *cls, uint32_t k, uint32_t M,
                   uint32_t *C) {
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint32_t *T = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    uint8_t *mark = (uint8_t *)malloc((size_t)k + 2);
    int rounds = 0;
    for (int64_t v = 0; v < n; v++)
        if (cls[v] == 0) C[v] = M + 1;
    for (;;) {
        int64_t moved = 0;
        for (int64_t v = 0; v < n; v++) {
            T[v] = C[v];
            if (cls[v] != 0) continue;
            int conf = 0;
            for (int64_t e = rp[v]; e < rp[v + 1] && !conf; e++)
                conf = cls[ci[e]] == 0 && ci[e] > v && C[ci[e]] == C[v];
            if (!conf) continue;
            memset(mark, 0, (size_t)k + 2);
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (cls[w] == 0 && C[w] > M && C[w] - M <= k + 1) mark[C[w] - M] = 1;
            }
            uint32_t c = 1;
            while (c <= k + 1 && mark[c]) c++;
            T[v] = M + c;
            moved++;
        }
        if (!moved) break;
        rounds++;
        memcpy(C, T, sizeof(uint32_t) * (size_t)n);
    }
    free(T);
    free(mark);
    return rounds;
}

/* the colour window: EB 32 bits; VB the average degree of the graph being coloured
   (admitted arcs / n, at least 1, at most 1024) */
static uint32_t spec_window(int64_t n, const int64_t *rp, const int32_t *ci, const uint32_t *cls, int admit, int vb) {
    if (!vb) return 32;
    int64_t a = 0;
    for (int64_t v = 0; v < n; v++)
        for (int64_t e = rp[v]; e < rp[v + 1]; e++) a += admitted(admit, cls[v], cls[ci[e]]);
    int64_t w = n > 0 ? a / n : 1;
    return (uint32_t)(w < 1 ? 1 : (w > 1024 ? 1024 : w));
}

/* COLOR flows with the paper's own subroutines (flags COLOR_EB / COLOR_VB; f3):
   the same flows as or_color with speculative colouring in place of LF-COL:
   NONE: spec(V, E).  RAND: C_IS = spec(V, intra); V' = both ends of monochromatic cross
   edges (or the lower ends with LOWER_ONLY); V' uncoloured; spec(all arcs) recolours
   every uncoloured vertex (a reset may uncolour a vertex outside V', which is then
   recoloured too).  DEGK: C_H = spec(V_H, E_H) with V_L held at colour 0 but not
   admitted (same-class arcs only, V_L coloured later); M = max C_H; then the literal
   G_L loop gl_loop.  W: EB 32; VB max(1, admitted arcs / n) of the graph being
   coloured.  Returns 0 (the rounds are not reported). */
void or_color_spec(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
                   uint32_t flags, uint32_t *colour) {
    uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, 0);
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    uint32_t *base = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    or_classes(n, rp, ci, kind, param, seed, cls);
    int vb = (flags & OR_F_COLOR_VB) != 0;
    for (int64_t v = 0; v < n; v++) {
        colour[v] = 0;
        base[v] = 1;
    }
    if (kind == OR_NONE) {
        spec_col(n, rp, ci, cls, 0, spec_window(n, rp, ci, cls, 0, vb), colour, base);
    } else if (kind == OR_DEGK) {
        /* C_H on G_H: V_L vertices are parked at a colour no H vertex can see (same-class
           arcs only) and excluded from the rounds by a temporary non-zero colour */
        for (int64_t v = 0; v < n; v++)
            if (cls[v] == 0) colour[v] = 0xFFFFFFFFu;
        spec_col(n, rp, ci, cls, 3, spec_window(n, rp, ci, cls, 3, vb), colour, base);
        uint32_t M = 0;
        for (int64_t v = 0; v < n; v++)
            if (cls[v] == 1 && colour[v] > M) M = colour[v];
        gl_loop(n, rp, ci, cls, param, M, colour);
    } else {
        spec_col(n, rp, ci, cls, 1, spec_window(n, rp, ci, cls, 1, vb), colour, base);  /* C_IS */
        uint8_t *S = (uint8_t *)calloc(nn, 1);
        for (int64_t v = 0; v < n; v++)
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (cls[w] != cls[v] && colour[w] == colour[v] &&
                    (!(flags & OR_F_LOWER_ONLY) || vgreater(key, w, (int32_t)v))) { S[v] = 1; break; }
            }
        for (int64_t v = 0; v < n; v++) {
            if (S[v]) colour[v] = 0;
            base[v] = 1;
        }
        spec_col(n, rp, ci, cls, 0, spec_window(n, rp, ci, cls, 0, vb), colour, base);  /* recolour against G */
        free(S);
    }
    free(cls);
    free(base);
}

/* ------------------------------------------------------------------ §ORD JP vertex orderings */
#define OR_F_ORDER_LF 0x400u  /* JP priority: largest degree first (Hasenplaugh et al. [14]) */
#define OR_F_ORDER_SF 0x800u  /* JP priority: smallest degree first ([14]) */

/* the (degree, pv, id) order of the colouring: LF compares the degree in G first
   (larger first), SF the degree (smaller first); ties by (pv, id) as everywhere */
static const int64_t *g_ord_rp;
static uint32_t g_ord_flags;
static int ord_greater(uint64_t key, int32_t a, int32_t b) {
    int64_t da = g_ord_rp[a + 1] - g_ord_rp[a], db = g_ord_rp[b + 1] - g_ord_rp[b];
    if (da != db) return (g_ord_flags & OR_F_ORDER_LF) ? da > db : da < db;
    return vgreater(key, a, b);
}
static int cmp_ord_desc(const void *x, const void *y) {
    int32_t a = *(const int32_t *)x, b = *(const int32_t *)y;
    if (a == b) return 0;
    return ord_greater(g_sort_key, a, b) ? -1 : 1;
}

/* LF-COL in the (degree, pv, id) order: first fit over the coloured admitted neighbours */
static void lf_col_ord(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *inS, const uint32_t *cls,
                       int admit, uint64_t key, uint32_t *C) {
    int64_t c = 0, maxd = 0;
    for (int64_t v = 0; v < n; v++) {
        c += inS[v] ? 1 : 0;
        if (rp[v + 1] - rp[v] > maxd) maxd = rp[v + 1] - rp[v];
    }
    int32_t *order = (int32_t *)malloc(sizeof(int32_t) * (size_t)(c > 0 ? c : 1));
    c = 0;
    for (int64_t v = 0; v < n; v++)
        if (inS[v]) order[c++] = (int32_t)v;
    g_sort_key = key;
    qsort(order, (size_t)c, sizeof(int32_t), cmp_ord_desc);
    uint8_t *mark = (uint8_t *)malloc((size_t)maxd + 2);
    for (int64_t i = 0; i < c; i++) C[order[i]] = mex_colour(rp, ci, order[i], cls, admit, C, mark);
    free(mark);
    free(order);
}

/* COLOR flows of or_color with JP's priority order replaced by LF / SF (the degree of
   the vertex in G; FIXED hash ties); COLOR-Rand's lower-endpoint variant compares in
   the same order.  Hasenplaugh et al. run JP with these orderings. */
void or_color_ord(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
                  uint32_t flags, uint32_t *colour) {
    uint64_t key = or_stream_key(seed, OR_TAG_VERTEX, 0);
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    uint8_t *S = (uint8_t *)calloc(nn, 1);
    g_ord_rp = rp;
    g_ord_flags = flags;
    or_classes(n, rp, ci, kind, param, seed, cls);
    for (int64_t v = 0; v < n; v++) colour[v] = 0;
    if (kind == OR_NONE) {
        for (int64_t v = 0; v < n; v++) S[v] = 1;
        lf_col_ord(n, rp, ci, S, cls, 0, key, colour);
    } else if (kind == OR_DEGK) {
        uint32_t *CL = (uint32_t *)calloc(nn, sizeof(uint32_t));
        for (int64_t v = 0; v < n; v++) S[v] = cls[v] == 1;
        lf_col_ord(n, rp, ci, S, cls, 1, key, colour);
        uint32_t M = 0;
        for (int64_t v = 0; v < n; v++)
            if (cls[v] == 1 && colour[v] > M) M = colour[v];
        for (int64_t v = 0; v < n; v++) S[v] = cls[v] == 0;
        lf_col_ord(n, rp, ci, S, cls, 1, key, CL);
        for (int64_t v = 0; v < n; v++)
            if (cls[v] == 0) colour[v] = M + CL[v];
        free(CL);
    } else {
        for (int64_t v = 0; v < n; v++) S[v] = 1;
        lf_col_ord(n, rp, ci, S, cls, 1, key, colour);
        for (int64_t v = 0; v < n; v++) {
            S[v] = 0;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (cls[w] != cls[v] && colour[w] == colour[v] &&
                    (!(flags & OR_F_LOWER_ONLY) || ord_greater(key, w, (int32_t)v))) { S[v] = 1; break; }
            }
        }
        for (int64_t v = 0; v < n; v++)
            if (S[v]) colour[v] = 0;
        lf_col_ord(n, rp, ci, S, cls, 0, key, colour);
    }
    free(cls);
    free(S);
}
