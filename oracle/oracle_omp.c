/*
 * oracle/oracle_omp.c -- CPU ORACLE, literal ROUND-BASED forms on all host cores
 * (OpenMP).  TEST INFRASTRUCTURE ONLY, like oracle.c: only tests/ and bench.py's
 * cpu_baseline / --impl reference legs may load it; the product never does.
 *
 * What it is: the paper's parallel algorithms written as synchronous rounds, the way
 * the paper states them, with the FIXED priorities of DESIGN §3 H (the hash helpers,
 * the decomposition classes and the admitted-arc predicate are oracle.c's, linked
 * into the same library):
 *   LubyMIS  every round, from a snapshot: an undecided vertex with an
 *                          In neighbour -> Out; one whose (pv, id) beats every
 *                          undecided neighbour -> In.
 *   LMAX / GM  every round: each free vertex picks its heaviest edge
 *                          (pe, other id) to a free neighbour; mutual picks match.
 *   JP      level by level: a vertex whose higher neighbours are all
 *                          coloured takes the smallest colour >= 1 not used by its
 *                          coloured neighbours (readiness by counters of uncoloured
 *                          higher neighbours, so each level touches only its vertices).
 * and the decomposition flows of oracle.c (MIS-Deg2 P:288, MIS-Rand P:286, MM-Rand
 * Alg 5, MM-Degk Alg 6, COLOR-Degk Alg 9, COLOR-Rand Alg 8) in the same phase order.
 * With fixed priorities each round form reaches the sequential greedy result
 * (Blelloch et al. [6]), so every output must equal or_mis /
 * or_mm / or_color bit for bit -- pinned in tests/test_oracle_omp.py.  Rounds are
 * synchronous (every decision of a round reads the previous round's state), so the
 * result does not depend on the thread count.
 *
 * This is the all-core CPU baseline of BASELINE.md §3 ("oracle_rounds_omp"); it is
 * not tuned beyond running each round's vertex loop in parallel.
 */
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* from oracle.c (same library) */
uint64_t or_stream_key(uint64_t seed, uint32_t tag, uint32_t round);
uint32_t or_pv(uint64_t key, uint32_t v);
uint32_t or_pe(uint64_t key, uint32_t lo, uint32_t hi);
void or_classes(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
                uint32_t *cls);

enum { K_NONE = 0, K_RAND = 1, K_DEGK = 2, K_BRIDGE = 3 };
enum { UNDEC = 0, IN = 1, OUT = 2 };

static int vgt(uint64_t key, int32_t a, int32_t b) { /* (pv, id) order */
    uint32_t pa = or_pv(key, (uint32_t)a), pb = or_pv(key, (uint32_t)b);
    return pa != pb ? pa > pb : a > b;
}

static int adm(int admit, uint32_t cu, uint32_t cw) { /* same codes as oracle.c admitted() */
    switch (admit) {
    case 0: return 1;
    case 1: return cu == cw;
    case 2: return cu != cw;
    case 3: return cu == 1 && cw == 1;
    case 4: return cu == 0 || cw == 0;
    }
    return 0;
}

int oro_threads(void) { return omp_get_max_threads(); }

/* ------------------------------------------------------------------ LubyMIS rounds */
/* MIS of G[S] by synchronous Luby rounds; st[v] for v in S: UNDEC on entry -> IN/OUT.
   Vertices outside S are not in the phase graph.  Returns the number of rounds. */
static int luby_rounds(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *S, uint64_t key,
                       uint8_t *st) {
    int32_t *fr = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    int32_t *nx = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    uint8_t *dec = (uint8_t *)malloc((size_t)(n > 0 ? n : 1));
    int64_t cnt = 0;
    for (int64_t v = 0; v < n; v++)
        if (S[v] && st[v] == UNDEC) fr[cnt++] = (int32_t)v;
    int rounds = 0;
    while (cnt > 0) {
        /* decisions from the snapshot st (written to dec, applied after the round) */
#pragma omp parallel for schedule(dynamic, 256)
        for (int64_t i = 0; i < cnt; i++) {
            int32_t v = fr[i];
            int has_in = 0, is_max = 1;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (!S[w]) continue;
                if (st[w] == IN) { has_in = 1; break; }
                if (st[w] == UNDEC && vgt(key, w, v)) is_max = 0;
            }
            dec[v] = has_in ? OUT : (is_max ? IN : UNDEC);
        }
        int64_t k = 0;
        for (int64_t i = 0; i < cnt; i++) {
            int32_t v = fr[i];
            st[v] = dec[v];
            if (dec[v] == UNDEC) nx[k++] = v;
        }
        int32_t *t = fr;
        fr = nx;
        nx = t;
        cnt = k;
        rounds++;
    }
    free(fr);
    free(nx);
    free(dec);
    return rounds;
}

/* MIS flows (oracle.c or_mis): NONE LubyMIS; DEGK MIS-Deg2; RAND MIS-Rand. */
void oro_mis(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
             uint8_t *in_set) {
    uint64_t key = or_stream_key(seed, 1, 0);
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    uint8_t *S = (uint8_t *)malloc(nn), *st = (uint8_t *)calloc(nn, 1);
    or_classes(n, rp, ci, kind, param, seed, cls);
    if (kind == K_NONE) {
        memset(S, 1, nn);
        luby_rounds(n, rp, ci, S, key, st);
    } else {
        /* first phase: V_L (DEGk) / the partition interiors V \ B (RAND) */
#pragma omp parallel for schedule(dynamic, 4096)
        for (int64_t v = 0; v < n; v++) {
            if (kind == K_DEGK) {
                S[v] = cls[v] == 0;
            } else {
                S[v] = 1;
                for (int64_t e = rp[v]; e < rp[v + 1]; e++)
                    if (cls[ci[e]] != cls[v]) { S[v] = 0; break; }
            }
        }
        luby_rounds(n, rp, ci, S, key, st);
        /* fix-up: the rest minus the neighbours of the first phase's In vertices */
        uint8_t *X = (uint8_t *)malloc(nn);
#pragma omp parallel for schedule(dynamic, 4096)
        for (int64_t v = 0; v < n; v++) {
            X[v] = 0;
            if (S[v]) continue;
            int killed = 0;
            for (int64_t e = rp[v]; e < rp[v + 1] && !killed; e++) killed = S[ci[e]] && st[ci[e]] == IN;
            if (killed) st[v] = OUT;
            else X[v] = 1;
        }
        luby_rounds(n, rp, ci, X, key, st);
        free(X);
    }
    for (int64_t v = 0; v < n; v++) in_set[v] = st[v] == IN;
    free(cls);
    free(S);
    free(st);
}

/* ------------------------------------------------------------------ LMAX rounds */
/* handshake rounds on the admitted edges among free vertices; returns rounds */
static int lmax_rounds(int64_t n, const int64_t *rp, const int32_t *ci, const uint32_t *cls, int admit,
                       uint64_t key, int32_t *mate) {
    int32_t *pick = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    int32_t *fr = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    int64_t cnt = 0;
    for (int64_t v = 0; v < n; v++) {
        pick[v] = -1;
        if (mate[v] < 0) fr[cnt++] = (int32_t)v;
    }
    int rounds = 0;
    for (;;) {
        int64_t live = 0;
#pragma omp parallel for schedule(dynamic, 256) reduction(+ : live)
        for (int64_t i = 0; i < cnt; i++) {
            int32_t v = fr[i];
            uint64_t best = 0;
            int32_t p = -1;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (mate[w] >= 0 || !adm(admit, cls[v], cls[w])) continue;
                uint32_t lo = v < w ? (uint32_t)v : (uint32_t)w, hi = v < w ? (uint32_t)w : (uint32_t)v;
                uint64_t k = ((uint64_t)or_pe(key, lo, hi) << 32) | (uint32_t)w;
                if (p < 0 || k > best) { best = k; p = w; }
            }
            pick[v] = p;
            live += p >= 0;
        }
        if (!live) break;
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < cnt; i++) {
            int32_t v = fr[i];
            if (pick[v] >= 0 && pick[pick[v]] == v) mate[v] = pick[v];
        }
        int64_t k = 0;
        for (int64_t i = 0; i < cnt; i++) {
            int32_t v = fr[i];
            if (mate[v] < 0 && pick[v] >= 0) fr[k++] = v; /* dead vertices (no pick) leave */
            pick[v] = -1;
        }
        cnt = k;
        rounds++;
    }
    free(pick);
    free(fr);
    return rounds;
}

/* MM flows (oracle.c or_mm): NONE LMAX; RAND MM-Rand (Alg 5); DEGK MM-Degk (Alg 6). */
void oro_mm(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
            int32_t *mate) {
    uint64_t key = or_stream_key(seed, 2, 0);
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(n > 0 ? n : 1));
    or_classes(n, rp, ci, kind, param, seed, cls);
    for (int64_t v = 0; v < n; v++) mate[v] = -1;
    if (kind == K_NONE) {
        lmax_rounds(n, rp, ci, cls, 0, key, mate);
    } else if (kind == K_RAND || kind == K_BRIDGE) {
        lmax_rounds(n, rp, ci, cls, 1, key, mate); /* intra edges */
        lmax_rounds(n, rp, ci, cls, 2, key, mate); /* cross edges among unmatched */
    } else {
        lmax_rounds(n, rp, ci, cls, 3, key, mate); /* G_H */
        lmax_rounds(n, rp, ci, cls, 4, key, mate); /* G_L u G_C among unmatched */
    }
    free(cls);
}

/* ------------------------------------------------------------------ JP levels */
/* JP on S over the admitted arcs; C holds the fixed colours of vertices outside S
   (0 = none) and 0 on S.  Level by level: the ready vertices (all higher admitted
   S-neighbours coloured) take the mex of their coloured admitted neighbours, then
   count down their lower S-neighbours.  Returns the number of levels. */
static int jp_levels(int64_t n, const int64_t *rp, const int32_t *ci, const uint8_t *S, const uint32_t *cls,
                     int admit, uint64_t key, uint32_t *C) {
    size_t nn = (size_t)(n > 0 ? n : 1);
    int64_t *pend = (int64_t *)malloc(sizeof(int64_t) * nn);
    int32_t *fr = (int32_t *)malloc(sizeof(int32_t) * nn), *nx = (int32_t *)malloc(sizeof(int32_t) * nn);
    int64_t cnt = 0;
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t v = 0; v < n; v++) {
        int64_t h = 0;
        if (S[v])
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                h += S[w] && adm(admit, cls[v], cls[w]) && vgt(key, w, (int32_t)v);
            }
        pend[v] = h;
    }
    int64_t maxd = 0;
    for (int64_t v = 0; v < n; v++) {
        if (S[v] && pend[v] == 0) fr[cnt++] = (int32_t)v;
        if (rp[v + 1] - rp[v] > maxd) maxd = rp[v + 1] - rp[v];
    }
    const int nt = omp_get_max_threads();
    uint8_t *marks = (uint8_t *)malloc((size_t)nt * (size_t)(maxd + 2)); /* one mex scratch per thread */
    int levels = 0;
    while (cnt > 0) {
        int64_t k = 0;
#pragma omp parallel
        {
            uint8_t *mark = marks + (size_t)omp_get_thread_num() * (size_t)(maxd + 2);
#pragma omp for schedule(dynamic, 64)
            for (int64_t i = 0; i < cnt; i++) {
                int32_t v = fr[i];
                int64_t d = rp[v + 1] - rp[v];
                memset(mark, 0, (size_t)d + 2);
                for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                    int32_t w = ci[e];
                    if (!adm(admit, cls[v], cls[w])) continue;
                    if (S[w] && !vgt(key, w, v)) continue; /* lower S-neighbours: not yet coloured */
                    if (C[w] != 0 && (int64_t)C[w] <= d + 1) mark[C[w]] = 1;
                }
                uint32_t c = 1;
                while (mark[c]) c++;
                C[v] = c;
            }
        }
        /* count down the lower S-neighbours; the ones reaching 0 form the next level */
#pragma omp parallel for schedule(dynamic, 64)
        for (int64_t i = 0; i < cnt; i++) {
            int32_t v = fr[i];
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (!S[w] || !adm(admit, cls[v], cls[w]) || !vgt(key, v, w)) continue;
                if (__atomic_sub_fetch(&pend[w], 1, __ATOMIC_RELAXED) == 0)
                    nx[__atomic_fetch_add(&k, 1, __ATOMIC_RELAXED)] = w;
            }
        }
        int32_t *t = fr;
        fr = nx;
        nx = t;
        cnt = k;
        levels++;
    }
    free(marks);
    free(pend);
    free(fr);
    free(nx);
    return levels;
}

/* COLOR flows (oracle.c or_color): NONE JP; DEGK COLOR-Degk (Alg 9); RAND COLOR-Rand (Alg 8). */
void oro_color(int64_t n, const int64_t *rp, const int32_t *ci, int kind, uint32_t param, uint64_t seed,
               uint32_t *colour) {
    uint64_t key = or_stream_key(seed, 1, 0);
    size_t nn = (size_t)(n > 0 ? n : 1);
    uint32_t *cls = (uint32_t *)malloc(sizeof(uint32_t) * nn);
    uint8_t *S = (uint8_t *)malloc(nn);
    or_classes(n, rp, ci, kind, param, seed, cls);
    for (int64_t v = 0; v < n; v++) colour[v] = 0;
    if (kind == K_NONE) {
        memset(S, 1, nn);
        jp_levels(n, rp, ci, S, cls, 0, key, colour);
    } else if (kind == K_DEGK) {
        uint32_t *CL = (uint32_t *)calloc(nn, sizeof(uint32_t));
        for (int64_t v = 0; v < n; v++) S[v] = cls[v] == 1;
        jp_levels(n, rp, ci, S, cls, 1, key, colour); /* C_H on G_H */
        uint32_t M = 0;
        for (int64_t v = 0; v < n; v++)
            if (cls[v] == 1 && colour[v] > M) M = colour[v];
        for (int64_t v = 0; v < n; v++) S[v] = cls[v] == 0;
        jp_levels(n, rp, ci, S, cls, 1, key, CL); /* C_L on G_L */
        for (int64_t v = 0; v < n; v++)
            if (cls[v] == 0) colour[v] = M + CL[v];
        free(CL);
    } else {
        memset(S, 1, nn);
        jp_levels(n, rp, ci, S, cls, 1, key, colour); /* C_IS on the induced subgraphs */
#pragma omp parallel for schedule(dynamic, 4096)
        for (int64_t v = 0; v < n; v++) { /* V' = both ends of monochromatic cross edges */
            S[v] = 0;
            for (int64_t e = rp[v]; e < rp[v + 1]; e++) {
                int32_t w = ci[e];
                if (cls[w] != cls[v] && colour[w] == colour[v]) { S[v] = 1; break; }
            }
        }
        for (int64_t v = 0; v < n; v++)
            if (S[v]) colour[v] = 0;
        jp_levels(n, rp, ci, S, cls, 0, key, colour); /* recolour V' against G */
    }
    free(cls);
    free(S);
}
