/*
 * synth.c - seeded synthetic inputs for the graph-H2TAP update path.
 *
 * This module is the ONLY code shared by the CUDA path and the oracle. It holds
 * no arithmetic of the method (no sorting, dedup, merge, CSR building): it only
 * draws graphs and update streams from a counter-based generator so that any
 * slice can be regenerated independently (SURVEY.md §8(d) "Concrete synthetic
 * inputs").
 *
 * Workload shapes:
 *  - RMAT (Graph500 parameters A,B,C,D = 0.57,0.19,0.19,0.05), vertex labels
 *    scrambled by a seeded bijection of [0, 2^scale), weights w = (r>>40)*2^-24
 *    (exactly representable in f32).  Configs C1 (scale 16), C3 (scale 24).
 *  - RMAT update batches: p_insert EDGE_INSERT of RMAT-sampled pairs, the rest
 *    EDGE_DELETE of uniformly chosen edges of the initial edge list, optional
 *    EDGE_WEIGHT and repeated keys (parity variant); timestamps monotone with a
 *    window-64 local shuffle; ops_per_txn ops share one timestamp.
 *  - LDBC-SNB-shaped property graph (config C2): 65,536 "Person" hubs with a
 *    heavy-tailed out-degree and low-degree "Message" vertices (out-degree 4);
 *    sparse u64 external IDs (type << 56) | index.  Update stream from the
 *    paper's query mix 66% insert relationship / 22% insert node / 11% delete
 *    relationship / 1% delete node (§6.3; query shapes
 *    §6.2).
 */
#include <stdint.h>
#include <stddef.h>
#include <string.h>

#define SYNTH_NODE_INSERT 0
#define SYNTH_NODE_DELETE 1
#define SYNTH_EDGE_INSERT 2
#define SYNTH_EDGE_DELETE 3
#define SYNTH_EDGE_WEIGHT 4

/* ---------------------------------------------------------------- RNG ---- */
static inline uint64_t sm64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}
/* counter-based: value depends only on (seed, stream, index) */
uint64_t synth_rand(uint64_t seed, uint64_t stream, uint64_t index) {
    return sm64(sm64(seed ^ sm64(stream * 0xD1B54A32D192ED03ull)) + index);
}
static inline double u01(uint64_t r) { return (double)(r >> 11) * (1.0 / 9007199254740992.0); }
static inline float weight_of(uint64_t r) { return (float)(r >> 40) * (1.0f / 16777216.0f); }

/* --------------------------------------------------- RMAT + scrambling ---- */
/* seeded bijection of [0, 2^scale): odd multiply / xor / rotate rounds mod 2^scale */
uint64_t synth_scramble(int scale, uint64_t seed, uint64_t v) {
    if (scale <= 0) return 0;
    const uint64_t mask = (scale >= 64) ? ~0ull : ((1ull << scale) - 1);
    uint64_t k1 = synth_rand(seed, 0x5C4A, 1) | 1ull, k2 = synth_rand(seed, 0x5C4A, 2);
    uint64_t k3 = synth_rand(seed, 0x5C4A, 3) | 1ull, k4 = synth_rand(seed, 0x5C4A, 4);
    uint64_t x = v & mask;
    x = (x * k1) & mask;
    x ^= k2 & mask;
    if (scale > 1) { int r = scale / 2; x = ((x << r) | (x >> (scale - r))) & mask; }
    x = (x * k3) & mask;
    x ^= k4 & mask;
    return x;
}

/* one RMAT pair for counter (stream, i); 16 bits of randomness per level */
static inline void rmat_pair(int scale, uint64_t seed, uint64_t stream, uint64_t i,
                             uint64_t* s, uint64_t* d) {
    const uint32_t tA = (uint32_t)(0.57 * 65536.0), tB = (uint32_t)(0.76 * 65536.0),
                   tC = (uint32_t)(0.95 * 65536.0);
    uint64_t u = 0, v = 0, r = 0;
    for (int lvl = 0; lvl < scale; ++lvl) {
        if ((lvl & 3) == 0) r = synth_rand(seed, stream, i * 16 + (uint64_t)(lvl >> 2));
        uint32_t q = (uint32_t)((r >> ((lvl & 3) * 16)) & 0xFFFF);
        uint64_t bu = 0, bv = 0;
        if (q < tA) { bu = 0; bv = 0; }
        else if (q < tB) { bu = 0; bv = 1; }
        else if (q < tC) { bu = 1; bv = 0; }
        else { bu = 1; bv = 1; }
        u = (u << 1) | bu;
        v = (v << 1) | bv;
    }
    *s = synth_scramble(scale, seed, u);
    *d = synth_scramble(scale, seed, v);
}

/* initial RMAT edge list slice [first, first+n) of stream 1 */
void synth_rmat_edges(int scale, uint64_t seed, uint64_t first, uint64_t n,
                      uint64_t* src, uint64_t* dst, float* w) {
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < (int64_t)n; ++k) {
        uint64_t i = first + (uint64_t)k;
        rmat_pair(scale, seed, 1, i, &src[k], &dst[k]);
        if (w) w[k] = weight_of(synth_rand(seed, 2, i));
    }
}

/* window-64 local shuffle of a monotone sequence: bijection of [0,64) per window */
static inline uint64_t shuffled_slot(uint64_t seed, uint64_t batch, uint64_t t) {
    uint64_t win = t >> 6, x = t & 63;
    uint64_t r = synth_rand(seed, 0x7500 + batch, win);
    uint64_t a = (r & 63) | 1, b = (r >> 8) & 63;
    return (win << 6) | ((a * x + b) & 63);
}

/*
 * RMAT update batch k.  Op i draws its kind from (p_insert, p_weight, rest =
 * delete); inserts are RMAT pairs of stream 100+k, deletes and weight updates
 * pick a uniformly random edge of the initial list (m_initial edges, stream 1)
 * so they mostly hit existing edges; with probability p_repeat the op reuses
 * the key of an earlier op of the same batch.  Ops are grouped into
 * transactions of ops_per_txn consecutive ops sharing one timestamp
 * ts = ts_base + 1 + shuffled(txn).
 */
void synth_rmat_batch(int scale, uint64_t seed, uint64_t k, uint64_t n, uint64_t m_initial,
                      double p_insert, double p_weight, double p_repeat, uint64_t ops_per_txn,
                      uint64_t ts_base, uint8_t* kind, uint64_t* src, uint64_t* dst, float* w,
                      uint64_t* ts) {
    if (ops_per_txn == 0) ops_per_txn = 1;
    for (uint64_t i = 0; i < n; ++i) {
        uint64_t r = synth_rand(seed, 200 + k, i);
        double c = u01(r);
        uint8_t kd = c < p_insert ? SYNTH_EDGE_INSERT
                   : (c < p_insert + p_weight ? SYNTH_EDGE_WEIGHT : SYNTH_EDGE_DELETE);
        uint64_t r2 = synth_rand(seed, 300 + k, i);
        if (i > 0 && p_repeat > 0 && u01(synth_rand(seed, 400 + k, i)) < p_repeat) {
            uint64_t j = r2 % i;
            src[i] = src[j];
            dst[i] = dst[j];
        } else if (kd == SYNTH_EDGE_INSERT || m_initial == 0) {
            rmat_pair(scale, seed, 100 + k, i, &src[i], &dst[i]);
        } else {
            uint64_t e = r2 % m_initial;
            rmat_pair(scale, seed, 1, e, &src[i], &dst[i]);
        }
        kind[i] = kd;
        w[i] = weight_of(synth_rand(seed, 500 + k, i));
        ts[i] = ts_base + 1 + shuffled_slot(seed, k, i / ops_per_txn);
    }
}

/* ---------------------------------------------------- LDBC-SNB shape ---- */
/* vertices: messages (1<<56)|m, persons (2<<56)|p; ascending (messages first).  The
 * Person type code is the larger one so that a new Person's ID (2<<56)|(n_person + j)
 * exceeds every existing ID, as Algorithm 2 assumes of new nodes. */
#define LDBC_MSG(m)    ((1ull << 56) | (uint64_t)(m))
#define LDBC_PERSON(p) ((2ull << 56) | (uint64_t)(p))

void synth_ldbc_vertices(uint64_t n_person, uint64_t n_msg, uint64_t* ids) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < (int64_t)(n_person + n_msg); ++i)
        ids[i] = (uint64_t)i < n_msg ? LDBC_MSG(i) : LDBC_PERSON((uint64_t)i - n_msg);
}

/* heavy-tailed person index: P(p) ~ p^(-2/3) (hub-first); lodeg mirrors it */
static inline uint64_t skewed_person(uint64_t n_person, uint64_t r, int lodeg) {
    double u = u01(r);
    uint64_t p = (uint64_t)((double)n_person * u * u * u);
    if (p >= n_person) p = n_person - 1;
    return lodeg ? n_person - 1 - p : p;
}

/*
 * LDBC-shaped edge e of the initial graph.  e < e_person: person -> (70% message
 * "likes", 30% person "knows"), source heavy-tailed; else message (e-e_person)/4
 * -> (50% person "hasCreator", 50% message "replyOf").
 */
static inline void ldbc_edge(uint64_t n_person, uint64_t n_msg, uint64_t e_person, uint64_t seed,
                             uint64_t e, uint64_t* s, uint64_t* d) {
    uint64_t r1 = synth_rand(seed, 11, e), r2 = synth_rand(seed, 12, e);
    if (e < e_person) {
        *s = LDBC_PERSON(skewed_person(n_person, r1, 0));
        *d = (r2 & 1023) < 717 ? LDBC_MSG((r2 >> 10) % n_msg) : LDBC_PERSON((r2 >> 10) % n_person);
    } else {
        uint64_t m = (e - e_person) >> 2;
        *s = LDBC_MSG(m % n_msg);
        *d = (r2 & 1) ? LDBC_PERSON((r2 >> 1) % n_person) : LDBC_MSG((r2 >> 1) % n_msg);
    }
}

void synth_ldbc_edges(uint64_t n_person, uint64_t n_msg, uint64_t e_person, uint64_t seed,
                      uint64_t first, uint64_t n, uint64_t* src, uint64_t* dst, float* w) {
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < (int64_t)n; ++k) {
        uint64_t e = first + (uint64_t)k;
        ldbc_edge(n_person, n_msg, e_person, seed, e, &src[k], &dst[k]);
        if (w) w[k] = weight_of(synth_rand(seed, 13, e));
    }
}

/*
 * LDBC-shaped update batch k: transactions drawn from the query mix until n_cap
 * ops are produced (returns the op count).  Each transaction has one commit
 * timestamp ts_base + 1 + txn.  Shapes:
 *   insert rel  : EDGE_INSERT person -> message
 *   insert node : NODE_INSERT new person, EDGE_INSERT existing person -> new
 *   delete rel  : EDGE_DELETE of an initial person edge
 *   delete node : NODE_DELETE person (+ the library cascades its relationships)
 * New person IDs are (2<<56) | (n_person + k*n_cap + txn): above every existing ID
 * (messages carry the smaller type code), as the paper's Algorithm 2 assumes of new
 * nodes.  Node deletes pick hubs first (the paper's HiDeg window,
 * P:L978-988), so every cycle cascades thousands of edges and the graph shrinks from
 * batch to batch (bench.py reports E before and after the timed region).
 */
uint64_t synth_ldbc_batch(uint64_t n_person, uint64_t n_msg, uint64_t e_person, uint64_t seed,
                          uint64_t k, uint64_t n_cap, int lodeg, uint64_t ts_base,
                          uint8_t* kind, uint64_t* src, uint64_t* dst, float* w, uint64_t* ts) {
    uint64_t n = 0, txn = 0;
    while (n + 2 <= n_cap) {
        uint64_t r = synth_rand(seed, 600 + k, txn), r2 = synth_rand(seed, 700 + k, txn);
        uint64_t q = r % 100;
        uint64_t t = ts_base + 1 + txn;
        float wt = weight_of(synth_rand(seed, 800 + k, txn));
        if (q < 66) {
            kind[n] = SYNTH_EDGE_INSERT;
            src[n] = LDBC_PERSON(skewed_person(n_person, r2, lodeg));
            dst[n] = LDBC_MSG((r2 >> 20) % n_msg);
            w[n] = wt; ts[n] = t; ++n;
        } else if (q < 88) {
            uint64_t nid = LDBC_PERSON(n_person + k * n_cap + txn);
            kind[n] = SYNTH_NODE_INSERT; src[n] = nid; dst[n] = 0; w[n] = 0.f; ts[n] = t; ++n;
            kind[n] = SYNTH_EDGE_INSERT;
            src[n] = LDBC_PERSON(skewed_person(n_person, r2, lodeg));
            dst[n] = nid; w[n] = wt; ts[n] = t; ++n;
        } else if (q < 99) {
            uint64_t s, d;
            ldbc_edge(n_person, n_msg, e_person, seed, r2 % (e_person ? e_person : 1), &s, &d);
            kind[n] = SYNTH_EDGE_DELETE; src[n] = s; dst[n] = d; w[n] = 0.f; ts[n] = t; ++n;
        } else {
            kind[n] = SYNTH_NODE_DELETE;
            src[n] = LDBC_PERSON(skewed_person(n_person, r2, lodeg));
            dst[n] = 0; w[n] = 0.f; ts[n] = t; ++n;
        }
        ++txn;
    }
    return n;
}

/* ------------------------------------------- tiny random streams (fuzz) ---- */
/*
 * Adversarial tiny op stream over vertex IDs [0, n_ids): all five kinds with
 * probabilities p[0..4], timestamps drawn from a small range so that equal
 * timestamps (same transaction) and out-of-order arrival are common.
 */
void synth_fuzz_batch(uint64_t seed, uint64_t k, uint64_t n, uint64_t n_ids, const double* p,
                      uint64_t ts_lo, uint64_t ts_span, uint8_t* kind, uint64_t* src,
                      uint64_t* dst, float* w, uint64_t* ts) {
    for (uint64_t i = 0; i < n; ++i) {
        double c = u01(synth_rand(seed, 900 + k, i)), acc = 0;
        uint8_t kd = 4;
        for (int j = 0; j < 5; ++j) { acc += p[j]; if (c < acc) { kd = (uint8_t)j; break; } }
        uint64_t r = synth_rand(seed, 1000 + k, i);
        kind[i] = kd;
        src[i] = (r & 0xFFFFFFFF) % n_ids;
        dst[i] = (kd <= SYNTH_NODE_DELETE) ? 0 : (r >> 32) % n_ids;
        w[i] = weight_of(synth_rand(seed, 1100 + k, i));
        ts[i] = ts_lo + (ts_span ? synth_rand(seed, 1200 + k, i) % ts_span : 0);
    }
}
