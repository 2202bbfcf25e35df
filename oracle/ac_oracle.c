/*
 * ac_oracle.c -- the CPU ORACLE for the Aho-Corasick matching scan.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * The product path (paper_conf_ipps_tranlhc13_b200/, libac.so) never links,
 * imports or calls anything in oracle/, and this file includes nothing from
 * the product tree.  The two share no code, headers, tables or helpers.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, cited as P:<line>):
 *   the multiset of all (end, pattern) occurrences of a dictionary in a text,
 *   reported in canonical order (start = end - len + 1 ascending, pattern id
 *   ascending) -- DESIGN.md reading R3.
 *
 * How: the textbook pattern matching machine of Aho & Corasick (ref [1],
 * P:321), exactly as the paper restates it in Section II:
 *   - goto function g      (Fig. 1a): a keyword trie; g(0,a) != fail
 *                                              for every symbol a
 *   - failure function f   (P:52,  Fig. 1b): consulted when g reports fail
 *   - output function: keywords recognised at a
 *                                              state, including those of f(s)
 *   - matching walk: "ushers" -> she, he at the same
 *                                     position, then hers.
 * The next-move function delta (the DFA form) is provided only as a
 * definition (AC'75 Alg. 4 semantics: delta(s,a) = g(s,a) if not fail, else
 * delta(f(s),a); delta(0,a) = g(0,a)) so tests can pin a DFA builder to it.
 *
 * Deliberately plain and slow: children are an unsorted singly linked edge
 * list scanned linearly, states are numbered in creation order while the
 * patterns are inserted in input order (reading R13), and nothing
 * is blocked, fused or reordered.
 *
 * Parity pins (tests/test_oracle.py): the printed worked example (P:55-58,
 * P:64-68), brute-force substring search on tiny random inputs, closed forms
 * (a^n with {a^1..a^K}; all k-mers), and invariants (count = sum of
 * per-pattern occurrences, chunking invariance, permutation equivariance,
 * shift under prefixing, concatenation with a separator).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define FAIL (-1)

typedef struct {
    uint8_t sym;
    uint32_t child;
    int64_t next; /* next edge of the same parent, -1 = end of list */
} edge_t;

typedef struct {
    int64_t first_edge; /* -1 = no children */
    uint32_t fail;
    uint32_t depth;
    uint32_t *out;      /* output(s): pattern ids */
    uint32_t n_out, cap_out;
} node_t;

typedef struct ac_oracle {
    int64_t root_goto[256]; /* g(0, a) as a total table: never FAIL */
    node_t *nodes;
    uint32_t n_nodes, cap_nodes;
    edge_t *edges;
    uint64_t n_edges, cap_edges;
    uint32_t n_patterns;
    uint32_t *lens; /* |pattern p| */
    uint32_t maxlen;
} ac_oracle;

static int push_out(node_t *nd, uint32_t pid) {
    if (nd->n_out == nd->cap_out) {
        uint32_t nc = nd->cap_out ? 2 * nd->cap_out : 2;
        uint32_t *p = (uint32_t *)realloc(nd->out, nc * sizeof(uint32_t));
        if (!p) return -1;
        nd->out = p;
        nd->cap_out = nc;
    }
    nd->out[nd->n_out++] = pid;
    return 0;
}

static int64_t new_node(ac_oracle *m, uint32_t depth) {
    if (m->n_nodes == m->cap_nodes) {
        uint32_t nc = m->cap_nodes ? 2 * m->cap_nodes : 64;
        node_t *p = (node_t *)realloc(m->nodes, (size_t)nc * sizeof(node_t));
        if (!p) return -1;
        m->nodes = p;
        m->cap_nodes = nc;
    }
    node_t *nd = &m->nodes[m->n_nodes];
    nd->first_edge = -1;
    nd->fail = 0;
    nd->depth = depth;
    nd->out = NULL;
    nd->n_out = nd->cap_out = 0;
    return (int64_t)m->n_nodes++;
}

/* The raw trie edge lookup: the child of s on symbol a, or FAIL. */
static int64_t trie_child(const ac_oracle *m, uint32_t s, uint8_t a) {
    for (int64_t e = m->nodes[s].first_edge; e >= 0; e = m->edges[e].next)
        if (m->edges[e].sym == a) return (int64_t)m->edges[e].child;
    return FAIL;
}

/* Goto function g.  The root never fails: g(0,a) = 0 when the trie
 * has no edge for a ("g(0, sigma) != fail for all sigma"). */
int64_t oracle_goto(const ac_oracle *m, uint32_t s, uint8_t a) {
    if (s == 0) return m->root_goto[a];
    return trie_child(m, s, a);
}

static int add_edge(ac_oracle *m, uint32_t parent, uint8_t a, uint32_t child) {
    if (m->n_edges == m->cap_edges) {
        uint64_t nc = m->cap_edges ? 2 * m->cap_edges : 64;
        edge_t *p = (edge_t *)realloc(m->edges, nc * sizeof(edge_t));
        if (!p) return -1;
        m->edges = p;
        m->cap_edges = nc;
    }
    edge_t *e = &m->edges[m->n_edges];
    e->sym = a;
    e->child = child;
    e->next = m->nodes[parent].first_edge; /* prepend: order is irrelevant */
    m->nodes[parent].first_edge = (int64_t)m->n_edges;
    m->n_edges++;
    return 0;
}

void oracle_free(ac_oracle *m) {
    if (!m) return;
    for (uint32_t i = 0; i < m->n_nodes; i++) free(m->nodes[i].out);
    free(m->nodes);
    free(m->edges);
    free(m->lens);
    free(m);
}

/*
 * Phase 1: construct the machine.  Returns NULL if any pattern is
 * empty (reading R6) or on allocation failure.
 */
ac_oracle *oracle_build(const uint8_t *const *pats, const uint32_t *lens, uint32_t np) {
    ac_oracle *m = (ac_oracle *)calloc(1, sizeof(ac_oracle));
    if (!m) return NULL;
    m->n_patterns = np;
    m->lens = (uint32_t *)malloc((np ? np : 1) * sizeof(uint32_t));
    if (!m->lens || new_node(m, 0) < 0) { oracle_free(m); return NULL; }

    /* Goto construction (AC'75 Alg. 2): insert each keyword in input order,
     * creating states in creation order; output(end state) gets the id. */
    for (uint32_t p = 0; p < np; p++) {
        if (lens[p] == 0) { oracle_free(m); return NULL; }
        m->lens[p] = lens[p];
        if (lens[p] > m->maxlen) m->maxlen = lens[p];
        uint32_t s = 0;
        for (uint32_t j = 0; j < lens[p]; j++) {
            int64_t t = trie_child(m, s, pats[p][j]);
            if (t == FAIL) {
                t = new_node(m, j + 1);
                if (t < 0 || add_edge(m, s, pats[p][j], (uint32_t)t) < 0) { oracle_free(m); return NULL; }
            }
            s = (uint32_t)t;
        }
        if (push_out(&m->nodes[s], p) < 0) { oracle_free(m); return NULL; }
    }
    /* AC'75 Alg. 2, last step: for all a with g(0,a) = fail, g(0,a) <- 0. */
    for (int a = 0; a < 256; a++) {
        int64_t t = trie_child(m, 0, (uint8_t)a);
        m->root_goto[a] = t == FAIL ? 0 : t;
    }

    /* Failure construction (AC'75 Alg. 3), breadth first.  Depth-1 states
     * fail to the root.  For r dequeued and each a with g(r,a) = s != fail:
     * state <- f(r); while g(state,a) = fail: state <- f(state);
     * f(s) <- g(state,a); output(s) <- output(s) U output(f(s)). */
    uint32_t *queue = (uint32_t *)malloc((size_t)m->n_nodes * sizeof(uint32_t));
    if (!queue) { oracle_free(m); return NULL; }
    uint64_t head = 0, tail = 0;
    for (int64_t e = m->nodes[0].first_edge; e >= 0; e = m->edges[e].next) {
        uint32_t s = m->edges[e].child;
        m->nodes[s].fail = 0;
        queue[tail++] = s;
    }
    while (head < tail) {
        uint32_t r = queue[head++];
        for (int64_t e = m->nodes[r].first_edge; e >= 0; e = m->edges[e].next) {
            uint8_t a = m->edges[e].sym;
            uint32_t s = m->edges[e].child;
            queue[tail++] = s;
            uint32_t state = m->nodes[r].fail;
            while (oracle_goto(m, state, a) == FAIL) state = m->nodes[state].fail;
            uint32_t fs = (uint32_t)oracle_goto(m, state, a);
            m->nodes[s].fail = fs;
            node_t *fn = &m->nodes[fs];
            for (uint32_t k = 0; k < fn->n_out; k++)
                if (push_out(&m->nodes[s], fn->out[k]) < 0) { free(queue); oracle_free(m); return NULL; }
        }
    }
    free(queue);
    return m;
}

uint32_t oracle_num_states(const ac_oracle *m) { return m->n_nodes; }
uint32_t oracle_maxlen(const ac_oracle *m) { return m->maxlen; }
uint32_t oracle_fail(const ac_oracle *m, uint32_t s) { return m->nodes[s].fail; }
uint32_t oracle_depth(const ac_oracle *m, uint32_t s) { return m->nodes[s].depth; }

/* output(s), ascending pattern id; returns |output(s)| (copies min(cap,|.|)). */
static int cmp_u32(const void *a, const void *b) {
    uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
    return (x > y) - (x < y);
}
uint32_t oracle_output(const ac_oracle *m, uint32_t s, uint32_t *pids, uint32_t cap) {
    const node_t *nd = &m->nodes[s];
    uint32_t k = nd->n_out < cap ? nd->n_out : cap;
    if (k) {
        memcpy(pids, nd->out, k * sizeof(uint32_t));
        if (k == nd->n_out) qsort(pids, k, sizeof(uint32_t), cmp_u32);
    }
    return nd->n_out;
}

/* Next-move function delta of the DFA form: g where defined, else
 * the move of the failure state.  Definition only; the walk below uses g/f. */
uint32_t oracle_delta(const ac_oracle *m, uint32_t s, uint8_t a) {
    for (;;) {
        int64_t t = oracle_goto(m, s, a);
        if (t != FAIL) return (uint32_t)t;
        s = m->nodes[s].fail;
    }
}

/*
 * Phase 2: the matching walk of P:55-58 (AC'75 Alg. 1) over
 * text[lo, hi), starting in state 0.  Each emitted occurrence is
 * (end = base + i, pid) for every pid in output(state) after consuming
 * text[i].  Occurrences whose start (end - len + 1 - base) is >= own_end are
 * dropped: this is the ownership rule of the chunked mode (reading R9); the
 * plain whole-text match passes own_end = hi.  Returns the number of owned
 * occurrences; stores the first `cap` of them (walk order) if ends != NULL.
 */
static uint64_t walk(const ac_oracle *m, const uint8_t *text, uint64_t lo, uint64_t hi,
                     uint64_t own_end, uint64_t base, uint64_t *ends, uint32_t *pids,
                     uint64_t cap, uint64_t count) {
    uint32_t state = 0;
    for (uint64_t i = lo; i < hi; i++) {
        uint8_t a = text[i];
        while (oracle_goto(m, state, a) == FAIL) state = m->nodes[state].fail;
        state = (uint32_t)oracle_goto(m, state, a);
        const node_t *nd = &m->nodes[state];
        for (uint32_t k = 0; k < nd->n_out; k++) {
            uint32_t p = nd->out[k];
            uint64_t start = i + 1 - m->lens[p];
            if (start >= own_end) continue;
            if (ends && count < cap) {
                ends[count] = base + i;
                pids[count] = p;
            }
            count++;
        }
    }
    return count;
}

uint64_t oracle_match(const ac_oracle *m, const uint8_t *text, uint64_t n, uint64_t base,
                      uint64_t *ends, uint32_t *pids, uint64_t cap) {
    return walk(m, text, 0, n, n, base, ends, pids, cap, 0);
}

/* One window of the chunked mode: the occurrences whose start lies in
 * [lo, own_hi), found by walking [lo, min(own_hi + maxlen - 1, n)) from
 * state 0.  Ends are reported as base + index.  Used to check sampled
 * windows of texts too large for a whole oracle pass. */
uint64_t oracle_match_window(const ac_oracle *m, const uint8_t *text, uint64_t n, uint64_t lo,
                             uint64_t own_hi, uint64_t base, uint64_t *ends, uint32_t *pids,
                             uint64_t cap) {
    uint64_t halo = m->maxlen ? m->maxlen - 1 : 0;
    if (own_hi > n) own_hi = n;
    if (lo >= own_hi) return 0;
    uint64_t hi = own_hi + halo < n ? own_hi + halo : n;
    return walk(m, text, lo, hi, own_hi, base, ends, pids, cap, 0);
}

/*
 * Chunked mode ("span each thread by adding X
 * characters after the chunk"): chunk [a,b) is walked from state 0 over
 * [a, min(b + maxlen - 1, n)) and keeps occurrences whose start is < b.
 * Used for the chunking-invariance pin and for multi-core timing.
 */
uint64_t oracle_match_chunked(const ac_oracle *m, const uint8_t *text, uint64_t n, uint64_t base,
                              uint64_t chunk, uint64_t *ends, uint32_t *pids, uint64_t cap) {
    uint64_t count = 0;
    if (chunk == 0) chunk = 1;
    uint64_t halo = m->maxlen ? m->maxlen - 1 : 0;
    for (uint64_t a = 0; a < n; a += chunk) {
        uint64_t b = a + chunk < n ? a + chunk : n;
        uint64_t hi = b + halo < n ? b + halo : n;
        /* occurrences starting before a belong to the previous chunk: they
         * cannot be seen here because the walk starts at a from state 0 and
         * a match ending at i >= a needs all its bytes read from a on. */
        count = walk(m, text, a, hi, b, base, ends, pids, cap, count);
    }
    return count;
}

/*
 * Transition counts of the walk of P:55-58 over text[0, n) (SURVEY 8(c)
 * pin P6, "O(n)"): out[0] = goto transitions (one per input symbol,
 * the root's self-loop g(0,a) = 0 included), out[1] = failure transitions
 * (state <- f(state)).  AC'75 bounds the failure transitions by the goto
 * transitions (each failure move strictly decreases the depth, which each
 * goto move raises by at most one), so the whole walk is O(n).
 */
void oracle_transitions(const ac_oracle *m, const uint8_t *text, uint64_t n, uint64_t *out) {
    uint64_t gotos = 0, fails = 0;
    uint32_t state = 0;
    for (uint64_t i = 0; i < n; i++) {
        uint8_t a = text[i];
        while (oracle_goto(m, state, a) == FAIL) {
            state = m->nodes[state].fail;
            fails++;
        }
        state = (uint32_t)oracle_goto(m, state, a);
        gotos++;
    }
    out[0] = gotos;
    out[1] = fails;
}

/* Canonical order (reading R3): start ascending, then pattern id ascending.
 * Each element carries its own start, so the comparator needs no shared state
 * and concurrent calls from several threads are safe. */
typedef struct { uint64_t start; uint64_t end; uint32_t pid; } occ_t;
static int cmp_occ(const void *x, const void *y) {
    const occ_t *a = (const occ_t *)x, *b = (const occ_t *)y;
    if (a->start != b->start) return a->start < b->start ? -1 : 1;
    return (a->pid > b->pid) - (a->pid < b->pid);
}
int oracle_canonical_sort(const ac_oracle *m, uint64_t *ends, uint32_t *pids, uint64_t count) {
    occ_t *v = (occ_t *)malloc((count ? count : 1) * sizeof(occ_t));
    if (!v) return -1;
    for (uint64_t i = 0; i < count; i++) {
        v[i].end = ends[i];
        v[i].pid = pids[i];
        v[i].start = ends[i] + 1 - m->lens[pids[i]];
    }
    qsort(v, count, sizeof(occ_t), cmp_occ);
    for (uint64_t i = 0; i < count; i++) { ends[i] = v[i].end; pids[i] = v[i].pid; }
    free(v);
    return 0;
}

/*
 * Multiset digest of the occurrences whose start lies in [lo, own_hi) (the
 * window of oracle_match_window, same walk), for texts whose full list is too
 * large to keep (SURVEY 8(c) "GPU parity": count, sum and xor of
 * splitmix64(key) over the occurrences, order independent).  key = start *
 * 2^24 + pid with start = base + end - len + 1 (the canonical (start, pid)
 * pair of reading R3 written as one integer; "at the end of position").
 * splitmix64 is the public constant-exact mixer (Steele, Lea, Flood 2014),
 * written out here on its own.  out[0] = count, out[1] = sum mod 2^64,
 * out[2] = xor.
 */
static uint64_t mix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
void oracle_digest_window(const ac_oracle *m, const uint8_t *text, uint64_t n, uint64_t lo, uint64_t own_hi,
                          uint64_t base, uint64_t *out) {
    uint64_t halo = m->maxlen ? m->maxlen - 1 : 0;
    uint64_t count = 0, sum = 0, x = 0;
    if (own_hi > n) own_hi = n;
    if (lo < own_hi) {
        uint64_t hi = own_hi + halo < n ? own_hi + halo : n;
        uint32_t state = 0;
        for (uint64_t i = lo; i < hi; i++) { /* the walk of P:55-58, as walk() above */
            uint8_t a = text[i];
            while (oracle_goto(m, state, a) == FAIL) state = m->nodes[state].fail;
            state = (uint32_t)oracle_goto(m, state, a);
            const node_t *nd = &m->nodes[state];
            for (uint32_t k = 0; k < nd->n_out; k++) {
                uint32_t p = nd->out[k];
                uint64_t start = i + 1 - m->lens[p];
                if (start >= own_hi) continue;
                uint64_t h = mix64(((base + start) << 24) | p);
                count++;
                sum += h;
                x ^= h;
            }
        }
    }
    out[0] = count;
    out[1] = sum;
    out[2] = x;
}
