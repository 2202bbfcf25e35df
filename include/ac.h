/*
 * ac.h -- C ABI of the B200-native Aho-Corasick matching scan (libac.so).
 *
 * Paper: N.-P. Tran, M. Lee, S. Hong, J. Choi, "High Throughput Parallel
 * Implementation of Aho-Corasick Algorithm on a GPU", IPDPS-W 2013.
 * Citations "P:<line>" refer to the paper text line numbers.
 *
 * The two calls follow the paper's problem statement: "In the first
 * phase, a pattern matching machine called AC automaton (machine) is
 * constructed from a finite set of patterns.  In the second phase, the input
 * text data is applied to the constructed AC machine in order to find the
 * locations that the patterns appear."
 *   - ac_build  : phase 1.  Host-side construction of the DFA (next-move
 *                 function delta with the failure function folded in) as a
 *                 State Transition Table (STT, Fig. 5), built once on
 *                 one CPU core and copied to device memory.  Untimed,
 *                 like the paper.
 *   - ac_match  : phase 2.  The data-parallel scan: one STT transition per
 *                 text byte (O(n)), every (position, pattern)
 *                 occurrence emitted, on an sm_100a GPU.
 *
 * Conventions:
 *   - Alphabet: raw bytes 0..255, binary safe, case sensitive (R7).
 *   - Pattern ids are the 0-based indices of the input array (R4);
 *     duplicate patterns are distinct ids (R5); empty patterns are rejected
 *     (R6).
 *   - Every occurrence is reported, overlapping and nested ones included
 *     (R19).
 *   - A match record is one 64-bit word:  (start << 24) | pattern
 *     where start is the 0-based index of the occurrence's first byte and
 *     end = start + len(pattern) - 1 is the paper's "end of position" (
 *     R2).  Canonical order = ascending record value = (start, pattern)
 *     ascending (R3).  Hence n < 2^40 and n_patterns < 2^24.
 *   - All functions are thread safe; an ac_stt is immutable after ac_build,
 *     so concurrent ac_match calls on different streams are allowed.
 *   - No C++ exception or abort crosses this ABI.  Errors are status codes;
 *     ac_last_error() returns a thread-local detail string.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default).
 *   - There is no CPU fallback: without a usable sm_100 device every device
 *     call returns AC_ERR_NO_DEVICE or AC_ERR_CUDA.
 */
#ifndef AC_H
#define AC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef uint64_t ac_match_t;
#define AC_MATCH_START(m) ((uint64_t)(m) >> 24)
#define AC_MATCH_PATTERN(m) ((uint32_t)((m) & 0xFFFFFFu))
#define AC_MAX_PATTERNS (1u << 24)
#define AC_MAX_TEXT ((uint64_t)1 << 40)

typedef enum {
    AC_OK = 0,
    AC_ERR_INVALID_ARG = 1,   /* NULL pointer, bad option, ...              */
    AC_ERR_EMPTY_PATTERN = 2, /* some lens[i] == 0 (reading R6)             */
    AC_ERR_TOO_LARGE = 3,     /* n_patterns >= 2^24, states >= 2^31, n >= 2^40 */
    AC_ERR_CAPACITY = 4,      /* list longer than cap: *count = needed size  */
    AC_ERR_NO_MEMORY = 5,     /* host or device allocation failed           */
    AC_ERR_CUDA = 6,          /* any CUDA runtime/driver error              */
    AC_ERR_NO_DEVICE = 7      /* no usable compute-capability-10.x device   */
} ac_status;

/* Opaque device STT handle: dense transition table + class map + output
 * CSR + pattern lengths, owned by the library, released by ac_free(). */
typedef struct ac_stt ac_stt;

/* Opaque HOST table (phase-1 result before upload); used by tests to check
 * the builder without a GPU. */
typedef struct ac_table ac_table;

/* STT residency tiers. */
/* SMEM: the dense table staged whole in shared memory.  HYBRID: its BFS
 * prefix in shared memory, the rest through L1/L2.  GLOBAL: L1/L2 only.
 * COMPACT: dense rows for shallow states + 8-byte default-transition records
 * for the others + an output table, all in shared memory (<= 32768 states,
 * <= 127 classes).  SPLIT: the hot BFS part of a
 * large automaton in shared memory -- dense 16-bit rows for the shallow
 * levels, 8-byte default-transition records for the next states -- and the
 * full 32-bit table in global memory (L1/L2) for the cold states (DESIGN.md
 * "SPLIT tier"; SURVEY 8(a)-a5 tier (ii)).  AUTO = SMEM if the dense table
 * fits, else COMPACT if that fits, else GLOBAL with the two-byte walk for
 * <= 8 classes, else SPLIT. */
enum {
    AC_TIER_AUTO = 0,
    AC_TIER_SMEM = 1,
    AC_TIER_HYBRID = 2,
    AC_TIER_GLOBAL = 3,
    AC_TIER_COMPACT = 4,
    AC_TIER_SPLIT = 5
};

typedef struct {
    uint32_t struct_size;  /* sizeof(ac_build_opts)                          */
    uint32_t entry_bytes;  /* 0 = auto (2 if states <= 32768 else 4), 2 or 4 */
    uint32_t tier;         /* AC_TIER_*                                      */
    uint32_t hot_rows;     /* HYBRID: rows kept in shared memory (0 = auto)  */
    uint32_t forward;      /* 0 (default) = automaton of the REVERSED
                              patterns, scanned right-to-left so that matches
                              come out in canonical (start, pattern) order;
                              1 = the paper's forward automaton (tests only:
                              ac_build rejects it, ac_compile accepts it)    */
    uint32_t stride;       /* bytes per dependent lookup in the staged scan:
                              0 = auto (2 for GLOBAL-tier automata with
                              <= 8 classes whose two-byte table fits 64 MiB),
                              1, or 2 (needs 32-bit
                              entries -- set entry_bytes = 4 for small S)    */
    uint32_t threads;      /* host threads for phase 1:
                              0 = $AC_BUILD_THREADS if set, else the
                              hardware concurrency (at most 32); the table
                              is identical for every value                  */
} ac_build_opts;

typedef struct {
    uint32_t n_patterns;
    uint32_t n_states;     /* S                                             */
    uint32_t n_classes;    /* C: class 0 = bytes in no pattern              */
    uint32_t row_stride;   /* entries per STT row (>= C, padded)            */
    uint32_t entry_bytes;  /* 2 or 4                                        */
    uint32_t tier;         /* resolved AC_TIER_*                            */
    uint32_t hot_rows;     /* rows resident in shared memory                */
    uint32_t maxlen;       /* longest pattern                               */
    uint32_t forward;
    uint32_t info_col;     /* entry index of each row's output summary: a u32
                              payload (the pattern id when |output| == 1,
                              else the CSR offset) followed by the count
                              (u16 saturating at 0xFFFF if entry_bytes == 2,
                              else u32)                                      */
    uint64_t stt_bytes;    /* S * row_stride * entry_bytes                  */
    uint64_t out_entries;  /* sum over states of |output(s)|                */
    /* COMPACT encoding (valid when compact_bytes != 0): byte layout
     * [dense rows: compact_dense x compact_dstride u16]
     * [sparse records at compact_sparse_off: (n_states - compact_dense) x 8 B,
     *  lo32 = 2 c1 | 2 c2 << 8 | fd << 16 (doubled classes, 0xFF = none),
     *  hi32 = t1 | t2 << 16]; every entry (dense row cell, t1, t2) is
     *  2 x + flag, x = compact id of the next state, flag = output(x) != {}
     * [output table at compact_out_off: (compact_od + compact_os) x
     *  (u32 payload, u32 count)], compact ids: 0 = root, then other dense
     * states, dense output states, sparse output states, other sparse: the
     * output states are ids [compact_dense - compact_od, compact_dense +
     * compact_os) and the output slot of id x is x - (compact_dense -
     * compact_od).                                                      */
    uint32_t compact_dense, compact_od, compact_os, compact_dstride;
    uint32_t compact_sparse_off, compact_out_off;
    uint64_t compact_bytes;
    uint32_t stride;       /* 1 or 2 (two-byte table present)                */
    uint32_t stride2_cols; /* row stride of the two-byte table (C*C, odd)   */
    uint64_t stt2_bytes;
    /* SPLIT tier (valid when split_bytes != 0): split_dense + 1 dense rows of
     * split_dstride u16 entries (row r = BFS state r for r < split_dense, the
     * last one -- the escape row -- all 0xFFFF), then one 8-byte CHILDREN
     * record per hot state split_dense <= s < split_records:
     * {lo32 = c1 | c2 << 8 | c3 << 16 | c4 << 24 (the classes of s's goto
     * children, ascending, the last one repeated),
     * hi32 = fd | flags << 12 | (2 first - 1) << 16}: delta(s, c) = first + k
     * (flag bit k) for the lowest k with c == c_k, else row[fd][c] (fd = f(s),
     * dense); dense states read row[s][c]; a u16 result is 2 x + flag, and a
     * value > 0xFFFD means "read the global table".  split_cold_records
     * records are cold (fd = the escape row, 2 first - 1 = 0xFFFD); states
     * >= split_records are read from the global table. */
    uint32_t split_dense, split_records, split_dstride, split_cold_records;
    uint64_t split_bytes;
} ac_stt_info;

/* Scan variants (SURVEY 8(f) NEXT-1 ablations are selectable here). */
enum {
    AC_KERNEL_AUTO = 0,
    AC_KERNEL_STAGED = 1, /* TMA-staged text tiles in shared memory, the
                             B200 form of the paper's "shared memory
                             approach"                           */
    AC_KERNEL_GLOBAL = 2  /* text read straight from global memory, the
                             paper's "global memory only approach" */
};

typedef struct {
    uint32_t struct_size;  /* sizeof(ac_match_opts)                          */
    uint32_t kernel;       /* AC_KERNEL_*                                    */
    uint32_t chain_bytes;  /* bytes owned per thread chain (0 = auto; STAGED:
                              rounded to the tile width)                     */
    uint32_t variant;      /* STAGED CTA shape, 0 = auto, 1..11 (DESIGN.md
                              "Staged variants": warps x chains/lane x tile
                              width x ring depth)                            */
    uint32_t scratch_slots;/* list mode: records each chain may park in its
                              scratch slot during the single emitting pass
                              (0 = auto from cap); chains with more are
                              re-scanned straight into place                 */
    uint32_t two_pass;     /* list mode: 0 = auto: single emitting pass;
                              when cap > n (room for more than one record
                              per text byte: dense outputs) the EVENTS
                              single pass unless the STT is COMPACT (one
                              parked event per output state reached,
                              expanded into records by the gather), else the
                              two passes -- also chosen when the scratch
                              budget cannot hold twice the expected records
                              per chain; single pass: chain
                              offsets computed inside the staged scan when
                              the text pointer is 16-byte aligned, else by
                              a separate offset scan); 1 = count pass + emit
                              pass (ablation / fallback); 2 = single pass
                              with the separate offset scan (ablation);
                              3 = single pass with 8-byte scratch records
                              (ablation of the 4-byte narrow records);
                              4 = the EVENTS single pass whenever the table
                              allows it (else as 0)                         */
    uint32_t stride;       /* 0 = the table's default, 1 = force one byte
                              per lookup even if a two-byte table exists     */
    uint32_t n_events;     /* pairs available in `events`                    */
    void **events;         /* optional cudaEvent_t[2 * n_events]: events[2i]
                              and events[2i+1] are recorded on the stream
                              right before / after kernel launch i, so a
                              caller can time each kernel (bench.py)         */
    uint32_t text_policy;  /* L2 policy of the staged kernel's text loads:
                              0 = auto (evict-first where the table lives in
                              L2: GLOBAL, HYBRID, SPLIT), 1 = evict-normal,
                              2 = evict-first, 3 = per 32-byte sector: the
                              half read first evict-normal, the second
                              evict-first (ablation knob)                   */
    uint32_t text_promotion; /* L2 promotion of the text's TMA misses:
                              0 = auto (256 B), 1 = none, 2 = 64 B,
                              3 = 128 B, 4 = 256 B (ablation knob)          */
    uint32_t l2_window_mib; /* > 0: the staged scan runs with a persisting L2
                              access-policy window over the first MiB of the
                              global table (GLOBAL/HYBRID/SPLIT tiers; capped
                              by the device's persisting-L2 limit, which the
                              first such call raises to its maximum -- a
                              process-wide setting).  0 = off (default)      */
} ac_match_opts;

/* Per-call device result written by the async entry points. */
typedef struct {
    uint64_t count;        /* total occurrences (always valid)               */
    uint32_t status;       /* AC_OK or AC_ERR_CAPACITY                       */
    uint32_t reserved;
} ac_result;

/* ---------------------------------------------------------------- phase 1
 * ac_build: patterns[i] points to lens[i] bytes (host memory, any bytes).
 * Builds the DFA on the host, uploads it to `device`, returns a
 * handle in *out.  Errors: AC_ERR_INVALID_ARG (NULL args, opts->forward),
 * AC_ERR_EMPTY_PATTERN, AC_ERR_TOO_LARGE, AC_ERR_NO_MEMORY, AC_ERR_CUDA,
 * AC_ERR_NO_DEVICE.  `opts` may be NULL (all auto). */
ac_status ac_build(const uint8_t *const *patterns, const uint32_t *lens, uint32_t n_patterns,
                   int device, const ac_build_opts *opts, ac_stt **out);
void ac_free(ac_stt *stt);
ac_status ac_stt_query(const ac_stt *stt, ac_stt_info *info);
/* Copies the n_patterns pattern lengths to host memory `lens`. */
ac_status ac_stt_pattern_lengths(const ac_stt *stt, uint32_t *lens);

/* ---------------------------------------------------------------- phase 2
 * ac_match: scans d_text[0, n) (DEVICE memory, any alignment, n may be 0)
 * and reports every occurrence.  The list is produced in one emitting pass
 * when cap <= n (at most one record per text byte of room), else in two
 * (count, then emit in place) -- cap is read as the caller's density bound,
 * no count pass is run to plan.
 *   d_out == NULL : count only; *count = number of occurrences.
 *   d_out != NULL : DEVICE buffer of `cap` records; on AC_OK it holds the
 *                   *count records in canonical order.  If the count exceeds
 *                   cap, returns AC_ERR_CAPACITY with *count = required size
 *                   and d_out contents unspecified.
 * The call is stream-ordered on `stream` and synchronises it before
 * returning (it must return the count).  Scratch space is taken from the
 * stream-ordered allocator (cudaMallocAsync). */
ac_status ac_match(const ac_stt *stt, const uint8_t *d_text, uint64_t n, ac_match_t *d_out,
                   uint64_t cap, uint64_t *count, void *stream);

/* ac_match_shard: one shard of a larger text.  d_text[0,
 * n_owned + n_halo) is readable; occurrences whose start lies in [0, n_owned)
 * are reported, with start + base in the records.  The caller passes
 * n_halo = min(maxlen - 1, n_total - (base + n_owned)) bytes of the next
 * shard so straddling occurrences are found exactly once (R8/R9). */
ac_status ac_match_shard(const ac_stt *stt, const uint8_t *d_text, uint64_t n_owned,
                         uint64_t n_halo, uint64_t base, ac_match_t *d_out, uint64_t cap,
                         uint64_t *count, void *stream);

/* Asynchronous form of ac_match_shard: enqueues the whole scan on `stream`
 * and returns without synchronising; the count and status land in the
 * DEVICE struct *d_result when the stream reaches that point.  `opts` may be
 * NULL.  Host-side argument errors are returned immediately. */
ac_status ac_match_async(const ac_stt *stt, const uint8_t *d_text, uint64_t n_owned,
                         uint64_t n_halo, uint64_t base, ac_match_t *d_out, uint64_t cap,
                         ac_result *d_result, void *stream, const ac_match_opts *opts);

/* ac_match_segments: a batch of independent texts -- e.g. network packets,
 * the NIDS workload of P:108 -- concatenated in d_text.
 * d_seg_off (DEVICE, n_seg + 1 ascending uint64, first 0) gives the
 * boundaries; segment i = d_text[d_seg_off[i], d_seg_off[i+1]) is scanned
 * from the start state on its own, so no occurrence crosses a boundary.
 * Records carry start offsets into d_text; the list is canonical.  Each
 * segment must be shorter than 2^31 / max|output(s)| bytes.  Asynchronous
 * like ac_match_async (count/status in *d_result); d_out == NULL = count
 * only. */
ac_status ac_match_segments(const ac_stt *stt, const uint8_t *d_text, const uint64_t *d_seg_off, uint64_t n_seg,
                            ac_match_t *d_out, uint64_t cap, ac_result *d_result, void *stream);

/* Number of kernel launches the last ac_match_async on this thread issued,
 * and the name of launch i (NULL if out of range). */
uint32_t ac_last_launch_count(void);
const char *ac_last_launch_name(uint32_t i);
/* Owned text bytes scan launch i walked (0 for non-scan launches: offsets,
 * gather, re-walk).  For per-kernel throughput accounting; halo re-walks are
 * not counted (reading R14). */
uint64_t ac_last_launch_text_bytes(uint32_t i);
/* Bytes per scratch record of the last list-mode ac_match_async on this
 * thread: 4 (narrow: offset in chain and pattern id share 32 bits), 8, or 0
 * (count mode / two-pass mode: no scratch).  For traffic accounting. */
uint32_t ac_last_scratch_record_bytes(void);

/* End-to-end entry with HOST buffers: copies h_text[0,n) to the device,
 * scans it, copies the count and (if h_out != NULL) the canonical list back
 * into h_out[0, cap).  Same status semantics as ac_match.  Device staging is
 * allocated on `stream`'s device with the stream-ordered allocator. */
ac_status ac_match_host(const ac_stt *stt, const uint8_t *h_text, uint64_t n, ac_match_t *h_out,
                        uint64_t cap, uint64_t *count, void *stream);

/* ----------------------------------------------------- host-only builder
 * ac_compile: phase 1 without a device (for tests and tooling).  hot_rows is
 * ignored; opts->forward selects the paper's forward automaton;
 * opts->tier == AC_TIER_COMPACT also builds the COMPACT encoding for the
 * default shared-memory budget (AC_ERR_TOO_LARGE if it cannot).
 * ac_table_export_compact copies it out (blob[compact_bytes], perm[S] =
 * compact id -> dense BFS id).  ac_table_export copies any non-NULL array:
 *   class_map[256]            byte -> class
 *   stt[S * row_stride]       entries of entry_bytes each: low bits = next
 *                             state, top bit (15 or 31) = output(next) != {};
 *                             columns >= info_col hold the output summary
 *   out_off[S + 1], out_ids[out_entries]   output CSR, ids ascending
 */
ac_status ac_compile(const uint8_t *const *patterns, const uint32_t *lens, uint32_t n_patterns,
                     const ac_build_opts *opts, ac_table **out);
ac_status ac_table_query(const ac_table *t, ac_stt_info *info);
ac_status ac_table_export(const ac_table *t, uint8_t *class_map, void *stt, uint32_t *out_off,
                          uint32_t *out_ids);
ac_status ac_table_export_compact(const ac_table *t, void *blob, uint32_t *perm);
/* opts->stride == 2 also builds the two-byte table (NEXT-4): n_states rows of
 * stride2_cols u32, column c1*C + c2 -> delta(delta(s,c1),c2) | bit 31 =
 * output(final) != {} | bit 30 = output(middle) != {}. */
ac_status ac_table_export_stride2(const ac_table *t, uint32_t *tab);
/* opts->tier == AC_TIER_SPLIT (ac_compile) builds the SPLIT shared-memory
 * part for the default budget (32-bit table); copies its split_bytes. */
ac_status ac_table_export_split(const ac_table *t, void *blob);
void ac_table_free(ac_table *t);

/* ------------------------------------------------------------ diagnostics */
const char *ac_status_string(ac_status s);
const char *ac_last_error(void);
/* Library build identification, e.g. "libac sm_100a". */
const char *ac_version(void);

#ifdef __cplusplus
}
#endif
#endif /* AC_H */
