/*
 * drgpum.h -- C ABI of the B200-native DrGPUM attribution library
 * (libdrgpum.so, built from paper_conf_asplos_linzs23_b200/csrc for sm_100a).
 *
 * The library implements the data-parallel hot path of DrGPUM's object-centric
 * analysis (Lin, Zhou, Su, ASPLOS '23).  "P:NNN" cites line NNN of the paper
 * text (/root/reference/PAPER.md at build time; the text is not needed at run
 * time).  Readings of the paper where it is silent or ambiguous are the
 * numbered items R1..R27 of DESIGN.md §"Readings".
 *
 *   objects + GPU-API timeline  --drgpum_objects_load-->  memory map M as a
 *       static segment index (§5.1)
 *   access records              --drgpum_trace_attribute--> per-object bitmap
 *       (§5.2), first/last use, accessing-API set (P:232,
 *       Def 3.6/3.7 P:164-168)
 *   per-object reductions       --drgpum_object_stats-->   accessed elements,
 *       span, largest unaccessed chunk (Eq. (1)), liveness
 *   patterns                    --drgpum_patterns-->       EA, LD, UA, ML, TI,
 *       DW, OA (+Frag) (Defs 3.1-3.8 P:124-174, rules P:244-249)
 *
 * Conventions for every call
 *   - Returns a drgpum_status; nothing throws across the ABI.  On failure the
 *     context keeps a message for drgpum_last_error() (with the index of the
 *     first offending object where relevant) and its state is unchanged.
 *   - "stream" is a cudaStream_t passed as void* (0 = legacy default stream).
 *     Device-side work is enqueued on it in call order; calls documented as
 *     "synchronous" synchronise that stream before returning.
 *   - Host input arrays are copied (or fully consumed) before the call
 *     returns; the caller may free them afterwards.  Device record buffers are
 *     BORROWED stream-ordered: keep them alive until the stream passes the call.
 *   - The workspace is caller-owned device memory (the Python binding takes it
 *     from torch.empty), bound once per trace; every device array the library
 *     uses lives inside it.  The library never allocates device memory except
 *     two tiny event/stream objects for drgpum_trace_attribute_host.
 *   - One context per device (per rank).  A context is not thread-safe.
 *   - Call order: create -> objects_load -> [set_features] [set_queue_capacity]
 *     -> workspace_bind -> { trace_attribute | trace_attribute_host }* ->
 *     one of the merges (multi-rank only):
 *       (a) merge_or ... (after an all-to-all) or merge_peers, between two
 *           barriers: afterwards every rank holds the whole merged shadow;
 *       (b) barrier, merge_peers_owned, barrier, finalize, barrier,
 *           gather_peers, barrier: afterwards every rank holds every
 *           object's stats and reports, but its shadow (bitmaps, hit rows,
 *           first/last) is merged for ITS OWN objects only;
 *     -> finalize / object_stats / patterns / NEXT-row queries.
 *     drgpum_reset starts a new trace on the same objects (and clears the
 *     owned-merge state).  Out-of-order calls return DRGPUM_ESTATE.
 *   - What a rank can read after an owned merge (b): object_stats, patterns
 *     (with the finalize's thresholds), consistency_errors and
 *     redundant_alloc are whole-trace results once gather_peers is done;
 *     dependency_graph and patterns_topo return ESTATE (they read every
 *     object's hit row); the bitmap / hit-row words, first/last of the other
 *     ranks' objects in the shadow view are this rank's partial ones.  The
 *     NEXT-2 / NEXT-3 results (drgpum_frequency, drgpum_structured) are never
 *     merged by any of the merges: they cover the records this rank
 *     attributed.
 */
#ifndef DRGPUM_H
#define DRGPUM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define DRGPUM_API __attribute__((visibility("default")))
#else
#define DRGPUM_API
#endif

/* t_free of an object that is never freed (memory leak, Def 3.5);
 * t_first of an object that is never accessed (unused, Def 3.4). */
#define DRGPUM_NEVER 0xFFFFFFFFu

/* GPU APIs of the timeline (footnote 1: allocation, deallocation, copy,
 * set, kernel launch).  Allocation/deallocation never access an object
 * (footnote 2). */
typedef enum {
  DRGPUM_API_ALLOC = 0, DRGPUM_API_FREE = 1, DRGPUM_API_MEMCPY = 2,
  DRGPUM_API_MEMSET = 3, DRGPUM_API_KERNEL = 4
} drgpum_api_kind;

typedef enum {
  DRGPUM_OK = 0,
  DRGPUM_EINVAL = 1,    /* malformed argument / object / timeline (rules below) */
  DRGPUM_EOVERLAP = 2,  /* two objects overlap in address AND in open lifetime [R5] */
  DRGPUM_ESTATE = 3,    /* call out of order */
  DRGPUM_ENOMEM = 4,    /* workspace too small / index would exceed limits */
  DRGPUM_ECUDA = 5      /* CUDA runtime error (message has cudaGetErrorString) */
} drgpum_status;

/* A data object ("a data object's lifetime, start address, and size").
 * 32 bytes.  Byte range [base, base+size); elements of elem_size bytes [R1];
 * open lifetime (t_alloc, t_free): live at ts iff t_alloc < ts < t_free. */
typedef struct {
  uint64_t base;
  uint64_t size;        /* > 0, multiple of elem_size, base+size must not overflow */
  uint32_t elem_size;   /* 1, 2, 4, 8 or 16 */
  uint32_t t_alloc;     /* timestamp of its ALLOC API */
  uint32_t t_free;      /* timestamp of its FREE API, or DRGPUM_NEVER */
  uint32_t user_id;     /* opaque, not interpreted */
} drgpum_object_t;

/* One instrumented access ("accessed memory range (i.e., start address
 * and size)") stamped with the timestamp T of the GPU API that issued it
 * (P:238).  16 bytes, little-endian; meta = ts | is_write << 31, ts < 2^31. */
typedef struct {
  uint64_t addr;
  uint32_t size;
  uint32_t meta;
} drgpum_record_t;

/* Per-object reductions, in the caller's load order.  56 bytes. */
typedef struct {
  uint64_t n_elems;                /* size / elem_size */
  uint64_t accessed;               /* popcount of the bitmap */
  uint64_t span_lo, span_hi;       /* lowest/highest accessed element; UINT64_MAX if none */
  uint64_t largest_unaccessed_run; /* longest run of 0 bits in [0, n_elems) (Eq. (1)) */
  uint32_t t_first, t_last;        /* T_first (DRGPUM_NEVER if unused), T_last (0 if unused) */
  uint32_t n_access_apis;          /* number of distinct GPU APIs that access the object */
  uint32_t _pad;
} drgpum_object_stats_t;

/* User-tunable thresholds.  Defaults {2, 80, 80}: TI X=2, OA 80%
 * (P:268), Frag 80%. */
typedef struct {
  uint32_t ti_min_idle;      /* TI if >= this many APIs lie between consecutive accesses */
  uint32_t oa_accessed_pct;  /* OA if 100*accessed < pct*n_elems (strict, [R10]) */
  uint32_t oa_frag_pct;      /* OA_ACTIONABLE if also Frag < pct (Eq. (1), [R11]) */
} drgpum_thresholds_t;

enum {
  DRGPUM_EA = 1,            /* early allocation      Def 3.1, rule P:244 */
  DRGPUM_LD = 2,            /* late deallocation     Def 3.2, rule P:245, never for ML [R8] */
  DRGPUM_UA = 4,            /* unused allocation     Def 3.4, rule P:246 */
  DRGPUM_ML = 8,            /* memory leak           Def 3.5, rule P:247 */
  DRGPUM_TI = 16,           /* temporary idleness    Def 3.6, rule P:248 */
  DRGPUM_DW = 32,           /* dead write            Def 3.7, rule P:249 [R12] */
  DRGPUM_OA = 64,           /* overallocation        Def 3.8, P:268 [R9] */
  DRGPUM_OA_ACTIONABLE = 128/* OA and Frag below threshold (Table 2) */
};

/* Pattern report per object (load order).  32 bytes.  Distances are
 * timestamp differences (inefficiency distance) and are 0 unless the
 * pattern fires; "APIs between" = distance - 1 [R6]. */
typedef struct {
  uint32_t flags;
  uint32_t ea_distance;     /* T_first - T_alloc when EA */
  uint32_t ld_distance;     /* T_free - T_last when LD */
  uint32_t ti_ranges;       /* number of idle gaps >= ti_min_idle */
  uint32_t ti_max_idle;     /* longest such gap, in APIs */
  uint32_t dw_pairs;        /* consecutive copy/set write pairs */
  uint64_t ti_total_idle;   /* sum of those gaps */
} drgpum_pattern_report_t;

/* Trace counters.  records = attributed + unattributed +
 * invalid; clipped <= attributed. */
typedef struct {
  uint64_t records;
  uint64_t attributed;      /* found a live object containing addr */
  uint64_t unattributed;    /* no live object contains addr [R4] */
  uint64_t clipped;         /* attributed but ran past the object's end [R3] */
  uint64_t invalid;         /* size 0, ts >= n_api, ts of ALLOC/FREE [R14], addr+size overflow */
} drgpum_counters_t;

/* Where the mergeable shadow state lives inside the workspace (byte offsets
 * from the workspace base), for multi-GPU exchange.  The OR-
 * mergeable words (bitmaps then hit rows) are ONE contiguous u32 array of
 * or_words words at or_off.  first/last are u32[n_obj]; counters u64[5]. */
typedef struct {
  uint64_t or_off, or_words;
  uint64_t bitmap_words, hit_words;   /* or_words = bitmap_words + hit_words */
  uint64_t first_off, last_off, counters_off;
  uint64_t n_obj;
} drgpum_shadow_view_t;

/* Per-object placement in the shadow (load order). */
typedef struct {
  uint64_t bitmap_word;   /* first u32 word of the object's bitmap (element e = bit e%32 of word bitmap_word + e/32) */
  uint64_t hit_word;      /* first u32 word of its hit row, relative to bitmap_words */
  uint32_t r_lo;          /* access-API rank of the first access API after t_alloc */
  uint32_t n_hit_apis;    /* access APIs inside (t_alloc, t_free); hit bit 2*(rank-r_lo)+is_write */
} drgpum_object_layout_t;

typedef struct drgpum_ctx drgpum_ctx;

/* Create a context on a CUDA device.  EINVAL if out is NULL; ECUDA if the
 * device cannot be selected. */
DRGPUM_API drgpum_status drgpum_create(int cuda_device, drgpum_ctx **out);

/* Load the object table and the GPU-API timeline (host arrays, copied).
 * Builds the memory map M as a static segment index valid for
 * every timestamp, the bitmap/hit-row layout and the access-API rank tables.
 * EINVAL: n_api >= 2^31; n_obj >= 2^32-1; an api kind > 4; per object: size
 * 0, elem_size not in {1,2,4,8,16}, size % elem_size, base+size overflow,
 * t_alloc >= n_api or not an ALLOC, t_free != NEVER and (>= n_api, <= t_alloc
 * or not a FREE).  EOVERLAP: two objects overlap in address and in open
 * lifetime [R5].  ENOMEM: the index would exceed 2^32-1 candidate entries.
 * Allowed after create, or again after a previous load (discards it). */
DRGPUM_API drgpum_status drgpum_objects_load(drgpum_ctx *ctx,
    const drgpum_object_t *h_objs, uint64_t n_obj,
    const uint8_t *h_api_kinds, uint32_t n_api);

/* Optional analyses.  Set after objects_load and
 * before workspace_size / workspace_bind (ESTATE otherwise); EINVAL on unknown
 * bits.  DRGPUM_FEATURE_STRUCTURED (NEXT-3, structured access, Def 3.10
 * l.200, §5.2 l.270) adds a u32 owner word per element of every object to the
 * workspace, and every trace_attribute call then also runs the structured-
 * access pass over its records. */
enum { DRGPUM_FEATURE_STRUCTURED = 1, DRGPUM_FEATURE_FREQUENCY = 2 };
DRGPUM_API drgpum_status drgpum_set_features(drgpum_ctx *ctx, uint32_t features);

/* Capacity of the device work queues, in entries (0 = keep the current
 * value; defaults 2^20 each).  range_entries sizes the A3b range-expansion
 * queue (16 B per entry, <= 4096 words each); aux_entries the wide-record
 * queues of the NEXT-2 / NEXT-3 passes.  A queue that fills up is never an
 * error: the records that do not fit are expanded in place by the warp that
 * found them (exact, slower), and the range-queue overflow is counted.
 * Smaller queues shrink the workspace; tests use tiny ones to drive the
 * overflow paths.  Set after objects_load and before workspace_size /
 * workspace_bind (ESTATE otherwise); EINVAL above 2^24 entries. */
DRGPUM_API drgpum_status drgpum_set_queue_capacity(drgpum_ctx *ctx, uint32_t range_entries,
                                                   uint32_t aux_entries);

/* NEXT-2 (DRGPUM_FEATURE_FREQUENCY) processes every attribute call in
 * sub-calls of at most records_per_call records (default 2^24); the
 * workspace holds 3 x records_per_call 8-byte event keys twice, plus the
 * digit histograms (~100 B per record of capacity).  The events of one API
 * that continues across calls are carried and must fit the capacity too
 * (ENOMEM at the query otherwise).  Set after objects_load, before
 * workspace_size / workspace_bind (ESTATE otherwise); EINVAL outside
 * [1024, 2^31]. */
DRGPUM_API drgpum_status drgpum_set_frequency_capacity(drgpum_ctx *ctx, uint64_t records_per_call);

/* Bytes of device workspace the loaded program needs (ESTATE before load). */
DRGPUM_API drgpum_status drgpum_workspace_size(const drgpum_ctx *ctx, uint64_t *bytes);

/* Bind caller-owned device memory (>= workspace_size bytes, 256-B aligned)
 * and enqueue on stream: upload of the static tables and zero-initialisation
 * of the shadow state (bitmaps/hit rows 0, first NEVER, last 0, counters 0).
 * ENOMEM if bytes is too small; EINVAL if d_ws is NULL or misaligned. */
DRGPUM_API drgpum_status drgpum_workspace_bind(drgpum_ctx *ctx, void *d_ws,
    uint64_t bytes, void *stream);

/* Enqueue re-zeroing of the shadow state: start a new trace over the same
 * objects and timeline (what one benchmark step does). */
DRGPUM_API drgpum_status drgpum_reset(drgpum_ctx *ctx, void *stream);

/* Attribute n device-resident records (d_recs 16-B aligned; n = 0 is a
 * no-op).  Asynchronous.  For every record: find the object live at its
 * timestamp that contains addr, set the bits of the touched elements, OR the
 * (API, read/write) hit bit, fold ts into first/last, count it (SURVEY §8(a)
 * A1-A5).  Records never fail the call; bad ones are counted as invalid.
 * Order-free: any permutation / chunking of the records gives identical
 * results.  EINVAL if d_recs is NULL (n > 0) or misaligned. */
DRGPUM_API drgpum_status drgpum_trace_attribute(drgpum_ctx *ctx,
    const drgpum_record_t *d_recs, uint64_t n, void *stream);

/* Same, from HOST memory: streams the records through two staging buffers
 * inside the workspace, overlapping host-to-device copies with attribution.
 * Synchronous w.r.t. the host buffer: returns once every record has been
 * copied (the attribution may still be running on stream).  Pinned memory
 * gives full PCIe/C2C bandwidth; pageable memory works but is slower. */
DRGPUM_API drgpum_status drgpum_trace_attribute_host(drgpum_ctx *ctx,
    const drgpum_record_t *h_recs, uint64_t n, void *stream);

/* Shadow-state locations inside the workspace (for merges), and per-object
 * placement (h_out has n_obj entries, load order). */
DRGPUM_API drgpum_status drgpum_shadow_view(const drgpum_ctx *ctx, drgpum_shadow_view_t *out);
DRGPUM_API drgpum_status drgpum_object_layout(const drgpum_ctx *ctx, drgpum_object_layout_t *h_out);

/* OR-merge: for w in [word_lo, word_hi) of the OR-mergeable
 * words, or_words[w] |= OR_{s<n_src} d_in[s*src_stride + (w - word_lo)].
 * d_in is device memory (e.g. the slices received by an all-to-all).
 * Asynchronous.  EINVAL if the range exceeds or_words. */
DRGPUM_API drgpum_status drgpum_merge_or(drgpum_ctx *ctx, const uint32_t *d_in,
    uint32_t n_src, uint64_t src_stride_words, uint64_t word_lo,
    uint64_t word_hi, void *stream);

/* Peer-memory merge ("P2P intermediate"; the exchange step of
 * the record-range sharding, §5.2 l.266-268 bitmaps and §5.1 l.242
 * first/last, merged by OR / MIN / MAX / SUM): ONE kernel per rank, over
 * NVLink peer pointers, instead of all-to-all + merge_or + all-gather.
 * h_peer_ws is a HOST array of n_peers device pointers: the workspace base of
 * every rank (index = rank; h_peer_ws[rank] must be this context's own
 * workspace), each bound to a context loaded with the same objects and
 * timeline (identical layouts) and addressable from this device -- the same
 * device, or mapped through NVLink (CUDA IPC / torch symmetric memory).
 * Rank r owns the r-th of n_peers equal slices of the OR words and of the
 * objects: it reads its slices from every peer, combines them and stores the
 * result into every peer's slices; rank 0 also sums the counters.  After ALL
 * ranks' calls have completed (the caller's barrier), every workspace holds
 * the merged shadow, bit-identical to a single-GPU run.  The caller must also
 * barrier BEFORE the call (every rank's attribution done).  Asynchronous.
 * EINVAL: n_peers == 0 or > 64, rank >= n_peers, a NULL / unaligned pointer,
 * or h_peer_ws[rank] != this workspace. */
DRGPUM_API drgpum_status drgpum_merge_peers(drgpum_ctx *ctx, void *const *h_peer_ws,
    uint32_t n_peers, uint32_t rank, void *stream);

/* Owned merge (the exchange step of the record-range sharding
 * with the finalize sharded by object, §5.2 l.266-268 bitmaps and
 * §5.1 l.242 first/last): rank r owns the objects [o_lo, o_hi) whose
 * boundaries split (bitmap words + objects) into n_peers near-equal parts;
 * ONE kernel reads those objects' bitmaps, hit rows and first/last from every
 * peer (h_peer_ws as for drgpum_merge_peers) and stores the OR / MIN / MAX
 * into THIS workspace only; rank 0 also sums the counters into every peer.
 * Then drgpum_finalize reduces and classifies only the owned objects, and
 * drgpum_gather_peers shares their stats and reports.  Compared with
 * drgpum_merge_peers, nothing is written to the peers' shadows (half the
 * NVLink traffic) and the finalize work is 1/n_peers per rank; the price is
 * that afterwards this workspace's shadow (bitmaps, hit rows, first/last) is
 * merged for the owned objects only.  Barriers as for drgpum_merge_peers
 * (before: all attribution done; after: all merges done).  Asynchronous.
 * EINVAL as for drgpum_merge_peers. */
DRGPUM_API drgpum_status drgpum_merge_peers_owned(drgpum_ctx *ctx, void *const *h_peer_ws,
    uint32_t n_peers, uint32_t rank, void *stream);

/* The same owned merge with NVLS (NVLink SHARP, SURVEY §8(e) "B200-native
 * stretch"): d_mc_ws is the NVSwitch multicast mapping of the ranks'
 * workspaces (torch symmetric memory's multicast_ptr; the workspace is the
 * symmetric buffer from its start).  Owned bitmap tiles and hit rows that at
 * least two OTHER ranks touched are read with multimem.ld_reduce...or, the
 * switch ORing every rank's copy (one read per word instead of one per
 * touching peer); the rest as drgpum_merge_peers_owned.  Needs NVSwitch
 * multicast (a multi-GPU NVLink box); untested on a single GPU, where torch
 * gives no multicast mapping.  EINVAL for a NULL / unaligned d_mc_ws, else
 * as drgpum_merge_peers_owned. */
DRGPUM_API drgpum_status drgpum_merge_peers_owned_nvls(drgpum_ctx *ctx, void *const *h_peer_ws,
    uint32_t n_peers, uint32_t rank, void *d_mc_ws, void *stream);

/* After drgpum_merge_peers_owned + drgpum_finalize on every rank (and a
 * barrier): stores this rank's objects' stats and pattern reports into every
 * peer's workspace and adds its consistency-violation count into every peer's
 * total.  After all ranks' calls have completed (barrier), object_stats,
 * patterns and consistency_errors return the single-GPU results on every
 * rank.  Asynchronous.  ESTATE without a preceding owned merge + finalize;
 * EINVAL for bad peers or an n_peers / rank different from the merge's.
 * object_stats / patterns after an owned merge return ESTATE until the
 * gather is done, and patterns with other thresholds than the finalize's
 * return ESTATE (a re-finalize would cover the owned objects only). */
DRGPUM_API drgpum_status drgpum_gather_peers(drgpum_ctx *ctx, void *const *h_peer_ws,
    uint32_t n_peers, uint32_t rank, void *stream);

/* Reduce-and-clear (default off).  While on, drgpum_finalize zeroes every
 * bitmap word it reduces (the per-object reductions of PAPER.md §5.2 l.268
 * read each word once), so the next drgpum_reset skips the bitmap tiles: one
 * pass over the shadow per trace instead of two.  After such a finalize the
 * bitmaps are CONSUMED: the shadow's bitmap words read back as zero,
 * drgpum_trace_attribute(_host) and the merge calls return DRGPUM_ESTATE
 * until drgpum_reset, while object_stats / patterns stay valid (other
 * thresholds re-run only the classification: the tile reductions are kept).
 * Hit rows, first / last and counters are untouched.  No effect after
 * drgpum_merge_peers_owned (the other ranks' objects are not finalized here).
 * Any time after create; on != 0 enables. */
DRGPUM_API drgpum_status drgpum_set_finalize_consume(drgpum_ctx *ctx, int on);

/* Enqueue the per-object reductions and the pattern classification on the
 * device (thresholds NULL = defaults).  Asynchronous; the results stay on
 * the device until object_stats / patterns copy them out. */
DRGPUM_API drgpum_status drgpum_finalize(drgpum_ctx *ctx,
    const drgpum_thresholds_t *th, void *stream);

/* Synchronous.  Runs finalize if the state changed since the last one, then
 * copies n_obj stats (load order) and the counters to the host.  Either
 * output pointer may be NULL. */
DRGPUM_API drgpum_status drgpum_object_stats(drgpum_ctx *ctx,
    drgpum_object_stats_t *h_out, drgpum_counters_t *h_ctr, void *stream);

/* Synchronous.  Finalizes with th (NULL = defaults) if needed and copies n_obj
 * pattern reports (load order) to the host. */
DRGPUM_API drgpum_status drgpum_patterns(drgpum_ctx *ctx,
    const drgpum_thresholds_t *th, drgpum_pattern_report_t *h_out, void *stream);

/* Number of internal consistency violations found by the last finalize
 * (first/last folded by atomics vs the hit rows; must be 0). */
DRGPUM_API drgpum_status drgpum_consistency_errors(drgpum_ctx *ctx,
    uint64_t *h_errors, void *stream);

/* NEXT-3 result (synchronous): h_sa[o] = 1 iff object o is accessed by at
 * least two GPU APIs and no element of o is touched by two different APIs
 * (each API touches its own slice, the slices do not overlap -- Def 3.10);
 * h_overlap[o] = 1 iff some element is touched by two APIs.  Either output
 * may be NULL.  ESTATE unless DRGPUM_FEATURE_STRUCTURED was enabled. */
DRGPUM_API drgpum_status drgpum_structured(drgpum_ctx *ctx, uint8_t *h_sa, uint8_t *h_overlap,
                                           void *stream);

/* API group of the NEXT-2 / NEXT-3 analyses [R22b, R23]: h_in_group[t] != 0
 * puts the GPU API at timestamp t in the group (NULL = every API, the
 * default after workspace_bind).  The paper reports structured access "at GPU
 * kernel gramschmidt_kernel3" (l.400): the group is then the invocations of
 * that kernel.  The structured-access pass of the following trace_attribute
 * calls only considers records of APIs in the group (set it before
 * attributing a trace); drgpum_structured counts the group's accessing APIs;
 * drgpum_slice_frequency uses the group at query time.  Synchronous (the
 * host array is consumed).  ESTATE before workspace_bind or without one of
 * the two features. */
DRGPUM_API drgpum_status drgpum_set_api_group(drgpum_ctx *ctx, const uint8_t *h_in_group, void *stream);

/* NEXT-2 results (synchronous; ESTATE unless DRGPUM_FEATURE_FREQUENCY, EINVAL
 * if the records were not in timestamp order).  For every (object O, access
 * API A in O's lifetime): n = elements A touched, S1 = sum of their access
 * frequencies, S2 = sum of squares [R22].  NUAF at A iff the population
 * coefficient of variation exceeds pct% (fn 3, l.222; X = 20% l.198), i.e.
 * (n*S2 - S1^2) * 100^2 > pct^2 * S1^2.  drgpum_frequency: per object the
 * number of APIs at which O matches (h_count) and the first one (h_first,
 * DRGPUM_NEVER if none).  drgpum_frequency_slots: the raw {n, S1, S2} triples,
 * u64[3 * n_slots], slots ordered by object (load order) then access API
 * (object o's slots start at sum of n_hit_apis of the objects before it). */
DRGPUM_API drgpum_status drgpum_frequency(drgpum_ctx *ctx, uint32_t pct, uint32_t *h_count,
                                          uint32_t *h_first, void *stream);
DRGPUM_API drgpum_status drgpum_frequency_slots(drgpum_ctx *ctx, uint64_t *h_acc,
                                                uint64_t *n_slots, void *stream);

/* Slice-level non-uniform access frequency [R22b] (Def 3.9 l.196 at the
 * granularity of §7.3 l.400, "the variance of access frequencies of
 * individual slices in R_gpu is 58%"): for object O, each API A of the group
 * (drgpum_set_api_group) that accesses O touches a slice of O whose access
 * frequency is F_A = S1 of slot (O, A) (the sum of its elements' counts).  O
 * matches iff the population coefficient of variation of {F_A} exceeds pct%,
 * exactly (n*S2 - S1^2) * 100^2 > pct^2 * S1^2 with n = number of such APIs,
 * S1 = sum F_A, S2 = sum F_A^2.  h_match u8[n_obj]; h_moments u64[4*n_obj] =
 * {n, S1, S2 low 64 bits, S2 high 64 bits} per object.  Either may be NULL.
 * Synchronous; errors as drgpum_frequency. */
DRGPUM_API drgpum_status drgpum_slice_frequency(drgpum_ctx *ctx, uint32_t pct, uint8_t *h_match,
                                                uint64_t *h_moments, void *stream);

/* Diagnostics (not part of the method): how many 32-record tiles took each
 * attribution path since the last reset -- out[0] affine run with one union
 * range, out[1] affine run with per-record words, out[2] per-tile fast path
 * (cached object and API), out[3] full per-lane path.  Synchronous. */
DRGPUM_API drgpum_status drgpum_path_stats(drgpum_ctx *ctx, uint64_t out[4], void *stream);

/* NEXT-1 redundant allocation (§5.1 l.253-260, Fig. 3; Def 3.3 l.154,
 * X = 10% l.156): the paper's one-pass pairing over the used objects' first
 * and last accessing APIs.  (reuser[k], donor[k]): object reuser[k] can reuse
 * donor[k]'s memory -- donor's last access precedes reuser's first (last after
 * first at equal timestamps), their sizes differ by at most pct% of the larger
 * [R19-R21], each donor is handed out once, pairs in the order the tail-to-head
 * walk finds them.  Up to cap pairs are written; *n_pairs is the total.
 *
 * drgpum_redundant_pairs is the host algorithm on plain arrays (sizes in
 * bytes, T_first, T_last, used flags; load order).  drgpum_redundant_alloc
 * runs it on the context's finalized stats (synchronous; finalizes if needed).
 * EINVAL on NULL outputs / pct > 100. */
DRGPUM_API drgpum_status drgpum_redundant_pairs(const uint64_t *sizes, const uint32_t *first,
    const uint32_t *last, const uint8_t *used, uint64_t n, uint32_t pct,
    uint32_t *reuser, uint32_t *donor, uint64_t cap, uint64_t *n_pairs);
DRGPUM_API drgpum_status drgpum_redundant_alloc(drgpum_ctx *ctx, uint32_t pct,
    uint32_t *reuser, uint32_t *donor, uint64_t cap, uint64_t *n_pairs, void *stream);

/* NEXT-4 multi-stream GPU applications (§5.3 l.273-297).
 *
 * Dependency graph G = (V, E) of Definition 5.1 (l.277-286): the vertices are
 * the timeline's APIs (timestamps 0..n_api-1 in invocation order, the value
 * access records carry [R24]); an edge i -> j exists when j is i's immediate
 * successor on the same stream (INTRA, l.281) or when, on some object, i
 * allocates/writes and j reads with no write in between (RAW, l.283), i
 * allocates/writes and j frees/writes with no access in between (WAW,
 * l.284), or i reads and j frees/writes with no write in between (WAR,
 * l.285).  Reads and writes are the per-(object, API) read/write sets the
 * attribution found [R25].  Kahn's algorithm with a global T (l.295) assigns
 * every vertex its topological level: T = 0 for in-degree-zero vertices, and
 * each round of deletions increments T. */
enum {
  DRGPUM_DEP_INTRA = 1,     /* same stream, immediate successor (l.281) */
  DRGPUM_DEP_RAW = 2,       /* read-after-write (l.283) */
  DRGPUM_DEP_WAW = 4,       /* write/free-after-write (l.284) */
  DRGPUM_DEP_WAR = 8        /* write/free-after-read (l.285) */
};

/* Kahn levels of an arbitrary edge list (src[k] -> dst[k], vertices < n_api;
 * duplicates allowed).  h_T: u32[n_api] out.  Host only, synchronous.
 * EINVAL on NULL pointers, an out-of-range vertex, or a cycle. */
DRGPUM_API drgpum_status drgpum_kahn_levels(uint32_t n_api, const uint32_t *src,
    const uint32_t *dst, uint64_t n_edges, uint32_t *h_T);

/* Build G for the trace attributed so far and level it.  h_stream: u32[n_api]
 * stream id of every API (any values; equal ids = same stream).  Outputs
 * (each may be NULL): h_T u32[n_api] the Kahn timestamps; up to cap edges in
 * (src, dst) order, duplicates merged with their labels OR-ed (h_src, h_dst
 * u32, h_label u8 DRGPUM_DEP_* bits); *n_edges (required) the edge count.
 * Synchronous (copies the hit rows to the host). */
DRGPUM_API drgpum_status drgpum_dependency_graph(drgpum_ctx *ctx, const uint32_t *h_stream,
    uint32_t *h_T, uint32_t *h_src, uint32_t *h_dst, uint8_t *h_label, uint64_t cap,
    uint64_t *n_edges, void *stream);

/* Pattern reports on topological timestamps h_T (u32[n_api], each < n_api,
 * e.g. drgpum_dependency_graph's).  EA / LD / TI / DW and their distances are
 * evaluated with an object's accesses ordered by (T, timestamp), "between"
 * counting every API whose T lies strictly between [R26], distances = T
 * differences (l.297); UA / ML / OA / OA_ACTIONABLE are time-free and equal
 * drgpum_patterns'.  With T = the invocation index this is drgpum_patterns.
 * Synchronous; EINVAL on NULL / out-of-range T. */
DRGPUM_API drgpum_status drgpum_patterns_topo(drgpum_ctx *ctx, const uint32_t *h_T,
    const drgpum_thresholds_t *th, drgpum_pattern_report_t *h_out, void *stream);

/* Message for the last failed call on ctx (never NULL). */
DRGPUM_API const char *drgpum_last_error(const drgpum_ctx *ctx);

/* Release host-side state (the workspace belongs to the caller). */
DRGPUM_API void drgpum_destroy(drgpum_ctx *ctx);

/* Number of kernel launches the library has enqueued on this context since
 * creation (evidence for benchmarks). */
DRGPUM_API uint64_t drgpum_launch_count(const drgpum_ctx *ctx);

#ifdef __cplusplus
}
#endif
#endif /* DRGPUM_H */
