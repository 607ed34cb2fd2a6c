/* wjindex.h — C ABI of the B200-native inverted-file indexer (Wei & JaJa, IPDPS 2011).
 *
 * PAPER.md = /root/reference/PAPER.md; "P:n" is its line n.  Readings S1..S19 of the paper are
 * listed in DESIGN.md §3.
 *
 * What the library computes (the paper's problem statement):
 *   * "parsing each document into a bag of words of the form <term, document ID> tuples, followed
 *     by constructing a postings list for each term such that each postings contains the ID of
 *     the document containing the term, term frequency";
 *   * postings "organized in a sorted order of document IDs", produced by consuming the
 *     documents in submission order;
 *   * a dictionary that maps every term to "the location of the postings list of each term and
 *     ... some related statistics": here df (u32) and cf (u64) (reading S11);
 *   * DocIDs are local id + global offset: 0-based u32 in global submission order (S9);
 *   * the dictionary is the paper's hybrid trie table (Table I) + per-collection B-trees
 *     of degree 16 with 512-byte nodes and 4-byte string caches (Table II).
 * Tokenisation (reading S1/S2/S4): maximal runs of [0-9A-Za-z] U [0x80-0xFF] inside one document,
 * ASCII A-Z folded, tokens longer than 255 bytes dropped and counted in n_dropped.
 * The result is unique (S18) and equals, byte for byte, the CPU oracle in oracle/.
 *
 * Every compute step runs in the library's sm_100a CUDA kernels.  There is no CPU fallback: a
 * call on a machine without a usable CUDA device fails with WJ_ERR_CUDA.
 *
 * Threading: one context per thread; a context is not thread-safe.  No exception crosses the ABI.
 * Error behaviour: every function returns a wj_status; on error index_last_error() describes it.
 * After a WJ_ERR_CUDA / WJ_ERR_NCCL error the context is unusable except for index_destroy.
 */
#ifndef WJINDEX_H
#define WJINDEX_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  WJ_OK = 0,
  WJ_NOT_FOUND = 1,            /* index_read_postings: term not in the dictionary (or not owned) */
  WJ_ERR_INVALID_ARG = -1,     /* NULL pointer, bad doc_off, n_bytes >= 2^32 in one call, ...     */
  WJ_ERR_STATE = -2,           /* call not allowed in the current state (see state machine)       */
  WJ_ERR_CUDA = -3,            /* CUDA runtime / kernel error, or no CUDA device                  */
  WJ_ERR_NCCL = -4,            /* NCCL error (world > 1)                                          */
  WJ_ERR_OOM = -5,             /* device allocation failed (or caller workspace exhausted)        */
  WJ_ERR_CAPACITY = -6,        /* > 2^32-1 documents or tokens; > 2^32-2 terms (one GPU) or 2^25 */
                               /* terms per slice (world > 1, stemming); > 2^25 distinct terms in  */
                               /* one index_add_stream call; string arena > 4 GiB                  */
  WJ_ERR_BUFFER_TOO_SMALL = -7 /* output buffer smaller than needed; *n_out holds the size needed */
} wj_status;

/* config.flags */
#define WJ_FLAG_PROFILE 0x1u   /* record CUDA events per phase (index_stats.phase_ms)               */
#define WJ_FLAG_LOOPBACK 0x2u  /* world > 1 inside one process: nccl_unique_id is a hub from        */
                               /* index_loopback_create; one host thread per rank context (tests)   */
#define WJ_FLAG_VBYTE 0x4u     /* finalize also encodes every postings list as d-gaps + variable-   */
                               /* byte code (reading S19) and            */
                               /* index_serialize writes the compressed file "WJINV002"             */
#define WJ_FLAG_HOST_PIPELINE 0x8u /* host-memory chunks are double-buffered: index_add_stream      */
                               /* enqueues the chunk's copy on a copy stream and indexes the        */
                               /* PREVIOUS host chunk meanwhile (Fig. 9 pipeline);       */
                               /* finalize (or a device-memory chunk) drains the pending chunk;     */
                               /* index_reset drops it.  Errors of a chunk may surface one call     */
                               /* late.  Use pinned host memory for the copy to overlap.            */
#define WJ_FLAG_BALANCED_OWNERS 0x10u /* world > 1: instead of b mod K, the first chunk's   */
                               /* 1 MiB samples are all-gathered and every rank bin-packs   */
                               /* the trie collections by sampled token count; the map is  */
                               /* kept for the context's lifetime, also across reset       */
#define WJ_FLAG_STEM 0x20u     /* parser Step 3 (reading S20): every term of   */
                               /* >= 3 bytes made only of a-z is replaced by its Porter (1980) stem */
                               /* before indexing; the dictionary holds stems (query by the stem)  */
#define WJ_FLAG_HOT_TERMS 0x80u /* opt-in: per chunk of >= 64 KiB the <= 127 most frequent terms of */
                               /* a 1 MiB sample are merged per       */
                               /* document in the tokenizer (one stream element with a count).      */
                               /* Same bytes; measured slower on config 2            */
#define WJ_FLAG_GLOBAL_STREAM 0x200u /* one GPU: instead of per-run partial postings lists (sorted  */
                               /* and run-length encoded per add_stream call beside the dictionary */
                               /* update, combined at finalize), keep one global      */
                               /* (term, docID) stream and sort it once at finalize.  Same bytes.   */
#define WJ_FLAG_STOPWORDS 0x40u /* parser Step 4 (reading S20): tokens whose (stemmed, with */
                               /* WJ_FLAG_STEM) term equals the (stemmed) form of a word of the     */
                               /* built-in 318-word English stop list are dropped; they count in    */
                               /* neither n_tokens nor n_dropped (index_stop_words lists the words) */

typedef struct wj_index wj_index; /* opaque; all index state is owned by the library */

typedef struct {
  int32_t device;            /* CUDA device ordinal                                               */
  int32_t rank, world;       /* world == 1: single GPU.  world > 1: see index_add_stream           */
  const void* nccl_unique_id;/* 128-byte ncclUniqueId when world > 1 (broadcast by the caller)     */
  void* stream;              /* cudaStream_t to launch on (e.g. torch's current stream); NULL =    */
                             /* the library creates its own non-blocking stream                    */
  uint64_t max_chunk_bytes;  /* hint: largest n_bytes of one index_add_stream call (0 = no hint)   */
  uint32_t flags;            /* WJ_FLAG_* ; other bits must be 0                                   */
  uint32_t reserved;         /* must be 0                                                          */
  void* workspace;           /* optional caller-owned device arena (e.g. a torch tensor's memory): */
  uint64_t workspace_bytes;  /* when non-NULL the library sub-allocates ALL its device buffers from */
                             /* it (first fit, 256-byte granules) and never calls cudaMalloc for    */
                             /* index state; the caller keeps it alive and unused until             */
                             /* index_destroy.  Exhausting it returns WJ_ERR_OOM.  NULL = the       */
                             /* library allocates with cudaMalloc.                                  */
} wj_config;

enum {
  WJ_PHASE_H2D = 0,      /* host -> device copy of a host-resident chunk (pre-processing)   */
  WJ_PHASE_TOKENIZE,     /* K1 count + emit: tokenise, normalise, chunk-local term dedup           */
  WJ_PHASE_UNIQUE,       /* unique-term compaction + Table I bucket + prefix strip     */
  WJ_PHASE_PROBE,        /* K3 B-tree probe of the chunk's unique terms                    */
  WJ_PHASE_INSERT,       /* K4 sort new terms, atomic termIDs, arena append, merge     */
  WJ_PHASE_REBUILD,      /* K4 bulk B-tree rebuild of the trie collections (Table II nodes)        */
  WJ_PHASE_STREAM,       /* (termID, docID) stream append (postings input)           */
  WJ_PHASE_LEXRANK,      /* finalize: global lexicographic order of the dictionary (S12)           */
  WJ_PHASE_SORT,         /* finalize: stable LSD radix sort of the stream by term rank             */
  WJ_PHASE_POSTINGS,     /* finalize: run-length (docID, tf), df, cf, post_off                     */
  WJ_PHASE_DICT,         /* finalize: term_off + term bytes of the final dictionary                */
  WJ_PHASE_EXCHANGE,     /* world > 1: all-to-all of the routed stream                             */
  WJ_PHASE_VBYTE,        /* finalize (WJ_FLAG_VBYTE): d-gap + variable-byte postings code  */
  WJ_PHASE_STEM,         /* WJ_FLAG_STEM/STOPWORDS: stem + stop-word test of the unique terms,     */
                         /* stem dedup, stop-word token compaction                     */
  WJ_PHASE_COUNT = 16
};

/* Individually timed kernels (WJ_FLAG_PROFILE): CUDA events bracket every launch of these. */
enum {
  WJ_KERNEL_TOKENIZE_COUNT = 0, /* K1 pass 1: classify bytes, count kept tokens per segment         */
  WJ_KERNEL_TOKENIZE_EMIT,      /* K1 pass 2: tokens -> chunk hash table -> (slot, docID) stream     */
  WJ_KERNEL_PROBE,              /* K3 warp-per-key B-tree descent                                   */
  WJ_KERNEL_SLOT_TO_TID,        /* stream slot -> termID                                           */
  WJ_KERNEL_MAP_RANK,           /* finalize: termID -> lexicographic rank                          */
  WJ_KERNEL_SORT_HIST,          /* radix digit histogram of the (term, docID) stream                */
  WJ_KERNEL_SORT_SCATTER,       /* stable radix scatter of the (term, docID) stream                 */
  WJ_KERNEL_RLE_EMIT,           /* run-length (docID, tf) emit of the sorted stream                 */
  WJ_KERNEL_COPY_PARTIALS,      /* finalize: copy each chunk's partial postings lists into place    */
  WJ_KERNEL_COUNT = 9
};

typedef struct {
  uint64_t n_docs, n_tokens, n_dropped, n_terms, n_postings, n_term_bytes;
  uint64_t n_chunks;               /* index_add_stream calls since init/reset                        */
  uint64_t kernel_launches;        /* kernels launched by the library since index_init (cumulative)  */
  uint64_t host_syncs;             /* stream synchronisations since index_init (cumulative)          */
  uint64_t unique_terms_last;      /* unique terms of the last chunk                                 */
  uint64_t new_terms_last;         /* terms inserted by the last chunk                               */
  uint64_t btree_nodes;            /* 512-byte B-tree nodes in the dictionary, and the tallest trie- */
  uint64_t btree_height_max;       /* collection B-tree, as of the last re-layout (done lazily before */
                                   /* the next chunk's probe or a retrieval)                          */
  uint64_t exchange_bytes;         /* world > 1: bytes this rank sent                                */
  uint64_t device_bytes;           /* device memory held by the context                              */
  uint64_t stream_elems;           /* (term, docID) stream elements of the index so far (tokens, and  */
                                   /* aggregated hot-term elements with WJ_FLAG_HOT_TERMS)            */
  uint64_t table_retries;          /* chunk hash-table probe overflows retried with a doubled table   */
                                   /* (cumulative since index_init)                                   */
  uint64_t hot_elems_saved;        /* stream elements merged away by the hot-term aggregation         */
                                   /* (cumulative since index_init)                                   */
  double exchange_ms;              /* world > 1: host wall time of the all-to-all-v rounds, device-    */
                                   /* synchronised (cumulative since index_init)                      */
  /* The fields below are cumulative since index_init (index_reset does not clear them).          */
  double phase_ms[WJ_PHASE_COUNT]; /* WJ_FLAG_PROFILE: accumulated CUDA-event time per phase        */
  uint64_t phase_launches[WJ_PHASE_COUNT];
  double kernel_ms[WJ_KERNEL_COUNT];      /* WJ_FLAG_PROFILE: accumulated time of each timed kernel  */
  uint64_t kernel_count[WJ_KERNEL_COUNT]; /* launches of each timed kernel                           */
} wj_stats;

/* Creates a context on cfg->device.  *out is set only on WJ_OK.  Ownership: the caller owns cfg
 * (read once); the library owns the context until index_destroy.
 * Errors: WJ_ERR_INVALID_ARG (NULL, bad rank/world, unknown flags), WJ_ERR_CUDA (no device),
 * WJ_ERR_NCCL, WJ_ERR_OOM. */
int index_init(wj_index** out, const wj_config* cfg);

/* Appends one chunk of documents ("a number of documents with a fixed total size").
 * Document i is bytes[doc_off[i] .. doc_off[i+1]), i < n_docs; doc_off has n_docs+1 entries,
 * doc_off[0] == 0, non-decreasing, doc_off[n_docs] == n_bytes; n_bytes < 2^32.  Empty documents
 * are allowed and consume a DocID (S16).  bytes and doc_off may each be host or device memory
 * (detected with cudaPointerGetAttributes); host memory is copied to the device on the context
 * stream (pinned memory makes the copy asynchronous).  Every document gets the next global
 * DocID in call order.
 * Stream-ordered: the call may return before the work finishes; the caller must keep the buffers
 * unchanged until the next index_* call on this context returns.
 * world > 1 (collective): every rank calls it the same number of times, each with its own
 * contiguous document range; rank r's documents follow rank r-1's within a call.
 * Errors: WJ_ERR_STATE (after finalize), WJ_ERR_INVALID_ARG, WJ_ERR_CAPACITY, WJ_ERR_CUDA, WJ_ERR_OOM. */
int index_add_stream(wj_index* ix, const void* bytes, uint64_t n_bytes, const uint64_t* doc_off,
                     uint64_t n_docs);

/* Builds the final inverted file on the device: dictionary in bytewise lexicographic order (S12),
 * postings (docID, tf) per term sorted by docID, df, cf.  Collective when world > 1.
 * Synchronises the context stream.  After it, index_add_stream returns WJ_ERR_STATE.
 * Errors: WJ_ERR_STATE (twice), WJ_ERR_CUDA, WJ_ERR_OOM. */
int index_finalize(wj_index* ix);

/* Retrieval: term -> trie index -> B-tree search -> postings.  term = normalised bytes
 * (ASCII lower case, 1..255 bytes), host memory.  docids/tfs: host arrays of cap entries.
 * Two-call sizing: if cap < df the call returns WJ_ERR_BUFFER_TOO_SMALL with *n_out = df.
 * Unknown term: WJ_NOT_FOUND, *n_out = 0.  Requires finalize (else WJ_ERR_STATE). */
int index_read_postings(wj_index* ix, const uint8_t* term, uint32_t len, uint32_t* docids,
                        uint32_t* tfs, uint64_t cap, uint64_t* n_out);

/* Canonical serialized inverted file (identical to the oracle's bytes), written to a
 * host buffer: "WJINV001", or with WJ_FLAG_VBYTE the compressed "WJINV002" (same header with
 * word 7 = code bytes, dictionary, df, cf; then u64 post_off[n_terms+1] in bytes and the code:
 * per posting vbyte(d-gap) then vbyte(tf), the first gap of a list = its docID; reading S19).  buf may be NULL (sizing call).  Requires finalize.  Errors: WJ_ERR_STATE,
 * WJ_ERR_BUFFER_TOO_SMALL (*n_out = size needed), WJ_ERR_CUDA. */
int index_serialize(wj_index* ix, uint8_t* buf, uint64_t cap, uint64_t* n_out);

/* Counters and per-phase times.  Synchronises the context stream. */
int index_stats(wj_index* ix, wj_stats* out);

/* Drops all documents and the dictionary but keeps device allocations (benchmark steps).  */
int index_reset(wj_index* ix);

/* Debug (tests only): tokenises one chunk exactly as index_add_stream does, without touching the
 * index, and writes the oracle's token-dump format to host memory: per kept token in text order
 * u32 docID (doc_base + local), u16 trie index (Table I), u8 len, len term bytes.
 * Two-call sizing on the byte count. */
int index_debug_tokens(wj_index* ix, const void* bytes, uint64_t n_bytes, const uint64_t* doc_off,
                       uint64_t n_docs, uint32_t doc_base, uint8_t* out, uint64_t cap, uint64_t* n_out);

/* Debug (tests only): copies the dictionary's B-tree state to host memory for the invariant checks
 * of the B-tree: nodes (512 B each, layout in DESIGN.md §5), per-collection
 * {root, n_keys, height} (3 x u32 per collection, 17,613 collections), and the string arena.
 * Any pointer may be NULL; *n_nodes, *arena_bytes are always set. */
int index_debug_btree(wj_index* ix, void* nodes, uint64_t node_cap, uint64_t* n_nodes,
                      uint32_t* collections, uint8_t* arena, uint64_t arena_cap,
                      uint64_t* arena_bytes);

/* Multi-GPU.  Rank r owns the trie collections b with b mod world == r
 * and builds that exclusive dictionary slice; every index_add_stream call is collective and
 * moves, per owner, the chunk's unique terms and (term, docID) token records with one all-to-all-v
 * (NCCL over NVLink, or the loopback hub).  index_serialize returns the rank's slice (its terms;
 * n_docs global, other header counts local); index_merge_serialized merges the slices of all ranks
 * into the canonical global file (host, untimed).  index_read_postings answers owned terms only. */

/* Writes a fresh 128-byte ncclUniqueId (rank 0 calls it and broadcasts the bytes).  WJ_ERR_NCCL if
 * libnccl.so.2 cannot be loaded (override the path with the WJ_NCCL_LIB environment variable). */
int index_nccl_unique_id(void* out128);

/* In-process transport for world ranks driven by world host threads on one device (tests). */
int index_loopback_create(int32_t world, void** hub);
void index_loopback_destroy(void* hub);

/* Merges k serialized slices (host memory) into the global serialized index; two-call sizing like
 * index_serialize.  WJ_ERR_INVALID_ARG if a slice does not parse or n_docs differ. */
int index_merge_serialized(int32_t k, const uint8_t* const* slices, const uint64_t* sizes, uint8_t* out, uint64_t cap,
                           uint64_t* n_out);

/* Host helper (no device): the balanced owner map's bin packing, exposed for tests.  Items (trie
 * collections) by count desc, index asc on ties, each to the least-loaded rank (lowest on ties);
 * count-0 items keep i mod world.  WJ_ERR_INVALID_ARG on NULL or world < 1. */
int index_balance_owners(const uint64_t* counts, uint32_t n, int32_t world, uint32_t* owner);

/* The built-in stop list of WJ_FLAG_STOPWORDS (parser Step 4; reading S20): 318 lowercase
 * words separated by single spaces, NUL-terminated, owned by the library (static storage). */
const char* index_stop_words(void);

/* Debug (tests): the device Porter stemmer (parser Step 3) on n host words.  Word i is
 * words[word_off[i] .. word_off[i+1]) (folded bytes, <= 255 each); its stem (reading S20: only
 * words of >= 3 bytes of a-z change) is written to out[word_off[i] ..] (a stem is never longer
 * than its word) with its length in out_len[i].  All pointers are host memory owned by the caller.
 * Runs on `device` with a temporary stream.  WJ_ERR_INVALID_ARG on NULL or a word > 255 bytes,
 * WJ_ERR_CUDA without a device. */
int index_debug_stem(int32_t device, const uint8_t* words, const uint32_t* word_off, uint32_t n, uint8_t* out,
                     uint32_t* out_len);

/* Owner rank of every trie collection (out: n >= 17613 entries): b mod world, or the balanced map
 * once the first chunk has built it (WJ_FLAG_BALANCED_OWNERS).  WJ_ERR_INVALID_ARG if n is small. */
int index_owner_map(wj_index* ix, uint32_t* out, uint32_t n);

const char* index_last_error(const wj_index* ix);
void index_destroy(wj_index* ix);

#ifdef __cplusplus
}
#endif
#endif /* WJINDEX_H */
