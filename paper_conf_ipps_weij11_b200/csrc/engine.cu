// Engine + C ABI (include/wjindex.h): owns device state, orders the kernels of one chunk and of
// finalize on the context stream, and turns CUDA errors into wj_status codes.
#include <algorithm>
#include <chrono>
#include <map>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "../../include/wjindex.h"
#include "common.cuh"
#include "dict.cuh"
#include "dist.cuh"
#include "hot.cuh"
#include "partials.cuh"
#include "exchange.h"
#include "postings.cuh"
#include "radix.cuh"
#include "scan.cuh"
#include "stem.cuh"
#include "tokenize.cuh"
#include "vbyte.cuh"

using namespace wj;

namespace {

struct StatusError {
  int code;
  std::string msg;
};

struct DevBuf {
  void* p = nullptr;
  size_t cap = 0;  // bytes
};

// Caller-owned device workspace (wj_config.workspace, e.g. a torch tensor): the library sub-allocates
// every device buffer from it, first fit with coalescing of freed neighbours, 256-byte granules.
struct Arena {
  uintptr_t base = 0;
  uint64_t bytes = 0;
  std::map<uint64_t, uint64_t> free_;  // offset -> size
  std::map<uint64_t, uint64_t> used_;  // offset -> size
  void init(void* p, uint64_t n) {
    const uintptr_t a = ((uintptr_t)p + 255) & ~(uintptr_t)255;
    base = a;
    bytes = n > (a - (uintptr_t)p) ? (n - (a - (uintptr_t)p)) & ~(uint64_t)255 : 0;
    free_.clear();
    used_.clear();
    if (bytes) free_[0] = bytes;
  }
  void* alloc(uint64_t n) {
    n = (n + 255) & ~(uint64_t)255;
    for (auto it = free_.begin(); it != free_.end(); ++it) {
      if (it->second < n) continue;
      const uint64_t off = it->first, sz = it->second;
      free_.erase(it);
      if (sz > n) free_[off + n] = sz - n;
      used_[off] = n;
      return (void*)(base + off);
    }
    return nullptr;
  }
  void release(void* p) {
    const uint64_t off = (uint64_t)((uintptr_t)p - base);
    auto u = used_.find(off);
    if (u == used_.end()) return;
    uint64_t o = off, n = u->second;
    used_.erase(u);
    auto nx = free_.lower_bound(o);
    if (nx != free_.end() && nx->first == o + n) {
      n += nx->second;
      nx = free_.erase(nx);
    }
    if (nx != free_.begin()) {
      auto pv = std::prev(nx);
      if (pv->first + pv->second == o) {
        o = pv->first;
        n += pv->second;
        free_.erase(pv);
      }
    }
    free_[o] = n;
  }
};

struct PhaseRec {
  int phase;
  cudaEvent_t a, b;
  uint64_t launches;
};
struct KernelRec {
  int k;
  cudaEvent_t a, b;
};

template <typename T>
__global__ void k_fill(T* p, uint64_t n, T v) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = v;
}

__global__ void k_update_counts(uint32_t* coll_n, const uint32_t* nlo, const uint32_t* nhi) {
  const uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b < kCollections) coll_n[b] += nhi[b] - nlo[b];
}
__global__ void k_iota_u32(uint32_t* p, uint32_t n) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = i;
}

// doc_off validation: doc_off[0]==0, non-decreasing, doc_off[n]==n_bytes
__global__ void k_check_docoff(const uint64_t* d, uint64_t n_docs, uint64_t n_bytes, uint32_t* bad) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i > n_docs) return;
  bool ok = true;
  if (i == 0) ok = d[0] == 0;
  else ok = d[i - 1] <= d[i];
  if (i == n_docs) ok = ok && d[i] == n_bytes;
  if (!ok) atomicExch(bad, 1u);
}

struct NonZeroSlot {
  const Slot* t;
  __device__ __forceinline__ uint32_t operator()(uint64_t i) const { return t[i].k0 != 0 ? 1u : 0u; }
};
struct IsMiss {
  const uint32_t* t;
  __device__ __forceinline__ uint32_t operator()(uint64_t i) const { return t[i] == kMiss ? 1u : 0u; }
};
struct ArenaSizeU {
  const uint32_t* u_tid;
  const uint32_t* u_len;
  const uint32_t* u_bucket;
  __device__ __forceinline__ uint32_t operator()(uint64_t u) const {
    return u_tid[u] == kMiss ? 1u + u_len[u] - bucket_plen(u_bucket[u]) : 0u;
  }
};

inline unsigned grid_for(uint64_t n, unsigned block) { return (unsigned)((n + block - 1) / block); }

}  // namespace

// Greedy longest-processing-time bin packing (host): items by count desc (index asc on ties), each
// to the least-loaded rank (lowest rank on ties); items with count 0 keep i mod K.
static void lpt_owner_map(const uint64_t* count, uint32_t n, int K, uint32_t* owner) {
  std::vector<uint32_t> order(n);
  for (uint32_t b = 0; b < n; ++b) {
    order[b] = b;
    owner[b] = b % (uint32_t)K;
  }
  std::stable_sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) { return count[a] > count[b]; });
  std::vector<uint64_t> load(K, 0);
  for (uint32_t b : order) {
    if (count[b] == 0) break;
    int best = 0;
    for (int r = 1; r < K; ++r)
      if (load[r] < load[best]) best = r;
    owner[b] = (uint32_t)best;
    load[best] += count[b];
  }
}

// Stop list of WJ_FLAG_STOPWORDS (parser Step 4; the paper names no list).  Reading S20:
// the 318-word English list scikit-learn ships as ENGLISH_STOP_WORDS (Glasgow IR group), sorted.
static const char kStopList[] =
    "a about above across after afterwards again against all almost alone along already also although "
    "always am among amongst amoungst amount an and another any anyhow anyone anything anyway anywhere are "
    "around as at back be became because become becomes becoming been before beforehand behind being below "
    "beside besides between beyond bill both bottom but by call can cannot cant co con could couldnt cry de "
    "describe detail do done down due during each eg eight either eleven else elsewhere empty enough etc "
    "even ever every everyone everything everywhere except few fifteen fifty fill find fire first five for "
    "former formerly forty found four from front full further get give go had has hasnt have he hence her "
    "here hereafter hereby herein hereupon hers herself him himself his how however hundred i ie if in inc "
    "indeed interest into is it its itself keep last latter latterly least less ltd made many may me "
    "meanwhile might mill mine more moreover most mostly move much must my myself name namely neither never "
    "nevertheless next nine no nobody none noone nor not nothing now nowhere of off often on once one only "
    "onto or other others otherwise our ours ourselves out over own part per perhaps please put rather re "
    "same see seem seemed seeming seems serious several she should show side since sincere six sixty so "
    "some somehow someone something sometime sometimes somewhere still such system take ten than that the "
    "their them themselves then thence there thereafter thereby therefore therein thereupon these they "
    "thick thin third this those though three through throughout thru thus to together too top toward "
    "towards twelve twenty two un under until up upon us very via was we well were what whatever when "
    "whence whenever where whereafter whereas whereby wherein whereupon wherever whether which while "
    "whither who whoever whole whom whose why will with within without would yet you your yours yourself "
    "yourselves";

struct wj_index {
  int device = 0;
  int rank = 0, world = 1;
  cudaStream_t st = nullptr;
  bool own_stream = false;
  // f3 host-streamed pipelining (WJ_FLAG_HOST_PIPELINE; Fig. 9): a host chunk is copied
  // on the copy stream `cs` into one of two staging slots while the previous chunk is indexed
  bool pipeline = false;
  cudaStream_t cs = nullptr;
  DevBuf pipe_text[2], pipe_off[2];
  cudaEvent_t pipe_copied[2] = {nullptr, nullptr}, pipe_done[2] = {nullptr, nullptr};
  bool pipe_used[2] = {false, false};
  bool pend = false;
  int pend_slot = 0, next_slot = 0;
  uint64_t pend_bytes = 0, pend_nd = 0;
  uint32_t flags = 0;
  std::string err;
  bool finalized = false;
  bool broken = false;

  // counters
  uint64_t n_elems = 0;  // stream length (tokens + hot-term elements + holes)
  uint64_t n_docs = 0, n_tokens = 0, n_dropped = 0, n_chunks = 0, launches = 0, syncs = 0;
  uint64_t unique_last = 0, new_last = 0, n_nodes = 0, height_max = 0;
  uint32_t V = 0;
  uint64_t arena_used = 0;
  // The first insert into an empty dictionary takes its arena size A from a bound (the chunk's text
  // bytes + U, set in dict_text_bytes by the caller; 0 = no bound) instead of a host round trip on the
  // dictionary stream; A stays on the device (dscal[4]) until settle_arena() reads it.
  uint64_t dict_text_bytes = 0;
  bool arena_pending = false;
  uint64_t table_est = 0;
  bool recs_by_tid = false;     // the records of run 0 are indexed by termID (chunk_partials)
  uint64_t table_retries = 0;  // chunk-table probe overflows retried with a larger table (cumulative)
  // chunk table capacity = table_pct% of the expected unique terms, any multiple of 4096 slots
  // (mulhi indexing).  On config 2 the emit kernel gets faster with capacity (2.82 / 2.45 /
  // 2.36 ms at 125 / 190 / 320%: shorter probe runs) while the slot -> rank gather of the first sort
  // pass and the slot scans get slower; 190-230% was the best step time (profiles/r01_README.md)
  uint64_t table_pct = 200;
  uint64_t P = 0, TB = 0, PB = 0;  // postings, term bytes, vbyte code bytes
  bool vbyte = false;              // WJ_FLAG_VBYTE
  bool balanced = false;           // WJ_FLAG_BALANCED_OWNERS
  bool owner_ready = false;        // owner_tab built (kept across index_reset: bound for the lifetime)
  std::vector<uint32_t> owner_h;   // collection -> rank (host copy)
  uint64_t exchange_bytes = 0;

  Transport* xport = nullptr;  // world > 1
  // sampled hot terms of the current chunk (hot.cuh): hot_slotb = hot id -> chunk-table slot
  DevBuf hot_samp, hot_slotb, hot_kb, hot_matb, hot_posb, hot_cfb, hot_nhb, samp_off, samp_slot, samp_doc, samp_cnt, samp_ck, samp_cv,
      samp_ck2, samp_cv2, samp_n;
  uint32_t hot_H = 0, hot_D = 0;  // hot terms of the current chunk (matrix rows), its documents
  bool stream_has_hot = false;  // some chunk appended hot-term elements (holes + counts > 1)
  // Partial postings per chunk (partials.cuh; single GPU, no stemming / stop words / hot terms): the
  // chunk's stream is sorted by slot and run-length encoded on side_st while the dictionary update
  // runs on st; finalize combines the partial lists.  WJ_PARTIALS=0: global stream
  // sorted at finalize instead.
  bool pm = false;
  // packed chunk stream (partials path without hot terms): the emit kernel writes one u64 per token,
  // slot << 32 | docID, into pc_key; the sort moves it as a value-less 64-bit key and the run-length
  // pass reads it back (one 8-byte access per element everywhere instead of two 4-byte ones)
  unsigned long long* emit_elem = nullptr;
  bool pc_packed = false;
  bool side_launched = false;  // the current chunk's side-stream work is enqueued (side_launch)
  cudaStream_t side_st = nullptr, hp_st = nullptr;  // side: lowest priority; hp: dictionary, highest
  cudaEvent_t ev_fork = nullptr, ev_side = nullptr, ev_dict = nullptr;
  cudaEvent_t ev_dfork = nullptr;  // the dictionary stream's fork (after the unique terms are gathered)
  DevBuf side_scan, side_hist, side_hist_scan;
  DevBuf mr_key, mr_idx, mr_key2, mr_idx2, mr_dst, mr_src;  // several runs: records in destination order
  DevBuf u_pack;  // per unique term {tid, info, insertion rank, arena offset} for k_ns_fill
  DevBuf pc_dig;  // packed stream: one digit byte per element for the next radix pass's upsweep
  DevBuf pc_key, pc_doc, pc_po, pc_cs, u_slot, pp_pair, x_pair, rec_tid, rec_start, rec_df, rec_cf, rec_aos, rec_before, df_totb,
      cf_totb;
  uint64_t pbase = 0, nrec = 0;      // partial postings / records of the chunks so far
  uint32_t rs_ctas = kRsCtas;        // radix downsweep CTAs (ranges) of sort_pairs
  uint32_t side_ctas = kRsCtas;      // ... for the side stream's sort (148 / 222 / 592 / 1184 measured slower)
  bool pc_pending = false;           // the last chunk's posting count is still on the device (dscal[13])
  bool pc_join = false;              // the last chunk's side-stream work is not joined yet
  uint64_t pc_U = 0, pc_Nc = 0;  // pc_Nc: tokens of the pending chunk
  bool pc_hot = false;                         // the pending chunk has hot-term lists
  bool pc_settle_hot = false;                  // ... the joined, unsettled chunk
  uint64_t pc_settle_tokens = 0;
  uint32_t doc_base_cur = 0;                   // first DocID of the chunk being indexed
  std::vector<uint64_t> rec_end;     // end of each chunk's records
  uint64_t sorted_elems = 0;    // stream elements the last finalize sorted (after hole compaction)
  // Sampled hot terms (hot.cuh) merged per document in the emit kernel: opt-in
  // (WJ_FLAG_HOT_TERMS, every chunk of >= 64 KiB); measured slower on config 2 (profiles/r02_README.md)
  uint64_t hot_min_bytes = ~0ull;
  uint64_t hot_elems_saved = 0;  // stream elements merged away by the hot-term aggregation (cumulative)
  uint64_t pm_merged = 0;        // ... of this index on the partials path (its stream_elems exclude them)
  DevBuf x_owner, x_iota, x_sorted, x_sorted2, x_owner2, x_xid, x_cnt, x_toff, x_boff, x_send, x_tkey, x_tidx, x_tkey2,
      x_tidx2, x_rkey, x_rdoc, x_keymap, x_recv_terms, x_recv_key, x_recv_doc, x_loc_slot, x_loc_doc, x_syn_slot, x_syn_doc, x_syn_off, x_roff, x_tbase,
      x_hdf, x_hcf, x_rhdf, x_rhcf, x_rpre, x_bnd;
  double exchange_ms = 0;  // host wall time inside the all-to-all-v calls (cumulative)
  // persistent dictionary
  // E = per-collection sorted key order: termID, info (Table I index | full length << 16), arena offset
  DevBuf nodes, coll_root, coll_n, coll_base, coll_base2, e_tid, e_bkt, e_tid2, e_bkt2, e_ar, e_ar2, arena, t_arena, t_cache,
      t_bucket;
  // device scalars: [0] tokens, [1] dropped, [2] U, [3] Nnew, [4] arena total, [5] overflow|bad,
  // [6] unused, [7] level count, [8] P, [9] TB, [10] bad doc_off, [11] rle tokens,
  DevBuf scal;
  uint64_t* h_scal = nullptr;  // pinned
  // token stream (termID, docID) of all chunks
  DevBuf g_tid, g_doc;
  // chunk scratch
  DevBuf text_stage, doc_stage, seg_cnt, table, uid, u_w, u_ref, u_len, u_bucket, u_cache, u_key, u_tid, u_rank, midx, nk_key,
      nk_val, nk_key2, nk_val2, aoff, ns_tid, ns_bucket, ns_rank, ns_info, ns_arena, nlo, nhi, nbase, lvA[4], lvB[4], child_off, root_idx,
      scan_scr, hist, hist_scan, kstart, slotref, dbg_start, dbg_len, dbg_off, dbg_out, dbg_slot, dbg_doc, lexg, lex_short, qbuf, qres;
  // finalize
  DevBuf rank_of, term_at, sk1, sv1, pidx, out_doc, out_tf, post_off, df, cf, term_off, term_bytes;
  DevBuf vb_first, vb_tiles, vb_code, vb_boff;  // f1 (WJ_FLAG_VBYTE)
  DevBuf samp_hist, owner_tab;                  // f2(i) (WJ_FLAG_BALANCED_OWNERS)
  // f4 parser Steps 3-4 (WJ_FLAG_STEM / WJ_FLAG_STOPWORDS; stem.cuh): the surface table is kept in
  // table_s / uid_s while table / uid / u_* describe the chunk's unique stems over the stem text
  bool stem_on = false, stop_on = false;
  uint32_t n_stop = 0;
  DevBuf table_s, uid_s, st_off, st_text, st_keep, st_tidx, st_m1, st_slot, st_doc, st_tiles, st_doff, stop_keys;
  std::vector<DevBuf> chunk_map;        // per chunk: slot -> termID (-> rank at finalize)
  std::vector<uint64_t> chunk_tok;      // per chunk: first token index in the stream
  std::vector<uint32_t> chunk_C;        // per chunk: table capacity
  DevBuf rle_look, rle_p0, rle_lead, rle_tok, cstart_b;
  uint32_t* f_key = nullptr;   // sorted keys (term ranks)
  uint32_t* f_doc = nullptr;   // sorted docIDs
  // profiling
  std::vector<PhaseRec> recs;
  std::vector<cudaEvent_t> ev_pool;
  size_t ev_used = 0;
  int cur_phase = -1;
  uint64_t phase_launch0 = 0;
  double phase_ms[WJ_PHASE_COUNT] = {0};
  uint64_t phase_launches[WJ_PHASE_COUNT] = {0};
  std::vector<KernelRec> krecs;
  double kernel_ms[WJ_KERNEL_COUNT] = {0};
  uint64_t kernel_count[WJ_KERNEL_COUNT] = {0};
  size_t device_bytes = 0;

  // ---------------------------------------------------------------- memory
  bool use_arena = false;  // wj_config.workspace given: every device buffer comes from it
  Arena arena_ws;
  void* dev_alloc(size_t n) {
    if (use_arena) {
      void* p = arena_ws.alloc(n);
      if (!p) throw StatusError{WJ_ERR_OOM, "workspace exhausted (" + std::to_string(n) + " more bytes needed)"};
      return p;
    }
    void* p = nullptr;
    cudaError_t e = cudaMalloc(&p, n);
    if (e != cudaSuccess) {
      cudaGetLastError();
      throw StatusError{WJ_ERR_OOM, "cudaMalloc(" + std::to_string(n) + ") failed: " + cudaGetErrorString(e)};
    }
    return p;
  }
  void dev_free(void* p) {
    if (!p) return;
    if (use_arena) arena_ws.release(p);
    else cudaFree(p);
  }
  void* grow(DevBuf& b, size_t bytes, bool keep = false, size_t keep_bytes = 0) {
    if (bytes <= b.cap && b.p) return b.p;
    size_t nc = std::max(bytes, b.cap + b.cap / 2);
    nc = (nc + 255) & ~(size_t)255;
    void* np = dev_alloc(nc);
    if (keep && b.p && keep_bytes) WJ_CUDA_CHECK(cudaMemcpyAsync(np, b.p, keep_bytes, cudaMemcpyDeviceToDevice, st));
    if (b.p) {
      // other streams (side / dictionary) may still read the old buffer: wait for the device
      WJ_CUDA_CHECK(cudaStreamSynchronize(st));
      if (side_st) WJ_CUDA_CHECK(cudaStreamSynchronize(side_st));
      if (hp_st) WJ_CUDA_CHECK(cudaStreamSynchronize(hp_st));
      dev_free(b.p);
      device_bytes -= b.cap;
    }
    b.p = np;
    b.cap = nc;
    device_bytes += nc;
    return np;
  }
  template <typename T>
  T* buf(DevBuf& b, uint64_t n) { return (T*)grow(b, std::max<uint64_t>(n, 1) * sizeof(T)); }
  template <typename T>
  T* buf_keep(DevBuf& b, uint64_t n, uint64_t used) {
    return (T*)grow(b, std::max<uint64_t>(n, 1) * sizeof(T), true, used * sizeof(T));
  }
  void free_all() {
    DevBuf* all[] = {&nodes, &coll_root, &coll_n, &coll_base, &coll_base2, &e_tid, &e_bkt, &e_tid2, &e_bkt2, &e_ar, &e_ar2, &arena,
                     &t_arena, &t_cache, &t_bucket, &scal, &g_tid, &g_doc, &text_stage, &doc_stage, &seg_cnt, &table,
                     &uid, &u_w, &u_ref, &u_len, &u_bucket, &u_cache, &u_key, &u_tid, &u_rank, &midx, &nk_key, &nk_val,
                     &nk_key2, &nk_val2, &aoff, &ns_tid, &ns_bucket, &ns_rank, &ns_info, &ns_arena, &nlo, &nhi, &nbase, &child_off,
                     &root_idx, &scan_scr, &hist, &hist_scan, &kstart, &slotref, &dbg_start, &dbg_len, &dbg_off, &dbg_out, &dbg_slot,
                     &dbg_doc, &lexg, &lex_short, &qbuf, &qres, &rank_of, &term_at, &sk1, &sv1, &pidx, &out_doc, &out_tf,
                     &post_off, &df, &cf, &term_off, &term_bytes, &vb_first, &vb_tiles, &vb_code, &vb_boff, &samp_hist, &owner_tab,
                     &table_s, &uid_s, &st_off, &st_text, &st_keep, &st_tidx, &st_m1, &st_slot, &st_doc, &st_tiles,
                     &st_doff, &stop_keys, &side_scan, &side_hist, &side_hist_scan, &pc_key, &pc_doc, &pc_po,
                     &pc_cs, &u_slot, &pp_pair, &x_pair, &mr_key, &mr_idx, &mr_key2, &mr_idx2, &mr_dst, &mr_src, &rec_tid, &rec_start, &rec_df, &rec_cf, &rec_aos, &rec_before, &df_totb,
                     &cf_totb, &pc_dig, &u_pack};
    for (DevBuf* b : all) {
      dev_free(b->p);
      b->p = nullptr;
      b->cap = 0;
    }
    DevBuf* hs[] = {&hot_samp, &hot_slotb, &hot_kb, &hot_matb, &hot_posb, &hot_cfb, &hot_nhb, &samp_off, &samp_slot, &samp_doc, &samp_cnt,
                    &samp_ck, &samp_cv, &samp_ck2, &samp_cv2, &samp_n};
    for (DevBuf* b : hs) { dev_free(b->p); *b = DevBuf{}; }
    DevBuf* xs[] = {&x_owner, &x_iota, &x_sorted, &x_sorted2, &x_owner2, &x_xid, &x_cnt, &x_toff, &x_boff, &x_send,
                    &x_tkey, &x_tidx, &x_tkey2, &x_tidx2, &x_rkey, &x_rdoc, &x_keymap, &x_recv_terms, &x_recv_key, &x_recv_doc, &x_loc_slot,
                    &x_loc_doc, &x_syn_slot, &x_syn_doc, &x_syn_off, &x_roff, &x_tbase, &x_hdf, &x_hcf, &x_rhdf,
                    &x_rhcf, &x_rpre, &x_bnd};
    for (DevBuf* b : xs) { dev_free(b->p); *b = DevBuf{}; }
    for (auto& b : chunk_map) dev_free(b.p);
    chunk_map.clear();
    for (DevBuf* b : {&rle_look, &rle_p0, &rle_lead, &rle_tok, &cstart_b}) { dev_free(b->p); *b = DevBuf{}; }
    for (int i = 0; i < 4; ++i) {
      dev_free(lvA[i].p);
      dev_free(lvB[i].p);
      lvA[i] = DevBuf{};
      lvB[i] = DevBuf{};
    }
  }

  void* scan_scratch(uint64_t n, size_t elem) {
    const uint64_t tiles = (n + kScanTile - 1) / kScanTile;
    return grow(scan_scr, (size_t)(tiles + 2) * elem * 2 + 1024);
  }

  // ---------------------------------------------------------------- launch bookkeeping
#ifdef WJ_DEBUG_LAUNCH  // debug build: every launch synchronised, a fault reported with its call site
  void launched(int n = 1, int line = __builtin_LINE()) {
    launches += n;
    cudaError_t e = cudaDeviceSynchronize();
    if (e == cudaSuccess) e = cudaGetLastError();
    if (e != cudaSuccess) throw CudaError(e, "kernel launch", __FILE__, line);
  }
#else
  void launched(int n = 1) {
    launches += n;
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) throw CudaError(e, "kernel launch", __FILE__, __LINE__);
  }
#endif
  void sync() {
    WJ_CUDA_CHECK(cudaStreamSynchronize(st));
    ++syncs;
  }
  cudaEvent_t ev() {
    if (ev_used == ev_pool.size()) {
      cudaEvent_t e;
      WJ_CUDA_CHECK(cudaEventCreate(&e));
      ev_pool.push_back(e);
    }
    return ev_pool[ev_used++];
  }
  void phase(int p) {
    if (!(flags & WJ_FLAG_PROFILE)) { cur_phase = p; return; }
    if (cur_phase >= 0) {
      PhaseRec& r = recs.back();
      WJ_CUDA_CHECK(cudaEventRecord(r.b, st));
      r.launches = launches - phase_launch0;
    }
    cur_phase = p;
    if (p >= 0) {
      PhaseRec r{p, ev(), ev(), 0};
      WJ_CUDA_CHECK(cudaEventRecord(r.a, st));
      recs.push_back(r);
      phase_launch0 = launches;
    }
  }
  // times one launch (or a few) of kernel k with CUDA events when profiling
  template <class F>
  void ktime(int k, F&& launch) {
    if (!(flags & WJ_FLAG_PROFILE)) { launch(); return; }
    KernelRec r{k, ev(), ev()};
    WJ_CUDA_CHECK(cudaEventRecord(r.a, st));
    launch();
    WJ_CUDA_CHECK(cudaEventRecord(r.b, st));
    krecs.push_back(r);
  }
  void collect_phases() {
    if (recs.empty() && krecs.empty()) return;
    if (cur_phase >= 0) phase(-1);
    sync();
    if (side_st) WJ_CUDA_CHECK(cudaStreamSynchronize(side_st));  // side-stream events (partials)
    for (auto& r : recs) {
      float ms = 0;
      WJ_CUDA_CHECK(cudaEventElapsedTime(&ms, r.a, r.b));
      phase_ms[r.phase] += ms;
      phase_launches[r.phase] += r.launches;
    }
    for (auto& r : krecs) {
      float ms = 0;
      WJ_CUDA_CHECK(cudaEventElapsedTime(&ms, r.a, r.b));
      kernel_ms[r.k] += ms;
      kernel_count[r.k] += 1;
    }
    recs.clear();
    krecs.clear();
    ev_used = 0;
  }
  uint64_t* dscal() { return (uint64_t*)scal.p; }
  void readback(int first, int count) {
    WJ_CUDA_CHECK(cudaMemcpyAsync(h_scal + first, dscal() + first, count * sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    sync();
  }

  template <typename T, typename F>
  void scan(F in, uint64_t n, T* out, T* d_total) {
    void* s = scan_scratch(n, sizeof(T));
    launched(0);
    launches += exclusive_scan<T, F>(in, n, out, d_total, s, st);
    launched(0);
  }

  // ---------------------------------------------------------------- init / reset
  void reset_state() {
    if (cs) WJ_CUDA_CHECK(cudaStreamSynchronize(cs));
    if (side_st) WJ_CUDA_CHECK(cudaStreamSynchronize(side_st));  // an unjoined chunk (partials)
    pend = false;  // a pending (copied, not yet indexed) host chunk is dropped
    collect_phases();
    chunk_tok.clear();
    chunk_C.clear();
    n_docs = n_tokens = n_dropped = n_chunks = n_elems = 0;
    stream_has_hot = false;
    sorted_elems = 0;
    pbase = nrec = 0;
    pm_merged = 0;
    pc_pending = pc_join = false;
    side_launched = false;
    rec_end.clear();
    unique_last = new_last = n_nodes = height_max = 0;
    btree_dirty = false;
    exchange_bytes = 0;
    V = 0;
    arena_used = 0;
    arena_pending = false;
    dict_text_bytes = 0;
    P = TB = PB = 0;
    finalized = false;
    f_key = f_doc = nullptr;
    cur_phase = -1;
    uint32_t* cn = buf<uint32_t>(coll_n, kCollections + 1);
    uint32_t* cb = buf<uint32_t>(coll_base, kCollections + 1);
    uint32_t* cr = buf<uint32_t>(coll_root, kCollections + 1);
    WJ_CUDA_CHECK(cudaMemsetAsync(cn, 0, (kCollections + 1) * 4, st));
    WJ_CUDA_CHECK(cudaMemsetAsync(cb, 0, (kCollections + 1) * 4, st));
    WJ_CUDA_CHECK(cudaMemsetAsync(cr, 0xFF, (kCollections + 1) * 4, st));
    buf<uint64_t>(scal, 16);
    WJ_CUDA_CHECK(cudaMemsetAsync(scal.p, 0, 16 * 8, st));
    sync();
  }

  // ---------------------------------------------------------------- chunk staging
  static bool is_device_ptr(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
  }

  void stage(const void* bytes, uint64_t n_bytes, const uint64_t* doc_off, uint64_t nd, const uint8_t** text_d,
             const uint64_t** off_d) {
    const bool dev_text = n_bytes == 0 || is_device_ptr(bytes);
    const bool dev_off = is_device_ptr(doc_off);
    if (!dev_off) {
      // host doc_off: validate here (cheap) before copying
      if (doc_off[0] != 0 || doc_off[nd] != n_bytes) throw StatusError{WJ_ERR_INVALID_ARG, "doc_off[0] must be 0 and doc_off[n_docs] == n_bytes"};
      for (uint64_t i = 0; i < nd; ++i)
        if (doc_off[i] > doc_off[i + 1]) throw StatusError{WJ_ERR_INVALID_ARG, "doc_off must be non-decreasing"};
    }
    const bool any_host = !dev_text || !dev_off;
    if (any_host) phase(WJ_PHASE_H2D);
    if (dev_text && ((uintptr_t)bytes & 15) == 0) {
      *text_d = (const uint8_t*)bytes;
    } else {
      uint8_t* t = buf<uint8_t>(text_stage, n_bytes + 16);
      if (n_bytes) WJ_CUDA_CHECK(cudaMemcpyAsync(t, bytes, n_bytes, dev_text ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, st));
      *text_d = t;
    }
    if (dev_off) {
      *off_d = doc_off;
    } else {
      uint64_t* o = buf<uint64_t>(doc_stage, nd + 1);
      WJ_CUDA_CHECK(cudaMemcpyAsync(o, doc_off, (nd + 1) * 8, cudaMemcpyHostToDevice, st));
      *off_d = o;
    }
    uint32_t* bad = (uint32_t*)(dscal() + 10);
    WJ_CUDA_CHECK(cudaMemsetAsync(bad, 0, 8, st));
    if (dev_off) {
      k_check_docoff<<<grid_for(nd + 1, 256), 256, 0, st>>>(*off_d, nd, n_bytes, bad);
      launched();
    }
  }

  // K1 count + scan; returns kept tokens of the chunk (host sync)
  uint64_t count_tokens(const ChunkView& cv, uint64_t n_segs) {
    const uint64_t ranges = (n_segs + kSegsPerWarp - 1) / kSegsPerWarp;
    const unsigned grid = (unsigned)((ranges + kTokWarps - 1) / kTokWarps);
    uint32_t* cnt = buf<uint32_t>(seg_cnt, ranges + 1);
    uint64_t* ks = buf<uint64_t>(kstart, ranges);
    k_warp_kstart<<<grid_for(ranges, 256), 256, 0, st>>>(cv, ranges, ks);
    launched();
    WJ_CUDA_CHECK(cudaMemsetAsync(dscal() + 1, 0, 8, st));
    ktime(WJ_KERNEL_TOKENIZE_COUNT, [&] {
      k_tok_count<<<grid, kTokThreads, 0, st>>>(cv, (uint32_t)n_segs, ks, cnt, (unsigned long long*)(dscal() + 1));
      launched();
    });
    scan<uint32_t>(ArrayIn<uint32_t>{cnt}, ranges, cnt, (uint32_t*)(dscal() + 0));
    readback(0, 11);  // kept tokens [0], dropped [1], doc_off check [10]: one round trip
    if ((uint32_t)h_scal[10]) throw StatusError{WJ_ERR_INVALID_ARG, "doc_off must start at 0, be non-decreasing and end at n_bytes"};
    return (uint32_t)h_scal[0];
  }

  void emit_tokens(const ChunkView& cv, uint64_t n_segs, uint32_t* slot_out, uint32_t* doc_out, uint32_t doc_base,
                   uint64_t C, uint32_t* dstart, uint32_t* dlen, bool use_hot = false, bool clear_table = true) {
    Slot* tab = buf<Slot>(table, C);
    uint32_t* sref = buf<uint32_t>(slotref, C);
    if (clear_table) WJ_CUDA_CHECK(cudaMemsetAsync(tab, 0, C * sizeof(Slot), st));
    WJ_CUDA_CHECK(cudaMemsetAsync(dscal() + 5, 0, 8, st));
    EmitOut eo;
    eo.hot_mat = (use_hot && hot_H) ? (uint32_t*)hot_matb.p : nullptr;
    eo.hot_docs = hot_D;
    eo.table = tab;
    eo.slot_ref = sref;
    eo.cap = (uint32_t)C;
    eo.parts = tab_parts;
    eo.part_cap = (uint32_t)(C / tab_parts);
    eo.owner_tab = owner_ready ? (const uint32_t*)owner_tab.p : nullptr;
    eo.doc_base = doc_base;
    eo.slot = slot_out;
    eo.doc = doc_out;
    eo.elem = use_hot ? nullptr : emit_elem;
    eo.dig0 = eo.elem ? (uint8_t*)pc_dig.p : nullptr;
    eo.dbg_start = dstart;
    eo.dbg_len = dlen;
    eo.overflow = (uint32_t*)(dscal() + 5);
    const uint64_t ranges = (n_segs + kSegsPerWarp - 1) / kSegsPerWarp;
    const unsigned grid = (unsigned)((ranges + kTokWarps - 1) / kTokWarps);
    ktime(WJ_KERNEL_TOKENIZE_EMIT, [&] {
      const uint64_t* ks = (const uint64_t*)kstart.p;
      const uint32_t* ro = (const uint32_t*)seg_cnt.p;
      if (eo.parts > 1)
        k_tok_emit<false, true><<<grid, kTokThreads, 0, st>>>(cv, (uint32_t)n_segs, ks, ro, eo);
      else if (eo.hot_mat)
        k_tok_emit<true, false><<<grid, kTokThreads, 0, st>>>(cv, (uint32_t)n_segs, ks, ro, eo);
      else
        k_tok_emit<false, false><<<grid, kTokThreads, 0, st>>>(cv, (uint32_t)n_segs, ks, ro, eo);
      launched();
    });
  }

  // Sampled popular terms of a chunk ("1MB out of every 1GB"): tokenise the first 1 MiB of
  // its documents with the same kernels, count terms, keep the <= 256 most frequent (>= 16
  // occurrences, <= 11 bytes) -> hot_kb (slot words).  Returns the number of hot terms.
  // The paper's sample, "1MB out of every 1GB": tokenise the first 1 MiB of the chunk's
  // documents into the chunk table and count tokens per slot (samp_cnt).  Returns the sample's
  // kept tokens (0: no usable sample); Cs = table capacity used.
  uint64_t sample_counts(const ChunkView& cv, uint64_t& Cs, uint64_t min_tokens) {
    Cs = 0;
    const uint64_t S = std::min<uint64_t>(cv.n_bytes, 1ull << 20);
    if (S == 0 || cv.n_docs == 0) return 0;
    uint64_t* sn = buf<uint64_t>(samp_n, 1);
    k_sample_docs<<<1, 32, 0, st>>>(cv.doc_off, cv.n_docs, S, nullptr, sn);
    launched();
    uint64_t nds = 0;
    WJ_CUDA_CHECK(cudaMemcpyAsync(&nds, sn, 8, cudaMemcpyDeviceToHost, st));
    sync();
    if (nds == 0) return 0;
    uint64_t* so = buf<uint64_t>(samp_off, nds + 1);
    k_sample_docs_copy<<<grid_for(nds + 1, 256), 256, 0, st>>>(cv.doc_off, nds, S, so);
    launched();
    ChunkView sv{cv.text, S, so, nds};
    const uint64_t n_segs = (S + kSegBytes - 1) / kSegBytes;
    const uint64_t Ns = count_tokens(sv, n_segs);
    if (Ns < std::max<uint64_t>(min_tokens, 1)) return 0;
    uint32_t* ss = buf<uint32_t>(samp_slot, Ns + 16);
    uint32_t* sd = buf<uint32_t>(samp_doc, Ns + 16);
    Cs = pow2_at_least(2 * Ns);
    emit_tokens(sv, n_segs, ss, sd, 0, Cs, nullptr, nullptr, false, true);
    readback(5, 1);
    if ((uint32_t)h_scal[5]) return 0;
    uint32_t* cnt = buf<uint32_t>(samp_cnt, Cs);
    WJ_CUDA_CHECK(cudaMemsetAsync(cnt, 0, Cs * 4, st));
    k_sample_count<<<grid_for(Ns, 256), 256, 0, st>>>(ss, Ns, cnt);
    launched();
    return Ns;
  }

  // f2(i): balanced owner map ("split these trie collections into N_I independent sets such
  // that each contains almost the same number of tokens"; bound for the lifetime).  Every
  // rank samples its first chunk, the per-collection token counts are all-gathered, and every rank
  // runs the same greedy longest-processing-time assignment (collections by count desc, then index;
  // each to the least-loaded rank, lowest rank on ties); unsampled collections keep b mod K.
  void build_owner_map(const ChunkView* cv) {
    const int K = world;
    std::vector<uint64_t> mine(kCollections, 0), all((size_t)kCollections * K);
    uint64_t Cs = 0;
    if (cv && sample_counts(*cv, Cs, 1) > 0) {
      uint64_t* h = buf<uint64_t>(samp_hist, kCollections);
      WJ_CUDA_CHECK(cudaMemsetAsync(h, 0, kCollections * 8, st));
      k_sample_buckets<<<grid_for(Cs, 256), 256, 0, st>>>((const Slot*)table.p, (const uint32_t*)slotref.p,
                                                          (const uint32_t*)samp_cnt.p, (uint32_t)Cs, cv->text,
                                                          (unsigned long long*)h);
      launched();
      WJ_CUDA_CHECK(cudaMemcpyAsync(mine.data(), h, kCollections * 8, cudaMemcpyDeviceToHost, st));
      sync();
    }
    xport->allgather(mine.data(), kCollections, all.data(), st);
    std::vector<uint64_t> tot(kCollections, 0);
    for (int r = 0; r < K; ++r)
      for (uint32_t b = 0; b < kCollections; ++b) tot[b] += all[(size_t)r * kCollections + b];
    owner_h.assign(kCollections, 0);
    lpt_owner_map(tot.data(), kCollections, K, owner_h.data());
    uint32_t* d = buf<uint32_t>(owner_tab, kCollections);
    WJ_CUDA_CHECK(cudaMemcpyAsync(d, owner_h.data(), kCollections * 4, cudaMemcpyHostToDevice, st));
    sync();
    owner_ready = true;
  }

  // Sampled hot terms of a chunk ("1MB out of every 1GB"), without a host round trip:
  // the first 1 MiB of the chunk is tokenised into a scratch table (documents past it are never
  // reached; a token cut at the edge occurs once and cannot reach kHotMinCount), tokens are counted per
  // slot, (count, slot) pairs sorted, and k_hot_pick keeps the <= Hmax most frequent terms with
  // >= kHotMinCount occurrences (<= 11 bytes) in hot_kb, their number in *hot_Hdev().
  uint32_t* hot_Hdev() { return (uint32_t*)(dscal() + 14) + 1; }
  void select_hot(const ChunkView& cv, uint32_t Hmax) {
    const uint64_t S = std::min<uint64_t>(cv.n_bytes, 1ull << 20);
    ChunkView sv{cv.text, S, cv.doc_off, cv.n_docs};
    const uint64_t n_segs = (S + kSegBytes - 1) / kSegBytes;
    const uint64_t ranges = (n_segs + kSegsPerWarp - 1) / kSegsPerWarp;
    uint32_t* cnt = buf<uint32_t>(seg_cnt, ranges + 1);
    uint64_t* ks = buf<uint64_t>(kstart, ranges);
    k_warp_kstart<<<grid_for(ranges, 256), 256, 0, st>>>(sv, ranges, ks);
    k_tok_count<<<(unsigned)((ranges + kTokWarps - 1) / kTokWarps), kTokThreads, 0, st>>>(
        sv, (uint32_t)n_segs, ks, cnt, (unsigned long long*)(dscal() + 15));  // (its dropped count is ignored)
    launched(2);
    uint32_t* ns = (uint32_t*)(dscal() + 14);  // sample tokens
    scan<uint32_t>(ArrayIn<uint32_t>{cnt}, ranges, cnt, ns);
    const uint64_t Nmax = S + 16;  // a kept token takes >= 1 byte
    uint32_t* ss = buf<uint32_t>(samp_slot, Nmax);
    uint32_t* sd = buf<uint32_t>(samp_doc, Nmax);
    const uint64_t Cs = pow2_at_least(2 * Nmax);  // at most half full: no probe overflow
    emit_tokens(sv, n_segs, ss, sd, 0, Cs, nullptr, nullptr, false, true);
    uint32_t* sc = buf<uint32_t>(samp_cnt, Cs);
    WJ_CUDA_CHECK(cudaMemsetAsync(sc, 0, Cs * 4, st));
    k_sample_count_dev<<<grid_for(Nmax, 256), 256, 0, st>>>(ss, ns, sc);
    uint32_t* ck = buf<uint32_t>(samp_ck, Cs + 16);
    uint32_t* cv2 = buf<uint32_t>(samp_cv, Cs + 16);
    uint32_t* ck2 = buf<uint32_t>(samp_ck2, Cs + 16);
    uint32_t* cvb = buf<uint32_t>(samp_cv2, Cs + 16);
    k_sample_cand<<<grid_for(Cs, 256), 256, 0, st>>>((const Slot*)table.p, sc, (uint32_t)Cs, ck, cv2);
    launched(2);
    int bits = 0;
    while ((1ull << bits) <= Nmax) ++bits;
    const bool in1 = sort_pairs<uint32_t>(ck, cv2, ck2, cvb, Cs, 0, bits, nullptr, false);
    ulonglong2* hk = (ulonglong2*)grow(hot_kb, kHotMax * sizeof(ulonglong2));
    k_hot_pick<<<1, kHotMax, 0, st>>>(in1 ? ck2 : ck, in1 ? cvb : cv2, (uint32_t)Cs, (const Slot*)table.p, Hmax, hk,
                                      hot_Hdev());
    launched();
    buf<uint32_t>(hot_slotb, kHotMax + 1);  // written by k_hot_seed
  }

  // L2 persisting access-policy window on the context stream (best effort; cleared with bytes == 0)
  size_t l2_persist_max = 0;
  void set_l2_window(void* p, size_t bytes) {
    if (l2_persist_max == 0) {
      int v = 0;
      cudaDeviceGetAttribute(&v, cudaDevAttrMaxPersistingL2CacheSize, device);
      l2_persist_max = v > 0 ? (size_t)v : 1;
      if (v > 0 && cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)v) != cudaSuccess) cudaGetLastError();
    }
    if (l2_persist_max <= 1) return;
    cudaStreamAttrValue a;
    memset(&a, 0, sizeof(a));
    if (bytes) {
      int maxw = 0;
      cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, device);
      const size_t win = std::min(bytes, (size_t)maxw);
      a.accessPolicyWindow.base_ptr = p;
      a.accessPolicyWindow.num_bytes = win;
      a.accessPolicyWindow.hitRatio = (float)std::min(1.0, (double)l2_persist_max / (double)win);
      a.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
      a.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    }
    if (cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &a) != cudaSuccess) cudaGetLastError();
    if (!bytes && cudaCtxResetPersistingL2Cache() != cudaSuccess) cudaGetLastError();
  }

  // chunk table capacity: a multiple of 4096 slots (mulhi indexing takes any capacity)
  uint64_t table_cap(uint64_t x) const { return std::max<uint64_t>((x + 4095) / 4096 * 4096, 4096); }
  static uint64_t pow2_at_least(uint64_t x) {
    uint64_t c = 1;
    while (c < x) c <<= 1;
    return c;
  }

  // ---------------------------------------------------------------- one chunk
  // K1 (count + emit + dedup): tokens of cv into (slot, docID) arrays given by out_alloc(Nc); unique
  // terms of the chunk into the u_* arrays.  Returns Nc; sets C (table capacity), U.
  // parts > 1 (multi-rank): the table is cut into `parts` equal partitions, partition o holding the
  // terms whose trie collection rank o owns, so slot order groups the unique terms and
  // the sorted stream by owner
  uint32_t tab_parts = 1;  // partitions of the table emit_tokens fills
  template <class F>
  uint64_t tokenize_dedup(const ChunkView& cv, uint32_t doc_base, F&& out_alloc, uint64_t& C, uint64_t& U,
                          uint32_t*& slot_out, uint32_t*& doc_out, bool allow_hot = false, uint32_t parts = 1) {
    const uint64_t n_segs = (cv.n_bytes + kSegBytes - 1) / kSegBytes;
    C = 0;
    U = 0;
    phase(WJ_PHASE_TOKENIZE);
    hot_H = 0;
    hot_D = (uint32_t)cv.n_docs;
    if (allow_hot && cv.n_bytes >= hot_min_bytes && cv.n_docs > 0) {
      // hot_H = rows of the (hot term x document) matrix (<= 256 MB); the picked count is on the device
      hot_H = (uint32_t)std::min<uint64_t>(kHotMax, (64ull << 20) / cv.n_docs);
      if (hot_H) select_hot(cv, hot_H);
    }
    const uint64_t Nc = count_tokens(cv, n_segs);
    n_dropped += h_scal[1];
    out_alloc(Nc, slot_out, doc_out);
    if (Nc == 0) return 0;
    // capacity ~1.5-3x the expected unique terms (U/N ~ 1/30 on Zipf text; the next chunk uses
    // the last U); a probe-sequence overflow retries with a doubled table
    uint64_t est = std::max<uint64_t>({table_est, Nc / 32, 4096});
    est = std::min<uint64_t>(est, Nc + 16);
    // stream elements carry the slot below the count bits (slot | count << kCountShift): C <= 2^25
    constexpr uint64_t kMaxC = (uint64_t)kRankMask + 1;
    uint64_t Cp = table_cap(est * table_pct / 100 / parts);  // slots per partition
    C = std::min<uint64_t>(Cp * parts, kMaxC / parts * parts);
    tab_parts = parts;
    uint32_t* slot_uid = nullptr;
    for (;;) {
      Slot* tab = buf<Slot>(table, C);
      uint32_t* sref = buf<uint32_t>(slotref, C);
      WJ_CUDA_CHECK(cudaMemsetAsync(tab, 0, C * sizeof(Slot), st));
      if (hot_H) {  // hot terms first: their slots in this table carry their hot ids
        uint32_t* mat = buf<uint32_t>(hot_matb, (uint64_t)hot_H * hot_D);
        WJ_CUDA_CHECK(cudaMemsetAsync(mat, 0, (uint64_t)hot_H * hot_D * 4, st));
        WJ_CUDA_CHECK(cudaMemsetAsync(dscal() + 5, 0, 8, st));
        k_hot_seed<<<1, 128, 0, st>>>((const ulonglong2*)hot_kb.p, hot_Hdev(), tab, sref, (uint32_t)C,
                                      (uint32_t*)hot_slotb.p, (uint32_t*)(dscal() + 5));
        launched();
      }
      emit_tokens(cv, n_segs, slot_out, doc_out, doc_base, C, nullptr, nullptr, hot_H > 0, false);
      if (pc_packed && Nc > 0) side_launch(Nc, C, false);  // the sort needs the stream only
      phase(WJ_PHASE_UNIQUE);
      slot_uid = buf<uint32_t>(uid, C);
      scan<uint32_t>(NonZeroSlot{(const Slot*)table.p}, C, slot_uid, (uint32_t*)(dscal() + 2));
      WJ_CUDA_CHECK(cudaMemsetAsync((uint32_t*)(dscal() + 2) + 1, 0, 4, st));
      readback(2, 4);
      U = (uint32_t)h_scal[2];
      if (((uint32_t)h_scal[5]) == 0) break;
      // probe sequence overflow: retry with a larger table (an early-forked sort reads the stream the
      // retry rewrites: drained first, then forked again)
      if (side_launched) {
        WJ_CUDA_CHECK(cudaStreamSynchronize(side_st));
        side_launched = false;
      }
      if (C >= kMaxC / parts * parts) {
        tab_parts = 1;
        throw StatusError{WJ_ERR_CAPACITY, "more than ~2^25 distinct terms in one index_add_stream call: pass smaller chunks"};
      }
      C = std::min<uint64_t>(C * 2, kMaxC / parts * parts);
      ++table_retries;
      phase(WJ_PHASE_TOKENIZE);
    }
    tab_parts = 1;
    unique_last = U;
    table_est = (U * 5) / 4;
    // unique terms: first occurrence, folded bytes, Table I bucket, stripped-suffix cache, sort key
    uint4* uw = buf<uint4>(u_w, U);
    uint32_t* ur = buf<uint32_t>(u_ref, U);
    uint32_t* ul = buf<uint32_t>(u_len, U);
    uint32_t* ub = buf<uint32_t>(u_bucket, U);
    uint32_t* uc = buf<uint32_t>(u_cache, U);
    uint64_t* uk = buf<uint64_t>(u_key, U);
    uint32_t* us = buf<uint32_t>(u_slot, U);
    k_unique_gather<<<grid_for(C, 256), 256, 0, st>>>((const Slot*)table.p, (const uint32_t*)slotref.p, (uint32_t)C,
                                                      slot_uid, cv.text, uw, ur, ul, ub, uc, uk, us);
    launched();
    return Nc;
  }

  // ---------------------------------------------------------------- f4: parser Steps 3-4
  // WJ_FLAG_STEM / WJ_FLAG_STOPWORDS (stem.cuh).  In: the surface dedup of a chunk
  // (table / uid / u_*: C1 slots, U1 unique terms over `text`) and its stream (slot, doc)[Nc].
  // Out: table_s / uid_s hold the surface table; table / uid / u_* the U2 unique stems over
  // `ntext`; st_m1[s] = unique-stem index of surface slot s; the stream is compacted in place
  // (stop-word tokens removed).  Returns the kept token count.
  uint64_t normalize(const uint8_t* text, uint64_t C1, uint64_t U1, uint32_t* slot, uint32_t* doc, uint64_t Nc,
                     uint64_t& U2, const uint8_t*& ntext) {
    phase(WJ_PHASE_STEM);
    U2 = 0;
    uint64_t* off = buf<uint64_t>(st_off, U1 + 1);
    scan<uint64_t>(LenPlus1{(const uint32_t*)u_len.p}, U1, off, off + U1);
    WJ_CUDA_CHECK(cudaMemcpyAsync(h_scal + 12, off + U1, 8, cudaMemcpyDeviceToHost, st));
    sync();
    const uint64_t B = h_scal[12];
    uint8_t* nt = (uint8_t*)grow(st_text, B + 32);
    uint32_t* keep = buf<uint32_t>(st_keep, U1 + 1);
    k_stem_terms<<<grid_for(U1, 256), 256, 0, st>>>((const uint4*)u_w.p, (const uint32_t*)u_ref.p,
                                                    (const uint32_t*)u_len.p, text, (uint32_t)U1, off, nt, stem_on ? 1 : 0,
                                                    stop_on ? (const ulonglong2*)stop_keys.p : nullptr, n_stop, keep);
    launched();
    uint32_t* tidx = buf<uint32_t>(st_tidx, U1 + 1);
    scan<uint32_t>(ArrayIn<uint32_t>{keep}, U1, tidx, tidx + U1);
    WJ_CUDA_CHECK(cudaMemcpyAsync(h_scal + 13, tidx + U1, 4, cudaMemcpyDeviceToHost, st));
    sync();
    const uint64_t Kk = (uint32_t)h_scal[13];
    std::swap(table, table_s);  // keep the surface table; the stem dedup reuses the scratch set
    std::swap(uid, uid_s);
    uint32_t* sslot = nullptr;
    if (Kk > 0) {
      uint64_t* so = buf<uint64_t>(st_doff, 2);
      const uint64_t h2[2] = {0, B};
      WJ_CUDA_CHECK(cudaMemcpyAsync(so, h2, 16, cudaMemcpyHostToDevice, st));
      ChunkView sv{nt, B, so, 1};
      const uint64_t est0 = table_est, dropped0 = n_dropped;
      uint64_t C2 = 0;
      uint32_t* sdoc = nullptr;
      const uint64_t Ns = tokenize_dedup(sv, 0, [&](uint64_t nc, uint32_t*& sp, uint32_t*& dp) {
        sp = buf<uint32_t>(st_slot, nc + 16);
        dp = buf<uint32_t>(st_doc, nc + 16);
      }, C2, U2, sslot, sdoc);
      table_est = est0;
      n_dropped = dropped0;
      unique_last = U1;
      if (Ns != Kk) throw StatusError{WJ_ERR_CUDA, "stem text: token count mismatch (internal)"};
      phase(WJ_PHASE_STEM);
    }
    uint32_t* m1 = buf<uint32_t>(st_m1, C1);
    k_norm_map<<<grid_for(C1, 256), 256, 0, st>>>((const Slot*)table_s.p, (const uint32_t*)uid_s.p, (uint32_t)C1, keep,
                                                  tidx, sslot, (const uint32_t*)uid.p, m1);
    launched();
    uint64_t kept = Nc;
    if (Kk < U1) {
      kept = drop_tokens(slot, doc, Nc, m1);
      k_clear_drop<<<grid_for(C1, 256), 256, 0, st>>>(m1, (uint32_t)C1);
      launched();
    }
    ntext = nt;
    return kept;
  }

  // stable in-place compaction of a (slot, doc) stream: drops elements whose m1[slot] has kDropBit
  uint64_t drop_tokens(uint32_t* slot, uint32_t* doc, uint64_t n, const uint32_t* m1) {
    if (n == 0) return 0;
    const uint64_t T = (n + kDropTile - 1) / kDropTile;
    uint32_t* tk = buf<uint32_t>(st_tiles, T + 1);
    k_drop_count<<<(unsigned)T, kDropThreads, 0, st>>>(slot, n, m1, tk);
    launched();
    scan<uint32_t>(ArrayIn<uint32_t>{tk}, T, tk, tk + T);
    WJ_CUDA_CHECK(cudaMemcpyAsync(h_scal + 14, tk + T, 4, cudaMemcpyDeviceToHost, st));
    uint32_t* s2 = buf<uint32_t>(sk1, n + 16);
    uint32_t* d2 = buf<uint32_t>(sv1, n + 16);
    k_drop_write<<<(unsigned)T, kDropThreads, 0, st>>>(slot, doc, n, m1, tk, s2, d2);
    launched();
    sync();
    const uint64_t kept = (uint32_t)h_scal[14];
    if (kept) {
      WJ_CUDA_CHECK(cudaMemcpyAsync(slot, s2, kept * 4, cudaMemcpyDeviceToDevice, st));
      WJ_CUDA_CHECK(cudaMemcpyAsync(doc, d2, kept * 4, cudaMemcpyDeviceToDevice, st));
    }
    return kept;
  }

  // stop keys (index_init, WJ_FLAG_STOPWORDS): the built-in list, stemmed on the device when
  // WJ_FLAG_STEM (Step 4 follows Step 3, S20), sorted and deduplicated on the host
  void build_stop_keys() {
    std::vector<uint8_t> words;
    std::vector<uint32_t> woff{0};
    for (const char* p = kStopList;; ++p) {
      if (*p == ' ' || *p == 0) {
        if (words.size() > woff.back()) woff.push_back((uint32_t)words.size());
        if (*p == 0) break;
      } else {
        words.push_back((uint8_t)*p);
      }
    }
    const uint32_t nw = (uint32_t)woff.size() - 1;
    uint8_t* dw = (uint8_t*)grow(st_text, words.size() + 32);
    uint32_t* doff = buf<uint32_t>(st_tidx, nw + 1);
    ulonglong2* dk = (ulonglong2*)grow(stop_keys, (size_t)nw * sizeof(ulonglong2));
    WJ_CUDA_CHECK(cudaMemcpyAsync(dw, words.data(), words.size(), cudaMemcpyHostToDevice, st));
    WJ_CUDA_CHECK(cudaMemcpyAsync(doff, woff.data(), woff.size() * 4, cudaMemcpyHostToDevice, st));
    k_stop_keys<<<grid_for(nw, 128), 128, 0, st>>>(dw, doff, nw, stem_on ? 1 : 0, dk);
    launched();
    std::vector<ulonglong2> hk(nw);
    WJ_CUDA_CHECK(cudaMemcpyAsync(hk.data(), dk, (size_t)nw * sizeof(ulonglong2), cudaMemcpyDeviceToHost, st));
    sync();
    auto less = [](const ulonglong2& a, const ulonglong2& b) { return a.x < b.x || (a.x == b.x && a.y < b.y); };
    std::sort(hk.begin(), hk.end(), less);
    hk.erase(std::unique(hk.begin(), hk.end(), [](const ulonglong2& a, const ulonglong2& b) { return a.x == b.x && a.y == b.y; }),
             hk.end());
    n_stop = (uint32_t)hk.size();
    WJ_CUDA_CHECK(cudaMemcpyAsync(dk, hk.data(), hk.size() * sizeof(ulonglong2), cudaMemcpyHostToDevice, st));
    sync();
  }

  // The B-trees are re-laid lazily: an insert only marks them stale; the next probe (the next chunk's
  // dictionary update) or a retrieval rebuilds them first, so the last chunk of an index never pays
  // for a rebuild that nothing reads (finalize ranks terms from E and the arena, not from the nodes).
  bool btree_dirty = false;
  void ensure_btrees() {
    if (!btree_dirty) return;
    btree_dirty = false;
    const int open = cur_phase;
    phase(WJ_PHASE_REBUILD);
    rebuild();
    phase(open);
  }

  // K3 probe + K4 insert of the chunk's unique terms (u_* arrays) -> u_tid
  void dictionary_update(const uint8_t* text, uint64_t U) {
    uint32_t* ut = buf<uint32_t>(u_tid, U);
    uint32_t* urk = buf<uint32_t>(u_rank, U);
    if (V > 0) ensure_btrees();
    phase(WJ_PHASE_PROBE);
    DictView dv{(const Node*)nodes.p, (const uint32_t*)coll_root.p, (const uint32_t*)coll_n.p, (const uint8_t*)arena.p};
    if (V > 0) {
      UniqueView uv{text, (const uint4*)u_w.p, (const uint32_t*)u_ref.p, (const uint32_t*)u_len.p,
                    (const uint32_t*)u_bucket.p, (const uint32_t*)u_cache.p};
      const unsigned blocks = (unsigned)std::min<uint64_t>((U + 8 * kProbeKeysPerWarp - 1) / (8 * kProbeKeysPerWarp),
                                                          148ull * 64);
      ktime(WJ_KERNEL_PROBE, [&] {
        k_probe4<<<blocks, 256, 0, st>>>(dv, uv, (uint32_t)U, ut, urk);
        launched();
      });
    } else {
      k_fill<uint32_t><<<grid_for(U, 256), 256, 0, st>>>(ut, U, kMiss);
      k_fill<uint32_t><<<grid_for(U, 256), 256, 0, st>>>(urk, U, 0u);
      launched(2);
    }
    phase(WJ_PHASE_INSERT);
    uint32_t* mi = buf<uint32_t>(midx, U);
    uint64_t Nn = U;
    if (V > 0) {
      scan<uint32_t>(IsMiss{ut}, U, mi, (uint32_t*)(dscal() + 3));
      WJ_CUDA_CHECK(cudaMemsetAsync((uint32_t*)(dscal() + 3) + 1, 0, 4, st));
      readback(3, 1);
      Nn = (uint32_t)h_scal[3];
    } else {  // an empty dictionary: every unique term is new, miss index = unique index (no round trip)
      k_iota_u32<<<grid_for(U, 256), 256, 0, st>>>(mi, (uint32_t)U);
      launched();
    }
    new_last = Nn;
    if (Nn > 0) {
      // the per-run partial lists carry u32 termIDs; the global-stream path (multi-rank, stemming)
      // sorts rank | count << kCountShift keys, so its dictionary slice is limited to 2^25 terms
      const uint64_t vmax = pm ? 0xFFFFFFFEull : (uint64_t)kRankMask + 1;
      if ((uint64_t)V + Nn > vmax)
        throw StatusError{WJ_ERR_CAPACITY, pm ? "more than 2^32-2 terms" : "more than 2^25 terms in one dictionary slice"};
      insert_new(text, U, Nn);
      btree_dirty = true;
    }
  }

  // run the following launches on side_st with its own scan / histogram scratch (no host syncs there)
  void swap_side() {
    std::swap(st, side_st);
    std::swap(scan_scr, side_scan);
    std::swap(hist, side_hist);
    std::swap(hist_scan, side_hist_scan);
    std::swap(rs_ctas, side_ctas);
  }

  // run-length pass over a sorted stream (postings.cuh): docid/tf into od/of, post_off / cstart at each
  // term's key (key & kRankMask); the posting count is left in dscal[8] (u32, no host round trip)
  // n_dev (optional): the actual element count on the device, N being an upper bound
  // pairs != nullptr: the postings go there as interleaved (docID, tf) pairs (per-run partial lists)
  // geometry of the plain-stream run-length pass (k_rlw_*): warp ranges of `per` elements, Wg warps
  void rlw_geometry(uint64_t N, uint64_t& per, uint32_t& grid, uint32_t& Wg) const {
    const uint64_t W = 148ull * 3 * kRlwWarps;  // one wave at 3 CTAs per SM
    per = rlw_per(N, W);
    const uint32_t Wn = (uint32_t)((N + per - 1) / per);
    grid = (Wn + kRlwWarps - 1) / kRlwWarps;
    Wg = grid * kRlwWarps;  // warps launched (ranges past N count 0)
  }
  // precounted: rle_p0 already holds each warp range's posting count (the last radix pass counted them)
  void rle(const uint32_t* key, const uint32_t* docs, uint64_t N, bool counts, uint32_t* od, uint32_t* of, uint64_t* po,
           uint64_t* csp, const uint32_t* n_dev = nullptr, uint2* pairs = nullptr,
           const unsigned long long* elem = nullptr, bool precounted = false) {
    const uint32_t ostride = pairs ? 2u : 1u;
    if (pairs) {
      od = (uint32_t*)pairs;
      of = (uint32_t*)pairs + 1;
    }
    if (N == 0) {  // e.g. every token of the chunk was a hot term
      WJ_CUDA_CHECK(cudaMemsetAsync(dscal() + 8, 0, 8, st));
      return;
    }
    if (elem && (counts || n_dev)) throw StatusError{WJ_ERR_STATE, "packed stream with counts"};
    if (!counts && !n_dev) {  // plain stream: one warp per range (k_rlw_*)
      uint64_t per;
      uint32_t grid, Wg;
      rlw_geometry(N, per, grid, Wg);
      uint32_t* rc = buf<uint32_t>(rle_p0, (uint64_t)Wg + 1);
      uint32_t* rl = buf<uint32_t>(rle_lead, (uint64_t)Wg + 1);
      ktime(WJ_KERNEL_RLE_EMIT, [&] {
        if (!precounted) {
          if (elem) k_rlw_count<true><<<grid, kRlwThreads, 0, st>>>(key, docs, elem, N, per, rc);
          else k_rlw_count<false><<<grid, kRlwThreads, 0, st>>>(key, docs, elem, N, per, rc);
          launched();
        }
        scan<uint32_t>(ArrayIn<uint32_t>{rc}, Wg, rc, (uint32_t*)(dscal() + 8));
        if (elem) k_rlw_write<true><<<grid, kRlwThreads, 0, st>>>(key, docs, elem, N, per, rc, od, of, ostride, po, csp, rl);
        else k_rlw_write<false><<<grid, kRlwThreads, 0, st>>>(key, docs, elem, N, per, rc, od, of, ostride, po, csp, rl);
        launched();
      });
      k_rle_fixup<<<grid_for(Wg, 256), 256, 0, st>>>(rc, rl, Wg, of, ostride);
      launched();
      WJ_CUDA_CHECK(cudaMemsetAsync((uint32_t*)(dscal() + 8) + 1, 0, 4, st));
      return;
    }
    uint64_t per = (N + 148 * 2 - 1) / (148 * 2);
    per = (per + kRleTile - 1) / kRleTile * kRleTile;
    const uint32_t G = (uint32_t)((N + per - 1) / per);
    uint32_t* rc = buf<uint32_t>(rle_p0, (uint64_t)G + 1);
    uint32_t* rl = buf<uint32_t>(rle_lead, (uint64_t)G + 1);
    uint64_t* rt = buf<uint64_t>(rle_tok, (uint64_t)G + 1);
    ktime(WJ_KERNEL_RLE_EMIT, [&] {
      if (counts) k_rle_count<true><<<G, kRleThreads, 0, st>>>(key, docs, N, per, rc, rt, n_dev);
      else k_rle_count<false><<<G, kRleThreads, 0, st>>>(key, docs, N, per, rc, rt, n_dev);
      launched();
      scan<uint32_t>(ArrayIn<uint32_t>{rc}, G, rc, (uint32_t*)(dscal() + 8));
      scan<uint64_t>(ArrayIn<uint64_t>{rt}, G, rt, (uint64_t*)(dscal() + 11));
      if (counts)
        k_rle_write_tma<true><<<G, kRleThreads, rle_smem_bytes(), st>>>(key, docs, N, per, rc, rt, od, of, ostride, po,
                                                                        csp, rl, n_dev);
      else
        k_rle_write_tma<false><<<G, kRleThreads, rle_smem_bytes(false), st>>>(key, docs, N, per, rc, rt, od, of, ostride,
                                                                          po, csp, rl, n_dev);
      launched();
    });
    k_rle_fixup<<<grid_for(G, 256), 256, 0, st>>>(rc, rl, G, of, ostride);
    launched();
    WJ_CUDA_CHECK(cudaMemsetAsync((uint32_t*)(dscal() + 8) + 1, 0, 4, st));
  }

  // the previous chunk's posting count (partials mode): read once its side-stream work is joined
  void settle_partials() {
    if (!pc_pending) return;
    sync();
    pbase += (uint32_t)h_scal[13];
    if (pc_settle_hot) {  // stream elements left after the hot tokens' holes were dropped
      const uint64_t left = (uint32_t)h_scal[14];
      hot_elems_saved += pc_settle_tokens - left;
      pm_merged += pc_settle_tokens - left;
    }
    pc_pending = false;
  }

  // Partials mode, one chunk: the stream (pc_key, pc_doc)[Nc] of C slots, U unique terms.  Sort by slot
  // + run-length on side_st (the partial lists of the run) while the dictionary update runs on
  // st; then one record per unique term.
  // hot: the stream holds merged hot-term elements (counts) and holes (hot.cuh)
  void chunk_partials(const uint8_t* text, uint64_t Nc, uint64_t C, uint64_t U, bool hot) {
    // the first chunk into an empty dictionary: every unique term is new and takes termID = its unique
    // index (k_new_terms), so its records (k_chunk_records, record u = unique term u) are indexed by termID
    recs_by_tid = nrec == 0 && V == 0 && !hot;
    if (!side_launched) side_launch(Nc, C, hot);
    side_launched = false;
    // the dictionary update (latency-bound small kernels with host round trips) on a high-priority
    // stream, so its CTAs are scheduled ahead of the side stream's whenever SMs free up; it forks here,
    // after the unique terms it reads are gathered (the side stream may have forked at the emit kernel)
    WJ_CUDA_CHECK(cudaEventRecord(ev_dfork, st));
    WJ_CUDA_CHECK(cudaStreamWaitEvent(hp_st, ev_dfork, 0));
    std::swap(st, hp_st);
    try {
      dictionary_update(text, U);
      phase(-1);
      WJ_CUDA_CHECK(cudaEventRecord(ev_dict, st));
    } catch (...) {
      std::swap(st, hp_st);
      throw;
    }
    std::swap(st, hp_st);
    WJ_CUDA_CHECK(cudaStreamWaitEvent(st, ev_dict, 0));
    pc_join = true;
    pc_U = U;
    pc_Nc = Nc;
    pc_hot = hot;
  }

  // The chunk's stream sorted by slot and run-length encoded on side_st (forked from st here).  The packed
  // path forks right after the emit kernel (tokenize_dedup), ahead of the unique-term scan and gather,
  // which the sort does not need.
  void side_launch(uint64_t Nc, uint64_t C, bool hot) {
    settle_partials();  // the previous chunk is joined (add_chunk), its posting count read here
    side_launched = true;
    const bool packed = pc_packed;
    uint32_t* kt = (uint32_t*)pc_key.p;
    uint32_t* dt = (uint32_t*)pc_doc.p;
    uint32_t* k1 = packed ? nullptr : buf<uint32_t>(sk1, Nc + 16);
    uint32_t* v1 = packed ? nullptr : buf<uint32_t>(sv1, Nc + 16);
    unsigned long long* e1 = packed ? buf<unsigned long long>(sk1, Nc + 16) : nullptr;
    uint2* pp = buf_keep<uint2>(pp_pair, pbase + Nc + 16, pbase);  // P_c <= N_c
    uint64_t* po = buf<uint64_t>(pc_po, C + 1);
    uint64_t* cs = buf<uint64_t>(pc_cs, C + 1);
    int bits = 0;
    while (bits < 32 && ((uint64_t)1 << bits) < C) ++bits;
    phase(-1);
    WJ_CUDA_CHECK(cudaEventRecord(ev_fork, st));
    WJ_CUDA_CHECK(cudaStreamWaitEvent(side_st, ev_fork, 0));
    swap_side();
    try {
      phase(WJ_PHASE_SORT);
      // holes (hot tokens, key 0) are dropped by the first pass; the count left stays on the device
      // (*ns_dev) and the later passes and the run-length pass are launched for the upper bound Nc
      uint32_t* ns_dev = hot ? (uint32_t*)(dscal() + 13) : nullptr;
      if (packed) {
        sort_rle_packed(Nc, bits, e1, po, cs, pp + pbase);
      } else {
        const bool in1 = sort_pairs<uint32_t>(kt, dt, k1, v1, Nc, 0, bits, nullptr, true, nullptr, kRankMask, hot, nullptr,
                                              true, nullptr, ns_dev);
        phase(WJ_PHASE_POSTINGS);
        rle(in1 ? k1 : kt, in1 ? v1 : dt, Nc, false, nullptr, nullptr, po, cs, ns_dev, pp + pbase);
      }
      if (hot) {  // the hot matrix rows -> the hot terms' partial lists, after the run-length postings
        const uint64_t HD = (uint64_t)hot_H * hot_D;
        uint32_t* hp = buf<uint32_t>(hot_posb, HD + 1);
        uint32_t* hcf = buf<uint32_t>(hot_cfb, hot_H);
        const uint32_t* mat = (const uint32_t*)hot_matb.p;
        scan<uint32_t>(NonZeroU32{mat}, HD, hp, hp + HD);
        k_hot_scatter<<<grid_for(HD, 256), 256, 0, st>>>(mat, HD, hot_D, hp, (const uint32_t*)(dscal() + 8),
                                                         doc_base_cur, pp + pbase);
        k_hot_rowsum<<<hot_H, 256, 0, st>>>(mat, hot_D, hcf);
        k_hot_total<<<1, 1, 0, st>>>(hp + HD, (uint32_t*)(dscal() + 8), (uint32_t*)(dscal() + 12));
        launched(3);
      }
      phase(-1);
      WJ_CUDA_CHECK(cudaEventRecord(ev_side, st));
    } catch (...) {
      swap_side();
      throw;
    }
    swap_side();
  }

  // The packed chunk stream (pc_key, Nc elements of C <= 2^bits slots) sorted by slot and run-length
  // encoded into partial lists at pp: value-less 64-bit radix passes (digits from bit 32, upsweeps over
  // the digit bytes in pc_dig), the last pass counting the run-length heads per warp range
  void sort_rle_packed(uint64_t Nc, int bits, unsigned long long* e1, uint64_t* po, uint64_t* cs, uint2* pp) {
    unsigned long long* e0 = (unsigned long long*)pc_key.p;
    uint64_t rper;
    uint32_t rgrid, Wg;
    rlw_geometry(Nc, rper, rgrid, Wg);
    uint32_t* rc = buf<uint32_t>(rle_p0, (uint64_t)Wg + 1);
    WJ_CUDA_CHECK(cudaMemsetAsync(rc, 0, ((size_t)Wg + 1) * 4, st));
    const bool in1 = sort_pairs<uint64_t>((uint64_t*)e0, nullptr, (uint64_t*)e1, nullptr, Nc, 32, 32 + std::max(bits, 1),
                                          nullptr, true, nullptr, ~0ull, false, nullptr, true, nullptr, nullptr, rc,
                                          (uint32_t)rper, (uint8_t*)pc_dig.p);
    phase(WJ_PHASE_POSTINGS);
    rle(nullptr, nullptr, Nc, false, nullptr, nullptr, po, cs, nullptr, pp, in1 ? e1 : e0, true);
  }

  // Join the last chunk's side-stream work and write its records; runs before the next chunk's
  // tokenizer reuses the chunk buffers, or in finalize after the work that does not need postings.
  void join_partials() {
    if (!pc_join) return;
    pc_join = false;
    const uint64_t U = pc_U, Nc = pc_Nc;
    phase(WJ_PHASE_STREAM);
    WJ_CUDA_CHECK(cudaStreamWaitEvent(st, ev_side, 0));
    const uint64_t* po = (const uint64_t*)pc_po.p;
    const uint64_t* cs = (const uint64_t*)pc_cs.p;
    uint32_t* rt = buf_keep<uint32_t>(rec_tid, nrec + U, nrec);
    uint64_t* rs = buf_keep<uint64_t>(rec_start, nrec + U, nrec);
    uint32_t* rd = buf_keep<uint32_t>(rec_df, nrec + U, nrec);
    uint32_t* rc = buf_keep<uint32_t>(rec_cf, nrec + U, nrec);
    const uint32_t* nh = nullptr;
    if (pc_hot) {  // records in partial-list order: non-hot terms (slot order), then the hot terms
      uint32_t* p = buf<uint32_t>(hot_nhb, U + 1);
      scan<uint32_t>(NotHotSlot{(const uint32_t*)u_slot.p, (const Slot*)table.p}, U, p, p + U);
      nh = p;
    }
    k_chunk_records<<<grid_for(U, 256), 256, 0, st>>>(
        (const uint32_t*)u_slot.p, (uint32_t)U, po, cs, (const uint32_t*)(dscal() + (pc_hot ? 12 : 8)), Nc,
        pc_hot ? (const uint32_t*)(dscal() + 13) : nullptr,
        (const uint32_t*)u_tid.p, pbase, rt + nrec, rs + nrec, rd + nrec, rc + nrec, (const Slot*)table.p,
        pc_hot ? (const uint32_t*)hot_posb.p : nullptr, (const uint32_t*)hot_cfb.p, hot_D, nh, hot_Hdev(),
        recs_by_tid ? buf<uint4>(rec_aos, U) : nullptr);
    launched();
    WJ_CUDA_CHECK(cudaMemcpyAsync(h_scal + 13, dscal() + 8, 8, cudaMemcpyDeviceToHost, st));
    if (pc_hot) WJ_CUDA_CHECK(cudaMemcpyAsync(h_scal + 14, dscal() + 13, 8, cudaMemcpyDeviceToHost, st));
    pc_pending = true;
    pc_settle_hot = pc_hot;
    pc_settle_tokens = Nc;
    nrec += U;
    rec_end.push_back(nrec);
    phase(-1);
  }

  // the chunk's (slot, docID) stream is the postings input; keep its slot -> termID map
  void register_chunk_map(uint64_t C, uint64_t tok_start) {
    phase(WJ_PHASE_STREAM);
    const size_t ci = chunk_tok.size();
    if (chunk_map.size() <= ci) chunk_map.emplace_back();
    uint32_t* cmap = buf<uint32_t>(chunk_map[ci], C);
    ktime(WJ_KERNEL_SLOT_TO_TID, [&] {
      k_slot_map<<<grid_for(C, 256), 256, 0, st>>>((const Slot*)table.p, (const uint32_t*)uid.p,
                                                    (const uint32_t*)u_tid.p, (uint32_t)C, cmap);
      launched();
    });
    chunk_tok.push_back(tok_start);
    chunk_C.push_back((uint32_t)C);
  }

  // ---------------------------------------------------------------- f3: host pipeline
  // Index the pending host chunk (its copy was enqueued by the previous call).
  void drain() {
    if (!pend) return;
    pend = false;
    const int s = pend_slot;
    WJ_CUDA_CHECK(cudaStreamWaitEvent(st, pipe_copied[s], 0));
    add_chunk(pipe_text[s].p, pend_bytes, (const uint64_t*)pipe_off[s].p, pend_nd);
    WJ_CUDA_CHECK(cudaEventRecord(pipe_done[s], st));
    pipe_used[s] = true;
  }

  // Host chunk with WJ_FLAG_HOST_PIPELINE: validate doc_off, enqueue its copy on the copy stream,
  // then index the previous chunk on the context stream while the copy engine moves this one.
  void add_stream_pipelined(const void* bytes, uint64_t n_bytes, const uint64_t* doc_off, uint64_t nd) {
    if (doc_off[0] != 0 || doc_off[nd] != n_bytes) throw StatusError{WJ_ERR_INVALID_ARG, "doc_off[0] must be 0 and doc_off[n_docs] == n_bytes"};
    for (uint64_t i = 0; i < nd; ++i)
      if (doc_off[i] > doc_off[i + 1]) throw StatusError{WJ_ERR_INVALID_ARG, "doc_off must be non-decreasing"};
    const int s = next_slot;
    if (pipe_used[s]) WJ_CUDA_CHECK(cudaStreamWaitEvent(cs, pipe_done[s], 0));  // slot consumed (chunk c-2)
    uint8_t* t = buf<uint8_t>(pipe_text[s], n_bytes + 16);
    uint64_t* o = buf<uint64_t>(pipe_off[s], nd + 1);
    if (n_bytes) WJ_CUDA_CHECK(cudaMemcpyAsync(t, bytes, n_bytes, cudaMemcpyHostToDevice, cs));
    WJ_CUDA_CHECK(cudaMemcpyAsync(o, doc_off, (nd + 1) * 8, cudaMemcpyHostToDevice, cs));
    WJ_CUDA_CHECK(cudaEventRecord(pipe_copied[s], cs));
    next_slot ^= 1;
    drain();
    pend = true;
    pend_slot = s;
    pend_bytes = n_bytes;
    pend_nd = nd;
  }

  void add_stream(const void* bytes, uint64_t n_bytes, const uint64_t* doc_off, uint64_t nd) {
    if (pipeline && !is_device_ptr(doc_off) && (n_bytes == 0 || !is_device_ptr(bytes))) {
      add_stream_pipelined(bytes, n_bytes, doc_off, nd);
      return;
    }
    drain();
    add_chunk(bytes, n_bytes, doc_off, nd);
  }

  void add_chunk(const void* bytes, uint64_t n_bytes, const uint64_t* doc_off_in, uint64_t nd) {
    const uint8_t* text = nullptr;
    const uint64_t* off = nullptr;
    if (pm) join_partials();  // the previous chunk's side work, before its buffers are reused
    stage(bytes, n_bytes, doc_off_in, nd, &text, &off);
    ++n_chunks;
    if (xport && pm) {
      add_chunk_dist_pl(text, nd ? n_bytes : 0, off, nd);
      phase(-1);
      return;
    }
    if (xport) {
      add_chunk_dist(text, nd ? n_bytes : 0, off, nd);
      phase(-1);
      return;
    }
    if (n_docs + nd > 0xFFFFFFFFull) throw StatusError{WJ_ERR_CAPACITY, "more than 2^32-1 documents"};
    const uint32_t doc_base = (uint32_t)n_docs;
    doc_base_cur = doc_base;
    if (nd == 0 || n_bytes == 0) {
      n_docs += nd;
      phase(-1);
      return;
    }
    ChunkView cv{text, n_bytes, off, nd};
    uint64_t C = 0, U = 0;
    uint32_t *so = nullptr, *dout = nullptr;
    const bool norm = stem_on || stop_on;
    emit_elem = nullptr;
    pc_packed = false;
    const uint64_t Nc = tokenize_dedup(cv, doc_base, [&](uint64_t nc, uint32_t*& sp, uint32_t*& dp) {
      if (pm) {  // the chunk's own stream; the previous chunk's side work is joined on st already
        if (nc > 0xFFFFFFFFull) throw StatusError{WJ_ERR_CAPACITY, "more than 2^32-1 tokens in one chunk"};
        pc_packed = !norm && hot_H == 0;
        if (pc_packed) {
          emit_elem = buf<unsigned long long>(pc_key, nc + 16);
          buf<uint8_t>(pc_dig, nc + 64);  // digit bytes of the radix passes (k_rs_up_bytes)
          sp = dp = nullptr;
          return;
        }
        sp = buf<uint32_t>(pc_key, nc + 16);  // +16: TMA round-up reads
        dp = buf<uint32_t>(pc_doc, nc + 16);
        return;
      }
      if (n_elems + nc > 0xFFFFFFFFull) throw StatusError{WJ_ERR_CAPACITY, "more than 2^32-1 stream elements"};
      sp = buf_keep<uint32_t>(g_tid, n_elems + nc + 16, n_elems) + n_elems;  // +16: TMA round-up reads
      dp = buf_keep<uint32_t>(g_doc, n_elems + nc + 16, n_elems) + n_elems;
    }, C, U, so, dout, pm && !norm);
    emit_elem = nullptr;
    if (Nc > 0 && norm) {  // f4: stems / stop words
      uint64_t U2 = 0;
      const uint8_t* ntext = nullptr;
      const uint64_t kept = normalize(text, C, U, so, dout, Nc, U2, ntext);
      if (kept > 0) {
        dictionary_update(ntext, U2);
        phase(WJ_PHASE_STREAM);
        const size_t ci = chunk_tok.size();
        if (chunk_map.size() <= ci) chunk_map.emplace_back();
        uint32_t* cmap = buf<uint32_t>(chunk_map[ci], C);
        k_norm_tid_map<<<grid_for(C, 256), 256, 0, st>>>((const uint32_t*)st_m1.p, (uint32_t)C, (const uint32_t*)u_tid.p,
                                                         cmap);
        launched();
        chunk_tok.push_back(n_elems);
        chunk_C.push_back((uint32_t)C);
        n_elems += kept;
        n_tokens += kept;
      }
    } else if (Nc > 0 && pm) {
      dict_text_bytes = n_bytes;
      chunk_partials(text, Nc, C, U, hot_H > 0);
      dict_text_bytes = 0;
      n_elems += Nc;
      n_tokens += Nc;
    } else if (Nc > 0) {
      dictionary_update(text, U);
      register_chunk_map(C, n_elems);
      if (hot_H) stream_has_hot = true;
      n_elems += Nc;
      n_tokens += Nc;
    }
    n_docs += nd;
    phase(-1);
  }

  // ---------------------------------------------------------------- one chunk, world > 1
  // Sender-side partial lists: every rank tokenises its own documents,
  // groups its unique terms by owner (collection b -> b mod K, or the balanced map) and
  // sends each owner its terms (folded bytes) first; then, overlapped, it sorts + run-length encodes its
  // stream by (owner, term) into (docID, tf) postings on the side stream while, as an owner, it
  // deduplicates the received terms and updates its exclusive dictionary slice on the
  // dictionary stream.  A second all-to-all-v moves a (df, cf) header per term and the postings grouped
  // per term; the owner appends one partial-list record per (source, term) in source-rank
  // order = docID order, and finalize is the single-GPU partial-list combine.
  void add_chunk_dist_pl(const uint8_t* text, uint64_t n_bytes, const uint64_t* off, uint64_t nd) {
    recs_by_tid = false;  // records per (source rank, term): not indexed by termID
    const int K = world;
    phase(WJ_PHASE_EXCHANGE);
    std::vector<uint64_t> ndall(K);
    const uint64_t mine = nd;
    xport->allgather(&mine, 1, ndall.data(), st);
    uint64_t base = n_docs, tot_docs = 0;
    for (int r = 0; r < K; ++r) {
      if (r < rank) base += ndall[r];
      tot_docs += ndall[r];
    }
    if (n_docs + tot_docs > 0xFFFFFFFFull) throw StatusError{WJ_ERR_CAPACITY, "more than 2^32-1 documents"};
    if (balanced && !owner_ready) {
      ChunkView cv0{text, n_bytes, off, nd};
      build_owner_map(nd > 0 && n_bytes > 0 ? &cv0 : nullptr);
      phase(WJ_PHASE_EXCHANGE);
    }
    // 1. local tokenize + dedup of this rank's documents (stream into pc_key / pc_doc)
    uint64_t C = 0, U = 0, Nc = 0;
    uint32_t *lslot = nullptr, *ldoc = nullptr;
    if (nd > 0 && n_bytes > 0) {
      ChunkView cv{text, n_bytes, off, nd};
      emit_elem = nullptr;
      Nc = tokenize_dedup(cv, (uint32_t)base, [&](uint64_t nc, uint32_t*& sp, uint32_t*& dp) {
        if (nc > 0xFFFFFFFFull) throw StatusError{WJ_ERR_CAPACITY, "more than 2^32-1 tokens in one chunk"};
        emit_elem = buf<unsigned long long>(pc_key, nc + 16);  // the packed stream (chunk_partials)
        buf<uint8_t>(pc_dig, nc + 64);
        sp = dp = nullptr;
      }, C, U, lslot, ldoc, false, (uint32_t)K);  // table partitioned by owner (slot order = owner order)
      emit_elem = nullptr;
    }
    std::vector<uint64_t> t_off(K + 1, 0), b_off(K + 1, 0), p_off(K + 1, 0), c_off(K + 1, 0);
    uint8_t* send_terms = (uint8_t*)grow(x_send, 16);
    uint64_t* toff_d = buf<uint64_t>(x_toff, K + 1);
    // the chunk's postings: K == 1 straight into the partial-list buffer; K > 1 into scratch, from where
    // every owner's range (the own one by a device copy) lands in the owners' partial-list buffers in
    // source-rank order, so each chunk's partial lists are back to back in record order
    uint2* opp = K == 1 ? buf_keep<uint2>(pp_pair, pbase + Nc + 16, pbase) + pbase : buf<uint2>(x_pair, Nc + 16);
    uint32_t* hdf = buf<uint32_t>(x_hdf, U + 1);
    uint32_t* hcf = buf<uint32_t>(x_hcf, U + 1);
    uint64_t* bnd = buf<uint64_t>(x_bnd, 2 * (K + 1));
    const bool solo = K == 1;  // one rank owns everything: no exchange, the local terms are the owner's
    if (U > 0 && solo) {
      t_off[1] = U;
      WJ_CUDA_CHECK(cudaMemcpyAsync(toff_d, t_off.data(), 2 * 8, cudaMemcpyHostToDevice, st));
    } else if (U > 0) {
      // 2. the unique terms are in owner order already: t_off = first unique term of each partition
      k_part_bounds<<<grid_for(K + 1, 256), 256, 0, st>>>((const uint32_t*)uid.p, (uint32_t)K, C / K,
                                                          (const uint32_t*)(dscal() + 2), toff_d);
      launched();
      uint64_t* boff = buf<uint64_t>(x_boff, U + 1);
      scan<uint64_t>(PackTermSize{nullptr, (const uint32_t*)u_len.p}, U, boff, boff + U);
      WJ_CUDA_CHECK(cudaMemcpyAsync(t_off.data(), toff_d, (K + 1) * 8, cudaMemcpyDeviceToHost, st));
      sync();
      for (int o = 0; o <= K; ++o)
        WJ_CUDA_CHECK(cudaMemcpyAsync(&b_off[o], boff + t_off[o], 8, cudaMemcpyDeviceToHost, st));
      sync();
      send_terms = (uint8_t*)grow(x_send, b_off[K] + 16);
      k_pack_terms<<<grid_for(U, 256), 256, 0, st>>>(nullptr, (uint32_t)U, boff, (const uint4*)u_w.p, text,
                                                    (const uint32_t*)u_ref.p, (const uint32_t*)u_len.p, send_terms);
      launched();
    }
    // 3. first exchange: the terms (folded bytes) to their owners
    std::vector<uint64_t> cnt(2 * K, 0), all(2 * K * K);
    for (int o = 0; o < K; ++o) {
      cnt[o] = t_off[o + 1] - t_off[o];
      cnt[K + o] = b_off[o + 1] - b_off[o];
    }
    if (!solo) xport->allgather(cnt.data(), 2 * K, all.data(), st);
    else all = cnt;
    std::vector<uint64_t> rt(K + 1, 0), rb(K + 1, 0);
    for (int s = 0; s < K; ++s) {
      const uint64_t* c = all.data() + (size_t)s * 2 * K;
      rt[s + 1] = rt[s] + c[rank];
      rb[s + 1] = rb[s] + c[K + rank];
    }
    const uint64_t RT = rt[K];
    uint8_t* recv_terms = (uint8_t*)grow(x_recv_terms, rb[K] + 32);
    const uint64_t t0 = xport->sent;
    double xms = 0;
    auto exchange = [&](auto&& f) {
      const auto tx = std::chrono::steady_clock::now();
      try {
        f();
      } catch (const ExchangeError& e) {
        throw StatusError{WJ_ERR_NCCL, e.msg};
      }
      WJ_CUDA_CHECK(cudaStreamSynchronize(st));
      xms += std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - tx).count();
    };
    if (!solo) exchange([&] { xport->alltoallv(send_terms, b_off.data(), recv_terms, rb.data(), st); });
    uint32_t* us = buf<uint32_t>(x_xid, U + 1);  // the local unique terms' slots (u_slot is reused by the owner)
    // 4. overlapped: side stream = the local stream sorted by slot (= by owner, then term) and
    //    run-length encoded, headers, per-owner bounds; dictionary stream = the owner's dictionary
    if (U > 0) {
      int bits = 0;
      while (bits < 32 && ((uint64_t)1 << bits) < C) ++bits;
      unsigned long long* e1 = buf<unsigned long long>(sk1, Nc + 16);
      uint64_t* po = buf<uint64_t>(pc_po, C + 1);
      uint64_t* cs = buf<uint64_t>(pc_cs, C + 1);
      WJ_CUDA_CHECK(cudaMemcpyAsync(us, u_slot.p, U * 4, cudaMemcpyDeviceToDevice, st));
      phase(-1);
      WJ_CUDA_CHECK(cudaEventRecord(ev_fork, st));
      WJ_CUDA_CHECK(cudaStreamWaitEvent(side_st, ev_fork, 0));
      swap_side();
      try {
        phase(WJ_PHASE_SORT);
        sort_rle_packed(Nc, bits, e1, po, cs, opp);
        k_term_hdr<<<grid_for(U, 256), 256, 0, st>>>(us, (uint32_t)U, po, cs, (const uint32_t*)(dscal() + 8), Nc, hdf, hcf);
        k_owner_bounds<<<grid_for(K + 1, 256), 256, 0, st>>>(us, po, cs, toff_d, (uint32_t)K, (uint32_t)U,
                                                            (const uint32_t*)(dscal() + 8), Nc, bnd, bnd + K + 1);
        launched(2);
        phase(-1);
        WJ_CUDA_CHECK(cudaEventRecord(ev_side, st));
      } catch (...) {
        swap_side();
        throw;
      }
      swap_side();
    } else {
      WJ_CUDA_CHECK(cudaMemsetAsync(bnd, 0, 2 * (K + 1) * 8, st));
      WJ_CUDA_CHECK(cudaEventRecord(ev_side, st));
    }
    uint32_t* sslot = nullptr;
    if (RT > 0) {  // the owner's dictionary on the high-priority stream
      WJ_CUDA_CHECK(cudaEventRecord(ev_fork, st));
      WJ_CUDA_CHECK(cudaStreamWaitEvent(hp_st, ev_fork, 0));
      std::swap(st, hp_st);
      try {
        if (solo) {  // the owner's terms are the local unique terms: no re-tokenisation
          dictionary_update(text, U);
          sslot = us;
        } else {
        uint64_t* so = buf<uint64_t>(x_syn_off, 2);
        const uint64_t h2[2] = {0, rb[K]};
        WJ_CUDA_CHECK(cudaMemcpyAsync(so, h2, 16, cudaMemcpyHostToDevice, st));
        ChunkView sv{recv_terms, rb[K], so, 1};
        uint64_t C2 = 0, U2 = 0;
        uint32_t* sdoc = nullptr;
        const uint64_t dropped0 = n_dropped;
        const uint64_t Ns2 = tokenize_dedup(sv, 0, [&](uint64_t nc, uint32_t*& sp2, uint32_t*& dp2) {
          sp2 = buf<uint32_t>(x_syn_slot, nc + 16);
          dp2 = buf<uint32_t>(x_syn_doc, nc + 16);
        }, C2, U2, sslot, sdoc);
        n_dropped = dropped0;
        if (Ns2 != RT) throw StatusError{WJ_ERR_CUDA, "received term text: token count mismatch (internal)"};
        dictionary_update(recv_terms, U2);
        }
        phase(-1);
        WJ_CUDA_CHECK(cudaEventRecord(ev_dict, st));
      } catch (...) {
        std::swap(st, hp_st);
        throw;
      }
      std::swap(st, hp_st);
      WJ_CUDA_CHECK(cudaStreamWaitEvent(st, ev_dict, 0));
    }
    WJ_CUDA_CHECK(cudaStreamWaitEvent(st, ev_side, 0));
    phase(WJ_PHASE_EXCHANGE);
    std::vector<uint64_t> hb(2 * (K + 1));
    WJ_CUDA_CHECK(cudaMemcpyAsync(hb.data(), bnd, hb.size() * 8, cudaMemcpyDeviceToHost, st));
    sync();
    for (int o = 0; o <= K; ++o) {
      p_off[o] = hb[o];
      c_off[o] = hb[K + 1 + o];
    }
    // 5. second exchange: per owner [postings, tokens]; then the headers and the postings
    std::vector<uint64_t> cnt2(2 * K, 0), all2(2 * K * K);
    for (int o = 0; o < K; ++o) {
      cnt2[o] = p_off[o + 1] - p_off[o];
      cnt2[K + o] = c_off[o + 1] - c_off[o];
    }
    if (!solo) xport->allgather(cnt2.data(), 2 * K, all2.data(), st);
    else all2 = cnt2;
    std::vector<uint64_t> rp(K + 1, 0);
    uint64_t my_tokens = 0;
    for (int s = 0; s < K; ++s) {
      const uint64_t* c = all2.data() + (size_t)s * 2 * K;
      rp[s + 1] = rp[s] + c[rank];
      my_tokens += c[K + rank];
    }
    const uint64_t RP = rp[K];  // postings of this owner's terms over all sources
    uint32_t* rhdf = solo ? hdf : buf<uint32_t>(x_rhdf, RT + 1);
    uint32_t* rhcf = solo ? hcf : buf<uint32_t>(x_rhcf, RT + 1);
    std::vector<uint64_t> s4(K + 1), r4(K + 1);
    for (int o = 0; o <= K; ++o) {
      s4[o] = t_off[o] * 4;
      r4[o] = rt[o] * 4;
    }
    if (!solo) exchange([&] {
      xport->alltoallv(hdf, s4.data(), rhdf, r4.data(), st);
      xport->alltoallv(hcf, s4.data(), rhcf, r4.data(), st);
      if (K > 1) {  // postings: owner o's range of the scratch -> o's partial-list buffer
        uint2* pd = buf_keep<uint2>(pp_pair, pbase + RP + 16, pbase) + pbase;
        std::vector<uint64_t> spb(K + 1), rpb(K + 1);
        for (int o = 0; o <= K; ++o) {
          spb[o] = p_off[o] * 8;
          rpb[o] = rp[o] * 8;
        }
        xport->alltoallv(opp, spb.data(), pd, rpb.data(), st);
      }
    });
    exchange_ms += xms;
    exchange_bytes += xport->sent - t0;
    // 6. owner side: one record per (source, term) in source-rank order
    if (RT > 0) {
      phase(WJ_PHASE_STREAM);
      uint64_t* pre = buf<uint64_t>(x_rpre, RT + 1);
      uint32_t* rtid = buf_keep<uint32_t>(rec_tid, nrec + RT, nrec);
      uint64_t* rst = buf_keep<uint64_t>(rec_start, nrec + RT, nrec);
      uint32_t* rdf = buf_keep<uint32_t>(rec_df, nrec + RT, nrec);
      uint32_t* rcf = buf_keep<uint32_t>(rec_cf, nrec + RT, nrec);
      for (int s = 0; s < K; ++s) {
        const uint64_t nt = rt[s + 1] - rt[s];
        if (nt == 0) continue;
        scan<uint64_t>(U32AsU64{rhdf + rt[s]}, nt, pre + rt[s], (uint64_t*)nullptr);
        k_recv_records<<<grid_for(nt, 256), 256, 0, st>>>(sslot + rt[s], (uint32_t)nt, (const Slot*)table.p,
                                                          (const uint32_t*)uid.p, (const uint32_t*)u_tid.p, rhdf + rt[s],
                                                          rhcf + rt[s], pre + rt[s], pbase + rp[s], rtid + nrec + rt[s],
                                                          rst + nrec + rt[s], rdf + nrec + rt[s], rcf + nrec + rt[s]);
        launched();
        rec_end.push_back(nrec + rt[s + 1]);
      }
      nrec += RT;
    }
    pbase += RP;
    n_tokens += my_tokens;
    n_elems += Nc;
    n_docs += tot_docs;
    sync();  // exchange buffers are reused by the next chunk
  }

  // ---------------------------------------------------------------- one chunk, world > 1, global stream
  // (stemming / stop words / WJ_FLAG_GLOBAL_STREAM): token records routed to the owners
  void add_chunk_dist(const uint8_t* text, uint64_t n_bytes, const uint64_t* off, uint64_t nd) {
    const int K = world;
    // DocID base = documents of earlier chunks + of lower ranks in this chunk
    std::vector<uint64_t> ndall(K);
    const uint64_t mine = nd;
    phase(WJ_PHASE_EXCHANGE);
    xport->allgather(&mine, 1, ndall.data(), st);
    uint64_t base = n_docs, tot_docs = 0;
    for (int r = 0; r < K; ++r) {
      if (r < rank) base += ndall[r];
      tot_docs += ndall[r];
    }
    if (n_docs + tot_docs > 0xFFFFFFFFull) throw StatusError{WJ_ERR_CAPACITY, "more than 2^32-1 documents"};
    if (balanced && !owner_ready) {  // first chunk: sampled, bin-packed owner map (collective)
      ChunkView cv0{text, n_bytes, off, nd};
      build_owner_map(nd > 0 && n_bytes > 0 ? &cv0 : nullptr);
      phase(WJ_PHASE_EXCHANGE);
    }
    // 1. local tokenize + dedup of this rank's documents
    uint64_t C = 0, U = 0, Nc = 0;
    uint32_t *lslot = nullptr, *ldoc = nullptr;
    if (nd > 0 && n_bytes > 0) {
      ChunkView cv{text, n_bytes, off, nd};
      Nc = tokenize_dedup(cv, (uint32_t)base, [&](uint64_t nc, uint32_t*& sp, uint32_t*& dp) {
        sp = buf<uint32_t>(x_loc_slot, nc + 16);
        dp = buf<uint32_t>(x_loc_doc, nc + 16);
      }, C, U, lslot, ldoc, false);
    }
    // f4: the unique stems (stop words removed) are the chunk's terms; tokens map to them via st_m1
    const Slot* tok_table = (const Slot*)table.p;
    const uint32_t* tok_uid = (const uint32_t*)uid.p;
    const uint8_t* term_text = text;
    if (Nc > 0 && (stem_on || stop_on)) {
      uint64_t U2 = 0;
      const uint8_t* ntext = nullptr;
      Nc = normalize(text, C, U, lslot, ldoc, Nc, U2, ntext);
      U = Nc > 0 ? U2 : 0;
      tok_table = (const Slot*)table_s.p;
      tok_uid = (const uint32_t*)st_m1.p;
      term_text = ntext;
    }
    // 2. pack per owner (collection b -> rank b mod K, or the balanced map)
    phase(WJ_PHASE_EXCHANGE);
    std::vector<uint64_t> cnt(3 * K, 0);  // [terms to o | term bytes to o | records to o]
    uint64_t* toff_d = buf<uint64_t>(x_toff, K + 1);
    std::vector<uint64_t> t_off(K + 1, 0), b_off(K + 1, 0), r_off(K + 1, 0);
    uint8_t* send_terms = nullptr;
    uint32_t *send_key = nullptr, *send_doc = nullptr;
    if (U > 0) {
      uint32_t* own = buf<uint32_t>(x_owner, U + 16);
      uint32_t* iota = buf<uint32_t>(x_iota, U + 16);
      uint32_t* own2 = buf<uint32_t>(x_owner2, U + 16);
      uint32_t* srt2 = buf<uint32_t>(x_sorted2, U + 16);
      uint32_t* oc = buf<uint32_t>(x_cnt, 2 * K);
      WJ_CUDA_CHECK(cudaMemsetAsync(oc, 0, 2 * K * 4, st));
      k_owner<<<grid_for(U, 256), 256, 0, st>>>((const uint32_t*)u_bucket.p, (uint32_t)U, (uint32_t)K,
                                                owner_ready ? (const uint32_t*)owner_tab.p : nullptr, own, iota, oc);
      launched();
      // keep u_owner intact for the token pass: sort a copy
      WJ_CUDA_CHECK(cudaMemcpyAsync(own2, own, U * 4, cudaMemcpyDeviceToDevice, st));
      int bits = 0;
      while ((1 << bits) < K) ++bits;
      uint32_t* srt1 = (uint32_t*)grow(x_sorted, (U + 16) * 4);
      const bool in1 = sort_pairs<uint32_t>(own2, iota, srt1, srt2, U, 0, bits, nullptr, false);
      const uint32_t* sorted_u = in1 ? srt2 : iota;
      std::vector<uint32_t> oc_h(K);
      WJ_CUDA_CHECK(cudaMemcpyAsync(oc_h.data(), oc, K * 4, cudaMemcpyDeviceToHost, st));
      sync();
      for (int o = 0; o < K; ++o) t_off[o + 1] = t_off[o] + oc_h[o];
      WJ_CUDA_CHECK(cudaMemcpyAsync(toff_d, t_off.data(), (K + 1) * 8, cudaMemcpyHostToDevice, st));
      uint32_t* xid = buf<uint32_t>(x_xid, U);
      k_xid<<<grid_for(U, 256), 256, 0, st>>>(sorted_u, (uint32_t)U, own, toff_d, xid);
      launched();
      uint64_t* boff = buf<uint64_t>(x_boff, U + 1);
      scan<uint64_t>(PackTermSize{sorted_u, (const uint32_t*)u_len.p}, U, boff, boff + U);
      // byte offsets at owner boundaries
      for (int o = 0; o <= K; ++o)
        WJ_CUDA_CHECK(cudaMemcpyAsync(&b_off[o], boff + t_off[o], 8, cudaMemcpyDeviceToHost, st));
      sync();
      send_terms = (uint8_t*)grow(x_send, b_off[K] + 16);
      k_pack_terms<<<grid_for(U, 256), 256, 0, st>>>(sorted_u, (uint32_t)U, boff, (const uint4*)u_w.p, term_text,
                                                    (const uint32_t*)u_ref.p, (const uint32_t*)u_len.p, send_terms);
      launched();
      // token records (key with xid, docID) partitioned by owner, stream (= docID) order kept
      uint32_t* rk = buf<uint32_t>(x_rkey, Nc + 16);
      uint32_t* rd = buf<uint32_t>(x_rdoc, Nc + 16);
      if (K <= 64) {  // one radix pass on the owner bits of the mapped key
        uint32_t* km = buf<uint32_t>(x_keymap, C);
        k_slot_xkey<<<grid_for(C, 256), 256, 0, st>>>(tok_table, (uint32_t)C, tok_uid, own, xid, km);
        launched();
        std::vector<std::pair<uint64_t, const uint32_t*>> segs{{0, km}};
        std::vector<uint64_t> ds;
        const bool in2 = sort_pairs<uint32_t>(lslot, ldoc, rk, rd, Nc, kOwnerShift, kOwnerShift + bits, nullptr, false,
                                              &segs, kXidMask, false, nullptr, false, &ds);
        if (!in2) {  // K == 1 or a single token: no pass, the map was applied in place
          rk = lslot;
          rd = ldoc;
        }
        if (ds.size() == 257) {
          for (int o = 0; o < K; ++o) r_off[o] = ds[o];
          r_off[K] = Nc;
        } else {
          uint32_t o1 = 0;  // owner of the single record (Nc == 1)
          if (K > 1) {
            uint32_t v = 0;
            WJ_CUDA_CHECK(cudaMemcpyAsync(&v, rk, 4, cudaMemcpyDeviceToHost, st));
            sync();
            o1 = v >> kOwnerShift;
          }
          for (int o = 0; o <= K; ++o) r_off[o] = (uint32_t)o > o1 ? Nc : 0;
        }
      } else {
        uint32_t* tk = buf<uint32_t>(x_tkey, Nc + 16);
        uint32_t* ti = buf<uint32_t>(x_tidx, Nc + 16);
        uint32_t* tk2 = buf<uint32_t>(x_tkey2, Nc + 16);
        uint32_t* ti2 = buf<uint32_t>(x_tidx2, Nc + 16);
        k_tok_owner<<<grid_for(Nc, 256), 256, 0, st>>>(lslot, Nc, tok_uid, own, (uint32_t)K, tk, ti, oc + K);
        launched();
        const bool in2 = sort_pairs<uint32_t>(tk, ti, tk2, ti2, Nc, 0, bits, nullptr, false);
        const uint32_t* sorted_t = in2 ? ti2 : ti;
        k_pack_tok<<<grid_for(Nc, 256), 256, 0, st>>>(sorted_t, Nc, lslot, ldoc, tok_uid, xid, rk, rd);
        launched();
        WJ_CUDA_CHECK(cudaMemcpyAsync(oc_h.data(), oc + K, K * 4, cudaMemcpyDeviceToHost, st));
        sync();
        for (int o = 0; o < K; ++o) r_off[o + 1] = r_off[o] + oc_h[o];
      }
      send_key = rk;
      send_doc = rd;
      for (int o = 0; o < K; ++o) {
        cnt[o] = t_off[o + 1] - t_off[o];
        cnt[K + o] = b_off[o + 1] - b_off[o];
        cnt[2 * K + o] = r_off[o + 1] - r_off[o];
      }
    }
    // 3. exchange: counts, then the term text and the token records
    std::vector<uint64_t> all(3 * K * K);
    xport->allgather(cnt.data(), 3 * K, all.data(), st);
    std::vector<uint64_t> rt_off(K + 1, 0), rb_off(K + 1, 0), rr_off(K + 1, 0);
    for (int s = 0; s < K; ++s) {
      const uint64_t* c = all.data() + (size_t)s * 3 * K;
      rt_off[s + 1] = rt_off[s] + c[rank];
      rb_off[s + 1] = rb_off[s] + c[K + rank];
      rr_off[s + 1] = rr_off[s] + c[2 * K + rank];
    }
    uint8_t* recv_terms = (uint8_t*)grow(x_recv_terms, rb_off[K] + 32);
    // records land directly in the (termID, docID) stream; per-source maps (xid -> termID) are
    // registered below, so no per-record translation pass is needed
    const uint64_t R = rr_off[K];
    if (n_elems + R > 0xFFFFFFFFull) throw StatusError{WJ_ERR_CAPACITY, "more than 2^32-1 stream elements"};
    uint32_t* recv_key = buf_keep<uint32_t>(g_tid, n_elems + R + 16, n_elems) + n_elems;
    uint32_t* recv_doc = buf_keep<uint32_t>(g_doc, n_elems + R + 16, n_elems) + n_elems;
    std::vector<uint64_t> rec_soff(K + 1), rec_roff(K + 1);
    for (int o = 0; o <= K; ++o) { rec_soff[o] = r_off[o] * 4; rec_roff[o] = rr_off[o] * 4; }
    const uint64_t t0 = xport->sent;
    try {
      xport->alltoallv(send_terms, b_off.data(), recv_terms, rb_off.data(), st);
      xport->alltoallv(send_key, rec_soff.data(), recv_key, rec_roff.data(), st);
      xport->alltoallv(send_doc, rec_soff.data(), recv_doc, rec_roff.data(), st);
    } catch (const ExchangeError& e) {
      throw StatusError{WJ_ERR_NCCL, e.msg};
    }
    exchange_bytes += xport->sent - t0;
    // 4. owner side: the received term text goes through the same tokenizer / dedup / dictionary
    if (rt_off[K] > 0) {
      uint64_t* so = buf<uint64_t>(x_syn_off, 2);
      const uint64_t h2[2] = {0, rb_off[K]};
      WJ_CUDA_CHECK(cudaMemcpyAsync(so, h2, 16, cudaMemcpyHostToDevice, st));
      ChunkView sv{recv_terms, rb_off[K], so, 1};
      uint64_t C2 = 0, U2 = 0;
      uint32_t *sslot = nullptr, *sdoc = nullptr;
      const uint64_t dropped0 = n_dropped;
      const uint64_t Ns = tokenize_dedup(sv, 0, [&](uint64_t nc, uint32_t*& sp, uint32_t*& dp) {
        sp = buf<uint32_t>(x_syn_slot, nc + 16);
        dp = buf<uint32_t>(x_syn_doc, nc + 16);
      }, C2, U2, sslot, sdoc);
      n_dropped = dropped0;
      if (Ns != rt_off[K]) throw StatusError{WJ_ERR_CUDA, "received term text: token count mismatch (internal)"};
      dictionary_update(recv_terms, U2);
      phase(WJ_PHASE_STREAM);
      // source s's records: key & kRankMask = xid = index into the terms s sent; map xid -> termID
      for (int src = 0; src < K; ++src) {
        const uint64_t nr = rr_off[src + 1] - rr_off[src], nt = rt_off[src + 1] - rt_off[src];
        if (nr == 0) continue;
        const size_t ci = chunk_tok.size();
        if (chunk_map.size() <= ci) chunk_map.emplace_back();
        uint32_t* m = buf<uint32_t>(chunk_map[ci], nt);
        k_xid_map<<<grid_for(nt, 256), 256, 0, st>>>(sslot + rt_off[src], (uint32_t)nt, (const Slot*)table.p,
                                                     (const uint32_t*)uid.p, (const uint32_t*)u_tid.p, m);
        launched();
        chunk_tok.push_back(n_elems + rr_off[src]);
        chunk_C.push_back((uint32_t)nt);
      }
      n_elems += R;
      n_tokens += R;
    }
    n_docs += tot_docs;
    sync();  // exchange buffers are reused by the next chunk
  }

  // the arena size of a deferred first insert (dscal[4], written by its ArenaSizeU scan)
  void settle_arena() {
    if (!arena_pending) return;
    readback(4, 1);
    arena_used = (uint32_t)h_scal[4];
    arena_pending = false;
  }

  void insert_new(const uint8_t* text, uint64_t U, uint64_t Nn) {
    settle_arena();
    uint64_t* kk = buf<uint64_t>(nk_key, Nn + 16);
    uint32_t* kv = buf<uint32_t>(nk_val, Nn + 16);
    uint64_t* kk2 = buf<uint64_t>(nk_key2, Nn + 16);
    uint32_t* kv2 = buf<uint32_t>(nk_val2, Nn + 16);
    k_miss_compact<<<grid_for(U, 256), 256, 0, st>>>((const uint32_t*)u_tid.p, (const uint32_t*)midx.p,
                                                     (const uint64_t*)u_key.p, (uint32_t)U, kk, kv);
    launched();
    // arena offsets, in unique order (only misses take space); the new terms' columns and arena bytes
    // need no sorted order, so they go ahead of the sort (the dictionary stream's tail is the step's
    // critical path once the side stream is done)
    uint32_t* ao = buf<uint32_t>(aoff, U);
    scan<uint32_t>(ArenaSizeU{(const uint32_t*)u_tid.p, (const uint32_t*)u_len.p, (const uint32_t*)u_bucket.p}, U, ao,
                   (uint32_t*)(dscal() + 4));
    WJ_CUDA_CHECK(cudaMemsetAsync((uint32_t*)(dscal() + 4) + 1, 0, 4, st));
    uint64_t A = 0;
    uint8_t* ar = nullptr;
    const bool defer = V == 0 && arena_used == 0 && dict_text_bytes > 0 && dict_text_bytes + U < 0xFFFFFFFFull;
    if (defer) {  // A <= sum over the unique terms of (1 + length) <= text bytes + U
      ar = buf_keep<uint8_t>(arena, dict_text_bytes + U, 0);
    } else {
      readback(4, 1);
      A = (uint32_t)h_scal[4];
      if (arena_used + A >= 0xFFFFFFFFull) throw StatusError{WJ_ERR_CAPACITY, "string arena exceeds 4 GiB"};
      ar = buf_keep<uint8_t>(arena, arena_used + A, arena_used);
    }
    const uint64_t Vn = (uint64_t)V + Nn;
    uint32_t* ta = buf_keep<uint32_t>(t_arena, Vn, V);
    uint32_t* tc = buf_keep<uint32_t>(t_cache, Vn, V);
    uint32_t* tb = buf_keep<uint32_t>(t_bucket, Vn, V);
    uint32_t* nt = buf<uint32_t>(ns_tid, Nn);
    uint32_t* nb = buf<uint32_t>(ns_bucket, Nn);
    uint32_t* nr = buf<uint32_t>(ns_rank, Nn);
    k_new_terms<<<grid_for(U, 256), 256, 0, st>>>((uint32_t)U, ao, arena_used, text, (const uint4*)u_w.p,
                                                  (const uint32_t*)u_ref.p, (const uint32_t*)u_len.p,
                                                  (const uint32_t*)u_bucket.p, (const uint32_t*)u_cache.p,
                                                  (uint32_t*)u_tid.p, (const uint32_t*)midx.p, V, ar, ta, tc, tb,
                                                  (const uint32_t*)u_rank.p, buf<uint4>(u_pack, U));
    launched();
    // sort new terms by (collection, suffix): 8-bit LSD over the kSortKeyBits-bit key, then tie runs
    const bool in2 = sort_pairs<uint64_t>(kk, kv, kk2, kv2, Nn, 0, kSortKeyBits, nullptr, false);
    uint64_t* sk = in2 ? kk2 : kk;
    uint32_t* sv = in2 ? kv2 : kv;
    k_tie_fix<<<grid_for(Nn, 256), 256, 0, st>>>(sk, sv, (uint32_t)Nn, text, (const uint4*)u_w.p, (const uint32_t*)u_ref.p,
                                                 (const uint32_t*)u_len.p);
    launched();
    uint32_t* ni = buf<uint32_t>(ns_info, Nn);
    uint32_t* na = buf<uint32_t>(ns_arena, Nn);
    k_ns_fill<<<grid_for(Nn, 256), 256, 0, st>>>(sv, (uint32_t)Nn, (const uint4*)u_pack.p, nt, nb, nr, ni, na);
    launched();
    if (defer) arena_pending = true;
    else arena_used += A;
    // merge into the sorted key order E of every collection
    uint32_t* lo = buf<uint32_t>(nlo, kCollections + 1);
    uint32_t* hi = buf<uint32_t>(nhi, kCollections + 1);
    WJ_CUDA_CHECK(cudaMemsetAsync(lo, 0, (kCollections + 1) * 4, st));
    WJ_CUDA_CHECK(cudaMemsetAsync(hi, 0, (kCollections + 1) * 4, st));
    k_new_ranges<<<grid_for(Nn, 256), 256, 0, st>>>(nb, (uint32_t)Nn, lo, hi);
    launched();
    uint32_t* cb2 = buf<uint32_t>(coll_base2, kCollections + 1);
    scan<uint32_t>(NewCount{(const uint32_t*)coll_n.p, lo, hi}, kCollections, cb2, cb2 + kCollections);
    uint32_t* et2 = buf<uint32_t>(e_tid2, Vn);
    uint32_t* eb2 = buf<uint32_t>(e_bkt2, Vn);
    uint32_t* ea2 = buf<uint32_t>(e_ar2, Vn);
    k_place_new<<<grid_for(Nn, 256), 256, 0, st>>>(nt, ni, na, nr, (uint32_t)Nn, lo, cb2, et2, eb2, ea2);
    launched();
    if (V > 0) {
      k_place_old<<<grid_for(V, 256), 256, 0, st>>>((const uint32_t*)e_tid.p, (const uint32_t*)e_bkt.p,
                                                    (const uint32_t*)e_ar.p, V, (const uint32_t*)coll_base.p, nr, lo, hi,
                                                    cb2, et2, eb2, ea2);
      launched();
    }
    k_update_counts<<<grid_for(kCollections, 256), 256, 0, st>>>((uint32_t*)coll_n.p, lo, hi);
    launched();
    std::swap(e_tid, e_tid2);
    std::swap(e_bkt, e_bkt2);
    std::swap(e_ar, e_ar2);
    std::swap(coll_base, coll_base2);
    V = (uint32_t)Vn;
  }

  void rebuild() {
    // level 0: one root per non-empty collection
    uint32_t* ri = buf<uint32_t>(root_idx, kCollections + 1);
    scan<uint32_t>(NonEmpty{(const uint32_t*)coll_n.p}, kCollections, ri, (uint32_t*)(dscal() + 7));
    WJ_CUDA_CHECK(cudaMemsetAsync((uint32_t*)(dscal() + 7) + 1, 0, 4, st));
    readback(7, 1);
    uint64_t L = (uint32_t)h_scal[7];
    // worst case nodes: every non-root node holds >= 15 keys
    const uint64_t max_nodes = (uint64_t)V / 15 + L + 16;
    Node* nd = (Node*)grow(nodes, max_nodes * sizeof(Node));
    DevBuf* cur = lvA;
    DevBuf* nxt = lvB;
    auto level = [&](DevBuf* lv, uint64_t n) {
      return Level{buf<uint32_t>(lv[0], n), buf<uint32_t>(lv[1], n), buf<uint32_t>(lv[2], n), buf<uint32_t>(lv[3], n)};
    };
    Level lc = level(cur, L);
    k_roots<<<grid_for(kCollections, 256), 256, 0, st>>>((const uint32_t*)coll_n.p, ri, (uint32_t*)coll_root.p, lc);
    launched();
    uint64_t base = 0;
    uint32_t depth = 0;
    while (L > 0) {
      ++depth;
      uint32_t* co = buf<uint32_t>(child_off, L + 1);
      scan<uint32_t>(ChildCount{lc.m, lc.h}, L, co, (uint32_t*)(dscal() + 7));
      WJ_CUDA_CHECK(cudaMemsetAsync((uint32_t*)(dscal() + 7) + 1, 0, 4, st));
      readback(7, 1);
      const uint64_t Ln = (uint32_t)h_scal[7];
      if (base + L + Ln > max_nodes) throw StatusError{WJ_ERR_CAPACITY, "B-tree node pool overflow (internal)"};
      Level ln = level(nxt, Ln);
      lc = level(cur, L);  // (re)fetch pointers: level() may not reallocate cur, but keep it explicit
      const unsigned blocks = (unsigned)std::min<uint64_t>((L + 7) / 8, 148ull * 64);
      k_build_level<<<blocks, 256, 0, st>>>(lc, (uint32_t)L, (uint32_t)base, co, (uint32_t)(base + L), ln,
                                            (const uint32_t*)e_tid.p, (const uint32_t*)coll_base.p,
                                            (const uint32_t*)t_arena.p, (const uint32_t*)t_cache.p, nd);
      launched();
      base += L;
      L = Ln;
      std::swap(cur, nxt);
      lc = ln;
    }
    n_nodes = base;
    height_max = depth;
  }

  // stable LSD radix sort driver (radix.cuh: per pass k_rs_up + scan + k_rs_down2).  Digits come
  // from key & kmask.  segs (optional): per stream segment a key map applied in place by the first
  // upsweep (slot -> rank).  skip0: elements with no bits above kmask are holes, dropped by the first
  // pass; *n_out = elements after the sort.
  template <typename K>
  bool sort_pairs(K* k0, uint32_t* v0, K* k1, uint32_t* v1, uint64_t n, int begin_bit, int end_bit,
                  const uint32_t* rank_of, bool timed,
                  const std::vector<std::pair<uint64_t, const uint32_t*>>* segs = nullptr, K kmask = ~K(0),
                  bool skip0 = false, uint64_t* n_out = nullptr, bool mask_digits = true,
                  std::vector<uint64_t>* digit_start = nullptr, uint32_t* holes_n_dev = nullptr,
                  uint32_t* head_cnt = nullptr, uint32_t head_per = 0, uint8_t* digits = nullptr) {
    if (n_out) *n_out = n;
    if (n == 0) return false;
    int passes = end_bit > begin_bit ? (end_bit - begin_bit + 7) / 8 : 0;
    if (skip0 && passes == 0) passes = 1;  // the first pass also compacts the holes
    const bool multi_map = segs && segs->size() > 1;
    if (segs && multi_map) {  // apply each chunk's map first (holes and count bits preserved)
      for (size_t i = 0; i < segs->size(); ++i) {
        const uint64_t off = (*segs)[i].first;
        const uint64_t end = i + 1 < segs->size() ? (*segs)[i + 1].first : n;
        if (end > off) {
          auto m = [&] {
            k_map_rank<<<grid_for(end - off, 256), 256, 0, st>>>((uint32_t*)(k0 + off), end - off, (*segs)[i].second);
            launched();
          };
          if (timed) ktime(WJ_KERNEL_SORT_HIST, m); else m();
        }
      }
    }
    if (passes == 0 || (n == 1 && !skip0)) {
      if (head_cnt) {  // no pass counts the run-length heads: a single element is one head
        if (n > 1) throw StatusError{WJ_ERR_STATE, "head counting needs a radix pass (internal)"};
        k_fill<uint32_t><<<1, 32, 0, st>>>(head_cnt, 1, 1u);
        launched();
      }
      if (segs && !multi_map) {
        k_map_rank<<<grid_for(n, 256), 256, 0, st>>>((uint32_t*)k0, n, (*segs)[0].second);
        launched();
      }
      return false;
    }
    const uint32_t* first_map = (segs && !multi_map) ? (*segs)[0].second : rank_of;
    bool in1 = false;
    uint64_t cur_n = n;
    // with holes_n_dev the count left by the first (hole-compacting) pass stays on the device: the
    // later passes are launched for the upper bound and read the count (no host round trip)
    const uint32_t* n_dev = nullptr;
    for (int p = 0; p < passes; ++p) {
      if (cur_n == 0) break;  // every element was a hole
      uint64_t per = (cur_n + rs_ctas - 1) / rs_ctas;
      per = (per + kOsTile - 1) / kOsTile * kOsTile;
      const uint32_t G = (uint32_t)((cur_n + per - 1) / per);
      uint32_t* h1 = buf<uint32_t>(hist, (uint64_t)256 * G);
      uint32_t* h2 = buf<uint32_t>(hist_scan, (uint64_t)256 * G + 1);
      K* ki = in1 ? k1 : k0;
      uint32_t* vi = in1 ? v1 : v0;
      K* ko = in1 ? k0 : k1;
      uint32_t* vo = in1 ? v0 : v1;
      const int shift = begin_bit + 8 * p;
      const uint32_t* mp = p == 0 ? first_map : nullptr;
      const bool holes = skip0 && p == 0;
      // the count bits of stream elements only reach a digit when passes cover bits >= 25
      const bool masked = mask_digits && kmask != ~K(0) && begin_bit + 8 * passes > kCountShift;
      auto up = [&] {
        WJ_CUDA_CHECK(cudaMemsetAsync(h1, 0, (size_t)256 * G * 4, st));
        const uint32_t GU = G * kRsUpSplit;
        if (digits) k_rs_up_bytes<<<GU, 256, 0, st>>>(digits, cur_n, per, h1);  // this pass's digit bytes
        else if (holes && masked) k_rs_up<K, true, true><<<GU, 256, 0, st>>>(ki, cur_n, per, shift, mp, h1, kmask, n_dev);
        else if (holes) k_rs_up<K, true, false><<<GU, 256, 0, st>>>(ki, cur_n, per, shift, mp, h1, kmask, n_dev);
        else if (masked) k_rs_up<K, false, true><<<GU, 256, 0, st>>>(ki, cur_n, per, shift, mp, h1, kmask, n_dev);
        else k_rs_up<K, false, false><<<GU, 256, 0, st>>>(ki, cur_n, per, shift, mp, h1, kmask, n_dev);
        launched();
      };
      if (timed) ktime(WJ_KERNEL_SORT_HIST, up); else up();
      scan<uint32_t>(ArrayIn<uint32_t>{h1}, (uint64_t)256 * G, h2, h2 + (uint64_t)256 * G);
      auto down = [&] {
        const size_t sm = v0 ? ds_smem_bytes<K>() : ds_smem_bytes<K, true>();
        if (!v0) {  // value-less keys (the packed stream): no holes, no masked digits
          if (holes || masked) throw StatusError{WJ_ERR_STATE, "value-less sort with holes / masked digits"};
          if (head_cnt && p == passes - 1) {  // the last pass also counts the run-length heads
            k_rs_down2<K, false, false, true, true><<<G, kDsThreads, sm, st>>>(ki, vi, ko, vo, cur_n, per, shift, h2, kmask,
                                                                              n_dev, head_cnt, head_per);
            k_head_fix<K><<<grid_for((uint64_t)256 * G, 256), 256, 0, st>>>(ko, h2, 256 * G, head_cnt, head_per);
            launched();
          } else {  // (digits: write the next pass's digit bytes)
            k_rs_down2<K, false, false, true><<<G, kDsThreads, sm, st>>>(ki, vi, ko, vo, cur_n, per, shift, h2, kmask, n_dev,
                                                                        nullptr, 0, digits);
          }
        } else if (holes && masked) k_rs_down2<K, true, true><<<G, kDsThreads, sm, st>>>(ki, vi, ko, vo, cur_n, per, shift, h2, kmask, n_dev);
        else if (holes) k_rs_down2<K, true, false><<<G, kDsThreads, sm, st>>>(ki, vi, ko, vo, cur_n, per, shift, h2, kmask, n_dev);
        else if (masked) k_rs_down2<K, false, true><<<G, kDsThreads, sm, st>>>(ki, vi, ko, vo, cur_n, per, shift, h2, kmask, n_dev);
        else k_rs_down2<K, false, false><<<G, kDsThreads, sm, st>>>(ki, vi, ko, vo, cur_n, per, shift, h2, kmask, n_dev);
        launched();
      };
      if (timed) ktime(WJ_KERNEL_SORT_SCATTER, down); else down();
      if (digit_start && passes == 1) {  // global start of every digit (single-pass partitions)
        std::vector<uint32_t> ds(257);
        WJ_CUDA_CHECK(cudaMemcpy2DAsync(ds.data(), 4, h2, (size_t)G * 4, 4, 256, cudaMemcpyDeviceToHost, st));
        WJ_CUDA_CHECK(cudaMemcpyAsync(&ds[256], h2 + (uint64_t)256 * G, 4, cudaMemcpyDeviceToHost, st));
        sync();
        digit_start->assign(ds.begin(), ds.end());
      }
      if (holes && holes_n_dev) {
        WJ_CUDA_CHECK(cudaMemcpyAsync(holes_n_dev, h2 + (uint64_t)256 * G, 4, cudaMemcpyDeviceToDevice, st));
        n_dev = holes_n_dev;
      } else if (holes) {  // elements that survive the compaction
        uint32_t tot = 0;
        WJ_CUDA_CHECK(cudaMemcpyAsync(&tot, h2 + (uint64_t)256 * G, 4, cudaMemcpyDeviceToHost, st));
        sync();
        cur_n = tot;
        if (n_out) *n_out = cur_n;
      }
      in1 = !in1;
    }
    return in1;
  }

  // final dictionary bytes: term_off by scan, restored trie prefix + stored suffix (needs ranks only)
  void dict_bytes() {
    const uint2* ta = (const uint2*)term_at.p;  // rank_info (k_lexrank)
    phase(WJ_PHASE_DICT);
    uint64_t* to = buf<uint64_t>(term_off, (uint64_t)V + 1);
    TB = 0;
    if (V > 0) {
      scan<uint64_t>(TermFullLen{ta},
                     V, to, to + V);
      WJ_CUDA_CHECK(cudaMemcpyAsync(h_scal + 9, to + V, 8, cudaMemcpyDeviceToHost, st));
      sync();
      TB = h_scal[9];
      uint8_t* tbp = buf<uint8_t>(term_bytes, TB);
      k_term_bytes<<<(unsigned)std::min<uint64_t>(grid_for(V, 256), 148ull * 2), 256, 0, st>>>(  // 2 CTAs per SM
          ta, V, (const uint8_t*)arena.p, to, tbp);
      launched();
    } else {
      WJ_CUDA_CHECK(cudaMemsetAsync(to, 0, 8, st));
    }
  }

  // ---------------------------------------------------------------- finalize
  void finalize() {
    drain();
    const uint64_t NE = n_elems;  // stream elements (tokens, aggregated hot entries, holes)
    uint32_t* ro = buf<uint32_t>(rank_of, V);
    uint2* ta = buf<uint2>(term_at, V);  // rank_info
    if (!pm && (uint64_t)V > (uint64_t)kRankMask + 1)  // enforced at insert already (dictionary_update)
      throw StatusError{WJ_ERR_CAPACITY, "more than 2^25 terms in one dictionary slice"};
    if (pm) join_partials();  // the last run's records (on st)
    // one run whose records are indexed by termID (the first chunk into an empty dictionary, chunk_partials):
    // k_lexrank gathers df / cf / list start per term and writes them by rank
    const bool by_tid = pm && recs_by_tid && rec_end.size() == 1 && nrec == V && V > 0;
    uint64_t* po = buf<uint64_t>(post_off, (uint64_t)V + 1);
    uint32_t* dfp = buf<uint32_t>(df, V);
    uint64_t* cfp = buf<uint64_t>(cf, V);
    uint64_t* csp = buf<uint64_t>(cstart_b, (uint64_t)V + 1);
    uint64_t* src_r = by_tid ? buf<uint64_t>(cf_totb, V) : nullptr;  // list start by rank (k_copy_by_rank)
    if (V > 0) {
      phase(WJ_PHASE_LEXRANK);
      LexGroups* g = (LexGroups*)grow(lexg, sizeof(LexGroups));
      k_lex_groups<<<1, kLexGroupThreads, 0, st>>>((const uint32_t*)e_tid.p, (const uint32_t*)coll_base.p,
                                     (const uint32_t*)coll_n.p, (const uint32_t*)t_cache.p, g);
      uint32_t* sle = buf<uint32_t>(lex_short, 17576);
      k_lex_short<<<grid_for(17576, 256), 256, 0, st>>>((const uint32_t*)e_tid.p, (const uint32_t*)coll_base.p,
                                                        (const uint32_t*)coll_n.p, (const uint8_t*)arena.p,
                                                        (const uint32_t*)t_arena.p, (const uint32_t*)t_bucket.p, sle);
      k_lexrank<<<grid_for(V, 256), 256, 0, st>>>(
          (const uint32_t*)e_tid.p, (const uint32_t*)e_bkt.p, (const uint32_t*)e_ar.p, V, (const uint32_t*)coll_base.p,
          (const uint32_t*)coll_n.p, g, (const uint8_t*)arena.p, (const uint32_t*)t_arena.p, (const uint32_t*)t_bucket.p,
          (const uint32_t*)t_cache.p, sle, ro, ta, by_tid ? (const uint4*)rec_aos.p : nullptr, dfp, cfp, src_r);
      launched(3);
    }
    P = 0;
    if (pm) {
      // combine the chunks' partial lists (partials.cuh): totals per term in chunk order, post_off in
      // rank order, one copy of every partial list to its place.  The dictionary bytes need no
      // postings: they run on the side stream (idle once the last chunk is joined) meanwhile.
      settle_partials();
      sorted_elems = n_elems - pm_merged;
      phase(-1);
      WJ_CUDA_CHECK(cudaEventRecord(ev_fork, st));  // ranks (k_lexrank) are ready in st order
      bool dict_started = false;
      auto side_dict = [&] {  // enqueue dict_bytes on side_st (its size readback waits for side_st only)
        if (dict_started) return;
        dict_started = true;
        const int open = cur_phase;
        phase(-1);
        WJ_CUDA_CHECK(cudaStreamWaitEvent(side_st, ev_fork, 0));
        swap_side();
        try {
          dict_bytes();
          phase(-1);
          WJ_CUDA_CHECK(cudaEventRecord(ev_side, st));
        } catch (...) {
          swap_side();
          throw;
        }
        swap_side();
        if (open >= 0) phase(open);
      };
      if (nrec > 0 && V > 0) {
        phase(WJ_PHASE_POSTINGS);
        uint32_t* dft = buf<uint32_t>(df_totb, V);
        uint64_t* cft = buf<uint64_t>(cf_totb, V);
        uint32_t* bef = buf<uint32_t>(rec_before, nrec);
        const uint32_t* rt = (const uint32_t*)rec_tid.p;
        const uint32_t* rd = (const uint32_t*)rec_df.p;
        if (rec_end.size() == 1) {  // one run: every partial list is its term's whole list
          if (!by_tid) {  // (by_tid: k_lexrank wrote df, cf and the list starts by rank already)
            k_rank_scatter_rec<<<grid_for(nrec, 256), 256, 0, st>>>(rt, rd, (const uint32_t*)rec_cf.p, nrec, ro, dfp, cfp,
                                                                    (const uint64_t*)rec_start.p, cft);
            launched();
          }
        } else {
          WJ_CUDA_CHECK(cudaMemsetAsync(dft, 0, (size_t)V * 4, st));
          WJ_CUDA_CHECK(cudaMemsetAsync(cft, 0, (size_t)V * 8, st));
          uint64_t lo = 0;
          for (const uint64_t hi : rec_end) {
            if (hi > lo) {
              k_rec_accum<<<grid_for(hi - lo, 256), 256, 0, st>>>(rt, rd, (const uint32_t*)rec_cf.p, lo, hi, dft, cft, bef);
              launched();
            }
            lo = hi;
          }
          k_rank_scatter<<<grid_for(V, 256), 256, 0, st>>>(ro, V, dft, cft, dfp, cfp);
          launched();
        }
        scan<uint64_t>(U32AsU64{dfp}, V, po, po + V);
        WJ_CUDA_CHECK(cudaMemcpyAsync(h_scal + 8, po + V, 8, cudaMemcpyDeviceToHost, st));
        side_dict();
        sync();
        P = h_scal[8];
        uint32_t* od = buf<uint32_t>(out_doc, P + 1);
        uint32_t* of = buf<uint32_t>(out_tf, P + 1);
        ktime(WJ_KERNEL_COPY_PARTIALS, [&] {
          if (rec_end.size() == 1) {  // one run: cft holds the list start of each rank
            k_copy_by_rank<<<grid_for((P + kCopyChunk - 1) / kCopyChunk * 32, 256), 256, 0, st>>>(
                cft, V, P, po, (const uint2*)pp_pair.p, od, of);
            launched();
            return;
          }
          // several runs: the records sorted into destination order (rank, then run: a stable sort by
          // rank), then the same rank-order copy (coalesced writes, each partial list one gathered read)
          uint32_t* rk = buf<uint32_t>(mr_key, nrec + 16);
          uint32_t* ri = buf<uint32_t>(mr_idx, nrec + 16);
          uint32_t* rk2 = buf<uint32_t>(mr_key2, nrec + 16);
          uint32_t* ri2 = buf<uint32_t>(mr_idx2, nrec + 16);
          k_rec_rank_key<<<grid_for(nrec, 256), 256, 0, st>>>(rt, nrec, ro, rk, ri);
          launched();
          int rbits = 0;
          while (rbits < 32 && ((uint64_t)1 << rbits) < V) ++rbits;
          const uint32_t* sorted = sort_pairs<uint32_t>(rk, ri, rk2, ri2, nrec, 0, std::max(rbits, 1), nullptr, false)
                                       ? ri2 : ri;
          uint64_t* dst = buf<uint64_t>(mr_dst, nrec + 1);
          uint64_t* src = buf<uint64_t>(mr_src, nrec + 1);
          k_rec_dest<<<grid_for(nrec, 256), 256, 0, st>>>(sorted, nrec, rt, bef, (const uint64_t*)rec_start.p, ro, po,
                                                          dst, src);
          k_copy_by_rank<<<grid_for((P + kCopyChunk - 1) / kCopyChunk * 32, 256), 256, 0, st>>>(
              src, nrec, P, dst, (const uint2*)pp_pair.p, od, of);
          launched(2);
        });
      } else {
        WJ_CUDA_CHECK(cudaMemsetAsync(po, 0, 8, st));
      }
      side_dict();
      WJ_CUDA_CHECK(cudaStreamWaitEvent(st, ev_side, 0));
    } else if (NE > 0 && V > 0) {
      phase(WJ_PHASE_SORT);
      uint32_t* kt = (uint32_t*)g_tid.p;
      uint32_t* dt = (uint32_t*)g_doc.p;
      uint32_t* k1 = buf<uint32_t>(sk1, NE + 16);
      uint32_t* v1 = buf<uint32_t>(sv1, NE + 16);
      int bits = 0;
      while (bits < 32 && ((uint64_t)1 << bits) < V) ++bits;
      // per chunk: slot -> termID -> rank map; applied in the histogram pass; the stable sort by
      // rank keeps docIDs ascending within every term; the first pass drops the holes
      std::vector<std::pair<uint64_t, const uint32_t*>> segs;
      for (size_t c = 0; c < chunk_tok.size(); ++c) {
        uint32_t* m = (uint32_t*)chunk_map[c].p;
        k_map_compose<<<grid_for(chunk_C[c], 256), 256, 0, st>>>(m, chunk_C[c], ro);
        launched();
        segs.emplace_back(chunk_tok[c], m);
      }
      uint64_t N = NE;
      const bool in1 =
          sort_pairs<uint32_t>(kt, dt, k1, v1, NE, 0, bits, nullptr, true, &segs, kRankMask, stream_has_hot, &N, true,
                               nullptr);
      sorted_elems = N;
      f_key = in1 ? k1 : kt;
      f_doc = in1 ? v1 : dt;

      phase(WJ_PHASE_POSTINGS);
      uint64_t per = (N + 148 * 2 - 1) / (148 * 2);
      per = (per + kRleTile - 1) / kRleTile * kRleTile;
      const uint32_t G = (uint32_t)((N + per - 1) / per);
      uint32_t* rc = buf<uint32_t>(rle_p0, (uint64_t)G + 1);
      uint32_t* rl = buf<uint32_t>(rle_lead, (uint64_t)G + 1);
      uint64_t* rt = buf<uint64_t>(rle_tok, (uint64_t)G + 1);
      // P <= N: size the outputs by N, no host round trip before the pass
      uint32_t* od = buf<uint32_t>(out_doc, N);
      uint32_t* of = buf<uint32_t>(out_tf, N);
      ktime(WJ_KERNEL_RLE_EMIT, [&] {
        if (stream_has_hot)
          k_rle_count<true><<<G, kRleThreads, 0, st>>>(f_key, f_doc, N, per, rc, rt, nullptr);
        else
          k_rle_count<false><<<G, kRleThreads, 0, st>>>(f_key, f_doc, N, per, rc, rt, nullptr);
        launched();
        scan<uint32_t>(ArrayIn<uint32_t>{rc}, G, rc, (uint32_t*)(dscal() + 8));
        scan<uint64_t>(ArrayIn<uint64_t>{rt}, G, rt, (uint64_t*)(dscal() + 11));
        if (stream_has_hot)
          k_rle_write_tma<true><<<G, kRleThreads, rle_smem_bytes(), st>>>(f_key, f_doc, N, per, rc, rt, od, of, 1u, po,
                                                                          csp, rl, nullptr);
        else
          k_rle_write_tma<false><<<G, kRleThreads, rle_smem_bytes(false), st>>>(f_key, f_doc, N, per, rc, rt, od, of, 1u,
                                                                            po, csp, rl, nullptr);
        launched();
      });
      k_rle_fixup<<<grid_for(G, 256), 256, 0, st>>>(rc, rl, G, of, 1u);
      launched();
      WJ_CUDA_CHECK(cudaMemsetAsync((uint32_t*)(dscal() + 8) + 1, 0, 4, st));
      readback(8, 1);
      P = (uint32_t)h_scal[8];
      k_df_cf<<<grid_for((uint64_t)V + 1, 256), 256, 0, st>>>(po, csp, V, P, n_tokens, dfp, cfp);
      launched();
    } else {
      WJ_CUDA_CHECK(cudaMemsetAsync(po, 0, 8, st));
    }
    PB = 0;
    if (vbyte) encode_vbyte();
    if (!pm) dict_bytes();
    phase(-1);
    sync();
    finalized = true;
  }

  // f1: d-gap + variable-byte code of the postings (vbyte.cuh, reading S19) ->
  // vb_code[PB], vb_boff[V+1] (byte offset of every list)
  void encode_vbyte() {
    phase(WJ_PHASE_VBYTE);
    uint64_t* pbo = buf<uint64_t>(vb_boff, (uint64_t)V + 1);
    if (P == 0) {
      WJ_CUDA_CHECK(cudaMemsetAsync(pbo, 0, 8 * ((uint64_t)V + 1), st));
      return;
    }
    uint32_t* fb = buf<uint32_t>(vb_first, P / 32 + 1);
    WJ_CUDA_CHECK(cudaMemsetAsync(fb, 0, 4 * (P / 32 + 1), st));
    k_vb_first<<<grid_for(V, 256), 256, 0, st>>>((const uint64_t*)post_off.p, V, fb);
    launched();
    const uint64_t G = (P + kVbTile - 1) / kVbTile;
    uint64_t* tb = buf<uint64_t>(vb_tiles, G + 1);
    const uint32_t* od = (const uint32_t*)out_doc.p;
    const uint32_t* of = (const uint32_t*)out_tf.p;
    k_vb_tile<<<(unsigned)G, kVbThreads, 0, st>>>(od, of, fb, P, tb);
    launched();
    scan<uint64_t>(ArrayIn<uint64_t>{tb}, G, tb, tb + G);
    WJ_CUDA_CHECK(cudaMemcpyAsync(h_scal + 13, tb + G, 8, cudaMemcpyDeviceToHost, st));
    sync();
    PB = h_scal[13];
    uint8_t* code = buf<uint8_t>(vb_code, PB + 16);
    k_vb_encode<<<(unsigned)G, kVbThreads, kVbMaxTileBytes, st>>>(od, of, fb, P, (const uint64_t*)post_off.p, V, tb,
                                                                  code, pbo);
    launched();
    WJ_CUDA_CHECK(cudaMemcpyAsync(pbo + V, tb + G, 8, cudaMemcpyDeviceToDevice, st));
  }

  // ---------------------------------------------------------------- serialize
  uint64_t serialized_size() const {
    auto pad8 = [](uint64_t x) { return (x + 7) & ~7ull; };
    return 64 + 8 * ((uint64_t)V + 1) + pad8(TB) + pad8(4ull * V) + 8ull * V + 8 * ((uint64_t)V + 1) +
           (vbyte ? pad8(PB) : pad8(4 * P) + pad8(4 * P));
  }
  void serialize(uint8_t* out) {
    auto pad8 = [](uint64_t x) { return (x + 7) & ~7ull; };
    uint64_t hdr[8];
    memcpy(hdr, vbyte ? "WJINV002" : "WJINV001", 8);
    hdr[1] = n_docs; hdr[2] = n_tokens; hdr[3] = n_dropped; hdr[4] = V; hdr[5] = P; hdr[6] = TB; hdr[7] = vbyte ? PB : 0;
    memcpy(out, hdr, 64);
    uint64_t p = 64;
    auto d2h = [&](const void* src, uint64_t bytes, uint64_t padded) {
      if (bytes) WJ_CUDA_CHECK(cudaMemcpyAsync(out + p, src, bytes, cudaMemcpyDeviceToHost, st));
      if (padded > bytes) memset(out + p + bytes, 0, padded - bytes);
      p += padded;
    };
    d2h(term_off.p, 8 * ((uint64_t)V + 1), 8 * ((uint64_t)V + 1));
    d2h(term_bytes.p, TB, pad8(TB));
    d2h(df.p, 4ull * V, pad8(4ull * V));
    d2h(cf.p, 8ull * V, 8ull * V);
    if (vbyte) {
      d2h(vb_boff.p, 8 * ((uint64_t)V + 1), 8 * ((uint64_t)V + 1));
      d2h(vb_code.p, PB, pad8(PB));
    } else {
      d2h(post_off.p, 8 * ((uint64_t)V + 1), 8 * ((uint64_t)V + 1));
      d2h(out_doc.p, 4 * P, pad8(4 * P));
      d2h(out_tf.p, 4 * P, pad8(4 * P));
    }
    sync();
  }
};

// ====================================================================== C ABI
namespace {

template <class F>
int guarded(wj_index* ix, F&& f) {
  try {
    if (ix->broken) {
      ix->err = "context unusable after an earlier CUDA error";
      return WJ_ERR_CUDA;
    }
    WJ_CUDA_CHECK(cudaSetDevice(ix->device));
    return f();
  } catch (const StatusError& e) {
    ix->err = e.msg;
    return e.code;
  } catch (const CudaError& e) {
    ix->err = std::string("CUDA error ") + cudaGetErrorString(e.err) + " at " + e.file + ":" + std::to_string(e.line) +
              " (" + e.expr + ")";
    if (e.err == cudaErrorMemoryAllocation) return WJ_ERR_OOM;
    ix->broken = true;
    return WJ_ERR_CUDA;
  } catch (const std::bad_alloc&) {
    ix->err = "host allocation failed";
    return WJ_ERR_OOM;
  }
}

thread_local std::string g_init_err;

}  // namespace

extern "C" {

int index_init(wj_index** out, const wj_config* cfg) {
  if (!out || !cfg) return WJ_ERR_INVALID_ARG;
  *out = nullptr;
  if (cfg->world < 1 || cfg->world > 1024 || cfg->rank < 0 || cfg->rank >= cfg->world || (cfg->flags & ~(WJ_FLAG_PROFILE | WJ_FLAG_LOOPBACK | WJ_FLAG_VBYTE | WJ_FLAG_HOST_PIPELINE | WJ_FLAG_BALANCED_OWNERS | WJ_FLAG_STEM | WJ_FLAG_STOPWORDS | WJ_FLAG_HOT_TERMS | WJ_FLAG_GLOBAL_STREAM)) || cfg->reserved) {
    g_init_err = "invalid config";
    return WJ_ERR_INVALID_ARG;
  }
  if (cfg->world > 1 && !cfg->nccl_unique_id) {
    g_init_err = "world > 1 needs nccl_unique_id (NCCL) or a loopback hub (WJ_FLAG_LOOPBACK)";
    return WJ_ERR_INVALID_ARG;
  }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    g_init_err = "no CUDA device";
    return WJ_ERR_CUDA;
  }
  if (cfg->device < 0 || cfg->device >= ndev) {
    g_init_err = "bad device ordinal";
    return WJ_ERR_INVALID_ARG;
  }
  wj_index* ix = new (std::nothrow) wj_index();
  if (!ix) return WJ_ERR_OOM;
  ix->device = cfg->device;
  ix->rank = cfg->rank;
  ix->world = cfg->world;
  ix->flags = cfg->flags;
  ix->vbyte = (cfg->flags & WJ_FLAG_VBYTE) != 0;
  ix->pipeline = (cfg->flags & WJ_FLAG_HOST_PIPELINE) != 0;
  ix->balanced = (cfg->flags & WJ_FLAG_BALANCED_OWNERS) != 0;
  ix->stem_on = (cfg->flags & WJ_FLAG_STEM) != 0;
  ix->stop_on = (cfg->flags & WJ_FLAG_STOPWORDS) != 0;
  if (cfg->workspace) {
    ix->use_arena = true;
    ix->arena_ws.init(cfg->workspace, cfg->workspace_bytes);
  }
  int rc = guarded(ix, [&]() {
    if (cfg->stream) {
      ix->st = (cudaStream_t)cfg->stream;
    } else {
      WJ_CUDA_CHECK(cudaStreamCreateWithFlags(&ix->st, cudaStreamNonBlocking));
      ix->own_stream = true;
    }
    WJ_CUDA_CHECK(cudaHostAlloc(&ix->h_scal, 16 * sizeof(uint64_t), cudaHostAllocDefault));
    if (ix->pipeline) {
      WJ_CUDA_CHECK(cudaStreamCreateWithFlags(&ix->cs, cudaStreamNonBlocking));
      for (int i = 0; i < 2; ++i) {
        WJ_CUDA_CHECK(cudaEventCreateWithFlags(&ix->pipe_copied[i], cudaEventDisableTiming));
        WJ_CUDA_CHECK(cudaEventCreateWithFlags(&ix->pipe_done[i], cudaEventDisableTiming));
      }
    }
    // per-run partial lists (one GPU) / sender-side partial lists (a transport: world > 1, or a
    // communicator at world 1); stemming / stop words and WJ_FLAG_GLOBAL_STREAM sort one global stream
    ix->pm = !ix->stem_on && !ix->stop_on;
    if (cfg->flags & WJ_FLAG_GLOBAL_STREAM) ix->pm = false;
    if (cfg->flags & WJ_FLAG_HOT_TERMS) ix->hot_min_bytes = 64ull << 10;
    if (ix->pm) {
      int least = 0, greatest = 0;
      WJ_CUDA_CHECK(cudaDeviceGetStreamPriorityRange(&least, &greatest));
      WJ_CUDA_CHECK(cudaStreamCreateWithPriority(&ix->side_st, cudaStreamNonBlocking, least));
      WJ_CUDA_CHECK(cudaStreamCreateWithPriority(&ix->hp_st, cudaStreamNonBlocking, greatest));
      WJ_CUDA_CHECK(cudaEventCreateWithFlags(&ix->ev_fork, cudaEventDisableTiming));
      WJ_CUDA_CHECK(cudaEventCreateWithFlags(&ix->ev_side, cudaEventDisableTiming));
      WJ_CUDA_CHECK(cudaEventCreateWithFlags(&ix->ev_dict, cudaEventDisableTiming));
      WJ_CUDA_CHECK(cudaEventCreateWithFlags(&ix->ev_dfork, cudaEventDisableTiming));
    }
    if (cfg->world > 1 || cfg->nccl_unique_id) {  // a transport at world 1 runs the same distributed path
      try {
        if (cfg->flags & WJ_FLAG_LOOPBACK)
          ix->xport = new LoopbackTransport((LoopbackHub*)cfg->nccl_unique_id, cfg->rank);
        else
          ix->xport = new NcclTransport(cfg->nccl_unique_id, cfg->rank, cfg->world);
      } catch (const ExchangeError& e) {
        throw StatusError{WJ_ERR_NCCL, e.msg};
      }
    }
#define WJ_DS_ATTR(K, H, M)                                                                           \
  WJ_CUDA_CHECK(cudaFuncSetAttribute(k_rs_down2<K, H, M>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                     (int)ds_smem_bytes<K>()))
    WJ_DS_ATTR(uint64_t, false, false); WJ_DS_ATTR(uint64_t, true, false); WJ_DS_ATTR(uint64_t, false, true);
    WJ_DS_ATTR(uint64_t, true, true); WJ_DS_ATTR(uint32_t, false, false); WJ_DS_ATTR(uint32_t, true, false);
    WJ_DS_ATTR(uint32_t, false, true); WJ_DS_ATTR(uint32_t, true, true);
#undef WJ_DS_ATTR
    WJ_CUDA_CHECK(cudaFuncSetAttribute(k_rs_down2<uint64_t, false, false, true, true>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ds_smem_bytes<uint64_t, true>()));
    WJ_CUDA_CHECK(cudaFuncSetAttribute(k_rs_down2<uint64_t, false, false, true>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ds_smem_bytes<uint64_t, true>()));
    WJ_CUDA_CHECK(cudaFuncSetAttribute(k_rle_write_tma<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)rle_smem_bytes()));
    WJ_CUDA_CHECK(cudaFuncSetAttribute(k_rle_write_tma<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)rle_smem_bytes()));
    ix->reset_state();
    if (ix->stop_on) ix->build_stop_keys();
    return WJ_OK;
  });
  if (rc != WJ_OK) {
    g_init_err = ix->err;
    index_destroy(ix);
    return rc;
  }
  *out = ix;
  return WJ_OK;
}

int index_add_stream(wj_index* ix, const void* bytes, uint64_t n_bytes, const uint64_t* doc_off, uint64_t n_docs) {
  if (!ix) return WJ_ERR_INVALID_ARG;
  return guarded(ix, [&]() {
    if (ix->finalized) throw StatusError{WJ_ERR_STATE, "index_add_stream after index_finalize"};
    if (!doc_off || (n_bytes && !bytes)) throw StatusError{WJ_ERR_INVALID_ARG, "NULL bytes or doc_off"};
    if (n_bytes >= 0xFFFFFFFFull) throw StatusError{WJ_ERR_INVALID_ARG, "n_bytes must be < 2^32 per call"};
    if (n_docs == 0 && n_bytes != 0) throw StatusError{WJ_ERR_INVALID_ARG, "n_bytes > 0 with no documents"};
    ix->add_stream(bytes, n_bytes, doc_off, n_docs);
    return WJ_OK;
  });
}

int index_finalize(wj_index* ix) {
  if (!ix) return WJ_ERR_INVALID_ARG;
  return guarded(ix, [&]() {
    if (ix->finalized) throw StatusError{WJ_ERR_STATE, "index_finalize called twice"};
    ix->finalize();
    return WJ_OK;
  });
}

int index_read_postings(wj_index* ix, const uint8_t* term, uint32_t len, uint32_t* docids, uint32_t* tfs, uint64_t cap,
                        uint64_t* n_out) {
  if (!ix || !n_out || (!term && len)) return WJ_ERR_INVALID_ARG;
  return guarded(ix, [&]() {
    if (!ix->finalized) throw StatusError{WJ_ERR_STATE, "index_read_postings before index_finalize"};
    *n_out = 0;
    if (len == 0 || len > kMaxTermLen || ix->V == 0) return (int)WJ_NOT_FOUND;
    for (uint32_t i = 0; i < len; ++i) {  // only token bytes can be terms (reading S1)
      const uint8_t c = term[i];
      const bool tok = (c >= '0' && c <= '9') || (c >= 'A' && c <= 'Z') || (c >= 'a' && c <= 'z') || c >= 0x80;
      if (!tok) return (int)WJ_NOT_FOUND;
    }
    ix->ensure_btrees();
    uint8_t* q = (uint8_t*)ix->grow(ix->qbuf, 512);
    QueryResult* r = (QueryResult*)ix->grow(ix->qres, sizeof(QueryResult));
    WJ_CUDA_CHECK(cudaMemcpyAsync(q, term, len, cudaMemcpyHostToDevice, ix->st));
    DictView dv{(const Node*)ix->nodes.p, (const uint32_t*)ix->coll_root.p, (const uint32_t*)ix->coll_n.p,
                (const uint8_t*)ix->arena.p};
    k_query<<<1, 32, 0, ix->st>>>(dv, q, len, (const uint32_t*)ix->rank_of.p, (const uint64_t*)ix->post_off.p, r);
    ix->launched();
    QueryResult h;
    WJ_CUDA_CHECK(cudaMemcpyAsync(&h, r, sizeof(h), cudaMemcpyDeviceToHost, ix->st));
    ix->sync();
    if (h.tid == kMiss) return (int)WJ_NOT_FOUND;
    const uint64_t df = h.hi - h.lo;
    *n_out = df;
    if (cap < df) return (int)WJ_ERR_BUFFER_TOO_SMALL;
    if (df && (!docids || !tfs)) throw StatusError{WJ_ERR_INVALID_ARG, "NULL output arrays"};
    if (df) {
      WJ_CUDA_CHECK(cudaMemcpyAsync(docids, (const uint32_t*)ix->out_doc.p + h.lo, df * 4, cudaMemcpyDeviceToHost, ix->st));
      WJ_CUDA_CHECK(cudaMemcpyAsync(tfs, (const uint32_t*)ix->out_tf.p + h.lo, df * 4, cudaMemcpyDeviceToHost, ix->st));
      ix->sync();
    }
    return (int)WJ_OK;
  });
}

int index_serialize(wj_index* ix, uint8_t* buf, uint64_t cap, uint64_t* n_out) {
  if (!ix || !n_out) return WJ_ERR_INVALID_ARG;
  return guarded(ix, [&]() {
    if (!ix->finalized) throw StatusError{WJ_ERR_STATE, "index_serialize before index_finalize"};
    const uint64_t n = ix->serialized_size();
    *n_out = n;
    if (!buf) return (int)WJ_OK;
    if (cap < n) return (int)WJ_ERR_BUFFER_TOO_SMALL;
    ix->serialize(buf);
    return (int)WJ_OK;
  });
}

int index_stats(wj_index* ix, wj_stats* out) {
  if (!ix || !out) return WJ_ERR_INVALID_ARG;
  return guarded(ix, [&]() {
    ix->collect_phases();
    ix->sync();
    memset(out, 0, sizeof(*out));
    out->n_docs = ix->n_docs;
    out->n_tokens = ix->n_tokens;
    out->n_dropped = ix->n_dropped;
    out->n_terms = ix->V;
    out->n_postings = ix->P;
    out->n_term_bytes = ix->TB;
    out->n_chunks = ix->n_chunks;
    out->kernel_launches = ix->launches;
    out->host_syncs = ix->syncs;
    out->unique_terms_last = ix->unique_last;
    out->new_terms_last = ix->new_last;
    out->btree_nodes = ix->n_nodes;
    out->btree_height_max = ix->height_max;
    out->exchange_bytes = ix->exchange_bytes;
    out->device_bytes = ix->device_bytes;
    out->stream_elems = ix->finalized ? ix->sorted_elems : ix->n_elems - ix->pm_merged;
    out->table_retries = ix->table_retries;
    out->hot_elems_saved = ix->hot_elems_saved;
    out->exchange_ms = ix->exchange_ms;
    for (int i = 0; i < WJ_PHASE_COUNT; ++i) {
      out->phase_ms[i] = ix->phase_ms[i];
      out->phase_launches[i] = ix->phase_launches[i];
    }
    for (int i = 0; i < WJ_KERNEL_COUNT; ++i) {
      out->kernel_ms[i] = ix->kernel_ms[i];
      out->kernel_count[i] = ix->kernel_count[i];
    }
    return (int)WJ_OK;
  });
}

int index_reset(wj_index* ix) {
  if (!ix) return WJ_ERR_INVALID_ARG;
  return guarded(ix, [&]() {
    ix->reset_state();
    return (int)WJ_OK;
  });
}

int index_debug_tokens(wj_index* ix, const void* bytes, uint64_t n_bytes, const uint64_t* doc_off, uint64_t n_docs,
                       uint32_t doc_base, uint8_t* out, uint64_t cap, uint64_t* n_out) {
  if (!ix || !n_out || !doc_off) return WJ_ERR_INVALID_ARG;
  return guarded(ix, [&]() {
    if (n_bytes >= 0xFFFFFFFFull) throw StatusError{WJ_ERR_INVALID_ARG, "n_bytes must be < 2^32"};
    *n_out = 0;
    if (n_docs == 0 || n_bytes == 0) return (int)WJ_OK;
    const uint8_t* text = nullptr;
    const uint64_t* off = nullptr;
    ix->stage(bytes, n_bytes, doc_off, n_docs, &text, &off);
    ChunkView cv{text, n_bytes, off, n_docs};
    const uint64_t n_segs = (n_bytes + kSegBytes - 1) / kSegBytes;
    const uint64_t Nc = ix->count_tokens(cv, n_segs);
    if (Nc == 0) return (int)WJ_OK;
    uint32_t* sl = ix->buf<uint32_t>(ix->dbg_slot, Nc);
    uint32_t* dd = ix->buf<uint32_t>(ix->dbg_doc, Nc);
    uint32_t* ds = ix->buf<uint32_t>(ix->dbg_start, Nc);
    uint32_t* dl = ix->buf<uint32_t>(ix->dbg_len, Nc);
    uint64_t C = wj_index::pow2_at_least(2 * Nc + 16);
    ix->emit_tokens(cv, n_segs, sl, dd, doc_base, C, ds, dl);
    uint64_t* doff = ix->buf<uint64_t>(ix->dbg_off, Nc + 1);
    ix->scan<uint64_t>(DumpSize{dl}, Nc, doff, doff + Nc);
    WJ_CUDA_CHECK(cudaMemcpyAsync(ix->h_scal + 9, doff + Nc, 8, cudaMemcpyDeviceToHost, ix->st));
    ix->sync();
    const uint64_t total = ix->h_scal[9];
    *n_out = total;
    if (!out) return (int)WJ_OK;
    if (cap < total) return (int)WJ_ERR_BUFFER_TOO_SMALL;
    uint8_t* dbo = ix->buf<uint8_t>(ix->dbg_out, total);
    k_dump_tokens<<<grid_for(Nc, 256), 256, 0, ix->st>>>(text, ds, dl, dd, Nc, doff, dbo);
    ix->launched();
    WJ_CUDA_CHECK(cudaMemcpyAsync(out, dbo, total, cudaMemcpyDeviceToHost, ix->st));
    ix->sync();
    return (int)WJ_OK;
  });
}

int index_debug_btree(wj_index* ix, void* nodes, uint64_t node_cap, uint64_t* n_nodes, uint32_t* collections,
                      uint8_t* arena, uint64_t arena_cap, uint64_t* arena_bytes) {
  if (!ix || !n_nodes || !arena_bytes) return WJ_ERR_INVALID_ARG;
  return guarded(ix, [&]() {
    ix->ensure_btrees();
    ix->settle_arena();
    ix->sync();
    *n_nodes = ix->n_nodes;
    *arena_bytes = ix->arena_used;
    if (nodes) {
      if (node_cap < ix->n_nodes) return (int)WJ_ERR_BUFFER_TOO_SMALL;
      if (ix->n_nodes) WJ_CUDA_CHECK(cudaMemcpy(nodes, ix->nodes.p, ix->n_nodes * sizeof(Node), cudaMemcpyDeviceToHost));
    }
    if (collections) {
      std::vector<uint32_t> r(kCollections), n(kCollections);
      WJ_CUDA_CHECK(cudaMemcpy(r.data(), ix->coll_root.p, kCollections * 4, cudaMemcpyDeviceToHost));
      WJ_CUDA_CHECK(cudaMemcpy(n.data(), ix->coll_n.p, kCollections * 4, cudaMemcpyDeviceToHost));
      for (uint32_t b = 0; b < kCollections; ++b) {
        collections[3 * b] = r[b];
        collections[3 * b + 1] = n[b];
        collections[3 * b + 2] = height_of(n[b]);
      }
    }
    if (arena) {
      if (arena_cap < ix->arena_used) return (int)WJ_ERR_BUFFER_TOO_SMALL;
      if (ix->arena_used) WJ_CUDA_CHECK(cudaMemcpy(arena, ix->arena.p, ix->arena_used, cudaMemcpyDeviceToHost));
    }
    return (int)WJ_OK;
  });
}

int index_balance_owners(const uint64_t* counts, uint32_t n, int32_t world, uint32_t* owner) {
  if (!counts || !owner || world < 1) return WJ_ERR_INVALID_ARG;
  lpt_owner_map(counts, n, world, owner);
  return WJ_OK;
}

int index_owner_map(wj_index* ix, uint32_t* out, uint32_t n) {
  if (!ix || !out || n < kCollections) return WJ_ERR_INVALID_ARG;
  for (uint32_t b = 0; b < kCollections; ++b)
    out[b] = ix->owner_ready ? ix->owner_h[b] : b % (uint32_t)ix->world;
  return WJ_OK;
}

const char* index_stop_words(void) { return kStopList; }

int index_debug_stem(int32_t device, const uint8_t* words, const uint32_t* word_off, uint32_t n, uint8_t* out,
                     uint32_t* out_len) {
  if (!words || !word_off || !out || !out_len) return WJ_ERR_INVALID_ARG;
  for (uint32_t i = 0; i < n; ++i)
    if (word_off[i + 1] < word_off[i] || word_off[i + 1] - word_off[i] > kMaxTermLen) return WJ_ERR_INVALID_ARG;
  if (n == 0) return WJ_OK;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0 || device < 0 || device >= ndev) {
    cudaGetLastError();
    return WJ_ERR_CUDA;
  }
  const uint64_t nb = word_off[n];
  uint8_t *dw = nullptr, *dout = nullptr;
  uint32_t *doff = nullptr, *dlen = nullptr;
  cudaStream_t s = nullptr;
  int prev = 0;
  cudaGetDevice(&prev);
  bool ok = cudaSetDevice(device) == cudaSuccess && cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) == cudaSuccess &&
            cudaMalloc(&dw, nb + 1) == cudaSuccess && cudaMalloc(&dout, nb + 1) == cudaSuccess &&
            cudaMalloc(&doff, (n + 1) * 4ull) == cudaSuccess && cudaMalloc(&dlen, n * 4ull) == cudaSuccess &&
            cudaMemcpyAsync(dw, words, nb, cudaMemcpyHostToDevice, s) == cudaSuccess &&
            cudaMemcpyAsync(doff, word_off, (n + 1) * 4ull, cudaMemcpyHostToDevice, s) == cudaSuccess;
  if (ok) {
    k_stem_words<<<(n + 127) / 128, 128, 0, s>>>(dw, doff, n, dout, dlen);
    ok = cudaGetLastError() == cudaSuccess &&
         cudaMemcpyAsync(out, dout, nb, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
         cudaMemcpyAsync(out_len, dlen, n * 4ull, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
         cudaStreamSynchronize(s) == cudaSuccess;
  }
  cudaFree(dw);
  cudaFree(dout);
  cudaFree(doff);
  cudaFree(dlen);
  if (s) cudaStreamDestroy(s);
  cudaSetDevice(prev);
  cudaGetLastError();
  return ok ? WJ_OK : WJ_ERR_CUDA;
}

const char* index_last_error(const wj_index* ix) { return ix ? ix->err.c_str() : g_init_err.c_str(); }

int index_nccl_unique_id(void* out128) {
  if (!out128) return WJ_ERR_INVALID_ARG;
  try {
    NcclApi& a = NcclApi::get();
    ncclUniqueId id;
    if (!a.GetUniqueId || a.GetUniqueId(&id) != ncclSuccess) {
      g_init_err = "ncclGetUniqueId failed";
      return WJ_ERR_NCCL;
    }
    memcpy(out128, &id, sizeof(id));
    return WJ_OK;
  } catch (const ExchangeError& e) {
    g_init_err = e.msg;
    return WJ_ERR_NCCL;
  }
}

int index_loopback_create(int32_t world, void** hub) {
  if (!hub || world < 1) return WJ_ERR_INVALID_ARG;
  *hub = new (std::nothrow) LoopbackHub(world);
  return *hub ? WJ_OK : WJ_ERR_OOM;
}

void index_loopback_destroy(void* hub) { delete (LoopbackHub*)hub; }

int index_merge_serialized(int32_t k, const uint8_t* const* slices, const uint64_t* sizes, uint8_t* out, uint64_t cap,
                           uint64_t* n_out) {
  if (k < 1 || !slices || !sizes || !n_out) return WJ_ERR_INVALID_ARG;
  std::vector<SliceView> v(k);
  uint64_t nt = 0, np = 0, ntb = 0, ntok = 0, ndrop = 0, npb = 0;
  for (int i = 0; i < k; ++i) {
    if (!slices[i] || !parse_slice(slices[i], sizes[i], v[i])) {
      g_init_err = "index_merge_serialized: slice " + std::to_string(i) + " is not a serialized index";
      return WJ_ERR_INVALID_ARG;
    }
    if (v[i].n_docs != v[0].n_docs || v[i].vb != v[0].vb) {
      g_init_err = "index_merge_serialized: slices disagree on n_docs or format";
      return WJ_ERR_INVALID_ARG;
    }
    nt += v[i].n_terms; np += v[i].n_postings; ntb += v[i].n_tb; ntok += v[i].n_tokens; ndrop += v[i].n_dropped;
    npb += v[i].n_pb;
  }
  const bool vb = v[0].vb;
  const uint64_t size = 64 + 8 * (nt + 1) + pad8(ntb) + pad8(4 * nt) + 8 * nt + 8 * (nt + 1) +
                        (vb ? pad8(npb) : 2 * pad8(4 * np));
  *n_out = size;
  if (!out) return WJ_OK;
  if (cap < size) return WJ_ERR_BUFFER_TOO_SMALL;
  memset(out, 0, size);
  uint64_t h[8];
  memcpy(h, vb ? "WJINV002" : "WJINV001", 8);
  h[1] = v[0].n_docs; h[2] = ntok; h[3] = ndrop; h[4] = nt; h[5] = np; h[6] = ntb; h[7] = vb ? npb : 0;
  memcpy(out, h, 64);
  uint64_t p = 64;
  uint64_t* term_off = (uint64_t*)(out + p); p += 8 * (nt + 1);
  uint8_t* tb = out + p; p += pad8(ntb);
  uint32_t* df = (uint32_t*)(out + p); p += pad8(4 * nt);
  uint64_t* cf = (uint64_t*)(out + p); p += 8 * nt;
  uint64_t* post_off = (uint64_t*)(out + p); p += 8 * (nt + 1);
  uint32_t* docid = nullptr;
  uint32_t* tf = nullptr;
  uint8_t* code = nullptr;
  if (vb) {
    code = out + p;
  } else {
    docid = (uint32_t*)(out + p); p += pad8(4 * np);
    tf = (uint32_t*)(out + p);
  }
  std::vector<uint64_t> cur(k, 0);
  auto term_less = [&](int a, int b) {
    const SliceView &x = v[a], &y = v[b];
    const uint8_t* s1 = x.term_bytes + x.term_off[cur[a]];
    const uint64_t l1 = x.term_off[cur[a] + 1] - x.term_off[cur[a]];
    const uint8_t* s2 = y.term_bytes + y.term_off[cur[b]];
    const uint64_t l2 = y.term_off[cur[b] + 1] - y.term_off[cur[b]];
    const int c = memcmp(s1, s2, l1 < l2 ? l1 : l2);
    return c != 0 ? c < 0 : l1 < l2;
  };
  uint64_t to = 0, po = 0;
  for (uint64_t t = 0; t < nt; ++t) {
    int best = -1;
    for (int i = 0; i < k; ++i)
      if (cur[i] < v[i].n_terms && (best < 0 || term_less(i, best))) best = i;
    SliceView& x = v[best];
    const uint64_t j = cur[best]++;
    const uint64_t l = x.term_off[j + 1] - x.term_off[j];
    term_off[t] = to;
    memcpy(tb + to, x.term_bytes + x.term_off[j], l);
    to += l;
    df[t] = x.df[j];
    cf[t] = x.cf[j];
    post_off[t] = po;
    const uint64_t a = x.post_off[j], b = x.post_off[j + 1];
    if (vb) {  // a list's code is self-contained (its first gap is the docID): copy it
      memcpy(code + po, x.code + a, b - a);
    } else {
      memcpy(docid + po, x.docid + a, 4 * (b - a));
      memcpy(tf + po, x.tf + a, 4 * (b - a));
    }
    po += b - a;
  }
  term_off[nt] = to;
  post_off[nt] = po;
  return WJ_OK;
}

void index_destroy(wj_index* ix) {
  if (!ix) return;
  cudaSetDevice(ix->device);
  if (ix->st) cudaStreamSynchronize(ix->st);
  if (ix->cs) cudaStreamSynchronize(ix->cs);
  ix->free_all();
  for (int i = 0; i < 2; ++i) {
    for (DevBuf* b : {&ix->pipe_text[i], &ix->pipe_off[i]})
      ix->dev_free(b->p);
    if (ix->pipe_copied[i]) cudaEventDestroy(ix->pipe_copied[i]);
    if (ix->pipe_done[i]) cudaEventDestroy(ix->pipe_done[i]);
  }
  if (ix->cs) cudaStreamDestroy(ix->cs);
  if (ix->side_st) {
    cudaStreamSynchronize(ix->side_st);
    cudaStreamDestroy(ix->side_st);
  }
  if (ix->hp_st) {
    cudaStreamSynchronize(ix->hp_st);
    cudaStreamDestroy(ix->hp_st);
  }
  if (ix->ev_dict) cudaEventDestroy(ix->ev_dict);
  if (ix->ev_dfork) cudaEventDestroy(ix->ev_dfork);
  if (ix->ev_fork) cudaEventDestroy(ix->ev_fork);
  if (ix->ev_side) cudaEventDestroy(ix->ev_side);
  delete ix->xport;
  for (auto e : ix->ev_pool) cudaEventDestroy(e);
  if (ix->h_scal) cudaFreeHost(ix->h_scal);
  if (ix->own_stream && ix->st) cudaStreamDestroy(ix->st);
  delete ix;
}

}  // extern "C"
