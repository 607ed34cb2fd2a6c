// Stable LSD radix sort of (key, u32 value) pairs with 8-bit digits: per pass an upsweep (per-CTA-range
// digit histogram, optionally applying a key map in place), a scan of the 256 x G counts and a
// TMA-prefetched downsweep (8-bit digits keep >= 16 elements per digit per 4096-element tile, so
// each digit's output run is a coalesced store; 12-bit digits were measured 2.8x slower per pass
// for exactly that reason, profiles/r02_README.md).
// Stability (equal keys keep input order) is what turns the docID-ordered token stream into
// docID-sorted postings: within one term, tokens stay in submission order.
#pragma once
#include <type_traits>
#include "common.cuh"
#include "scan.cuh"
#include "tma.cuh"

namespace wj {

constexpr int kOsThreads = 256;
constexpr int kOsWarps = kOsThreads / 32;
constexpr int kOsItems = 16;
constexpr int kOsTile = kOsThreads * kOsItems;  // 4096

// Lanes holding the same 8-bit digit (a warp-wide multi-split with 8 ballots: cheaper than
// MATCH.ANY on sm_100a); `valid` lanes only.
#ifndef WJ_PEERS_ASM
#define WJ_PEERS_ASM 1
#endif
__device__ __forceinline__ uint32_t digit_peers(uint32_t d, bool valid) {
  uint32_t peers = __ballot_sync(0xffffffffu, valid);
#if WJ_PEERS_ASM
  // The integer ALU pipe issues one warp instruction every 2 cycles per SMSP (B300_MICROARCH.md
  // "fma vs alu split") and this loop is ~45% of the downsweep's instructions: one predicate test, the
  // ballot and one predicated LOP3 per bit (the C form compiles to shift, test, a second compare, ballot,
  // select and LOP3).
  uint32_t m[8];
#pragma unroll
  for (int b = 0; b < 8; ++b)  // m[b] = lanes whose bit b equals this lane's
    asm("{\n\t.reg .pred p;\n\t.reg .b32 t;\n\t"
        "and.b32 t, %1, %2;\n\t"
        "setp.ne.u32 p, t, 0;\n\t"
        "vote.sync.ballot.b32 %0, p, 0xffffffff;\n\t"
        "@!p not.b32 %0, %0;\n\t}"
        : "=r"(m[b])
        : "r"(d), "r"(1u << b));
  uint32_t a, b2, c;  // the AND of 9 masks as 4 three-input LOP3s (ptxas keeps 2-input ANDs otherwise)
  asm("lop3.b32 %0, %1, %2, %3, 0x80;" : "=r"(a) : "r"(peers), "r"(m[0]), "r"(m[1]));
  asm("lop3.b32 %0, %1, %2, %3, 0x80;" : "=r"(b2) : "r"(m[2]), "r"(m[3]), "r"(m[4]));
  asm("lop3.b32 %0, %1, %2, %3, 0x80;" : "=r"(c) : "r"(m[5]), "r"(m[6]), "r"(m[7]));
  asm("lop3.b32 %0, %1, %2, %3, 0x80;" : "=r"(peers) : "r"(a), "r"(b2), "r"(c));
#else
#pragma unroll
  for (int b = 0; b < 8; ++b) {
    const bool bit = (d >> b) & 1u;
    const uint32_t m = __ballot_sync(0xffffffffu, bit);
    peers &= bit ? m : ~m;
  }
#endif
  return peers;
}

// Same result through a per-warp table of 256 lane masks in shared memory (all zero on entry and
// on exit): one shared atomic OR per lane instead of 8 ballots.
__device__ __forceinline__ uint32_t digit_peers_smem(uint32_t* bins, uint32_t d, bool valid) {
  const uint32_t lane = lane_id();
  if (valid) atomicOr(&bins[d], 1u << lane);
  __syncwarp();
  const uint32_t peers = valid ? bins[d] : 0u;
  __syncwarp();
  if (valid && (peers & ((1u << lane) - 1u)) == 0) bins[d] = 0u;  // the lowest peer clears
  __syncwarp();
  return peers;
}

// ------------------------------------------------------------------ reduce-then-scan, TMA ring
// Pass = upsweep (per-CTA-range digit histogram) + scan of the 256 x G counts (digit-major) +
// downsweep: CTA c walks its contiguous range tile by tile with exact running digit offsets (no
// look-back), the next tile's keys/values streaming into the other half of a 2-stage smem ring by
// cp.async.bulk while the current tile is ranked, staged in digit order and written out.
constexpr int kRsCtas = 148 * 2;

// Digits come from (key & kmask) (the count bits of a stream element ride along unsorted); with skip0
// the elements whose bits above kmask are 0 are holes (not counted, dropped by the downsweep).  A map
// (slot -> rank) is applied in place to the masked part: key = map[key & kmask] | (key & ~kmask).
// HOLES / MASK are compile-time so the common path (no holes, digits below the count bits) is the
// plain branch-free kernel.
template <typename K, bool HOLES>
__device__ __forceinline__ bool rs_hole(K k, K kmask) { return HOLES && (k & ~kmask) == 0; }
template <typename K, bool MASK>
__device__ __forceinline__ K rs_dkey(K k, K kmask) { return MASK ? (k & kmask) : k; }

// kRsUpSplit CTAs share one downsweep range (each a contiguous quarter), adding their counts to the
// range's histogram column with global atomics (hist zeroed by the caller): 4x the warps in flight for
// the map gather of the first pass, which is L2-latency bound at 2 CTAs/SM.
constexpr int kRsUpSplit = 4;

// elements per CTA range for n elements over G ranges (a multiple of the 4096-element tile); the
// host uses the same cut (engine.cu sort_pairs)
__host__ __device__ __forceinline__ uint64_t rs_per(uint64_t n, uint64_t G) {
  const uint64_t per = (n + G - 1) / G;
  return (per + kOsTile - 1) / kOsTile * kOsTile;
}

template <typename K, bool HOLES, bool MASK>
__global__ void __launch_bounds__(256) k_rs_up(K* keys, uint64_t n, uint64_t per, int shift,
                                               const uint32_t* __restrict__ map, uint32_t* hist, K kmask,
                                               const uint32_t* __restrict__ n_dev) {
  if (n_dev) {  // elements left by an earlier hole-compacting pass: ranges re-cut for that count
    n = min(n, (uint64_t)*n_dev);
    per = rs_per(n, gridDim.x / kRsUpSplit);
  }
  __shared__ uint32_t h[kOsWarps][256];
  const int w = threadIdx.x >> 5;
  for (int x = 0; x < kOsWarps; ++x) h[x][threadIdx.x] = 0;
  __syncthreads();
  const uint32_t range = blockIdx.x / kRsUpSplit, part = blockIdx.x % kRsUpSplit;
  const uint32_t n_ranges = gridDim.x / kRsUpSplit;
  const uint64_t sub = per / kRsUpSplit;  // per is a multiple of the 4096-element tile
  const uint64_t rhi = (uint64_t)range * per + per < n ? (uint64_t)range * per + per : n;
  const uint64_t lo0 = (uint64_t)range * per + part * sub;  // 16-byte aligned
  const uint64_t lo = lo0 < rhi ? lo0 : rhi;
  const uint64_t hi = (part + 1 == kRsUpSplit) ? rhi : (lo0 + sub < rhi ? lo0 + sub : rhi);
  constexpr int V = 16 / sizeof(K);  // keys per 16-byte vector
  const uint64_t nvec = (hi - lo) / V;
  typedef typename std::conditional<sizeof(K) == 4, uint4, ulonglong2>::type Vec;
  Vec* vp = (Vec*)(keys + lo);
  constexpr int U = 4;  // vectors in flight per thread
  uint64_t v0 = threadIdx.x;
  for (; v0 + (U - 1) * 256 < nvec; v0 += U * 256) {
    Vec x[U];
#pragma unroll
    for (int u = 0; u < U; ++u) x[u] = vp[v0 + u * 256];
    // all U * V map gathers are issued before any histogram update (the gathers are L2-latency
    // bound; interleaving them with shared atomics serialised them)
    if (map) {
#pragma unroll
      for (int u = 0; u < U; ++u) {
        K* kk = (K*)&x[u];
#pragma unroll
        for (int j = 0; j < V; ++j)
          if (!rs_hole<K, HOLES>(kk[j], kmask)) kk[j] = (K)__ldg(&map[(uint32_t)(kk[j] & kmask)]) | (kk[j] & ~kmask);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      K* kk = (K*)&x[u];
#pragma unroll
      for (int j = 0; j < V; ++j) {
        // a mapped hole stays a hole: map values keep the bits above kmask of a non-hole
        const bool hole = rs_hole<K, HOLES>(kk[j], kmask);
        if (!hole) atomicAdd(&h[w][(uint32_t)(rs_dkey<K, MASK>(kk[j], kmask) >> shift) & 255u], 1u);
      }
      if (map) vp[v0 + u * 256] = x[u];
    }
  }
  for (uint64_t v = v0; v < nvec; v += 256) {
    Vec x = vp[v];
    K* kk = (K*)&x;
#pragma unroll
    for (int j = 0; j < V; ++j) {
      const bool hole = rs_hole<K, HOLES>(kk[j], kmask);
      if (map && !hole) kk[j] = (K)__ldg(&map[(uint32_t)(kk[j] & kmask)]) | (kk[j] & ~kmask);
      if (!hole) atomicAdd(&h[w][(uint32_t)(rs_dkey<K, MASK>(kk[j], kmask) >> shift) & 255u], 1u);
    }
    if (map) vp[v] = x;
  }
  for (uint64_t i = lo + nvec * V + threadIdx.x; i < hi; i += 256) {
    K k = keys[i];
    if (rs_hole<K, HOLES>(k, kmask)) continue;
    if (map) {
      k = (K)__ldg(&map[(uint32_t)(k & kmask)]) | (k & ~kmask);
      keys[i] = k;
    }
    atomicAdd(&h[w][(uint32_t)(rs_dkey<K, MASK>(k, kmask) >> shift) & 255u], 1u);
  }
  __syncthreads();
  uint32_t t = 0;
#pragma unroll
  for (int x = 0; x < kOsWarps; ++x) t += h[x][threadIdx.x];
  if (t) atomicAdd(&hist[(uint64_t)threadIdx.x * n_ranges + range], t);
}

// Upsweep over a digit byte array (the packed stream's passes: the emit kernel / the previous downsweep
// wrote each element's digit of this pass as one byte at the element's position): reads 1 B per element
// instead of the 8-byte element.  Same ranges and histogram layout as k_rs_up.
__global__ void __launch_bounds__(256) k_rs_up_bytes(const uint8_t* __restrict__ dig, uint64_t n, uint64_t per,
                                                     uint32_t* hist) {
  __shared__ uint32_t h[kOsWarps][256];
  const int w = threadIdx.x >> 5;
  for (int x = 0; x < kOsWarps; ++x) h[x][threadIdx.x] = 0;
  __syncthreads();
  const uint32_t range = blockIdx.x / kRsUpSplit, part = blockIdx.x % kRsUpSplit;
  const uint32_t n_ranges = gridDim.x / kRsUpSplit;
  const uint64_t sub = per / kRsUpSplit;  // a multiple of 1024: 16-byte aligned parts
  const uint64_t rhi = (uint64_t)range * per + per < n ? (uint64_t)range * per + per : n;
  const uint64_t lo0 = (uint64_t)range * per + part * sub;
  const uint64_t lo = lo0 < rhi ? lo0 : rhi;
  const uint64_t hi = (part + 1 == kRsUpSplit) ? rhi : (lo0 + sub < rhi ? lo0 + sub : rhi);
  const uint64_t nvec = (hi - lo) / 16;
  const uint4* vp = (const uint4*)(dig + lo);
  for (uint64_t v = threadIdx.x; v < nvec; v += 256) {
    const uint4 x = __ldcs(vp + v);
    const uint32_t wd[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
    for (int q = 0; q < 4; ++q)
#pragma unroll
      for (int b = 0; b < 4; ++b) atomicAdd(&h[w][(wd[q] >> (8 * b)) & 255u], 1u);
  }
  for (uint64_t i = lo + nvec * 16 + threadIdx.x; i < hi; i += 256) atomicAdd(&h[w][dig[i]], 1u);
  __syncthreads();
  uint32_t t = 0;
#pragma unroll
  for (int x = 0; x < kOsWarps; ++x) t += h[x][threadIdx.x];
  if (t) atomicAdd(&hist[(uint64_t)threadIdx.x * n_ranges + range], t);
}

// Downsweep v2: 512 threads x 8 items (tile 4096); the tile is never copied inside shared memory:
// ranks produce an inverse permutation (u16) and the write-out gathers keys/values from the TMA
// stage through it, so keys/values need no registers across barriers (occupancy: 32 warps/SM).
constexpr int kDsThreads = 512;
constexpr int kDsWarps = kDsThreads / 32;
constexpr int kDsItems = 8;
static_assert(kDsThreads * kDsItems == kOsTile, "tile");

template <typename K, bool NOVAL = false>
inline size_t ds_smem_bytes() { return 2 * (size_t)kOsTile * (sizeof(K) + (NOVAL ? 0 : sizeof(uint32_t))) + kOsTile * 2; }

// NOVAL: keys only (the packed stream: u64 slot << 32 | docID, digits from the slot bits), one TMA load,
// one shared-memory gather and one 8-byte store per element instead of two of each
// HEADS (the last pass over a packed stream, NOVAL): also counts run-length heads -- elements whose
// (slot, docID) differs from the previous one in the final order -- per run-length range of rper elements
// into rcnt (zeroed by the caller), which replaces the run-length count pass.  The predecessor is the
// previous lane's element (a shuffle), the previous warp's last one, or the digit's last element of an
// earlier tile (carry); a block's first element is counted as a head and k_head_fix corrects it.
template <typename K, bool HOLES, bool MASK, bool NOVAL = false, bool HEADS = false>
// 64 registers (__launch_bounds__(512, 2)): with the lazy B-tree re-layout the dictionary stream
// no longer needs room beside the persistent downsweep; the earlier 48-register cap
// (WJ_DS_MAXREG=48) is 2.93 -> 3.09 ms for the three passes, step 8.98 vs 9.00-9.02 ms (A/B x2)
#ifndef WJ_DS_MAXREG
#define WJ_DS_MAXREG 0
#endif
#if WJ_DS_MAXREG > 0
#define WJ_DS_BOUNDS __maxnreg__(WJ_DS_MAXREG)
#else
#define WJ_DS_BOUNDS __launch_bounds__(kDsThreads, 2)
#endif
__global__ void WJ_DS_BOUNDS k_rs_down2(const K* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                         K* __restrict__ kout, uint32_t* __restrict__ vout, uint64_t n,
                                                         uint64_t per, int shift, const uint32_t* __restrict__ offs,
                                                         K kmask, const uint32_t* __restrict__ n_dev,
                                                         uint32_t* __restrict__ rcnt = nullptr, uint32_t rper = 0,
                                                         uint8_t* __restrict__ dnext = nullptr) {
  if (n_dev) {
    n = min(n, (uint64_t)*n_dev);
    per = rs_per(n, gridDim.x);
  }
  extern __shared__ __align__(128) unsigned char os_smem[];
  __shared__ __align__(8) uint64_t bar[2];
  __shared__ uint32_t wcnt[kDsWarps][256];
  constexpr bool kSmemPeers = sizeof(K) == 8 && !NOVAL;  // 64-bit (all distinct) keys: shared-memory masks
  __shared__ uint32_t wbins[kSmemPeers ? kDsWarps : 1][256];
  __shared__ uint32_t dig_off[256];
  __shared__ uint32_t dig_glob[256];
  __shared__ uint32_t run_base[256];
  __shared__ uint32_t wtot[8];
  __shared__ uint32_t s_tvalid;
  __shared__ __align__(8) K carry[HEADS ? 2 : 1][HEADS ? 256 : 1];  // per digit: last element of an earlier tile
  const uint32_t rmagic = HEADS ? (uint32_t)(0xFFFFFFFFull / rper + 1) : 0u;  // q = umulhi(pos, m), -1 fix
  uint32_t tile_par = 0;
  const size_t stage_bytes = (size_t)kOsTile * (sizeof(K) + (NOVAL ? 0 : sizeof(uint32_t)));
  auto skey = [&](int s) { return (K*)(os_smem + s * stage_bytes); };
  auto sval = [&](int s) { return (uint32_t*)(os_smem + s * stage_bytes + (size_t)kOsTile * sizeof(K)); };
  uint16_t* inv = (uint16_t*)(os_smem + 2 * stage_bytes);
  const uint32_t lane = lane_id();
  const int w = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  const uint64_t lo = (uint64_t)blockIdx.x * per;
  const uint64_t hi = lo + per < n ? lo + per : n;
  if (lo >= hi) return;

  auto issue = [&](int s, uint64_t base) {  // thread 0
    const uint32_t cnt = (uint32_t)((hi - base) < (uint64_t)kOsTile ? (hi - base) : (uint64_t)kOsTile);
    const uint32_t bk = (uint32_t)((cnt * sizeof(K) + 15) & ~(size_t)15);
    const uint32_t bv = (cnt * 4 + 15) & ~15u;
    fence_proxy_async_smem();
    mbar_arrive_expect_tx(&bar[s], bk + (NOVAL ? 0u : bv));
    tma_load_1d(skey(s), kin + base, bk, &bar[s]);
    if (!NOVAL) tma_load_1d(sval(s), vin + base, bv, &bar[s]);
  };

  if (threadIdx.x == 0) {
    mbar_init(&bar[0], 1);
    mbar_init(&bar[1], 1);
    fence_mbar_init();
  }
  for (int i = threadIdx.x; i < kDsWarps * 256; i += kDsThreads) {
    (&wcnt[0][0])[i] = 0;
    if (kSmemPeers) (&wbins[0][0])[i] = 0;
  }
  if (threadIdx.x < 256) run_base[threadIdx.x] = offs[(uint64_t)threadIdx.x * gridDim.x + blockIdx.x];
  if (HEADS && threadIdx.x < 256) carry[0][threadIdx.x] = carry[HEADS ? 1 : 0][threadIdx.x] = ~K(0);  // none
  __syncthreads();
  if (threadIdx.x == 0) issue(0, lo);
  uint32_t parity = 0u;
  int s = 0;
  for (uint64_t base = lo; base < hi; base += kOsTile) {
    if (threadIdx.x == 0 && base + kOsTile < hi) issue(s ^ 1, base + kOsTile);
    mbar_wait(&bar[s], (parity >> s) & 1u);
    parity ^= 1u << s;
    const uint32_t tn = (uint32_t)((hi - base) < (uint64_t)kOsTile ? (hi - base) : (uint64_t)kOsTile);
    const K* sk = skey(s);
    const uint32_t* sv = sval(s);
    uint32_t dg[kDsItems], rank[kDsItems];
    uint32_t vmask = 0;  // valid items of this thread (in range, not a hole)
#pragma unroll
    for (int k = 0; k < kDsItems; ++k) {
      const uint32_t li = w * (32 * kDsItems) + k * 32 + lane;
      const K kv = sk[li];
      const bool valid = li < tn && !rs_hole<K, HOLES>(kv, kmask);
      vmask |= (valid ? 1u : 0u) << k;
      dg[k] = (uint32_t)((rs_dkey<K, MASK>(kv, kmask) >> shift) & 255u);
      // 64-bit keys (all distinct: new-term sort): shared-memory masks; 32-bit keys (Zipf-skewed
      // ranks, many equal digits per warp -> atomic conflicts): ballots
      // (shared-memory masks for the 32-bit stream keys too: 3.31 vs 3.09 ms for the three passes)
      rank[k] = kSmemPeers ? digit_peers_smem(wbins[kSmemPeers ? w : 0], dg[k], valid) : digit_peers(dg[k], valid);
    }
#pragma unroll
    for (int k = 0; k < kDsItems; ++k) {
      const bool valid = (vmask >> k) & 1u;
      const uint32_t peers = rank[k];
      const int leader = valid ? __ffs(peers) - 1 : (int)lane;
      uint32_t old = 0;
      if (valid && (int)lane == leader) {
        old = wcnt[w][dg[k]];
        wcnt[w][dg[k]] = old + __popc(peers);
      }
      old = __shfl_sync(0xffffffffu, old, leader);
      rank[k] = old + __popc(peers & lt);
      __syncwarp();
    }
    __syncthreads();
    // per digit (threads 0..255): offsets across warps, tile count, tile-exclusive digit offset
    uint32_t cnt = 0, inc = 0;
    if (threadIdx.x < 256) {
      const uint32_t d = threadIdx.x;
#pragma unroll
      for (int x = 0; x < kDsWarps; ++x) {
        const uint32_t t = wcnt[x][d];
        wcnt[x][d] = cnt;
        cnt += t;
      }
      inc = warp_inclusive_sum<uint32_t>(cnt);
      if (lane == 31) wtot[w] = inc;
    }
    __syncthreads();
    if (threadIdx.x < 256) {
      const uint32_t d = threadIdx.x;
      uint32_t wp = 0;
      for (int x = 0; x < w; ++x) wp += wtot[x];
      const uint32_t toff = wp + inc - cnt;
      dig_off[d] = toff;
      const uint32_t rb = run_base[d];
      dig_glob[d] = rb - toff;
      run_base[d] = rb + cnt;
      if (d == 255) s_tvalid = toff + cnt;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kDsItems; ++k) {
      const uint32_t li = w * (32 * kDsItems) + k * 32 + lane;
      if ((vmask >> k) & 1u) inv[dig_off[dg[k]] + wcnt[w][dg[k]] + rank[k]] = (uint16_t)li;
    }
    __syncthreads();
    const uint32_t tvalid = HOLES ? s_tvalid : tn;  // valid (non-hole) items of the tile
    if (HEADS) {
      const K* cprev = carry[(tile_par ^ 1) & (HEADS ? 1u : 0u)];
      for (uint32_t j0 = 0; j0 < kOsTile; j0 += kDsThreads) {
        const uint32_t j = j0 + threadIdx.x;
        const bool valid = j < tvalid;
        const K kk = valid ? sk[inv[j]] : ~K(0);
        const uint32_t d = (uint32_t)(kk >> shift) & 255u;
        const uint32_t pos = dig_glob[d] + j;
        if (valid) kout[pos] = kk;
        K pk = (K)__shfl_up_sync(0xffffffffu, (unsigned long long)kk, 1);
        if (lane == 0) pk = (valid && j > 0) ? sk[inv[j - 1]] : ~K(0);  // (inv past tvalid is stale)
        // the previous element of the final order: in this tile's run of digit d, else the carry
        const K pred = (j > 0 && ((uint32_t)(pk >> shift) & 255u) == d) ? pk : cprev[d];
        const bool head = valid && pred != kk;
        uint32_t q = valid ? __umulhi(pos, rmagic) : 0xFFFFFFFFu;
        if (valid && (uint64_t)q * rper > pos) --q;
        const uint32_t qp = __shfl_up_sync(0xffffffffu, q, 1);
        const bool leader = valid && (lane == 0 || qp != q);
        const uint32_t lm = __ballot_sync(0xffffffffu, leader), hm = __ballot_sync(0xffffffffu, head);
        if (leader) {
          const uint32_t later = lm & ~((2u << lane) - 1u);
          const uint32_t seg = (later ? (1u << (__ffs(later) - 1)) - 1u : 0xFFFFFFFFu) & ~((1u << lane) - 1u);
          const uint32_t hc = __popc(hm & seg);
          if (hc) atomicAdd(&rcnt[q], hc);
        }
      }
    } else {
      for (uint32_t j = threadIdx.x; j < tvalid; j += kDsThreads) {
        const uint32_t li = inv[j];
        const K kk = sk[li];
        const uint32_t pos = dig_glob[(uint32_t)((rs_dkey<K, MASK>(kk, kmask) >> shift) & 255u)] + j;
        kout[pos] = kk;
        if (!NOVAL) vout[pos] = sv[li];
        if (NOVAL && dnext) dnext[pos] = (uint8_t)(kk >> (shift + 8));  // the next pass's digit
      }
    }
    if (HEADS && threadIdx.x < 256) {  // this tile's last element of each digit (or the earlier carry)
      K* cur = carry[tile_par & (HEADS ? 1u : 0u)];
      const K* prv = carry[(tile_par ^ 1) & (HEADS ? 1u : 0u)];
      cur[threadIdx.x] = cnt ? sk[inv[dig_off[threadIdx.x] + cnt - 1]] : prv[threadIdx.x];
    }
    tile_par ^= 1u;
    for (int i = threadIdx.x; i < kDsWarps * 256; i += kDsThreads) (&wcnt[0][0])[i] = 0;
    __syncthreads();
    s ^= 1;
  }
}

// HEADS correction: a non-empty block (d, c) of the last pass starts at offs[d][c]; its first element was
// counted as a head without seeing its predecessor out[pos - 1]
template <typename K>
__global__ void k_head_fix(const K* __restrict__ out, const uint32_t* __restrict__ offs, uint32_t blocks,
                           uint32_t* rcnt, uint32_t rper) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= blocks) return;
  const uint32_t p = offs[i];
  if (offs[i + 1] == p || p == 0) return;
  if (out[p - 1] == out[p]) atomicSub(&rcnt[p / rper], 1u);
}

}  // namespace wj
