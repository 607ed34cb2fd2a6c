// wjgen — deterministic synthetic corpus generator (shared test/bench input module).
//
// This module is shared by the CPU oracle tests and the CUDA path tests/bench.  It holds
// NONE of the indexing method's arithmetic (no tokenisation, no trie bucket, no dictionary):
// it only emits document bytes and document offsets.  Recipe (DESIGN.md "Input recipe",
// SURVEY.md §8(d)):
//   * RNG: splitmix64 for seeding, xoshiro256** for streams; every document has its own seed
//     splitmix(seed, chunk, doc) so any thread can generate any document.
//   * Vocabulary ranks 1..V: length clamp(floor(3.8 + 0.45 ln r) + J, 2, 24), J in {-1,0,1};
//     letters i.i.d. from English unigram frequencies; 3% pure numbers (1-6 digits), 1%
//     digit-led alphanumerics, 0.5% containing one 2-byte UTF-8 Latin letter; duplicates are
//     regenerated.  Token-weighted mean length ~6.6.
//   * Zipf(s=1) over ranks with integer weights floor(2^40 / r), sampled by mulhi + search of
//     u64 prefix sums (bit-reproducible).
//   * Surface text: first letter upper-case 8%, whole token upper-case 0.5%; separators
//     " " 90%, ", " 4%, ". " 4%, "\n" 2%; 0.1% of documents start with one 300-letter token
//     (dropped by the >255-byte rule); optional hapax fraction of fresh random
//     6-14-letter strings (Library-of-Congress-shaped config, high new-term insert rate).
//   * Document lengths: uniform [lo,hi] or lognormal(mean, sigma) clamped to [lo,hi] bytes.
// Build: g++ -O2 -ffp-contract=off -fPIC -shared -pthread (the same binary on every box).
#include <cmath>
#include <cstdint>
#include <cstring>
#include <string>
#include <thread>
#include <unordered_set>
#include <vector>
#include <algorithm>
#include <atomic>

namespace {

inline uint64_t splitmix64(uint64_t& x) {
  uint64_t z = (x += 0x9E3779B97F4A7C15ull);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
inline uint64_t mix3(uint64_t a, uint64_t b, uint64_t c) {
  uint64_t x = a;
  uint64_t h = splitmix64(x);
  x = h ^ (b * 0xD6E8FEB86659FD93ull);
  h = splitmix64(x);
  x = h ^ (c * 0xA0761D6478BD642Full);
  return splitmix64(x);
}

struct Xoshiro {
  uint64_t s[4];
  explicit Xoshiro(uint64_t seed) {
    uint64_t x = seed;
    for (auto& v : s) v = splitmix64(x);
  }
  static inline uint64_t rotl(uint64_t x, int k) { return (x << k) | (x >> (64 - k)); }
  inline uint64_t next() {
    const uint64_t result = rotl(s[1] * 5, 7) * 9;
    const uint64_t t = s[1] << 17;
    s[2] ^= s[0]; s[3] ^= s[1]; s[1] ^= s[2]; s[0] ^= s[3];
    s[2] ^= t; s[3] = rotl(s[3], 45);
    return result;
  }
  // uniform in [0, n)
  inline uint64_t below(uint64_t n) { return (uint64_t)(((unsigned __int128)next() * n) >> 64); }
  // uniform double in [0,1)
  inline double unif() { return (double)(next() >> 11) * (1.0 / 9007199254740992.0); }
  // per-mille Bernoulli
  inline bool permille(uint32_t p) { return below(1000) < p; }
  inline bool per100k(uint32_t p) { return below(100000) < p; }
};

// English unigram letter frequencies (per 10,000), a..z.
const uint32_t kLetterW[26] = {817, 149, 278, 425, 1270, 223, 202, 609, 697, 15, 77, 403, 241,
                               675, 751, 193, 10,  599, 633, 906, 276, 98,  236, 15,  197, 7};

struct LetterTable {
  uint32_t cum[26];
  uint32_t total;
  LetterTable() {
    uint32_t c = 0;
    for (int i = 0; i < 26; ++i) { c += kLetterW[i]; cum[i] = c; }
    total = c;
  }
  inline char draw(Xoshiro& r) const {
    uint32_t u = (uint32_t)r.below(total);
    int i = 0;
    while (cum[i] <= u) ++i;
    return (char)('a' + i);
  }
};
const LetterTable kLetters;

// Two-byte UTF-8 Latin letters: é ñ ö ü ç à è á í ó
const uint8_t kUtf8[10][2] = {{0xC3, 0xA9}, {0xC3, 0xB1}, {0xC3, 0xB6}, {0xC3, 0xBC}, {0xC3, 0xA7},
                              {0xC3, 0xA0}, {0xC3, 0xA8}, {0xC3, 0xA1}, {0xC3, 0xAD}, {0xC3, 0xB3}};

std::string make_term(uint64_t seed, uint64_t rank, uint32_t attempt) {
  Xoshiro r(mix3(seed ^ 0x5EED0F7E4Dull, rank, attempt));
  uint32_t kind = (uint32_t)r.below(1000);  // 30 numbers, 10 digit-led, 5 utf8, rest words
  std::string s;
  if (kind < 30) {
    int n = 1 + (int)r.below(6);
    for (int i = 0; i < n; ++i) s.push_back((char)('0' + r.below(10)));
    return s;
  }
  double lr = std::log((double)rank);
  int L = (int)std::floor(3.8 + 0.45 * lr) + (int)r.below(3) - 1;
  if (L < 2) L = 2;
  if (L > 24) L = 24;
  if (kind < 40) {
    s.push_back((char)('0' + r.below(10)));
    for (int i = 1; i < L; ++i) {
      if (r.below(4) == 0) s.push_back((char)('0' + r.below(10)));
      else s.push_back(kLetters.draw(r));
    }
    // guarantee a letter so it is not a pure number
    bool has_letter = false;
    for (char c : s) has_letter |= (c >= 'a' && c <= 'z');
    if (!has_letter) s.push_back(kLetters.draw(r));
    return s;
  }
  for (int i = 0; i < L; ++i) s.push_back(kLetters.draw(r));
  if (kind < 45) {
    int pos = (int)r.below((uint64_t)L + 1);
    const uint8_t* u = kUtf8[r.below(10)];
    s.insert(s.begin() + pos, (char)u[1]);
    s.insert(s.begin() + pos, (char)u[0]);
  }
  return s;
}

struct Vocab {
  std::vector<uint32_t> off;   // V+1
  std::vector<char> bytes;
  std::vector<uint64_t> cum;   // Zipf prefix sums, V
  std::vector<uint32_t> guide; // 65537 entries
  uint64_t total = 0;
  uint32_t V = 0;

  void build(uint64_t seed, uint32_t v, int threads) {
    V = v;
    std::vector<std::string> cand(V);
    auto work = [&](uint32_t lo, uint32_t hi) {
      for (uint32_t i = lo; i < hi; ++i) cand[i] = make_term(seed, (uint64_t)i + 1, 0);
    };
    std::vector<std::thread> th;
    uint32_t step = (V + threads - 1) / threads;
    for (int t = 0; t < threads; ++t) {
      uint32_t lo = std::min<uint32_t>(V, t * step), hi = std::min<uint32_t>(V, lo + step);
      th.emplace_back(work, lo, hi);
    }
    for (auto& t : th) t.join();
    std::unordered_set<std::string> seen;
    seen.reserve((size_t)V * 2);
    for (uint32_t i = 0; i < V; ++i) {
      uint32_t attempt = 0;
      while (!seen.insert(cand[i]).second) cand[i] = make_term(seed, (uint64_t)i + 1, ++attempt);
    }
    off.resize((size_t)V + 1);
    size_t tot = 0;
    for (uint32_t i = 0; i < V; ++i) { off[i] = (uint32_t)tot; tot += cand[i].size(); }
    off[V] = (uint32_t)tot;
    bytes.resize(tot);
    for (uint32_t i = 0; i < V; ++i) memcpy(bytes.data() + off[i], cand[i].data(), cand[i].size());
    cum.resize(V);
    uint64_t c = 0;
    for (uint32_t i = 0; i < V; ++i) { c += (1ull << 40) / ((uint64_t)i + 1); cum[i] = c; }
    total = c;
    guide.resize(65537);
    uint32_t r = 0;
    for (uint32_t k = 0; k <= 65536; ++k) {
      uint64_t thr = (uint64_t)(((unsigned __int128)total * k) >> 16);
      while (r < V - 1 && cum[r] <= thr) ++r;
      guide[k] = r;
    }
  }
  // smallest r with cum[r] > u
  inline uint32_t sample(Xoshiro& rng) const {
    uint64_t u = (uint64_t)(((unsigned __int128)rng.next() * total) >> 64);
    uint32_t k = (uint32_t)(((unsigned __int128)u << 16) / total);
    uint32_t lo = guide[k], hi = guide[std::min<uint32_t>(k + 1, 65536)];
    if (lo > 0) --lo;
    while (lo < hi) {
      uint32_t mid = (lo + hi) >> 1;
      if (cum[mid] > u) hi = mid; else lo = mid + 1;
    }
    return lo;
  }
};

}  // namespace

extern "C" {

typedef struct {
  uint64_t seed;
  uint64_t chunk;         // chunk index (part of each document's seed)
  uint64_t n_docs;        // if > 0: exactly this many documents
  uint64_t target_bytes;  // if n_docs == 0: documents until this many bytes (last one clipped)
  uint32_t len_dist;      // 0 = uniform [len_lo, len_hi]; 1 = lognormal(len_mean, len_sigma) clamped
  uint32_t vocab;         // V
  double len_mean, len_sigma;
  uint64_t len_lo, len_hi;
  uint32_t hapax_per100k; // fresh random terms per 100k tokens
  uint32_t long_permille; // documents (per mille) that start with one 300-letter token
  uint32_t threads;
  uint32_t reserved;
} wjgen_params;

// Computes document lengths (and therefore n_docs and n_bytes) without generating text.
// doc_off may be NULL (sizing call).  Returns 0 on success, -1 if doc_cap too small.
int wjgen_layout(const wjgen_params* p, uint64_t* doc_off, uint64_t doc_cap, uint64_t* n_docs,
                 uint64_t* n_bytes) {
  Xoshiro r(mix3(p->seed ^ 0xD0C1E7ull, p->chunk, 0x1A40u));
  uint64_t total = 0, d = 0;
  const double mu = std::log(p->len_mean > 1 ? p->len_mean : 1.0) - 0.5 * p->len_sigma * p->len_sigma;
  for (;;) {
    if (p->n_docs > 0 && d >= p->n_docs) break;
    if (p->n_docs == 0 && total >= p->target_bytes) break;
    uint64_t len;
    if (p->len_dist == 0) {
      len = p->len_lo + r.below(p->len_hi - p->len_lo + 1);
    } else {
      double u1 = r.unif(), u2 = r.unif();
      if (u1 < 1e-300) u1 = 1e-300;
      double z = std::sqrt(-2.0 * std::log(u1)) * std::cos(6.283185307179586 * u2);
      double x = std::exp(mu + p->len_sigma * z);
      if (x < (double)p->len_lo) x = (double)p->len_lo;
      if (x > (double)p->len_hi) x = (double)p->len_hi;
      len = (uint64_t)x;
    }
    if (p->n_docs == 0 && total + len > p->target_bytes) len = p->target_bytes - total;
    if (doc_off) {
      if (d + 1 >= doc_cap) return -1;
      doc_off[d] = total;
    }
    total += len;
    ++d;
  }
  if (doc_off) {
    if (d >= doc_cap) return -1;
    doc_off[d] = total;
  }
  *n_docs = d;
  *n_bytes = total;
  return 0;
}

// Generates text for documents laid out by wjgen_layout (doc_off must hold n_docs+1 entries).
int wjgen_fill(const wjgen_params* p, const uint64_t* doc_off, uint64_t n_docs, uint8_t* text) {
  static const char* kSep[4] = {" ", ", ", ". ", "\n"};
  Vocab voc;
  int threads = p->threads ? (int)p->threads : (int)std::max(1u, std::thread::hardware_concurrency());
  voc.build(p->seed, p->vocab ? p->vocab : 1000, threads);
  auto gen_doc = [&](uint64_t d) {
    Xoshiro r(mix3(p->seed, p->chunk, d + 1));
    uint8_t* out = text + doc_off[d];
    const uint64_t len = doc_off[d + 1] - doc_off[d];
    uint64_t pos = 0;
    auto put = [&](const char* s, size_t n) {
      for (size_t i = 0; i < n && pos < len; ++i) out[pos++] = (uint8_t)s[i];
    };
    if (p->long_permille && r.permille(p->long_permille)) {
      char buf[300];
      for (int i = 0; i < 300; ++i) buf[i] = kLetters.draw(r);
      put(buf, 300);
      put(" ", 1);
    }
    char tb[64];
    while (pos < len) {
      const char* src;
      size_t n;
      if (p->hapax_per100k && r.per100k(p->hapax_per100k)) {
        n = 6 + (size_t)r.below(9);
        for (size_t i = 0; i < n; ++i) tb[i] = kLetters.draw(r);
        src = tb;
      } else {
        uint32_t k = voc.sample(r);
        n = voc.off[k + 1] - voc.off[k];
        memcpy(tb, voc.bytes.data() + voc.off[k], n);
        src = tb;
        uint32_t c = (uint32_t)r.below(1000);
        if (c < 5) {
          for (size_t i = 0; i < n; ++i) if (tb[i] >= 'a' && tb[i] <= 'z') tb[i] -= 32;
        } else if (c < 85) {
          if (tb[0] >= 'a' && tb[0] <= 'z') tb[0] -= 32;
        }
      }
      put(src, n);
      uint32_t s = (uint32_t)r.below(100);
      const char* sep = s < 90 ? kSep[0] : s < 94 ? kSep[1] : s < 98 ? kSep[2] : kSep[3];
      put(sep, strlen(sep));
    }
  };
  std::vector<std::thread> th;
  const uint64_t grain = 64;
  std::atomic_uint64_t next{0};
  for (int t = 0; t < threads; ++t) {
    th.emplace_back([&]() {
      for (;;) {
        uint64_t lo = next.fetch_add(grain);
        if (lo >= n_docs) break;
        uint64_t hi = std::min(n_docs, lo + grain);
        for (uint64_t d = lo; d < hi; ++d) gen_doc(d);
      }
    });
  }
  for (auto& t : th) t.join();
  return 0;
}

// Closed-form corpus (SURVEY.md §8(c) "Closed form"): term j = base26 5-letter string of
// (j*7919 + 12345) mod 26^5; document d holds term j exactly 1 + ((d+j) mod 3) times when
// d mod (j+1) == 0, space separated, terms in increasing j.  Two-call sizing: text may be NULL.
int wjgen_closed_form(uint64_t n_docs, uint32_t n_terms, uint8_t* text, uint64_t* doc_off,
                      uint64_t* n_bytes) {
  uint64_t pos = 0;
  for (uint64_t d = 0; d < n_docs; ++d) {
    if (doc_off) doc_off[d] = pos;
    for (uint32_t j = 0; j < n_terms; ++j) {
      if (d % ((uint64_t)j + 1) != 0) continue;
      uint32_t reps = 1 + (uint32_t)((d + j) % 3);
      uint32_t code = (uint32_t)(((uint64_t)j * 7919u + 12345u) % 11881376u);
      char w[5];
      for (int k = 4; k >= 0; --k) { w[k] = (char)('a' + code % 26); code /= 26; }
      for (uint32_t t = 0; t < reps; ++t) {
        if (text) { memcpy(text + pos, w, 5); text[pos + 5] = ' '; }
        pos += 6;
      }
    }
  }
  if (doc_off) doc_off[n_docs] = pos;
  *n_bytes = pos;
  return 0;
}

}  // extern "C"
