// tracegen — seeded synthetic CUDAAdvisor-style traces.
//
// INPUT GENERATOR ONLY.  This module emits trace records the way the paper's
// instrumentation would (Record() per active lane of a memory instruction,
// passBasicBlock() per active lane entering a basic block: PAPER.md L235-237,
// L322, L345).  It holds none of the analysis arithmetic (no cache lines, no
// reuse distances, no divergence counting) and is shared by the oracle side
// and the CUDA side of the tests and of bench.py.
//
// Record layout (SoA, one element per record):
//   addr  u64  effective byte address (0 for basic-block records)
//   cta   u32  linearised CTA id, unique across the launches of one trace
//   tid   u16  linearised thread id inside the CTA
//   site  u32  static instruction id (memory op) or basic-block id
//   winst u32  per-(cta, warp32, family) dynamic warp-instruction counter;
//              family = memory (load/store) or basic block
//   meta  u8   kind (0 load, 1 store, 2 BB) | log2(access bytes) << 2
//
// Virtual scheduler: 15 SMs (K40c-like), <= 16 CTAs and
// <= 64 warps per SM; CTAs are dispatched in order; every step each resident
// warp issues one warp-instruction; the active lanes of one warp-instruction
// are emitted contiguously in ascending lane order.  Launches are independent
// (each starts on an empty machine) so they are generated in parallel.
#include <algorithm>
#include <atomic>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <map>
#include <memory>
#include <stdexcept>
#include <string>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {

constexpr uint8_t K_LOAD = 0, K_STORE = 1, K_BB = 2;
constexpr uint64_t VA_BASE = 0x7f0000000000ull;

inline uint64_t splitmix64(uint64_t x) {
  x += 0x9e3779b97f4a7c15ull;
  x = (x ^ (x >> 30)) * 0xbf58476d1ce4e5b9ull;
  x = (x ^ (x >> 27)) * 0x94d049bb133111ebull;
  return x ^ (x >> 31);
}

struct Rng {
  uint64_t s;
  explicit Rng(uint64_t seed) : s(splitmix64(seed ^ 0x5851f42d4c957f2dull)) {}
  uint64_t next() { s += 0x9e3779b97f4a7c15ull; return splitmix64(s); }
  uint32_t below(uint32_t n) { return (uint32_t)(next() % n); }
  double uni() { return (next() >> 11) * (1.0 / 9007199254740992.0); }
};

inline uint8_t log2b(uint32_t bytes) {
  uint8_t l = 0;
  while ((1u << l) < bytes) ++l;
  return l;
}
inline uint8_t mk_meta(uint8_t kind, uint32_t bytes) { return (uint8_t)(kind | (log2b(bytes) << 2)); }

// One warp-level instruction: a memory op or a basic-block entry.
struct WInstr {
  uint8_t meta;
  uint32_t site;
  uint32_t mask;
  uint64_t addr[32];
};
using WarpProg = std::vector<WInstr>;

struct Prog {
  WarpProg* p;
  void bb(uint32_t site, uint32_t mask) {
    if (!mask) return;
    WInstr w; w.meta = K_BB; w.site = site; w.mask = mask;
    std::memset(w.addr, 0, sizeof(w.addr));
    p->push_back(w);
  }
  // f(lane) -> address for active lanes
  template <class F> void mem(uint8_t kind, uint32_t bytes, uint32_t site, uint32_t mask, F f) {
    if (!mask) return;
    WInstr w; w.meta = mk_meta(kind, bytes); w.site = site; w.mask = mask;
    for (int l = 0; l < 32; ++l) w.addr[l] = (mask >> l & 1u) ? (uint64_t)f(l) : 0;
    p->push_back(w);
  }
};

struct Launch {
  uint32_t ncta = 0, nthreads = 0;
  uint32_t cta_base = 0;
  std::function<void(uint32_t cta, uint32_t warp, Prog&)> gen;
  uint64_t count = 0, offset = 0;
};

// Bump allocator of the synthetic kernel's arrays; every allocation is
// recorded as a data object [base, base + bytes) (the allocation map the
// paper's data-centric profiler builds from the malloc family).
struct Alloc {
  uint64_t next = VA_BASE;
  std::vector<std::pair<uint64_t, uint64_t>>* objs = nullptr;
  explicit Alloc(std::vector<std::pair<uint64_t, uint64_t>>* o = nullptr) : objs(o) {}
  uint64_t get(uint64_t bytes) {
    uint64_t a = next;
    if (objs) objs->push_back({a, bytes});
    next += (bytes + 4095) & ~4095ull;
    next += 4096;  // guard page between arrays
    return a;
  }
};

struct Sink {
  uint64_t *addr; uint32_t *cta; uint16_t *tid; uint32_t *site; uint32_t *winst; uint8_t *meta;
  uint64_t lo, hi;  // global positions written: [lo, hi)
};

struct Trace {
  std::string name, info;
  std::vector<Launch> launches;
  uint32_t nsites = 0;
  uint32_t nctas = 0;
  uint64_t n = 0;
  std::vector<std::pair<uint64_t, uint64_t>> objs;  // allocated arrays (base, bytes), ascending
  // state shared by the generator closures
  std::vector<std::shared_ptr<void>> keep;
  uint64_t limit = 0;  // > 0: the trace is truncated to its first `limit` records (C5)
  int scramble = 0;
  uint64_t scramble_seed = 0;
};

inline uint32_t lane_mask_threads(uint32_t warp, uint32_t nthreads) {
  uint32_t first = warp * 32;
  if (first >= nthreads) return 0;
  uint32_t k = std::min<uint32_t>(32, nthreads - first);
  return k == 32 ? 0xffffffffu : ((1u << k) - 1);
}

uint64_t count_launch(const Launch& L) {
  uint32_t nw = (L.nthreads + 31) / 32;
  uint64_t total = 0;
#pragma omp parallel for schedule(dynamic, 16) reduction(+ : total)
  for (int64_t c = 0; c < (int64_t)L.ncta; ++c) {
    WarpProg wp;
    Prog p{&wp};
    for (uint32_t w = 0; w < nw; ++w) {
      wp.clear();
      L.gen((uint32_t)c, w, p);
      for (auto& i : wp) total += __builtin_popcount(i.mask);
    }
  }
  return total;
}

// Runs the virtual scheduler over one launch and writes its records.
void simulate(const Launch& L, const Sink& S) {
  const int NSM = 15;
  const uint32_t nw = (L.nthreads + 31) / 32;
  int slots = (int)std::min<uint32_t>(16, std::max<uint32_t>(1, 64 / std::max<uint32_t>(1, nw)));
  struct Cta {
    uint32_t id;
    std::vector<WarpProg> warps;
    std::vector<size_t> pc;
    std::vector<uint32_t> wmem, wbb;
    uint32_t live;
  };
  std::vector<std::vector<std::unique_ptr<Cta>>> sm(NSM);
  for (auto& s : sm) s.resize(slots);
  uint32_t next = 0;
  auto make = [&](uint32_t id) {
    auto c = std::make_unique<Cta>();
    c->id = id;
    c->warps.resize(nw);
    c->pc.assign(nw, 0);
    c->wmem.assign(nw, 0);
    c->wbb.assign(nw, 0);
    c->live = 0;
    for (uint32_t w = 0; w < nw; ++w) {
      Prog p{&c->warps[w]};
      L.gen(id, w, p);
      if (!c->warps[w].empty()) c->live++;
    }
    return c;
  };
  for (int s = 0; s < slots; ++s)
    for (int m = 0; m < NSM; ++m)
      if (next < L.ncta) sm[m][s] = make(next++);
  uint64_t pos = L.offset;
  bool any = true;
  while (any) {
    any = false;
    for (int m = 0; m < NSM; ++m) {
      for (int s = 0; s < slots; ++s) {
        Cta* c = sm[m][s].get();
        if (!c) continue;
        any = true;
        for (uint32_t w = 0; w < nw; ++w) {
          if (c->pc[w] >= c->warps[w].size()) continue;
          const WInstr& I = c->warps[w][c->pc[w]++];
          uint32_t wi = ((I.meta & 3) == K_BB) ? c->wbb[w]++ : c->wmem[w]++;
          for (int l = 0; l < 32; ++l) {
            if (!(I.mask >> l & 1u)) continue;
            if (pos >= S.lo && pos < S.hi) {
              uint64_t o = pos - S.lo;
              S.addr[o] = I.addr[l];
              S.cta[o] = L.cta_base + c->id;
              S.tid[o] = (uint16_t)(w * 32 + l);
              S.site[o] = I.site;
              S.winst[o] = wi;
              S.meta[o] = I.meta;
            }
            ++pos;
          }
          if (c->pc[w] == c->warps[w].size()) {
            c->live--;
            WarpProg().swap(c->warps[w]);
          }
        }
      }
      for (int s = 0; s < slots; ++s) {
        if (sm[m][s] && sm[m][s]->live == 0) {
          sm[m][s].reset();
          if (next < L.ncta) { sm[m][s] = make(next++); any = true; }
        }
      }
    }
  }
  if (pos != L.offset + L.count) {
    fprintf(stderr, "tracegen: internal count mismatch (%llu vs %llu)\n",
            (unsigned long long)(pos - L.offset), (unsigned long long)L.count);
    abort();
  }
}

// ---------------------------------------------------------------- params
struct Params {
  std::map<std::string, std::string> kv;
  explicit Params(const char* s) {
    std::string str = s ? s : "";
    size_t i = 0;
    while (i < str.size()) {
      size_t j = str.find(',', i);
      if (j == std::string::npos) j = str.size();
      std::string item = str.substr(i, j - i);
      size_t e = item.find('=');
      if (e != std::string::npos) kv[item.substr(0, e)] = item.substr(e + 1);
      i = j + 1;
    }
  }
  int64_t i(const char* k, int64_t d) const {
    auto it = kv.find(k);
    return it == kv.end() ? d : strtoll(it->second.c_str(), nullptr, 0);
  }
  double f(const char* k, double d) const {
    auto it = kv.find(k);
    return it == kv.end() ? d : strtod(it->second.c_str(), nullptr);
  }
};

// ---------------------------------------------------------------- workloads
// Site numbering: each workload hands out ids from a counter.

// C1: vecAdd, 1 CTA x 64 threads, grid-stride loop over N fp32.
void wl_vecadd(Trace& T, const Params& P) {
  uint32_t N = (uint32_t)P.i("n", 683), NT = (uint32_t)P.i("threads", 64);
  int bb = (int)P.i("bb", 1);
  Alloc A(&T.objs);
  uint64_t a = A.get(N * 4ull), b = A.get(N * 4ull), c = A.get(N * 4ull);
  enum { S_ENTRY, S_HDR, S_BODY, S_EXIT, S_LDA, S_LDB, S_STC, S_N };
  T.nsites = S_N;
  Launch L;
  L.ncta = 1; L.nthreads = NT;
  L.gen = [=](uint32_t, uint32_t w, Prog& p) {
    uint32_t all = lane_mask_threads(w, NT);
    if (bb) p.bb(S_ENTRY, all);
    uint32_t in = all;
    for (uint32_t k = 0;; ++k) {
      if (bb) p.bb(S_HDR, in);
      uint32_t take = 0;
      for (int l = 0; l < 32; ++l)
        if ((in >> l & 1u) && (w * 32 + l) + k * NT < N) take |= 1u << l;
      if (!take) break;
      if (bb) p.bb(S_BODY, take);
      auto idx = [=](int l) { return (uint64_t)(w * 32 + l) + (uint64_t)k * NT; };
      p.mem(K_LOAD, 4, S_LDA, take, [&](int l) { return a + 4 * idx(l); });
      p.mem(K_LOAD, 4, S_LDB, take, [&](int l) { return b + 4 * idx(l); });
      p.mem(K_STORE, 4, S_STC, take, [&](int l) { return c + 4 * idx(l); });
      in = take;
    }
    if (bb) p.bb(S_EXIT, all);
  };
  T.launches.push_back(L);
}

// C2: SGEMM n x n x n, 16x16 CTAs; naive launch then shared-memory-tiled launch.
void wl_sgemm(Trace& T, const Params& P) {
  uint32_t n = (uint32_t)P.i("n", 256);
  const uint32_t TS = 16;
  int naive = (int)P.i("naive", 1), tiled = (int)P.i("tiled", 1), bb = (int)P.i("bb", 0);
  Alloc A(&T.objs);
  uint64_t a = A.get(4ull * n * n), b = A.get(4ull * n * n), c = A.get(4ull * n * n);
  uint32_t g = n / TS;
  uint32_t site = 0;
  if (naive) {
    uint32_t s_ld_a = site++, s_ld_b = site++, s_st_c = site++;
    uint32_t s_entry = site++, s_hdr = site++, s_body = site++, s_exit = site++;
    Launch L; L.ncta = g * g; L.nthreads = TS * TS;
    L.gen = [=](uint32_t cta, uint32_t w, Prog& p) {
      uint32_t bx = cta % g, by = cta / g, all = 0xffffffffu;
      auto row = [=](int l) { return (uint64_t)by * TS + (w * 32 + l) / TS; };
      auto col = [=](int l) { return (uint64_t)bx * TS + (w * 32 + l) % TS; };
      if (bb) p.bb(s_entry, all);
      for (uint32_t k = 0; k < n; ++k) {
        if (bb) { p.bb(s_hdr, all); p.bb(s_body, all); }
        p.mem(K_LOAD, 4, s_ld_a, all, [&](int l) { return a + 4 * (row(l) * n + k); });
        p.mem(K_LOAD, 4, s_ld_b, all, [&](int l) { return b + 4 * ((uint64_t)k * n + col(l)); });
      }
      if (bb) p.bb(s_hdr, all);
      p.mem(K_STORE, 4, s_st_c, all, [&](int l) { return c + 4 * (row(l) * n + col(l)); });
      if (bb) p.bb(s_exit, all);
    };
    T.launches.push_back(L);
  }
  if (tiled) {
    uint32_t s_ld_a = site++, s_ld_b = site++, s_st_c = site++;
    uint32_t s_entry = site++, s_hdr = site++, s_body = site++, s_exit = site++;
    Launch L; L.ncta = g * g; L.nthreads = TS * TS;
    L.gen = [=](uint32_t cta, uint32_t w, Prog& p) {
      uint32_t bx = cta % g, by = cta / g, all = 0xffffffffu;
      auto ty = [=](int l) { return (uint64_t)(w * 32 + l) / TS; };
      auto tx = [=](int l) { return (uint64_t)(w * 32 + l) % TS; };
      if (bb) p.bb(s_entry, all);
      for (uint32_t t = 0; t < n / TS; ++t) {
        if (bb) { p.bb(s_hdr, all); p.bb(s_body, all); }
        p.mem(K_LOAD, 4, s_ld_a, all,
              [&](int l) { return a + 4 * (((uint64_t)by * TS + ty(l)) * n + t * TS + tx(l)); });
        p.mem(K_LOAD, 4, s_ld_b, all,
              [&](int l) { return b + 4 * (((uint64_t)t * TS + ty(l)) * n + (uint64_t)bx * TS + tx(l)); });
      }
      if (bb) p.bb(s_hdr, all);
      p.mem(K_STORE, 4, s_st_c, all,
            [&](int l) { return c + 4 * (((uint64_t)by * TS + ty(l)) * n + (uint64_t)bx * TS + tx(l)); });
      if (bb) p.bb(s_exit, all);
    };
    T.launches.push_back(L);
  }
  T.nsites = site;
}

// Polybench BICG (NX x NY), 256-thread CTAs; accumulators kept in registers,
// so only the loop loads are traced (SURVEY 8(c) "MD BICG shape").
void wl_bicg(Trace& T, const Params& P) {
  uint32_t nx = (uint32_t)P.i("nx", 1024), ny = (uint32_t)P.i("ny", 1024), NT = 256;
  int final_store = (int)P.i("store", 0);
  Alloc A(&T.objs);
  uint64_t a = A.get(4ull * nx * ny), r = A.get(4ull * nx), p_ = A.get(4ull * ny);
  uint64_t s = A.get(4ull * ny), q = A.get(4ull * nx);
  enum { S_K1_A, S_K1_R, S_K1_S, S_K2_A, S_K2_P, S_K2_Q, S_N };
  T.nsites = S_N;
  Launch L1; L1.ncta = (ny + NT - 1) / NT; L1.nthreads = NT;
  L1.gen = [=](uint32_t cta, uint32_t w, Prog& p) {
    uint32_t m = 0;
    for (int l = 0; l < 32; ++l) if ((uint64_t)cta * NT + w * 32 + l < ny) m |= 1u << l;
    auto j = [=](int l) { return (uint64_t)cta * NT + w * 32 + l; };
    for (uint32_t i = 0; i < nx; ++i) {
      p.mem(K_LOAD, 4, S_K1_A, m, [&](int l) { return a + 4 * ((uint64_t)i * ny + j(l)); });
      p.mem(K_LOAD, 4, S_K1_R, m, [&](int) { return r + 4ull * i; });
    }
    if (final_store) p.mem(K_STORE, 4, S_K1_S, m, [&](int l) { return s + 4 * j(l); });
  };
  Launch L2; L2.ncta = (nx + NT - 1) / NT; L2.nthreads = NT;
  L2.gen = [=](uint32_t cta, uint32_t w, Prog& p) {
    uint32_t m = 0;
    for (int l = 0; l < 32; ++l) if ((uint64_t)cta * NT + w * 32 + l < nx) m |= 1u << l;
    auto i = [=](int l) { return (uint64_t)cta * NT + w * 32 + l; };
    for (uint32_t j = 0; j < ny; ++j) {
      p.mem(K_LOAD, 4, S_K2_A, m, [&](int l) { return a + 4 * (i(l) * ny + j); });
      p.mem(K_LOAD, 4, S_K2_P, m, [&](int) { return p_ + 4ull * j; });
    }
    if (final_store) p.mem(K_STORE, 4, S_K2_Q, m, [&](int l) { return q + 4 * i(l); });
  };
  T.launches.push_back(L1);
  T.launches.push_back(L2);
}

// Polybench SYRK / SYR2K: 32x8 CTAs, thread (i = row, j = col); a loop of
// (broadcast a[i][k], strided a[j][k]) pairs, then one coalesced c store.
void wl_syrk(Trace& T, const Params& P, bool two) {
  uint32_t ni = (uint32_t)P.i("ni", 8), nj = (uint32_t)P.i("nj", 32), M = (uint32_t)P.i("m", 1024);
  uint32_t N = (uint32_t)std::max(ni, nj);
  Alloc A(&T.objs);
  uint64_t a = A.get(4ull * N * M), b = A.get(4ull * N * M), c = A.get(4ull * N * N);
  enum { S_AI, S_BJ, S_BI, S_AJ, S_C, S_N };
  T.nsites = S_N;
  const uint32_t BX = 32, BY = 8;
  uint32_t gx = (nj + BX - 1) / BX, gy = (ni + BY - 1) / BY;
  Launch L; L.ncta = gx * gy; L.nthreads = BX * BY;
  L.gen = [=](uint32_t cta, uint32_t w, Prog& p) {
    uint32_t bx = cta % gx, by = cta / gx;
    uint64_t i = (uint64_t)by * BY + w;  // one row of the CTA per warp
    uint32_t m = 0;
    for (int l = 0; l < 32; ++l) if (i < ni && (uint64_t)bx * BX + l < nj) m |= 1u << l;
    auto j = [=](int l) { return (uint64_t)bx * BX + l; };
    for (uint32_t k = 0; k < M; ++k) {
      p.mem(K_LOAD, 4, S_AI, m, [&](int) { return a + 4 * (i * M + k); });
      p.mem(K_LOAD, 4, two ? S_BJ : S_AJ, m, [&](int l) { return (two ? b : a) + 4 * (j(l) * M + k); });
      if (two) {
        p.mem(K_LOAD, 4, S_BI, m, [&](int) { return b + 4 * (i * M + k); });
        p.mem(K_LOAD, 4, S_AJ, m, [&](int l) { return a + 4 * (j(l) * M + k); });
      }
    }
    p.mem(K_STORE, 4, S_C, m, [&](int l) { return c + 4 * (i * N + j(l)); });
  };
  T.launches.push_back(L);
}

// C3: Rodinia-shaped BFS (512-thread CTAs = 16 warps, Table 2), random graph
// with out-degree uniform in {dmin..dmax}; Kernel / Kernel2 per level.
void wl_bfs(Trace& T, const Params& P) {
  uint32_t N = (uint32_t)P.i("nodes", 1000000);
  uint32_t dmin = (uint32_t)P.i("dmin", 2), dmax = (uint32_t)P.i("dmax", 10);
  uint64_t seed = (uint64_t)P.i("seed", 42);
  int bb = (int)P.i("bb", 1);
  const uint32_t NT = 512;
  struct G {
    std::vector<uint32_t> start, ne, edges;
    std::vector<std::vector<uint8_t>> mask, visited, updating;  // per level
  };
  auto g = std::make_shared<G>();
  Rng rng(seed);
  g->start.resize(N); g->ne.resize(N);
  uint64_t tot = 0;
  for (uint32_t v = 0; v < N; ++v) {
    g->start[v] = (uint32_t)tot;
    g->ne[v] = dmin + rng.below(dmax - dmin + 1);
    tot += g->ne[v];
  }
  g->edges.resize(tot);
  for (auto& e : g->edges) e = rng.below(N);
  std::vector<uint8_t> mask(N, 0), vis(N, 0), upd(N, 0);
  mask[0] = 1; vis[0] = 1;
  for (;;) {
    g->mask.push_back(mask);
    g->visited.push_back(vis);
    bool over = false;
    for (uint32_t v = 0; v < N; ++v) {
      if (!mask[v]) continue;
      mask[v] = 0;
      for (uint32_t k = 0; k < g->ne[v]; ++k) {
        uint32_t id = g->edges[g->start[v] + k];
        if (!vis[id]) upd[id] = 1;
      }
    }
    g->updating.push_back(upd);
    for (uint32_t v = 0; v < N; ++v)
      if (upd[v]) { mask[v] = 1; vis[v] = 1; over = true; upd[v] = 0; }
    if (!over) break;
  }
  Alloc A(&T.objs);
  uint64_t nodes = A.get(8ull * N), edges = A.get(4ull * tot), gmask = A.get(N), gupd = A.get(N);
  uint64_t gvis = A.get(N), cost = A.get(4ull * N), overp = A.get(4);
  enum {
    K1_ENTRY, K1_COND, K1_THEN, K1_HDR, K1_BODY, K1_IF, K1_INC, K1_EXIT,
    K1_LD_MASK, K1_ST_MASK, K1_LD_START, K1_LD_NE, K1_LD_EDGE, K1_LD_VIS, K1_LD_COST, K1_ST_COST, K1_ST_UPD,
    K2_ENTRY, K2_COND, K2_THEN, K2_EXIT,
    K2_LD_UPD, K2_ST_MASK, K2_ST_VIS, K2_ST_OVER, K2_ST_UPD, S_N
  };
  T.nsites = S_N;
  uint32_t ncta = (N + NT - 1) / NT;
  for (size_t lev = 0; lev < g->mask.size(); ++lev) {
    Launch L1; L1.ncta = ncta; L1.nthreads = NT;
    L1.gen = [=](uint32_t cta, uint32_t w, Prog& p) {
      const auto& mk = g->mask[lev];
      const auto& vs = g->visited[lev];
      uint32_t all = 0xffffffffu, in = 0, fr = 0;
      auto tid = [=](int l) { return (uint64_t)cta * NT + w * 32 + l; };
      for (int l = 0; l < 32; ++l) if (tid(l) < N) in |= 1u << l;
      for (int l = 0; l < 32; ++l) if ((in >> l & 1u) && mk[tid(l)]) fr |= 1u << l;
      if (bb) p.bb(K1_ENTRY, all);
      if (bb) p.bb(K1_COND, in);
      p.mem(K_LOAD, 1, K1_LD_MASK, in, [&](int l) { return gmask + tid(l); });
      if (fr) {
        if (bb) p.bb(K1_THEN, fr);
        p.mem(K_STORE, 1, K1_ST_MASK, fr, [&](int l) { return gmask + tid(l); });
        p.mem(K_LOAD, 4, K1_LD_START, fr, [&](int l) { return nodes + 8 * tid(l); });
        p.mem(K_LOAD, 4, K1_LD_NE, fr, [&](int l) { return nodes + 8 * tid(l) + 4; });
        uint32_t inl = fr;
        for (uint32_t k = 0;; ++k) {
          if (bb) p.bb(K1_HDR, inl);
          uint32_t cont = 0;
          for (int l = 0; l < 32; ++l) if ((inl >> l & 1u) && k < g->ne[tid(l)]) cont |= 1u << l;
          if (!cont) break;
          if (bb) p.bb(K1_BODY, cont);
          auto eidx = [&](int l) { return (uint64_t)g->start[tid(l)] + k; };
          p.mem(K_LOAD, 4, K1_LD_EDGE, cont, [&](int l) { return edges + 4 * eidx(l); });
          p.mem(K_LOAD, 1, K1_LD_VIS, cont, [&](int l) { return gvis + g->edges[eidx(l)]; });
          uint32_t unv = 0;
          for (int l = 0; l < 32; ++l) if ((cont >> l & 1u) && !vs[g->edges[eidx(l)]]) unv |= 1u << l;
          if (unv) {
            if (bb) p.bb(K1_IF, unv);
            p.mem(K_LOAD, 4, K1_LD_COST, unv, [&](int l) { return cost + 4 * tid(l); });
            p.mem(K_STORE, 4, K1_ST_COST, unv, [&](int l) { return cost + 4ull * g->edges[eidx(l)]; });
            p.mem(K_STORE, 1, K1_ST_UPD, unv, [&](int l) { return gupd + g->edges[eidx(l)]; });
          }
          if (bb) p.bb(K1_INC, cont);
          inl = cont;
        }
      }
      if (bb) p.bb(K1_EXIT, all);
    };
    T.launches.push_back(L1);
    Launch L2; L2.ncta = ncta; L2.nthreads = NT;
    L2.gen = [=](uint32_t cta, uint32_t w, Prog& p) {
      const auto& up = g->updating[lev];
      uint32_t all = 0xffffffffu, in = 0, u = 0;
      auto tid = [=](int l) { return (uint64_t)cta * NT + w * 32 + l; };
      for (int l = 0; l < 32; ++l) if (tid(l) < N) in |= 1u << l;
      for (int l = 0; l < 32; ++l) if ((in >> l & 1u) && up[tid(l)]) u |= 1u << l;
      if (bb) p.bb(K2_ENTRY, all);
      if (bb) p.bb(K2_COND, in);
      p.mem(K_LOAD, 1, K2_LD_UPD, in, [&](int l) { return gupd + tid(l); });
      if (u) {
        if (bb) p.bb(K2_THEN, u);
        p.mem(K_STORE, 1, K2_ST_MASK, u, [&](int l) { return gmask + tid(l); });
        p.mem(K_STORE, 1, K2_ST_VIS, u, [&](int l) { return gvis + tid(l); });
        p.mem(K_STORE, 1, K2_ST_OVER, u, [&](int) { return overp; });
        p.mem(K_STORE, 1, K2_ST_UPD, u, [&](int l) { return gupd + tid(l); });
      }
      if (bb) p.bb(K2_EXIT, all);
    };
    T.launches.push_back(L2);
  }
  T.keep.push_back(g);
  char buf[128];
  snprintf(buf, sizeof buf, "\"levels\": %zu, \"edges\": %llu", g->mask.size(), (unsigned long long)tot);
  T.info = buf;
}

// C4: Rodinia-shaped SRAD (srad_v2), rows x cols fp32, 16x16 CTAs (8 warps).
// Kernel 1: 5 loads (J at p and 4 clamped neighbours) + 5 stores (c, dN, dS,
// dW, dE).  Kernel 2: 8 loads (c at p, south, east; dN..dE at p; J at p) + 1
// store (J).  Basic blocks: entry, border clamps, body, a data-dependent
// saturation branch (hashed per pixel and iteration), tail.
void wl_srad(Trace& T, const Params& P) {
  uint32_t R = (uint32_t)P.i("rows", 2048), C = (uint32_t)P.i("cols", 2048);
  uint32_t iters = (uint32_t)P.i("iters", 6);
  int bb = (int)P.i("bb", 1);
  uint64_t seed = (uint64_t)P.i("seed", 42);
  const uint32_t TS = 16;
  uint32_t gx = (C + TS - 1) / TS, gy = (R + TS - 1) / TS;
  Alloc A(&T.objs);
  uint64_t sz = 4ull * R * C;
  uint64_t J = A.get(sz), Cc = A.get(sz), dN = A.get(sz), dS = A.get(sz), dW = A.get(sz), dE = A.get(sz);
  enum {
    K1_ENTRY, K1_CLN, K1_CLS, K1_CLW, K1_CLE, K1_BODY, K1_SAT, K1_TAIL,
    K1_LD_J, K1_LD_JN, K1_LD_JS, K1_LD_JW, K1_LD_JE, K1_ST_C, K1_ST_DN, K1_ST_DS, K1_ST_DW, K1_ST_DE,
    K2_ENTRY, K2_CLS, K2_CLE, K2_BODY,
    K2_LD_C, K2_LD_CS, K2_LD_CE, K2_LD_DN, K2_LD_DS, K2_LD_DW, K2_LD_DE, K2_LD_J, K2_ST_J, S_N
  };
  T.nsites = S_N;
  for (uint32_t it = 0; it < iters; ++it) {
    for (int k = 0; k < 2; ++k) {
      Launch L; L.ncta = gx * gy; L.nthreads = TS * TS;
      L.gen = [=](uint32_t cta, uint32_t w, Prog& p) {
        uint32_t bx = cta % gx, by = cta / gx;
        auto r = [=](int l) { return (uint64_t)by * TS + (w * 32 + l) / TS; };
        auto c = [=](int l) { return (uint64_t)bx * TS + (w * 32 + l) % TS; };
        uint32_t all = 0, cn = 0, cs = 0, cw = 0, ce = 0, sat = 0;
        for (int l = 0; l < 32; ++l) {
          if (r(l) >= R || c(l) >= C) continue;
          all |= 1u << l;
          if (r(l) == 0) cn |= 1u << l;
          if (r(l) == R - 1) cs |= 1u << l;
          if (c(l) == 0) cw |= 1u << l;
          if (c(l) == C - 1) ce |= 1u << l;
          if ((splitmix64(seed * 0x100000001b3ull + (r(l) * C + c(l)) * 64 + it) & 7) == 0) sat |= 1u << l;
        }
        auto at = [=](uint64_t base, uint64_t rr, uint64_t cc) { return base + 4 * (rr * C + cc); };
        auto nr = [=](int l) { return r(l) == 0 ? 0 : r(l) - 1; };
        auto sr = [=](int l) { return r(l) == R - 1 ? (uint64_t)R - 1 : r(l) + 1; };
        auto wc = [=](int l) { return c(l) == 0 ? 0 : c(l) - 1; };
        auto ec = [=](int l) { return c(l) == C - 1 ? (uint64_t)C - 1 : c(l) + 1; };
        if (k == 0) {
          if (bb) { p.bb(K1_ENTRY, all); p.bb(K1_CLN, cn); p.bb(K1_CLS, cs); p.bb(K1_CLW, cw); p.bb(K1_CLE, ce); p.bb(K1_BODY, all); }
          p.mem(K_LOAD, 4, K1_LD_J, all, [&](int l) { return at(J, r(l), c(l)); });
          p.mem(K_LOAD, 4, K1_LD_JN, all, [&](int l) { return at(J, nr(l), c(l)); });
          p.mem(K_LOAD, 4, K1_LD_JS, all, [&](int l) { return at(J, sr(l), c(l)); });
          p.mem(K_LOAD, 4, K1_LD_JW, all, [&](int l) { return at(J, r(l), wc(l)); });
          p.mem(K_LOAD, 4, K1_LD_JE, all, [&](int l) { return at(J, r(l), ec(l)); });
          if (bb) { p.bb(K1_SAT, sat); p.bb(K1_TAIL, all); }
          p.mem(K_STORE, 4, K1_ST_C, all, [&](int l) { return at(Cc, r(l), c(l)); });
          p.mem(K_STORE, 4, K1_ST_DN, all, [&](int l) { return at(dN, r(l), c(l)); });
          p.mem(K_STORE, 4, K1_ST_DS, all, [&](int l) { return at(dS, r(l), c(l)); });
          p.mem(K_STORE, 4, K1_ST_DW, all, [&](int l) { return at(dW, r(l), c(l)); });
          p.mem(K_STORE, 4, K1_ST_DE, all, [&](int l) { return at(dE, r(l), c(l)); });
        } else {
          if (bb) { p.bb(K2_ENTRY, all); p.bb(K2_CLS, cs); p.bb(K2_CLE, ce); p.bb(K2_BODY, all); }
          p.mem(K_LOAD, 4, K2_LD_C, all, [&](int l) { return at(Cc, r(l), c(l)); });
          p.mem(K_LOAD, 4, K2_LD_CS, all, [&](int l) { return at(Cc, sr(l), c(l)); });
          p.mem(K_LOAD, 4, K2_LD_CE, all, [&](int l) { return at(Cc, r(l), ec(l)); });
          p.mem(K_LOAD, 4, K2_LD_DN, all, [&](int l) { return at(dN, r(l), c(l)); });
          p.mem(K_LOAD, 4, K2_LD_DS, all, [&](int l) { return at(dS, r(l), c(l)); });
          p.mem(K_LOAD, 4, K2_LD_DW, all, [&](int l) { return at(dW, r(l), c(l)); });
          p.mem(K_LOAD, 4, K2_LD_DE, all, [&](int l) { return at(dE, r(l), c(l)); });
          p.mem(K_LOAD, 4, K2_LD_J, all, [&](int l) { return at(J, r(l), c(l)); });
          p.mem(K_STORE, 4, K2_ST_J, all, [&](int l) { return at(J, r(l), c(l)); });
        }
      };
      T.launches.push_back(L);
    }
  }
}

// Rodinia-shaped backprop (Table 2: 8 warps/CTA): bpnn_layerforward (16x16
// CTAs over in x hid) and bpnn_adjust_weights.
void wl_backprop(Trace& T, const Params& P) {
  uint32_t in = (uint32_t)P.i("in", 65536), hid = 16;
  int bb = (int)P.i("bb", 1);
  const uint32_t TS = 16;
  Alloc A(&T.objs);
  uint64_t inp = A.get(4ull * (in + 1)), w = A.get(4ull * (in + 1) * (hid + 1));
  uint64_t part = A.get(4ull * (in / TS) * hid), delta = A.get(4ull * (hid + 1)), oldw = A.get(4ull * (in + 1) * (hid + 1));
  enum { F_ENTRY, F_TX0, F_RED, F_RED_IF, F_TAIL, F_LD_IN, F_LD_W, F_ST_W, F_ST_PART,
         W_ENTRY, W_IF, W_LD_D, W_LD_IN, W_LD_OW, W_LD_W, W_ST_W, W_ST_OW, S_N };
  T.nsites = S_N;
  uint32_t gy = in / TS;
  Launch L1; L1.ncta = gy; L1.nthreads = TS * TS;
  L1.gen = [=](uint32_t by, uint32_t wp, Prog& p) {
    uint32_t all = 0xffffffffu, tx0 = 0;
    auto ty = [=](int l) { return (uint64_t)(wp * 32 + l) / TS; };
    auto tx = [=](int l) { return (uint64_t)(wp * 32 + l) % TS; };
    for (int l = 0; l < 32; ++l) if (tx(l) == 0) tx0 |= 1u << l;
    auto idx = [=](int l) { return (hid + 1) * (TS * by + ty(l) + 1) + tx(l) + 1; };
    if (bb) { p.bb(F_ENTRY, all); p.bb(F_TX0, tx0); }
    p.mem(K_LOAD, 4, F_LD_IN, tx0, [&](int l) { return inp + 4 * ((uint64_t)TS * by + ty(l) + 1); });
    p.mem(K_LOAD, 4, F_LD_W, all, [&](int l) { return w + 4 * (uint64_t)idx(l); });
    p.mem(K_STORE, 4, F_ST_W, all, [&](int l) { return w + 4 * (uint64_t)idx(l); });
    for (uint32_t i = 1; i <= 4; ++i) {  // log2(16) reduction steps in shared memory
      uint32_t pw = 1u << i, m = 0;
      for (int l = 0; l < 32; ++l) if (ty(l) % pw == 0) m |= 1u << l;
      if (bb) { p.bb(F_RED, all); p.bb(F_RED_IF, m); }
    }
    uint32_t t0 = 0;
    for (int l = 0; l < 32; ++l) if (ty(l) == 0) t0 |= 1u << l;
    if (bb) p.bb(F_TAIL, t0);
    p.mem(K_STORE, 4, F_ST_PART, t0, [&](int l) { return part + 4 * ((uint64_t)by * hid + tx(l)); });
  };
  T.launches.push_back(L1);
  Launch L2; L2.ncta = gy; L2.nthreads = TS * TS;
  L2.gen = [=](uint32_t by, uint32_t wp, Prog& p) {
    uint32_t all = 0xffffffffu, f = 0;
    auto ty = [=](int l) { return (uint64_t)(wp * 32 + l) / TS; };
    auto tx = [=](int l) { return (uint64_t)(wp * 32 + l) % TS; };
    auto idx = [=](int l) { return (hid + 1) * (TS * by + ty(l) + 1) + tx(l) + 1; };
    if (bb) p.bb(W_ENTRY, all);
    p.mem(K_LOAD, 4, W_LD_D, all, [&](int l) { return delta + 4 * (tx(l) + 1); });
    p.mem(K_LOAD, 4, W_LD_IN, all, [&](int l) { return inp + 4 * ((uint64_t)TS * by + ty(l) + 1); });
    p.mem(K_LOAD, 4, W_LD_OW, all, [&](int l) { return oldw + 4 * (uint64_t)idx(l); });
    p.mem(K_LOAD, 4, W_LD_W, all, [&](int l) { return w + 4 * (uint64_t)idx(l); });
    p.mem(K_STORE, 4, W_ST_W, all, [&](int l) { return w + 4 * (uint64_t)idx(l); });
    p.mem(K_STORE, 4, W_ST_OW, all, [&](int l) { return oldw + 4 * (uint64_t)idx(l); });
    for (int l = 0; l < 32; ++l) if (ty(l) == 0 && by == 0) f |= 1u << l;
    if (bb) p.bb(W_IF, f);
    p.mem(K_LOAD, 4, W_LD_D, f, [&](int l) { return delta + 4 * (tx(l) + 1); });
    p.mem(K_LOAD, 4, W_LD_W, f, [&](int l) { return w + 4 * (tx(l) + 1); });
    p.mem(K_STORE, 4, W_ST_W, f, [&](int l) { return w + 4 * (tx(l) + 1); });
  };
  T.launches.push_back(L2);
}

// Needleman-Wunsch-shaped CTA (Rodinia nw: 16-thread CTAs = 1 warp with 16
// launched lanes, Table 2): basic-block trace only (BD closed form).
void wl_nw(Trace& T, const Params& P) {
  uint32_t ncta = (uint32_t)P.i("ctas", 4);
  const uint32_t B = 16;
  enum { ENTRY, IF_TX0, LA_HDR, LA_BODY, MID, L1_HDR, L1_IF, L1_LATCH, L2_HDR, L2_IF, L2_LATCH,
         L3_HDR, L3_BODY, EXIT, S_N };
  T.nsites = S_N;
  Launch L; L.ncta = ncta; L.nthreads = B;
  L.gen = [=](uint32_t, uint32_t, Prog& p) {
    uint32_t all = (1u << B) - 1;
    p.bb(ENTRY, all);
    p.bb(IF_TX0, 1u);
    for (uint32_t t = 0; t < B; ++t) { p.bb(LA_HDR, all); p.bb(LA_BODY, all); }
    p.bb(LA_HDR, all);
    p.bb(MID, all);
    for (uint32_t m = 0; m < B; ++m) {
      p.bb(L1_HDR, all);
      p.bb(L1_IF, (uint32_t)((2ull << m) - 1));  // tx <= m
      p.bb(L1_LATCH, all);
    }
    p.bb(L1_HDR, all);
    for (int m = (int)B - 2; m >= 0; --m) {
      p.bb(L2_HDR, all);
      p.bb(L2_IF, (uint32_t)((2ull << m) - 1));
      p.bb(L2_LATCH, all);
    }
    p.bb(L2_HDR, all);
    for (uint32_t t = 0; t < B; ++t) { p.bb(L3_HDR, all); p.bb(L3_BODY, all); }
    p.bb(L3_HDR, all);
    p.bb(EXIT, all);
  };
  T.launches.push_back(L);
}

// Random well-formed traces for fuzzing / adversarial parity cases.
//   ctas, threads, instrs (per warp), lines (address pool, in 128 B units),
//   pstore, pbb, pfull (full-warp mask), launches, seed, stride,
//   msites / bsites (number of memory / basic-block site ids, default 16 / 8),
//   lanes=asc|perm (lane order inside a warp-instruction)
void wl_rand(Trace& T, const Params& P) {
  uint32_t ncta = (uint32_t)P.i("ctas", 4), NT = (uint32_t)P.i("threads", 64);
  uint32_t ninstr = (uint32_t)P.i("instrs", 16), lines = (uint32_t)P.i("lines", 64);
  uint32_t nlaunch = (uint32_t)P.i("launches", 1);
  double pstore = P.f("pstore", 0.2), pbb = P.f("pbb", 0.3), pfull = P.f("pfull", 0.5);
  uint64_t seed = (uint64_t)P.i("seed", 1);
  uint32_t nmsite = (uint32_t)P.i("msites", 16), nbsite = (uint32_t)P.i("bsites", 8);
  if (!nmsite) nmsite = 1;
  if (!nbsite) nbsite = 1;
  T.nsites = nmsite + nbsite;
  Alloc A(&T.objs);
  uint64_t pool = A.get(128ull * lines + 4096);
  uint64_t pool2 = A.get(128ull * lines * 64 + 4096);
  for (uint32_t li = 0; li < nlaunch; ++li) {
    Launch L; L.ncta = ncta; L.nthreads = NT;
    L.gen = [=](uint32_t cta, uint32_t w, Prog& p) {
      Rng r(splitmix64(seed * 1000003ull + li) ^ splitmix64(((uint64_t)cta << 20) + w));
      uint32_t live = lane_mask_threads(w, NT);
      if (!live) return;
      uint32_t ni = ninstr ? 1 + r.below(2 * ninstr) : 0;
      for (uint32_t k = 0; k < ni; ++k) {
        uint32_t m = live;
        if (r.uni() >= pfull) { m = (uint32_t)r.next() & live; if (!m) m = live & (0u - live); }
        if (r.uni() < pbb) { p.bb(nmsite + r.below(nbsite), m); continue; }
        uint8_t kind = r.uni() < pstore ? K_STORE : K_LOAD;
        uint32_t bytes = 1u << r.below(5);
        uint32_t site = r.below(nmsite);
        uint32_t pat = r.below(5);
        uint64_t base = pool + (uint64_t)r.below(lines) * 128;
        uint64_t stride = (uint64_t)bytes << r.below(8);
        uint64_t rnd[32];
        for (int l = 0; l < 32; ++l) {
          uint64_t span = 128ull * lines / bytes;
          rnd[l] = pool + (r.next() % span) * bytes;
        }
        p.mem(kind, bytes, site, m, [&](int l) -> uint64_t {
          switch (pat) {
            case 0: return (base / bytes) * bytes + (uint64_t)l * bytes;    // coalesced
            case 1: return (base / bytes) * bytes;                          // broadcast
            case 2: return pool2 + ((base - pool) / bytes) * bytes + (uint64_t)l * stride;  // strided
            default: return rnd[l];                                         // random
          }
        });
      }
    };
    T.launches.push_back(L);
  }
}

// Hand-written explicit sequence: "seq=A,B,C" is not expressible in the k=v
// syntax, so the literal sequence workload takes lines as a '.'-separated list
// of element indices (one CTA, one thread, 4-byte loads; 's' suffix = store).
void wl_literal(Trace& T, const Params& P) {
  auto it = P.kv.find("seq");
  std::string s = it == P.kv.end() ? "" : it->second;
  std::vector<std::pair<uint64_t, bool>> ops;
  size_t i = 0;
  while (i < s.size()) {
    size_t j = s.find('.', i);
    if (j == std::string::npos) j = s.size();
    std::string tok = s.substr(i, j - i);
    bool st = !tok.empty() && tok.back() == 's';
    if (st) tok.pop_back();
    if (!tok.empty()) ops.push_back({strtoull(tok.c_str(), nullptr, 10), st});
    i = j + 1;
  }
  uint32_t elem = (uint32_t)P.i("elem", 4);
  T.nsites = 2;
  Alloc A(&T.objs);
  uint64_t base = A.get(1 << 20);
  Launch L; L.ncta = 1; L.nthreads = 1;
  L.gen = [=](uint32_t, uint32_t, Prog& p) {
    for (auto& o : ops)
      p.mem(o.second ? K_STORE : K_LOAD, elem, o.second ? 1 : 0, 1u, [&](int) { return base + o.first * elem; });
  };
  T.launches.push_back(L);
}

// C5: the launches of several Rodinia-shaped workloads back
// to back -- SRAD 4096^2 x 3 iterations, backprop 2^23, SGEMM-naive 512^3,
// BFS 4M nodes, tiled SGEMM 2048^3, then SRAD 4096^2 iterations -- until
// exactly `records` (default 4.0e9) records, the last launch truncated.
// Part k uses seed 42 + k.  CTA ids continue across launches; each part's
// site ids are offset past the previous parts'.  C5 is the memory trace of
// the mix (bb=0: the 4.0e9 records are loads/stores, so that the recipe's
// five parts (3.60e9 records) are followed by SRAD iterations as it states;
// with BB records the parts alone would exceed 4.0e9; reading R20).
// div=k divides every linear size by k (edge sizes by sqrt-ish factors) for
// small parity tests of the mixing and truncation logic.
void build(Trace& T, const std::string& name, const Params& P);
uint64_t count_launch(const Launch& L);

void wl_mixed(Trace& T, const Params& P) {
  const uint64_t limit = (uint64_t)P.i("records", 4000000000ll);
  const uint32_t d = (uint32_t)P.i("div", 1);
  auto sq = [&](uint32_t x) { uint32_t r = x; for (uint32_t k = 1; k * k < d && r > 16; k *= 2) r /= 2; return r; };
  std::vector<std::pair<std::string, std::string>> parts;
  char b[256];
  snprintf(b, sizeof b, "rows=%u,cols=%u,iters=3,bb=0,seed=42", sq(4096), sq(4096)); parts.push_back({"srad", b});
  snprintf(b, sizeof b, "in=%u,bb=0", (1u << 23) / d); parts.push_back({"backprop", b});
  snprintf(b, sizeof b, "n=%u,tiled=0,bb=0", sq(512)); parts.push_back({"sgemm", b});
  snprintf(b, sizeof b, "nodes=%u,seed=45,bb=0", 4000000u / d); parts.push_back({"bfs", b});
  snprintf(b, sizeof b, "n=%u,naive=0,bb=0", sq(2048)); parts.push_back({"sgemm", b});
  uint32_t site_base = 0;
  uint64_t total = 0;
  auto add = [&](const std::string& nm, const std::string& ps) {
    Trace sub;
    build(sub, nm, Params(ps.c_str()));
    for (auto& L : sub.launches) {
      Launch L2 = L;
      const uint32_t sb = site_base;
      auto g = L.gen;
      L2.gen = [g, sb](uint32_t c, uint32_t w, Prog& p) {
        size_t st = p.p->size();
        g(c, w, p);
        for (size_t k = st; k < p.p->size(); ++k) (*p.p)[k].site += sb;
      };
      total += count_launch(L);
      T.launches.push_back(L2);
    }
    for (auto& k : sub.keep) T.keep.push_back(k);
    site_base += sub.nsites;
  };
  for (auto& pr : parts) add(pr.first, pr.second);
  if (limit && total < limit) {  // SRAD iterations until the limit (records=0: the five parts only)
    Trace one;
    snprintf(b, sizeof b, "rows=%u,cols=%u,iters=1,bb=0,seed=47", sq(4096), sq(4096));
    build(one, "srad", Params(b));
    uint64_t per = 0;
    for (auto& L : one.launches) per += count_launch(L);
    const uint64_t it = (limit - total + per - 1) / per;
    if (it > 4096) throw std::runtime_error("mixed: records too large for the SRAD fill");
    snprintf(b, sizeof b, "rows=%u,cols=%u,iters=%llu,bb=0,seed=47", sq(4096), sq(4096), (unsigned long long)it);
    add("srad", b);
  }
  T.nsites = site_base;
  T.limit = limit;
}

void build(Trace& T, const std::string& name, const Params& P) {
  T.name = name;
  if (name == "vecadd") wl_vecadd(T, P);
  else if (name == "sgemm") wl_sgemm(T, P);
  else if (name == "bicg") wl_bicg(T, P);
  else if (name == "syrk") wl_syrk(T, P, false);
  else if (name == "syr2k") wl_syrk(T, P, true);
  else if (name == "bfs") wl_bfs(T, P);
  else if (name == "srad") wl_srad(T, P);
  else if (name == "backprop") wl_backprop(T, P);
  else if (name == "nw") wl_nw(T, P);
  else if (name == "rand") wl_rand(T, P);
  else if (name == "literal") wl_literal(T, P);
  else if (name == "mixed") wl_mixed(T, P);
  else throw std::runtime_error("unknown workload " + name);
}

}  // namespace

extern "C" {

struct tg_trace;

tg_trace* tg_plan(const char* workload, const char* params, char* err, int errlen) {
  try {
    auto* T = new Trace();
    Params P(params);
    build(*T, workload, P);
    T->scramble = (int)P.i("scramble", 0);
    T->scramble_seed = (uint64_t)P.i("scramble_seed", 7);
    uint32_t cb = 0;
    uint64_t off = 0;
    for (auto& L : T->launches) {
      L.cta_base = cb;
      cb += L.ncta;
      L.count = count_launch(L);
      L.offset = off;
      off += L.count;
    }
    T->nctas = cb;
    T->n = off;
    if (T->limit && T->n > T->limit) {  // truncation: launches that start past the limit go
      while (!T->launches.empty() && T->launches.back().offset >= T->limit) T->launches.pop_back();
      T->n = T->limit;
    }
    return reinterpret_cast<tg_trace*>(T);
  } catch (std::exception& e) {
    if (err && errlen > 0) snprintf(err, errlen, "%s", e.what());
    return nullptr;
  }
}

uint64_t tg_num_records(const tg_trace* t) { return reinterpret_cast<const Trace*>(t)->n; }
uint32_t tg_num_sites(const tg_trace* t) { return reinterpret_cast<const Trace*>(t)->nsites; }
uint32_t tg_num_ctas(const tg_trace* t) { return reinterpret_cast<const Trace*>(t)->nctas; }
uint32_t tg_num_launches(const tg_trace* t) { return (uint32_t)reinterpret_cast<const Trace*>(t)->launches.size(); }
const char* tg_info(const tg_trace* t) { return reinterpret_cast<const Trace*>(t)->info.c_str(); }

// First record position of every launch, plus the total (nlaunches + 1 values).
void tg_launch_offsets(const tg_trace* t, uint64_t* out) {
  const Trace* T = reinterpret_cast<const Trace*>(t);
  for (size_t k = 0; k < T->launches.size(); ++k) out[k] = T->launches[k].offset;
  out[T->launches.size()] = T->n;
}

// Data objects of the workload (its allocated arrays, ascending base):
// returns their number; fills base[] / bytes[] when non-NULL.  The mixed
// workload reuses the address range per sub-workload and reports none.
uint32_t tg_objects(const tg_trace* t, uint64_t* base, uint64_t* bytes) {
  const Trace* T = reinterpret_cast<const Trace*>(t);
  for (size_t k = 0; k < T->objs.size(); ++k) {
    if (base) base[k] = T->objs[k].first;
    if (bytes) bytes[k] = T->objs[k].second;
  }
  return (uint32_t)T->objs.size();
}

// Writes records [lo, hi) of the trace into the caller's arrays (indexed from 0).
int tg_fill_range(tg_trace* t, uint64_t lo, uint64_t hi, uint64_t* addr, uint32_t* cta, uint16_t* tid,
                  uint32_t* site, uint32_t* winst, uint8_t* meta) {
  Trace* T = reinterpret_cast<Trace*>(t);
  if (hi > T->n || lo > hi) return 1;
  if (T->scramble && (lo != 0 || hi != T->n)) return 2;
  Sink S{addr, cta, tid, site, winst, meta, lo, hi};
  std::vector<size_t> todo;
  for (size_t k = 0; k < T->launches.size(); ++k) {
    const Launch& L = T->launches[k];
    if (L.offset < hi && L.offset + L.count > lo) todo.push_back(k);
  }
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t k = 0; k < (int64_t)todo.size(); ++k) simulate(T->launches[todo[k]], S);
  if (T->scramble) {
    // Non-warp-contiguous variant: a random merge of the per-(cta, warp32)
    // record streams (each stream keeps its own order).
    uint64_t n = T->n;
    std::vector<uint64_t> key(n);
    std::vector<uint32_t> idx(n);
    Rng r(T->scramble_seed);
    std::vector<double> tms(n);
    for (uint64_t i = 0; i < n; ++i) tms[i] = r.uni();
    // per-stream sorted times: group records by stream, sort each group's times
    std::map<uint64_t, std::vector<uint64_t>> streams;
    for (uint64_t i = 0; i < n; ++i) streams[((uint64_t)cta[i] << 5) | (tid[i] >> 5)].push_back(i);
    for (auto& kv : streams) {
      std::vector<double> tt;
      for (auto i : kv.second) tt.push_back(tms[i]);
      std::sort(tt.begin(), tt.end());
      for (size_t q = 0; q < kv.second.size(); ++q) tms[kv.second[q]] = tt[q];
    }
    std::vector<uint64_t> ord(n);
    for (uint64_t i = 0; i < n; ++i) ord[i] = i;
    std::stable_sort(ord.begin(), ord.end(), [&](uint64_t a, uint64_t b) { return tms[a] < tms[b]; });
    std::vector<uint64_t> a2(n); std::vector<uint32_t> c2(n), s2(n), w2(n); std::vector<uint16_t> t2(n); std::vector<uint8_t> m2(n);
    for (uint64_t q = 0; q < n; ++q) {
      uint64_t i = ord[q];
      a2[q] = addr[i]; c2[q] = cta[i]; t2[q] = tid[i]; s2[q] = site[i]; w2[q] = winst[i]; m2[q] = meta[i];
    }
    std::copy(a2.begin(), a2.end(), addr); std::copy(c2.begin(), c2.end(), cta);
    std::copy(t2.begin(), t2.end(), tid); std::copy(s2.begin(), s2.end(), site);
    std::copy(w2.begin(), w2.end(), winst); std::copy(m2.begin(), m2.end(), meta);
  }
  return 0;
}

int tg_fill(tg_trace* t, uint64_t* addr, uint32_t* cta, uint16_t* tid, uint32_t* site, uint32_t* winst,
            uint8_t* meta) {
  return tg_fill_range(t, 0, reinterpret_cast<Trace*>(t)->n, addr, cta, tid, site, winst, meta);
}

void tg_free(tg_trace* t) { delete reinterpret_cast<Trace*>(t); }

}  // extern "C"
