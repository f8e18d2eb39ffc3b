// oracle — plain, slow, obviously-correct CPU reference for the CUDAAdvisor
// trace analyses.  TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke()
// and bench.py's cpu_baseline / --impl reference legs may load this library.
// It shares no code, header, table or helper with the CUDA path
// (paper_conf_cgo_shensll18_b200/); the only common input is the record
// layout produced by tracegen/.
//
// Each function follows the paper's definition step by step (PAPER.md =
// /root/reference/PAPER.md; "P:Lnnn" = its line):
//   * reuse distance: "the number of distinctive data elements accessed
//     between two consecutive uses of the same element", with the write tweak
//     "once an address A is written, we will restart its reuse distance
//     counting as another address A'" and ∞ = "never reused ... or
//     before the next write"; per CTA after regrouping by CTA id
//     (P:L237); memory-element or cache-line model; streaming
//     accesses "never reused by the same CTA".
//       - oracle_reuse: explicit LRU stack of renamed (line, write-epoch) keys.
//       - oracle_reuse_brute: literal O(n^2) definition (tiny traces only).
//       - oracle_reuse_fenwick: Fenwick-tree (Bennett-Kruskal) distinct
//         counts, O(n log n) per scope (large traces, kernel scope).
//   * memory divergence: "the number of unique cache lines touched by each
//     instruction", per dynamic warp-level instruction, a std::set
//     of lines per group (group identity = (cta, tid / W, winst), DESIGN.md
//     reading R9); degree = weighted average left to the caller.
//     A group's records must share kind and site (one static instruction,
//     P:L235 / P:L345; reading R19), else BAD_TRACE.
//   * branch divergence: how many times a block executes, how many threads,
//     how often it makes the warp diverge; divergent = fewer active
//     lanes than launched lanes of that warp (reading R12).
//
// Parity status: every function here is pinned by tests/test_oracle_pins.py
// (paper-printed values, closed forms, brute force, invariants); see DESIGN.md
// "Oracle pins".
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <map>
#include <set>
#include <tuple>
#include <unordered_map>
#include <utility>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {

enum { OK = 0, INVALID_ARG = 1, BAD_TRACE = 2 };
enum { KIND_LOAD = 0, KIND_STORE = 1, KIND_BB = 2 };
enum { SCOPE_CTA = 0, SCOPE_KERNEL = 1 };
enum { BINS_LINEAR = 0, BINS_LOG2 = 1 };

bool pow2(uint32_t x) { return x && !(x & (x - 1)); }

// Per-record validity (include/cadv.h "Per-record validity"), checked over
// the columns an analysis reads: kind <= 2, reserved meta bits 5..7 zero;
// memory records: log2 bytes <= 4, naturally aligned (when the address column
// is read; any 64-bit effective address, "Record(i8* addr, ...)");
// tid < 1024 (when the tid column is read).
bool record_ok(const uint64_t* addr, const uint16_t* tid, const uint8_t* meta, uint64_t i) {
  uint32_t kind = meta[i] & 3u;
  if (kind == 3 || (meta[i] >> 5) != 0) return false;
  if (tid && tid[i] >= 1024) return false;
  if (kind != KIND_BB) {
    uint32_t lg = (meta[i] >> 2) & 7u;
    if (lg > 4) return false;
    if (addr) {
      uint64_t bytes = 1ull << lg;
      if (addr[i] % bytes != 0) return false;
    }
  }
  return true;
}

bool check_all(const uint64_t* addr, const uint16_t* tid, const uint8_t* meta, uint64_t n) {
  for (uint64_t i = 0; i < n; ++i)
    if (!record_ok(addr, tid, meta, i)) return false;
  return true;
}

// Group invariant (include/cadv.h "Group validity", reading R19):
// the records of one dynamic warp-level instruction (cta, tid / 32, winst)
// of a family (memory or basic block) come from ONE static instruction
// (P:L235 one Record() call site per instrumented load/store; P:L345 one
// passBasicBlock() per block), so they share kind and site.  Checked by the
// divergence analyses over the family they analyse.
bool groups_uniform(const uint32_t* cta, const uint16_t* tid, const uint32_t* winst, const uint32_t* site,
                    const uint8_t* meta, uint64_t n, bool bb_family) {
  std::map<std::tuple<uint32_t, uint32_t, uint32_t>, std::pair<uint32_t, uint32_t>> first;  // -> (kind, site)
  for (uint64_t i = 0; i < n; ++i) {
    const uint32_t kind = meta[i] & 3u;
    if ((kind == KIND_BB) != bb_family) continue;
    auto key = std::make_tuple(cta[i], (uint32_t)tid[i] / 32u, winst[i]);
    auto it = first.find(key);
    if (it == first.end()) first.emplace(key, std::make_pair(kind, site[i]));
    else if (it->second.first != kind || it->second.second != site[i]) return false;
  }
  return true;
}

// Histogram index for a finite reuse distance d.
uint32_t bin_of(uint64_t d, int binning, uint32_t nbins) {
  if (binning == BINS_LINEAR) return d <= nbins - 3 ? (uint32_t)d : nbins - 2;
  if (d == 0) return 0;
  uint32_t k = 0;                      // k = floor(log2 d) + 1
  while ((d >> k) != 0) ++k;
  return k <= nbins - 3 ? k : nbins - 2;
}

struct KeyHash {
  size_t operator()(const std::pair<uint64_t, uint64_t>& k) const {
    return std::hash<uint64_t>()(k.first * 0x9e3779b97f4a7c15ull ^ k.second);
  }
};
using RKey = std::pair<uint64_t, uint64_t>;  // renamed key: (line, write epoch)

// Record indices of memory records, grouped by scope, trace order kept.
std::vector<std::vector<uint64_t>> scopes_of(const uint32_t* cta, const uint8_t* meta, uint64_t n, int scope) {
  std::map<uint32_t, std::vector<uint64_t>> m;
  for (uint64_t i = 0; i < n; ++i) {
    if ((meta[i] & 3u) == KIND_BB) continue;
    m[scope == SCOPE_CTA ? cta[i] : 0u].push_back(i);
  }
  std::vector<std::vector<uint64_t>> out;
  out.reserve(m.size());
  for (auto& kv : m) out.push_back(std::move(kv.second));
  return out;
}

int check_reuse_args(uint32_t line_bytes, int scope, int binning, uint32_t nbins) {
  if (!pow2(line_bytes) || line_bytes > 4096) return INVALID_ARG;
  if (scope != SCOPE_CTA && scope != SCOPE_KERNEL) return INVALID_ARG;
  if (binning != BINS_LINEAR && binning != BINS_LOG2) return INVALID_ARG;
  if (nbins < 3) return INVALID_ARG;
  return OK;
}

// One scope's records walked with an explicit LRU stack (top = back()).
// rd[k] = reuse distance of the k-th record of the scope, or -1 for ∞.
void lru_scope(const std::vector<uint64_t>& idx, const uint64_t* addr, const uint8_t* meta, uint32_t line_bytes,
               std::vector<int64_t>& rd, uint64_t& streaming) {
  std::vector<RKey> stack;
  std::unordered_map<uint64_t, uint64_t> epoch;            // e(s, line): stores seen so far
  std::unordered_map<RKey, uint64_t, KeyHash> occurrences;  // per renamed key
  std::vector<RKey> keys(idx.size());
  rd.assign(idx.size(), -1);
  for (size_t k = 0; k < idx.size(); ++k) {
    uint64_t i = idx[k];
    uint64_t line = addr[i] / line_bytes;
    bool store = (meta[i] & 3u) == KIND_STORE;
    if (store) {
      uint64_t e = ++epoch[line];
      RKey key{line, e};
      stack.push_back(key);      // fresh key "A'": first access, RD = ∞
      keys[k] = key;
      rd[k] = -1;
    } else {
      RKey key{line, epoch[line]};
      keys[k] = key;
      int64_t found = -1;
      for (size_t d = 0; d < stack.size(); ++d) {
        if (stack[stack.size() - 1 - d] == key) { found = (int64_t)d; break; }
      }
      if (found >= 0) {
        stack.erase(stack.end() - 1 - found);
        rd[k] = found;
      } else {
        rd[k] = -1;
      }
      stack.push_back(key);
    }
    occurrences[keys[k]]++;
  }
  streaming = 0;
  for (size_t k = 0; k < idx.size(); ++k)
    if (occurrences[keys[k]] == 1) streaming++;
}

}  // namespace

extern "C" {

// Reuse-distance histogram (LRU-stack oracle).  hist[nbins]; stats[5] =
// {accesses, inf, streaming, overflow, sum of the finite distances} (the last
// gives Eq. (1)'s average reuse distance).  Returns 0 / 1 (invalid arg) / 2 (bad trace).
int oracle_reuse(const uint64_t* addr, const uint32_t* cta, const uint16_t* tid, const uint8_t* meta, uint64_t n,
                 uint32_t line_bytes, int scope, int binning, uint32_t nbins, uint64_t* hist, uint64_t* stats) {
  int rc = check_reuse_args(line_bytes, scope, binning, nbins);
  if (rc) return rc;
  if (!check_all(addr, nullptr, meta, n)) return BAD_TRACE;
  auto sc = scopes_of(cta, meta, n, scope);
  std::vector<uint64_t> h(nbins, 0);
  uint64_t streaming = 0, fsum = 0;
#pragma omp parallel
  {
    std::vector<uint64_t> hl(nbins, 0);
    uint64_t sl = 0, fl = 0;
    std::vector<int64_t> rd;
#pragma omp for schedule(dynamic, 1)
    for (int64_t s = 0; s < (int64_t)sc.size(); ++s) {
      uint64_t st = 0;
      lru_scope(sc[s], addr, meta, line_bytes, rd, st);
      sl += st;
      for (int64_t d : rd) {
        hl[d < 0 ? nbins - 1 : bin_of((uint64_t)d, binning, nbins)]++;
        if (d > 0) fl += (uint64_t)d;
      }
    }
#pragma omp critical
    {
      for (uint32_t b = 0; b < nbins; ++b) h[b] += hl[b];
      streaming += sl;
      fsum += fl;
    }
  }
  uint64_t acc = 0;
  for (uint32_t b = 0; b < nbins; ++b) { hist[b] = h[b]; acc += h[b]; }
  stats[0] = acc;
  stats[1] = h[nbins - 1];
  stats[2] = streaming;
  stats[3] = h[nbins - 2];
  stats[4] = fsum;
  return OK;
}

// Per-record reuse distance (LRU-stack oracle): rd[i] = distance, -1 = ∞,
// -2 = not a memory record.
int oracle_reuse_rd(const uint64_t* addr, const uint32_t* cta, const uint16_t* tid, const uint8_t* meta, uint64_t n,
                    uint32_t line_bytes, int scope, int64_t* rd_out) {
  int rc = check_reuse_args(line_bytes, scope, BINS_LINEAR, 3);
  if (rc) return rc;
  if (!check_all(addr, nullptr, meta, n)) return BAD_TRACE;
  for (uint64_t i = 0; i < n; ++i) rd_out[i] = -2;
  auto sc = scopes_of(cta, meta, n, scope);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t s = 0; s < (int64_t)sc.size(); ++s) {
    std::vector<int64_t> rd;
    uint64_t st;
    lru_scope(sc[s], addr, meta, line_bytes, rd, st);
    for (size_t k = 0; k < rd.size(); ++k) rd_out[sc[s][k]] = rd[k];
  }
  return OK;
}

// Literal O(n^2) definition: for each access, find the previous use
// of the same renamed element in the same scope and count the distinct
// renamed elements of that scope accessed strictly in between.
int oracle_reuse_brute(const uint64_t* addr, const uint32_t* cta, const uint16_t* tid, const uint8_t* meta,
                       uint64_t n, uint32_t line_bytes, int scope, int binning, uint32_t nbins, uint64_t* hist,
                       uint64_t* stats, int64_t* rd_out) {
  int rc = check_reuse_args(line_bytes, scope, binning, nbins);
  if (rc) return rc;
  if (!check_all(addr, nullptr, meta, n)) return BAD_TRACE;
  // renamed element of every access: (scope, line, number of stores to that
  // (scope, line) at positions <= i)
  std::vector<std::tuple<uint32_t, uint64_t, uint64_t>> key(n);
  std::vector<bool> mem(n);
  for (uint64_t i = 0; i < n; ++i) {
    mem[i] = (meta[i] & 3u) != KIND_BB;
    if (!mem[i]) continue;
    uint32_t s = scope == SCOPE_CTA ? cta[i] : 0u;
    uint64_t line = addr[i] / line_bytes;
    uint64_t stores = 0;
    for (uint64_t j = 0; j <= i; ++j)
      if (mem[j] && (meta[j] & 3u) == KIND_STORE && (scope == SCOPE_CTA ? cta[j] : 0u) == s &&
          addr[j] / line_bytes == line)
        stores++;
    key[i] = std::make_tuple(s, line, stores);
  }
  std::vector<uint64_t> h(nbins, 0);
  uint64_t fsum = 0;
  for (uint64_t i = 0; i < n; ++i) {
    if (!mem[i]) { if (rd_out) rd_out[i] = -2; continue; }
    int64_t rd = -1;
    if ((meta[i] & 3u) == KIND_LOAD) {
      for (int64_t j = (int64_t)i - 1; j >= 0; --j) {
        if (mem[j] && key[j] == key[i]) {
          std::set<std::tuple<uint32_t, uint64_t, uint64_t>> between;
          for (uint64_t m = (uint64_t)j + 1; m < i; ++m)
            if (mem[m] && std::get<0>(key[m]) == std::get<0>(key[i])) between.insert(key[m]);
          rd = (int64_t)between.size();
          break;
        }
      }
    }
    if (rd_out) rd_out[i] = rd;
    h[rd < 0 ? nbins - 1 : bin_of((uint64_t)rd, binning, nbins)]++;
    if (rd > 0) fsum += (uint64_t)rd;
  }
  uint64_t streaming = 0;
  for (uint64_t i = 0; i < n; ++i) {
    if (!mem[i]) continue;
    uint64_t c = 0;
    for (uint64_t j = 0; j < n; ++j) if (mem[j] && key[j] == key[i]) c++;
    if (c == 1) streaming++;
  }
  uint64_t acc = 0;
  for (uint32_t b = 0; b < nbins; ++b) { hist[b] = h[b]; acc += h[b]; }
  stats[0] = acc; stats[1] = h[nbins - 1]; stats[2] = streaming; stats[3] = h[nbins - 2]; stats[4] = fsum;
  return OK;
}

// Reuse-distance histogram, large-trace variant ("the
// Fenwick-tree (Bennett-Kruskal) CPU variant ... cross-checked == LRU"):
// the same definition as oracle_reuse (P:L248 distinct elements between two
// consecutive uses; the write rule of P:L248/L252 renames the element), with
// the distinct count taken from a Fenwick tree over the scope's positions
// that holds a 1 at the LAST access of every renamed element seen so far:
// RD(k) = number of marks strictly between the previous use p and k (each
// marked position is a distinct element used in the window, and every
// element used in the window has its last use there).  O(n log n) per scope
// instead of the stack walk's O(n * depth), so kernel scope at full size
// finishes.  Same outputs and error codes as oracle_reuse.
namespace {
void fenwick_scope(const std::vector<uint64_t>& idx, const uint64_t* addr, const uint8_t* meta, uint32_t line_bytes,
                   int binning, uint32_t nbins, std::vector<uint64_t>& h, uint64_t& streaming, uint64_t& fsum) {
  const size_t m = idx.size();
  std::vector<uint32_t> bit(m + 1, 0);  // Fenwick tree, 1-based
  auto add = [&](size_t pos, int32_t v) { for (size_t x = pos + 1; x <= m; x += x & (0 - x)) bit[x] += (uint32_t)v; };
  auto prefix = [&](size_t pos) {  // marks at positions < pos
    uint64_t r = 0;
    for (size_t x = pos; x > 0; x -= x & (0 - x)) r += bit[x];
    return r;
  };
  // per line: its CURRENT renamed element (the one a load would use: the
  // latest store's, or the never-written one) -> (last position, uses);
  // an element replaced by a store is never used again, so only its use
  // count (streaming) is settled then -- its mark stays in the tree
  struct Cur { uint64_t last, uses; };
  std::unordered_map<uint64_t, Cur> cur;
  for (size_t k = 0; k < m; ++k) {
    const uint64_t i = idx[k];
    const uint64_t line = addr[i] / line_bytes;
    const bool store = (meta[i] & 3u) == KIND_STORE;
    auto it = cur.find(line);
    if (store || it == cur.end()) {           // first use of a (renamed) element: ∞
      h[nbins - 1]++;
      if (it == cur.end()) {
        cur.emplace(line, Cur{(uint64_t)k, 1});
      } else {
        if (it->second.uses == 1) streaming++;  // the replaced element was used once
        it->second = Cur{(uint64_t)k, 1};
      }
    } else {
      const uint64_t p = it->second.last;
      const uint64_t d = prefix(k) - prefix(p + 1);
      h[bin_of(d, binning, nbins)]++;
      fsum += d;
      add(p, -1);
      it->second.last = k;
      it->second.uses++;
    }
    add(k, 1);
  }
  for (auto& kv : cur) if (kv.second.uses == 1) streaming++;
}
}  // namespace

extern "C" int oracle_reuse_fenwick(const uint64_t* addr, const uint32_t* cta, const uint16_t* tid, const uint8_t* meta,
                                    uint64_t n, uint32_t line_bytes, int scope, int binning, uint32_t nbins,
                                    uint64_t* hist, uint64_t* stats) {
  int rc = check_reuse_args(line_bytes, scope, binning, nbins);
  if (rc) return rc;
  if (!check_all(addr, nullptr, meta, n)) return BAD_TRACE;
  auto sc = scopes_of(cta, meta, n, scope);
  std::vector<uint64_t> h(nbins, 0);
  uint64_t streaming = 0, fsum = 0;
#pragma omp parallel
  {
    std::vector<uint64_t> hl(nbins, 0);
    uint64_t sl = 0, fl = 0;
#pragma omp for schedule(dynamic, 1)
    for (int64_t s = 0; s < (int64_t)sc.size(); ++s) fenwick_scope(sc[s], addr, meta, line_bytes, binning, nbins, hl, sl, fl);
#pragma omp critical
    {
      for (uint32_t b = 0; b < nbins; ++b) h[b] += hl[b];
      streaming += sl;
      fsum += fl;
    }
  }
  uint64_t acc = 0;
  for (uint32_t b = 0; b < nbins; ++b) { hist[b] = h[b]; acc += h[b]; }
  stats[0] = acc; stats[1] = h[nbins - 1]; stats[2] = streaming; stats[3] = h[nbins - 2]; stats[4] = fsum;
  return OK;
}

// Memory divergence: per dynamic warp-level load/store, the number
// of unique cache lines touched.  Group = (cta, tid / W, winst) over memory
// records.  hist[2][W+1] (row 0 loads, row 1 stores; column = degree);
// per_site[nsites][2] = {groups, sum of degrees} (nullable).
int oracle_mem_div(const uint64_t* addr, const uint32_t* cta, const uint16_t* tid, const uint32_t* winst,
                   const uint32_t* site, const uint8_t* meta, uint64_t n, uint32_t line_bytes, uint32_t warp_size,
                   uint32_t nsites, uint64_t* hist, uint64_t* per_site) {
  if (!pow2(line_bytes) || line_bytes > 4096) return INVALID_ARG;
  if (!pow2(warp_size) || warp_size > 32) return INVALID_ARG;
  if (!check_all(addr, tid, meta, n)) return BAD_TRACE;
  if (!groups_uniform(cta, tid, winst, site, meta, n, false)) return BAD_TRACE;
  for (uint64_t i = 0; i < n; ++i)
    if ((meta[i] & 3u) != KIND_BB && per_site && site[i] >= nsites) return INVALID_ARG;
  const uint32_t W = warp_size;
  // bucket memory records by CTA (trace order kept inside each bucket)
  std::map<uint32_t, std::vector<uint64_t>> by_cta;
  for (uint64_t i = 0; i < n; ++i)
    if ((meta[i] & 3u) != KIND_BB) by_cta[cta[i]].push_back(i);
  std::vector<const std::vector<uint64_t>*> lists;
  for (auto& kv : by_cta) lists.push_back(&kv.second);
  std::vector<uint64_t> H(2 * (W + 1), 0), S(per_site ? 2ull * nsites : 0, 0);
  int bad = 0;
#pragma omp parallel
  {
    std::vector<uint64_t> Hl(2 * (W + 1), 0), Sl(per_site ? 2ull * nsites : 0, 0);
#pragma omp for schedule(dynamic, 4)
    for (int64_t c = 0; c < (int64_t)lists.size(); ++c) {
      struct Group { uint64_t first; std::set<uint64_t> lines; std::set<uint32_t> lanes; uint64_t count = 0; };
      std::map<std::pair<uint32_t, uint32_t>, Group> groups;  // (tid / W, winst)
      for (uint64_t i : *lists[c]) {
        auto key = std::make_pair((uint32_t)(tid[i] / W), winst[i]);
        auto it = groups.find(key);
        if (it == groups.end()) { it = groups.emplace(key, Group()).first; it->second.first = i; }
        it->second.lines.insert(addr[i] / line_bytes);
        it->second.lanes.insert(tid[i] % W);
        it->second.count++;
      }
      for (auto& kv : groups) {
        const Group& g = kv.second;
        if (g.lanes.size() != g.count) {
#pragma omp atomic write
          bad = 1;
          continue;
        }
        uint64_t deg = g.lines.size();
        uint32_t kind = meta[g.first] & 3u;
        Hl[kind * (W + 1) + deg]++;
        if (per_site) { Sl[2ull * site[g.first]] += 1; Sl[2ull * site[g.first] + 1] += deg; }
      }
    }
#pragma omp critical
    {
      for (size_t k = 0; k < H.size(); ++k) H[k] += Hl[k];
      for (size_t k = 0; k < S.size(); ++k) S[k] += Sl[k];
    }
  }
  if (bad) return BAD_TRACE;
  std::memcpy(hist, H.data(), H.size() * 8);
  if (per_site) std::memcpy(per_site, S.data(), S.size() * 8);
  return OK;
}

// Branch divergence (Table 3): per dynamic warp-level basic-block
// execution g = (cta, tid / W, winst) over BB records:
//   active(g) = number of distinct lanes (tid % W) in g
//   live(g)   = clamp(T_c - w*W, 0, W), T_c = 1 + max tid over CTA c's BB records
//   divergent = active < live
// per_site[nsites][3] = {exec, divergent, threads}; totals[3] = their sums.
int oracle_branch_div(const uint32_t* cta, const uint16_t* tid, const uint32_t* winst, const uint32_t* site,
                      const uint8_t* meta, uint64_t n, uint32_t warp_size, uint32_t nsites, uint64_t* per_site,
                      uint64_t* totals) {
  if (!pow2(warp_size) || warp_size > 32) return INVALID_ARG;
  if (!check_all(nullptr, tid, meta, n)) return BAD_TRACE;
  if (!groups_uniform(cta, tid, winst, site, meta, n, true)) return BAD_TRACE;
  for (uint64_t i = 0; i < n; ++i)
    if ((meta[i] & 3u) == KIND_BB && per_site && site[i] >= nsites) return INVALID_ARG;
  const uint32_t W = warp_size;
  std::map<uint32_t, std::vector<uint64_t>> by_cta;
  for (uint64_t i = 0; i < n; ++i)
    if ((meta[i] & 3u) == KIND_BB) by_cta[cta[i]].push_back(i);
  std::vector<const std::vector<uint64_t>*> lists;
  for (auto& kv : by_cta) lists.push_back(&kv.second);
  std::vector<uint64_t> S(per_site ? 3ull * nsites : 0, 0);
  uint64_t T[3] = {0, 0, 0};
  int bad = 0;
#pragma omp parallel
  {
    std::vector<uint64_t> Sl(S.size(), 0);
    uint64_t Tl[3] = {0, 0, 0};
#pragma omp for schedule(dynamic, 4)
    for (int64_t c = 0; c < (int64_t)lists.size(); ++c) {
      uint32_t Tc = 0;
      for (uint64_t i : *lists[c]) Tc = std::max<uint32_t>(Tc, (uint32_t)tid[i] + 1);
      struct Group { uint64_t first; std::set<uint32_t> lanes; uint64_t count = 0; };
      std::map<std::pair<uint32_t, uint32_t>, Group> groups;
      for (uint64_t i : *lists[c]) {
        auto key = std::make_pair((uint32_t)(tid[i] / W), winst[i]);
        auto it = groups.find(key);
        if (it == groups.end()) { it = groups.emplace(key, Group()).first; it->second.first = i; }
        it->second.lanes.insert(tid[i] % W);
        it->second.count++;
      }
      for (auto& kv : groups) {
        const Group& g = kv.second;
        if (g.lanes.size() != g.count) {
#pragma omp atomic write
          bad = 1;
          continue;
        }
        uint64_t w = kv.first.first;
        int64_t live = (int64_t)Tc - (int64_t)(w * W);
        if (live < 0) live = 0;
        if (live > (int64_t)W) live = W;
        uint64_t active = g.lanes.size();
        uint64_t div = (int64_t)active < live ? 1 : 0;
        Tl[0] += 1; Tl[1] += div; Tl[2] += active;
        if (per_site) {
          uint32_t s = site[g.first];
          Sl[3ull * s] += 1; Sl[3ull * s + 1] += div; Sl[3ull * s + 2] += active;
        }
      }
    }
#pragma omp critical
    {
      for (size_t k = 0; k < S.size(); ++k) S[k] += Sl[k];
      for (int k = 0; k < 3; ++k) T[k] += Tl[k];
    }
  }
  if (bad) return BAD_TRACE;
  if (per_site) std::memcpy(per_site, S.data(), S.size() * 8);
  for (int k = 0; k < 3; ++k) totals[k] = T[k];
  return OK;
}

// Data-centric attribution (the profiler "associates the memory
// accesses in GPU kernels with the data allocation ... utilizes this
// effective address to associate the memory access with data object"),
// applied to the two memory analyses (reading R18):
//   objects: nobj allocations [base[k], base[k] + bytes[k]), bytes > 0, in
//     ascending order; at line granularity a line belongs to the object whose
//     byte range it intersects, and no line may intersect two objects (else
//     INVALID_ARG).  Lines in no object belong to row nobj ("unattributed").
//   rd_hist[(nobj + 1) * nbins] (nullable): every memory access's reuse
//     distance exactly as oracle_reuse (same scope / binning), counted in the
//     row of the object of the access's line.
//   md_hist[(nobj + 1) * 2 * (W + 1)] (nullable): every group (cta, tid / W,
//     winst) exactly as oracle_mem_div, counted in the row of the object of
//     its first record's line.
// Rows are found by a linear scan over the table (the definition).
int oracle_data_centric(const uint64_t* addr, const uint32_t* cta, const uint16_t* tid, const uint32_t* winst,
                        const uint32_t* site, const uint8_t* meta, uint64_t n, const uint64_t* obj_base, const uint64_t* obj_bytes,
                        uint32_t nobj, uint32_t line_bytes, int scope, int binning, uint32_t nbins,
                        uint32_t warp_size, uint64_t* rd_hist, uint64_t* md_hist) {
  if (!rd_hist && !md_hist) return INVALID_ARG;
  int rc = check_reuse_args(line_bytes, scope, binning, rd_hist ? nbins : 3);
  if (rc) return rc;
  if (md_hist && (!pow2(warp_size) || warp_size > 32)) return INVALID_ARG;
  const uint64_t L = line_bytes;
  for (uint32_t k = 0; k < nobj; ++k) {
    if (obj_bytes[k] == 0 || obj_base[k] + obj_bytes[k] < obj_base[k]) return INVALID_ARG;
    // the last line of object k-1 must lie strictly before the first line of object k
    if (k > 0 && (obj_base[k - 1] + obj_bytes[k - 1] - 1) / L >= obj_base[k] / L) return INVALID_ARG;
  }
  if (!check_all(addr, md_hist ? tid : nullptr, meta, n)) return BAD_TRACE;
  if (md_hist && !groups_uniform(cta, tid, winst, site, meta, n, false)) return BAD_TRACE;
  auto row_of_line = [&](uint64_t line) -> uint32_t {
    const uint64_t lo = line * L, hi = lo + L;  // the line's bytes [lo, hi)
    for (uint32_t k = 0; k < nobj; ++k)
      if (lo < obj_base[k] + obj_bytes[k] && obj_base[k] < hi) return k;
    return nobj;
  };
  const uint64_t R = (uint64_t)nobj + 1;
  if (rd_hist) {
    std::vector<int64_t> rd(n);
    rc = oracle_reuse_rd(addr, cta, tid, meta, n, line_bytes, scope, rd.data());
    if (rc) return rc;
    std::vector<uint64_t> h(R * nbins, 0);
    for (uint64_t i = 0; i < n; ++i) {
      if (rd[i] == -2) continue;  // not a memory record
      const uint32_t b = rd[i] < 0 ? nbins - 1 : bin_of((uint64_t)rd[i], binning, nbins);
      h[row_of_line(addr[i] / L) * nbins + b]++;
    }
    std::memcpy(rd_hist, h.data(), h.size() * 8);
  }
  if (md_hist) {
    const uint32_t W = warp_size;
    std::map<uint32_t, std::vector<uint64_t>> by_cta;
    for (uint64_t i = 0; i < n; ++i)
      if ((meta[i] & 3u) != KIND_BB) by_cta[cta[i]].push_back(i);
    std::vector<const std::vector<uint64_t>*> lists;
    for (auto& kv : by_cta) lists.push_back(&kv.second);
    std::vector<uint64_t> H(R * 2 * (W + 1), 0);
    int bad = 0;
#pragma omp parallel
    {
      std::vector<uint64_t> Hl(H.size(), 0);
#pragma omp for schedule(dynamic, 4)
      for (int64_t c = 0; c < (int64_t)lists.size(); ++c) {
        struct Group { uint64_t first; std::set<uint64_t> lines; std::set<uint32_t> lanes; uint64_t count = 0; };
        std::map<std::pair<uint32_t, uint32_t>, Group> groups;  // (tid / W, winst)
        for (uint64_t i : *lists[c]) {
          auto key = std::make_pair((uint32_t)(tid[i] / W), winst[i]);
          auto it = groups.find(key);
          if (it == groups.end()) { it = groups.emplace(key, Group()).first; it->second.first = i; }
          it->second.lines.insert(addr[i] / L);
          it->second.lanes.insert(tid[i] % W);
          it->second.count++;
        }
        for (auto& kv : groups) {
          const Group& g = kv.second;
          if (g.lanes.size() != g.count) {
#pragma omp atomic write
            bad = 1;
            continue;
          }
          const uint32_t kind = meta[g.first] & 3u;
          Hl[(row_of_line(addr[g.first] / L) * 2 + kind) * (W + 1) + g.lines.size()]++;
        }
      }
#pragma omp critical
      for (size_t k = 0; k < H.size(); ++k) H[k] += Hl[k];
    }
    if (bad) return BAD_TRACE;
    std::memcpy(md_hist, H.data(), H.size() * 8);
  }
  return OK;
}

int oracle_num_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

// Thread count of the following calls (bench.py's 1-thread baseline); 0 = all cores.
void oracle_set_num_threads(int k) {
#ifdef _OPENMP
  static const int all = omp_get_max_threads();
  omp_set_num_threads(k > 0 ? k : all);
#else
  (void)k;
#endif
}

}  // extern "C"
