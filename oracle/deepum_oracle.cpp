// oracle/deepum_oracle.cpp
//
// TEST INFRASTRUCTURE ONLY.  This is the plain, slow, sequential CPU oracle of
// DeepUM's correlation-prefetch and migration engine.  Only tests/,
// __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
// may load it.  It shares no code, header, table or constant generator with the
// CUDA path in paper_conf_asplos_jungkl23_b200/csrc/, and neither includes the
// other.
//
// It executes the method in the paper's order and notation (the method is a
// heuristic with sequential state; there is no closed-form definition it
// reaches):
//   * execution ID table ............ PAPER.md L136 (Sec. 3.1)
//   * execution ID correlation table  PAPER.md L176, L208-L210 (Sec. 4.2, Fig. 6)
//   * UM block correlation tables ... PAPER.md L164-L174 (Sec. 4.1, Fig. 5),
//                                     L212-L216 (Sec. 4.2, Fig. 7)
//   * prefetch walk and chaining .... PAPER.md L156, L218-L224 (Sec. 4.2)
//   * pre-eviction / invalidation ... PAPER.md L236-L243 (Sec. 5.1), L285 (Sec. 5.2)
//   * migration ..................... PAPER.md L124 (Sec. 2.3)
// Where the paper is silent or garbled the readings D1-D22 of SURVEY.md
// Sec. 8(c) (restated in DESIGN.md "Readings") are followed; each use is tagged
// with its D-number below.
//
// Data structures are deliberately naive: std::vector sets searched linearly,
// std::unordered_map for the execution ID table.
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <map>
#include <set>
#include <thread>
#include <unordered_map>
#include <unordered_set>
#include <vector>

namespace {

constexpr uint32_t NONE = 0xFFFFFFFFu;  // D1

enum { ORC_OK = 0, ORC_EINVAL = -1, ORC_ECAPACITY = -2, ORC_ESTATE = -5 };

struct Row {                      // one way of a set: tag + NumSuccs successors
  uint32_t tag;
  std::vector<uint32_t> succ;     // MRU first
};
using Set = std::vector<Row>;     // ways, MRU first (D8)

struct BlockTable {               // one per execution ID
  std::vector<Set> sets;          // NumRows sets
  uint32_t start = NONE, end = NONE;
};

struct CorrRec {                  // (h1,h2,h3 -> succ)
  uint32_t h1, h2, h3, succ;
};

struct Staged {
  uint64_t k;
  uint32_t e;
  std::vector<uint32_t> L;
};

struct Oracle {
  uint32_t R, A, S, N, W, C, row_index;
  // execution ID table
  std::unordered_map<uint64_t, uint32_t> exec_map;
  std::vector<uint64_t> exec_hash;
  // execution ID correlation table
  std::vector<std::vector<CorrRec>> corr;
  uint32_t hist[4] = {NONE, NONE, NONE, NONE};  // oldest first (D4)
  uint64_t k = 0;                                // launches recorded
  // UM block correlation tables, allocated when an exec ID first faults (P L358)
  std::map<uint32_t, BlockTable> tbl;
  std::vector<Staged> staged;
  // residency
  std::vector<uint32_t> frame_of, block_of;
  std::vector<uint64_t> stamp;
  std::vector<uint8_t> inactive;
  std::set<uint32_t> free_frames;
  uint64_t mig_counter = 0;
  uint32_t threads = 1;                          // predict/select query ranges per thread (orc_set_threads)

  uint32_t idx(uint32_t b) const {               // D7
    if (row_index == 1) {
      uint32_t h = b;
      h ^= h >> 16; h *= 0x85ebca6bu; h ^= h >> 13; h *= 0xc2b2ae35u; h ^= h >> 16;
      return h & (R - 1);
    }
    return b & (R - 1);
  }

  BlockTable &table(uint32_t e) {
    auto it = tbl.find(e);
    if (it == tbl.end()) {
      BlockTable t;
      t.sets.resize(R);
      it = tbl.emplace(e, std::move(t)).first;
    }
    return it->second;
  }
  const BlockTable *table_if(uint32_t e) const {
    auto it = tbl.find(e);
    return it == tbl.end() ? nullptr : &it->second;
  }

  static int find_way(const Set &s, uint32_t b) {
    for (size_t w = 0; w < s.size(); ++w)
      if (s[w].tag == b) return (int)w;
    return -1;
  }

  // TOUCH(T,b): the faulted block's row is (re)allocated and becomes MRU.
  // Fig. 5(a) "Last ... points to c" before c has successors => a row is
  // allocated on every miss (D10); LRU way replacement (D8).
  void touch(BlockTable &T, uint32_t b) {
    Set &s = T.sets[idx(b)];
    int w = find_way(s, b);
    if (w >= 0) {
      Row r = s[w];
      s.erase(s.begin() + w);
      s.insert(s.begin(), r);
    } else {
      s.insert(s.begin(), Row{b, {}});
      if (s.size() > A) s.resize(A);
    }
  }

  // INSERT(T,p,s): s becomes the MRU successor of p ("NumSucc
  // entries are MRU ordered from left to right"; D9).
  void insert(BlockTable &T, uint32_t p, uint32_t sc) {
    if (sc == p) return;
    Set &s = T.sets[idx(p)];
    int w = find_way(s, p);
    if (w < 0) return;  // cannot happen: p was TOUCHed by the previous op
    Row r = s[w];
    s.erase(s.begin() + w);
    auto it = std::find(r.succ.begin(), r.succ.end(), sc);
    if (it != r.succ.end()) r.succ.erase(it);
    r.succ.insert(r.succ.begin(), sc);
    if (r.succ.size() > S) r.succ.resize(S);
    s.insert(s.begin(), r);
  }

  // a1 + a2: record_faults (PAPER.md L124 step (2): "removes the duplicate
  // addresses and groups them according to their UM blocks"; D2 keeps the first
  // occurrence) and exec-ID assignment in first-seen order (D3).
  void record(const uint64_t *hash, const uint64_t *off, uint32_t n, const uint32_t *faults,
              uint32_t *out_exec) {
    for (uint32_t i = 0; i < n; ++i) {
      std::vector<uint32_t> L;
      std::unordered_set<uint32_t> seen;
      for (uint64_t j = off[i]; j < off[i + 1]; ++j) {
        uint32_t b = faults[j];
        if (seen.insert(b).second) L.push_back(b);
      }
      uint32_t e;
      auto it = exec_map.find(hash[i]);
      if (it != exec_map.end()) {
        e = it->second;
      } else {
        e = (uint32_t)exec_hash.size();
        exec_map.emplace(hash[i], e);
        exec_hash.push_back(hash[i]);
        corr.emplace_back();
      }
      if (out_exec) out_exec[i] = e;
      staged.push_back(Staged{k, e, std::move(L)});
      ++k;
    }
  }

  // a3: "Each set consists of four execution IDs. The first three IDs
  // represent the previously executed kernels right before the last kernel
  // (currently executing kernel when updating the table). ... the last ID
  // represents the next kernel".  D5: the record is written at
  // launch k into entry e_{k-1}, key (e_{k-4}, e_{k-3}, e_{k-2}), successor
  // e_k; unique on the key; the last observed successor wins; first-seen order.
  void corr_upsert(uint32_t owner, uint32_t h1, uint32_t h2, uint32_t h3, uint32_t succ) {
    auto &v = corr[owner];
    for (auto &r : v) {
      if (r.h1 == h1 && r.h2 == h2 && r.h3 == h3) {
        r.succ = succ;
        return;
      }
    }
    v.push_back(CorrRec{h1, h2, h3, succ});
  }

  // a3-a5: build_tables applies every staged launch in order.
  void build() {
    for (auto &st : staged) {
      if (hist[3] != NONE) corr_upsert(hist[3], hist[0], hist[1], hist[2], st.e);
      hist[0] = hist[1]; hist[1] = hist[2]; hist[2] = hist[3]; hist[3] = st.e;
      if (st.L.empty()) continue;              // D11: no faults -> start/end unchanged
      BlockTable &T = table(st.e);
      uint32_t last = NONE;                    // "Last" resets per launch (D10, P L216)
      for (uint32_t b : st.L) {
        if (last != NONE) insert(T, last, b);
        touch(T, b);
        last = b;
      }
      // Start = first fault after the exec-ID transition, End =
      // last fault before the next transition (D11: fault-based reading).
      T.start = st.L.front();
      T.end = st.L.back();
    }
    staged.clear();
  }

  // A9: predict the next kernel from (current exec ID, previous three).
  uint32_t lookup(uint32_t e, uint32_t h1, uint32_t h2, uint32_t h3) const {
    if (e >= corr.size()) return NONE;
    for (auto &r : corr[e])
      if (r.h1 == h1 && r.h2 == h2 && r.h3 == h3) return r.succ;
    return NONE;
  }

  // WALK (D13, D14): prefetch all blocks correlated to the
  // current block, chaining row to row until a successor equals End.
  std::vector<uint32_t> walk(uint32_t e, uint32_t anchor) const {
    std::vector<uint32_t> out;
    const BlockTable *T = table_if(e);
    uint32_t start = T ? T->start : NONE, end = T ? T->end : NONE;
    if (anchor == NONE && start == NONE) return out;
    uint32_t x = anchor != NONE ? anchor : start;
    std::unordered_set<uint32_t> seen{x}, chained{x};
    if (anchor == NONE) out.push_back(x);
    if (x == end) return out;
    for (;;) {
      if (!T) break;
      const Set &s = T->sets[idx(x)];
      int w = find_way(s, x);                  // read-only: no recency update (D8)
      if (w < 0) break;
      bool hit = false;
      uint32_t nxt = NONE;
      for (uint32_t sc : s[w].succ) {          // MRU first
        if (!seen.count(sc)) { out.push_back(sc); seen.insert(sc); }
        if (sc == end) hit = true;
        if (nxt == NONE && !chained.count(sc)) nxt = sc;
      }
      if (hit || nxt == NONE) break;
      chained.insert(nxt);
      x = nxt;
    }
    return out;
  }

  // a7: PREDICT (D15-D17).
  void predict_one(uint32_t e0, uint32_t h1, uint32_t h2, uint32_t h3, uint32_t anchor, uint32_t n,
                   std::vector<uint32_t> &pairs, std::vector<uint32_t> &kern_off,
                   std::vector<uint32_t> &chain) const {
    std::vector<uint32_t> kernels{e0};
    uint32_t cur = e0, a = h1, b = h2, c = h3;
    if (e0 < exec_hash.size()) {
      for (uint32_t i = 0; i < n; ++i) {
        uint32_t nx = lookup(cur, a, b, c);
        if (nx == NONE) break;
        kernels.push_back(nx);
        a = b; b = c; c = cur;                 // D16: shift register over predicted IDs
        cur = nx;
      }
    } else {
      kernels.clear();                         // unknown exec ID: empty window
    }
    std::unordered_set<uint32_t> Sset;
    if (anchor != NONE) Sset.insert(anchor);
    kern_off.assign(N + 2, 0);
    chain.assign(N + 1, NONE);
    uint32_t cnt = 0;
    for (size_t d = 0; d < kernels.size(); ++d) {
      chain[d] = kernels[d];
      for (uint32_t blk : walk(kernels[d], d == 0 ? anchor : NONE)) {
        if (!Sset.count(blk)) {                // D17: first occurrence wins
          pairs.push_back(blk);
          pairs.push_back(kernels[d]);
          Sset.insert(blk);
          ++cnt;
        }
      }
      kern_off[d + 1] = cnt;
    }
    for (size_t d = kernels.size(); d <= N; ++d) kern_off[d + 1] = cnt;
  }

  // a8: SELECT (victims are least recently migrated AND not
  // expected in the current + next N kernels; L285: victims in inactive PT
  // blocks are invalidated; D18-D20).
  void select_one(const uint32_t *pairs, uint64_t npairs, uint32_t anchor,
                  std::vector<uint32_t> &wb, std::vector<uint32_t> &inv) const {
    std::unordered_set<uint32_t> window;
    uint64_t nonres = 0;
    for (uint64_t i = 0; i < npairs; ++i) {
      uint32_t b = pairs[2 * i];
      window.insert(b);
      if (b >= W || frame_of[b] == NONE) ++nonres;
    }
    if (anchor != NONE) window.insert(anchor);
    uint64_t nfree = free_frames.size();
    uint64_t need = nonres > nfree ? nonres - nfree : 0;
    std::vector<std::pair<uint64_t, uint32_t>> res;
    for (uint32_t f = 0; f < C; ++f)
      if (block_of[f] != NONE) res.push_back({stamp[block_of[f]], block_of[f]});
    std::sort(res.begin(), res.end());
    uint64_t taken = 0;
    for (auto &p : res) {
      if (taken >= need) break;
      if (window.count(p.second)) continue;
      ++taken;
      if (inactive[p.second]) inv.push_back(p.second);
      else wb.push_back(p.second);
    }
  }

  std::vector<uint32_t> lrm_list() const {
    std::vector<std::pair<uint64_t, uint32_t>> res;
    for (uint32_t f = 0; f < C; ++f)
      if (block_of[f] != NONE) res.push_back({stamp[block_of[f]], block_of[f]});
    std::sort(res.begin(), res.end());
    std::vector<uint32_t> out;
    for (auto &p : res) out.push_back(p.second);
    return out;
  }

  // a9 migration bookkeeping (PAPER.md L124 steps (4)-(7), L158; D19, D21).
  int migrate(int dir, const uint32_t *blocks, const uint32_t *dst, uint32_t n) {
    if (dir == 0) {  // H2D: lowest free frame first, in list order
      if (n > free_frames.size()) return ORC_ECAPACITY;
      std::unordered_set<uint32_t> uniq;
      for (uint32_t i = 0; i < n; ++i) {
        uint32_t b = blocks[i];
        if (b >= W || frame_of[b] != NONE || !uniq.insert(b).second) return ORC_EINVAL;
      }
      for (uint32_t i = 0; i < n; ++i) {
        uint32_t b = blocks[i];
        uint32_t f = *free_frames.begin();
        free_frames.erase(free_frames.begin());
        frame_of[b] = f;
        block_of[f] = b;
        stamp[b] = mig_counter++;
      }
      return ORC_OK;
    }
    if (dir == 1 || dir == 2) {  // D2H write-back / invalidate: free the frame
      std::unordered_set<uint32_t> uniq;
      for (uint32_t i = 0; i < n; ++i) {
        uint32_t b = blocks[i];
        if (b >= W || frame_of[b] == NONE || !uniq.insert(b).second) return ORC_EINVAL;
      }
      for (uint32_t i = 0; i < n; ++i) {
        uint32_t b = blocks[i];
        uint32_t f = frame_of[b];
        block_of[f] = NONE;
        frame_of[b] = NONE;
        free_frames.insert(f);
      }
      return ORC_OK;
    }
    if (dir == 3) {  // D2D
      if (blocks == nullptr) {
        // compaction: highest-indexed occupied frames move into the lowest
        // free frames so that the free region becomes a contiguous tail.
        uint32_t nres = 0;
        for (uint32_t f = 0; f < C; ++f) nres += block_of[f] != NONE;
        std::vector<uint32_t> holes, movers;
        for (uint32_t f = 0; f < nres; ++f)
          if (block_of[f] == NONE) holes.push_back(f);
        for (uint32_t f = C; f-- > nres;)
          if (block_of[f] != NONE) movers.push_back(f);
        for (size_t i = 0; i < holes.size(); ++i) {
          uint32_t src = movers[i], d = holes[i], b = block_of[src];
          block_of[d] = b;
          block_of[src] = NONE;
          frame_of[b] = d;
          free_frames.erase(d);
          free_frames.insert(src);
        }
        return ORC_OK;
      }
      std::unordered_set<uint32_t> ub, uf;
      for (uint32_t i = 0; i < n; ++i) {
        uint32_t b = blocks[i], f = dst[i];
        if (b >= W || frame_of[b] == NONE || f >= C || block_of[f] != NONE || !ub.insert(b).second ||
            !uf.insert(f).second)
          return ORC_EINVAL;
      }
      for (uint32_t i = 0; i < n; ++i) {
        uint32_t b = blocks[i], f = dst[i];
        uint32_t src = frame_of[b];
        block_of[src] = NONE;
        free_frames.insert(src);
        block_of[f] = b;
        free_frames.erase(f);
        frame_of[b] = f;
      }
      return ORC_OK;
    }
    return ORC_EINVAL;
  }

  int load_residency(const uint32_t *lrm, uint32_t n) {
    if (n > C) return ORC_ECAPACITY;
    std::unordered_set<uint32_t> uniq;
    for (uint32_t i = 0; i < n; ++i)
      if (lrm[i] >= W || !uniq.insert(lrm[i]).second) return ORC_EINVAL;
    std::fill(frame_of.begin(), frame_of.end(), NONE);
    std::fill(block_of.begin(), block_of.end(), NONE);
    free_frames.clear();
    for (uint32_t i = 0; i < n; ++i) {
      frame_of[lrm[i]] = i;
      block_of[i] = lrm[i];
      stamp[lrm[i]] = i;
    }
    for (uint32_t f = n; f < C; ++f) free_frames.insert(f);
    mig_counter = n;
    return ORC_OK;
  }

  // canonical dump (SURVEY Sec. 8c "Canonical dump byte format")
  void put32(std::vector<uint8_t> &o, uint32_t v) const {
    for (int i = 0; i < 4; ++i) o.push_back((v >> (8 * i)) & 0xFF);
  }
  void put64(std::vector<uint8_t> &o, uint64_t v) const {
    for (int i = 0; i < 8; ++i) o.push_back((v >> (8 * i)) & 0xFF);
  }
  std::vector<uint8_t> dump(uint32_t what) const {
    std::vector<uint8_t> o;
    uint32_t E = (uint32_t)exec_hash.size();
    if (what & 1) {
      put32(o, E);
      for (auto h : exec_hash) put64(o, h);
    }
    if (what & 2) {
      for (uint32_t e = 0; e < E; ++e) {
        put32(o, (uint32_t)corr[e].size());
        for (auto &r : corr[e]) { put32(o, r.h1); put32(o, r.h2); put32(o, r.h3); put32(o, r.succ); }
      }
    }
    if (what & 4) {
      for (uint32_t e = 0; e < E; ++e) {
        const BlockTable *T = table_if(e);
        for (uint32_t r = 0; r < R; ++r) {
          for (uint32_t w = 0; w < A; ++w) {
            const Row *row = (T && w < T->sets[r].size()) ? &T->sets[r][w] : nullptr;
            put32(o, row ? row->tag : NONE);
            for (uint32_t j = 0; j < S; ++j) put32(o, (row && j < row->succ.size()) ? row->succ[j] : NONE);
          }
        }
        put32(o, T ? T->start : NONE);
        put32(o, T ? T->end : NONE);
      }
    }
    if (what & 8) {
      for (uint32_t e = 0; e < E; ++e) {
        auto wl = walk(e, NONE);
        put32(o, (uint32_t)wl.size());
        for (auto b : wl) put32(o, b);
      }
    }
    if (what & 16) {
      put32(o, C);
      for (uint32_t f = 0; f < C; ++f) put32(o, block_of[f]);
      auto l = lrm_list();
      put32(o, (uint32_t)l.size());
      for (auto b : l) put32(o, b);
    }
    if (what & 32) {
      for (int i = 0; i < 4; ++i) put32(o, hist[i]);
      put64(o, k);
    }
    return o;
  }
};

}  // namespace

extern "C" {

void *orc_create(uint32_t R, uint32_t A, uint32_t S, uint32_t N, uint32_t W, uint32_t C, uint32_t row_index) {
  if (R == 0 || (R & (R - 1)) || A == 0 || S == 0 || W == 0) return nullptr;
  Oracle *o = new Oracle();
  o->R = R; o->A = A; o->S = S; o->N = N; o->W = W; o->C = C; o->row_index = row_index;
  o->frame_of.assign(W, NONE);
  o->block_of.assign(C, NONE);
  o->stamp.assign(W, 0);
  o->inactive.assign(W, 0);
  for (uint32_t f = 0; f < C; ++f) o->free_frames.insert(f);
  return o;
}

void orc_destroy(void *h) { delete static_cast<Oracle *>(h); }

int orc_record_faults(void *h, const uint64_t *hash, const uint64_t *off, uint32_t n, const uint32_t *faults,
                      uint32_t *out_exec) {
  static_cast<Oracle *>(h)->record(hash, off, n, faults, out_exec);
  return ORC_OK;
}

int orc_build_tables(void *h) {
  static_cast<Oracle *>(h)->build();
  return ORC_OK;
}

uint32_t orc_num_exec(void *h) { return (uint32_t)static_cast<Oracle *>(h)->exec_hash.size(); }

// queries: n x 6 u32 (exec, h1, h2, h3, anchor, n).  Outputs: CSR offsets
// (pairs), pairs (2 u32 each), kern_off n*(N+2), chain n*(N+1).
int orc_predict(void *h, const uint32_t *q, uint32_t nq, uint64_t *out_off, uint32_t *out_pairs,
                uint64_t cap_pairs, uint32_t *kern_off, uint32_t *chain, uint64_t *needed) {
  Oracle *o = static_cast<Oracle *>(h);
  // queries are independent pure functions of the state (no ordering between
  // them): with threads > 1 contiguous query ranges run on separate threads
  // and their outputs are concatenated in query order -- the same bytes.
  const uint32_t T = std::max<uint32_t>(1, std::min<uint32_t>(o->threads, nq ? nq : 1));
  std::vector<std::vector<uint32_t>> pairs(T);
  std::vector<std::vector<uint64_t>> cnt(T);
  auto run = [&](uint32_t t) {
    const uint32_t a = (uint64_t)nq * t / T, b = (uint64_t)nq * (t + 1) / T;
    std::vector<uint32_t> ko, ch;
    for (uint32_t i = a; i < b; ++i) {
      const uint32_t *x = q + 6 * i;
      o->predict_one(x[0], x[1], x[2], x[3], x[4], std::min(x[5], o->N), pairs[t], ko, ch);
      cnt[t].push_back(pairs[t].size() / 2);
      std::memcpy(kern_off + (uint64_t)i * (o->N + 2), ko.data(), 4 * (o->N + 2));
      std::memcpy(chain + (uint64_t)i * (o->N + 1), ch.data(), 4 * (o->N + 1));
    }
  };
  std::vector<std::thread> th;
  for (uint32_t t = 1; t < T; ++t) th.emplace_back(run, t);
  run(0);
  for (auto &x : th) x.join();
  out_off[0] = 0;
  uint64_t base = 0, i = 0;
  for (uint32_t t = 0; t < T; ++t) {
    for (uint64_t c : cnt[t]) out_off[++i] = base + c;
    base += pairs[t].size() / 2;
  }
  *needed = base;
  if (base > cap_pairs) return ORC_ECAPACITY;
  uint64_t w = 0;
  for (uint32_t t = 0; t < T; ++t) {
    if (!pairs[t].empty()) std::memcpy(out_pairs + w, pairs[t].data(), 4 * pairs[t].size());
    w += pairs[t].size();
  }
  return ORC_OK;
}

// select: per query i, pairs[qoff[i]..qoff[i+1]) (2 u32 each).  Outputs two
// CSR lists (write-back, invalidate) with offsets wb_off/inv_off (nq+1).
int orc_select(void *h, const uint64_t *qoff, const uint32_t *pairs, uint32_t nq, const uint32_t *anchors,
               uint32_t *wb, uint64_t *wb_off, uint32_t *inv, uint64_t *inv_off, uint64_t cap, uint64_t *needed) {
  Oracle *o = static_cast<Oracle *>(h);
  const uint32_t T = std::max<uint32_t>(1, std::min<uint32_t>(o->threads, nq ? nq : 1));
  std::vector<std::vector<uint32_t>> W(T), I(T);
  std::vector<std::vector<std::pair<uint64_t, uint64_t>>> cnt(T);
  auto run = [&](uint32_t t) {
    const uint32_t a = (uint64_t)nq * t / T, b = (uint64_t)nq * (t + 1) / T;
    for (uint32_t i = a; i < b; ++i) {
      o->select_one(pairs + 2 * qoff[i], qoff[i + 1] - qoff[i], anchors ? anchors[i] : NONE, W[t], I[t]);
      cnt[t].push_back({W[t].size(), I[t].size()});
    }
  };
  std::vector<std::thread> th;
  for (uint32_t t = 1; t < T; ++t) th.emplace_back(run, t);
  run(0);
  for (auto &x : th) x.join();
  wb_off[0] = 0;
  inv_off[0] = 0;
  uint64_t bw = 0, bi = 0, i = 0;
  for (uint32_t t = 0; t < T; ++t) {
    for (auto &c : cnt[t]) {
      ++i;
      wb_off[i] = bw + c.first;
      inv_off[i] = bi + c.second;
    }
    bw += W[t].size();
    bi += I[t].size();
  }
  *needed = std::max(bw, bi);
  if (bw > cap || bi > cap) return ORC_ECAPACITY;
  uint64_t pw = 0, pi = 0;
  for (uint32_t t = 0; t < T; ++t) {
    if (!W[t].empty()) std::memcpy(wb + pw, W[t].data(), 4 * W[t].size());
    if (!I[t].empty()) std::memcpy(inv + pi, I[t].data(), 4 * I[t].size());
    pw += W[t].size();
    pi += I[t].size();
  }
  return ORC_OK;
}

void orc_set_threads(void *h, uint32_t n) { static_cast<Oracle *>(h)->threads = n ? n : 1; }

int orc_mark_inactive(void *h, const uint32_t *blocks, uint32_t n, int flag) {
  Oracle *o = static_cast<Oracle *>(h);
  for (uint32_t i = 0; i < n; ++i) {
    if (blocks[i] >= o->W) return ORC_EINVAL;
    o->inactive[blocks[i]] = flag ? 1 : 0;
  }
  return ORC_OK;
}

int orc_load_residency(void *h, const uint32_t *lrm, uint32_t n) {
  return static_cast<Oracle *>(h)->load_residency(lrm, n);
}

int orc_migrate(void *h, int dir, const uint32_t *blocks, const uint32_t *dst, uint32_t n) {
  return static_cast<Oracle *>(h)->migrate(dir, blocks, dst, n);
}

uint32_t orc_free_frames(void *h) { return (uint32_t)static_cast<Oracle *>(h)->free_frames.size(); }

int orc_dump(void *h, uint32_t what, void *buf, uint64_t cap, uint64_t *needed) {
  auto o = static_cast<Oracle *>(h)->dump(what);
  *needed = o.size();
  if (o.size() > cap) return ORC_ECAPACITY;
  if (!o.empty()) std::memcpy(buf, o.data(), o.size());
  return ORC_OK;
}

}  // extern "C"
