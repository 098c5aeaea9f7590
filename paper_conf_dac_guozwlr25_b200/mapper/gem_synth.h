// gem_synth.h -- depth-oriented E-AIG synthesis (§III-B, P:93-95:
// "we want the depth of AIG to be as low as possible ... we run timing-driven
// synthesis as depth minimization").  Included by gem_map.cpp
// after `Graph` and `build_graph`; shares no code with oracle/.
//
// Two function-preserving rewrites of the strashed graph, each followed by
// structural hashing and cone-of-influence pruning:
//
//  1. AND-tree balancing.  A "supergate" is a maximal tree of AND nodes joined
//     by non-complemented edges whose inner nodes have exactly one reference;
//     its leaves are re-associated into a tree that always combines the two
//     earliest-arriving operands first (Huffman order on logic level), which
//     minimises the supergate's output level for the given leaf levels.
//
//  2. Chain lookahead.  A "link" is an AND node one of whose fanins (the
//     chain edge) arrives at least `chain_slack` levels after the other (the
//     side input); following each link to its most critical link user gives
//     disjoint chains n_1 .. n_m (carry / priority / comparator chains: the
//     deep, long-tailed paths of P:83).  Link j computes
//         c_j = (c_{j-1} xor s_j) and y_j        (s_j = chain-edge inversion)
//     i.e. c_j = M_j(c_{j-1}) with M_j(c) = E ? (c xor K) : D, (E,K,D) =
//     (y_j, s_j, 0).  Such maps are closed under composition:
//         M2 o M1 = (E1 E2,  K1 xor K2,  D)      with D = D2 or (E2 and (D1 xor K2))
//     (kept in the form D and E = 0, so the value is (E and (c xor K)) or D),
//     so every needed prefix c_j = P_{1..j}(c_0) is built by a parallel-prefix
//     (segment-tree) network of depth O(log m) over the side inputs instead of
//     the m-level ripple.  Only chain nodes with a reference outside the chain
//     ("taps": other AND users or endpoints) are rebuilt; a chain is rewritten
//     only if its estimated last-tap level improves.
//
// Both rewrites trade AND gates for depth.  Results are unchanged (every
// rewrite is an identity of Boolean algebra), which the ISA-interpreter and
// GPU parity tests check against the oracle on the ORIGINAL netlist.

struct SynthStats {
  uint64_t and_in = 0, and_balanced = 0, and_out = 0;
  uint32_t level_in = 0, level_balanced = 0, level_out = 0;
  uint32_t chains = 0, chain_links = 0, chain_taps = 0;
};

// Builder of a new Graph with the same sources: strash + constant folding.
struct GraphBuilder {
  Graph g;
  std::unordered_map<uint64_t, uint32_t> strash;
  explicit GraphBuilder(const Graph& src) {
    size_t ns = 0;
    while (ns < src.kind.size() && src.kind[ns] != K_AND) ns++;
    g.n_pi = src.n_pi; g.n_flops = src.n_flops; g.n_po = src.n_po; g.n_rams = src.n_rams;
    g.kind.assign(src.kind.begin(), src.kind.begin() + ns);
    g.a.assign(ns, 0); g.b.assign(ns, 0);
    g.gbit.assign(src.gbit.begin(), src.gbit.begin() + ns);
    g.level.assign(ns, 0);
    g.flop_init = src.flop_init;
    strash.reserve(src.kind.size() * 2 + 16);
  }
  uint32_t lev(uint32_t l) const { return g.level[l >> 1]; }
  uint32_t AND(uint32_t x, uint32_t y) {
    if (x > y) std::swap(x, y);
    if (x == 0) return 0;
    if (x == 1) return y;
    if (x == y) return x;
    if (x == (y ^ 1)) return 0;
    const uint64_t key = ((uint64_t)x << 32) | y;
    auto it = strash.find(key);
    if (it != strash.end()) return it->second;
    const uint32_t id = (uint32_t)g.kind.size();
    g.kind.push_back(K_AND); g.a.push_back(x); g.b.push_back(y); g.gbit.push_back(0);
    g.level.push_back(1 + std::max(g.level[x >> 1], g.level[y >> 1]));
    strash.emplace(key, 2 * id);
    return 2 * id;
  }
  uint32_t OR(uint32_t x, uint32_t y) { return AND(x ^ 1, y ^ 1) ^ 1; }
};

// live ANDs and max level of the cone of influence of all endpoints
static void finish_graph(Graph& g) {
  std::vector<uint8_t> live(g.kind.size(), 0);
  auto mark = [&](uint32_t l) { live[l >> 1] = 1; };
  for (auto l : g.flop_next) mark(l);
  for (auto l : g.po) mark(l);
  for (auto& rr : g.rams) for (int p = 0; p < 4; p++) for (int k = 0; k < 32; k++) mark(rr.port[p][k]);
  for (size_t i = g.kind.size(); i-- > 0;)
    if (live[i] && g.kind[i] == K_AND) { live[g.a[i] >> 1] = 1; live[g.b[i] >> 1] = 1; }
  g.n_and_live = 0;
  g.max_level = 0;
  for (size_t i = 0; i < g.kind.size(); i++)
    if (live[i] && g.kind[i] == K_AND) { g.n_and_live++; g.max_level = std::max(g.max_level, g.level[i]); }
}

// Copy endpoints through a node map (old node -> new literal).
static void map_endpoints(const Graph& src, Graph& dst, const std::vector<uint32_t>& m) {
  auto L = [&](uint32_t l) { return m[l >> 1] ^ (l & 1u); };
  dst.flop_next.resize(src.flop_next.size());
  for (size_t j = 0; j < src.flop_next.size(); j++) dst.flop_next[j] = L(src.flop_next[j]);
  dst.po.resize(src.po.size());
  for (size_t k = 0; k < src.po.size(); k++) dst.po[k] = L(src.po[k]);
  dst.rams = src.rams;
  for (auto& rr : dst.rams) for (int p = 0; p < 4; p++) for (int k = 0; k < 32; k++) rr.port[p][k] = L(rr.port[p][k]);
}

// reference counts (AND fanins + endpoints) and "referenced complemented" flags
static void ref_counts(const Graph& g, std::vector<uint32_t>& refs, std::vector<uint8_t>& comp_ref,
                       std::vector<uint8_t>& endpoint) {
  refs.assign(g.kind.size(), 0);
  comp_ref.assign(g.kind.size(), 0);
  endpoint.assign(g.kind.size(), 0);
  auto use = [&](uint32_t l, bool ep) {
    refs[l >> 1]++;
    if (l & 1u) comp_ref[l >> 1] = 1;
    if (ep) endpoint[l >> 1] = 1;
  };
  for (size_t i = 0; i < g.kind.size(); i++)
    if (g.kind[i] == K_AND) { use(g.a[i], false); use(g.b[i], false); }
  for (auto l : g.flop_next) use(l, true);
  for (auto l : g.po) use(l, true);
  for (auto& rr : g.rams) for (int p = 0; p < 4; p++) for (int k = 0; k < 32; k++) use(rr.port[p][k], true);
}

// ---------------------------------------------------------------- 1. balancing
static Graph balance_ands(const Graph& g) {
  std::vector<uint32_t> refs;
  std::vector<uint8_t> comp, ep;
  ref_counts(g, refs, comp, ep);
  auto absorbed = [&](uint32_t v) { return g.kind[v] == K_AND && refs[v] == 1 && !comp[v] && !ep[v]; };
  GraphBuilder B(g);
  std::vector<uint32_t> m(g.kind.size(), 0);
  for (size_t i = 0; i < g.kind.size(); i++)
    if (g.kind[i] != K_AND) m[i] = 2 * (uint32_t)i;
  std::vector<uint32_t> leaves, stack;
  for (size_t i = 0; i < g.kind.size(); i++) {
    if (g.kind[i] != K_AND || absorbed((uint32_t)i)) continue;
    leaves.clear();
    stack.assign({g.a[i], g.b[i]});
    while (!stack.empty()) {
      const uint32_t l = stack.back();
      stack.pop_back();
      if (!(l & 1u) && absorbed(l >> 1)) {
        stack.push_back(g.a[l >> 1]);
        stack.push_back(g.b[l >> 1]);
      } else {
        leaves.push_back(m[l >> 1] ^ (l & 1u));
      }
    }
    // earliest two first (ties: lower literal), as a min-heap on (level, literal)
    auto later = [&](uint32_t x, uint32_t y) {
      const uint32_t lx = B.lev(x), ly = B.lev(y);
      return lx != ly ? lx > ly : x > y;
    };
    std::make_heap(leaves.begin(), leaves.end(), later);
    while (leaves.size() > 1) {
      std::pop_heap(leaves.begin(), leaves.end(), later);
      const uint32_t x = leaves.back();
      leaves.pop_back();
      std::pop_heap(leaves.begin(), leaves.end(), later);
      const uint32_t y = leaves.back();
      leaves.pop_back();
      leaves.push_back(B.AND(x, y));
      std::push_heap(leaves.begin(), leaves.end(), later);
    }
    m[i] = leaves[0];
  }
  map_endpoints(g, B.g, m);
  finish_graph(B.g);
  return std::move(B.g);
}

// ---------------------------------------------------------------- 2. chain lookahead
// A link's map c -> c_j.  Two forms:
//  * cheap (tab = 0): (E, K, D) with K a constant and D and E = 0,
//      value(c) = (E and (c xor K)) or D;
//  * table (tab = 1): the two cofactors, value(c) = c ? F1 : F0 (fields E = F0, D = F1).
// A simple link (one AND with a late fanin) is cheap: (y, s, 0).  A complex
// link (a small cone whose only late leaf is the chain input, e.g. a
// majority/carry cell) gets its cofactors F0 = cone|c=0, F1 = cone|c=1 built
// by re-evaluating the cone with the chain input tied to a constant (strash
// folds the constants); it is cheap again whenever a cofactor is constant.
struct ChainMap {
  uint8_t tab;
  uint32_t E, K, D;
};

// Level-only stand-in for GraphBuilder (dry run of a chain rewrite): literal
// 0/1 = constants, 2 + 2*level (+1 = complemented) = a signal of that level.
// No structural hashing, so levels are upper bounds of the real rewrite.
struct LevelBuilder {
  static uint32_t sig(uint32_t level) { return 2 + 2 * level; }
  static uint32_t level(uint32_t l) { return l < 2 ? 0 : (l - 2) >> 1; }
  uint32_t AND(uint32_t x, uint32_t y) {
    if (x == 0 || y == 0) return 0;
    if (x == 1) return y;
    if (y == 1) return x;
    return sig(1 + std::max(level(x), level(y)));
  }
  uint32_t OR(uint32_t x, uint32_t y) { return AND(x ^ 1, y ^ 1) ^ 1; }
};

template <class BLD>
static ChainMap as_table(BLD& B, const ChainMap& x) {
  if (x.tab) return x;
  // F0 = value(0) = (E and K) or D, F1 = value(1) = (E and not K) or D
  const uint32_t f0 = x.K ? B.OR(x.E, x.D) : x.D;
  const uint32_t f1 = x.K ? x.D : B.OR(x.E, x.D);
  return {1, f0, 0, f1};
}

static ChainMap from_cofactors(uint32_t f0, uint32_t f1) {
  if (f0 == 0) return {0, f1, 0, 0};
  if (f1 == 0) return {0, f0, 1, 0};
  if (f0 == 1) return {0, f1 ^ 1, 1, f1};
  if (f1 == 1) return {0, f0 ^ 1, 0, f0};
  return {1, f0, 0, f1};
}

template <class BLD>
static uint32_t mux(BLD& B, uint32_t s, uint32_t a1, uint32_t a0) {
  return B.OR(B.AND(s, a1), B.AND(s ^ 1, a0));
}

template <class BLD>
static ChainMap compose_maps(BLD& B, const ChainMap& inner, const ChainMap& outer) {
  if (inner.tab || outer.tab) {
    // (G0, G1) o (F0, F1) = (F0 ? G1 : G0, F1 ? G1 : G0)
    const ChainMap f = as_table(B, inner), g = as_table(B, outer);
    return from_cofactors(mux(B, f.E, g.D, g.E), mux(B, f.D, g.D, g.E));
  }
  ChainMap r;
  r.tab = 0;
  r.E = B.AND(inner.E, outer.E);
  r.K = inner.K ^ outer.K;
  // outer(inner(c)) = (E2 and (inner(c) xor K2)) or D2
  if (!outer.K) {
    // inner(c) = (E1 and c') or D1  ->  D = (E2 and D1) or D2
    r.D = B.OR(B.AND(outer.E, inner.D), outer.D);
  } else {
    // not inner(c) = (E1 and not c') or (not E1 and not D1)  (D1 E1 = 0)
    // ->  D = (E2 and not (E1 or D1)) or D2
    r.D = B.OR(B.AND(outer.E, B.OR(inner.E, inner.D) ^ 1), outer.D);
  }
  return r;
}

template <class BLD>
static uint32_t apply_map(BLD& B, const ChainMap& P, uint32_t c) {
  if (P.tab) return mux(B, c, P.D, P.E);
  return B.OR(B.AND(P.E, c ^ P.K), P.D);
}

// One chain's lookahead network on builder BLD: the link maps, the memoised
// maps of aligned power-of-two link segments (a segment tree), and the prefix
// map of links 0..j as the balanced composition of the canonical cover of
// [0, j].  `leaf(old literal)` gives a literal of the side logic on BLD.
struct ChainDef {
  std::vector<uint32_t> nodes;                 // n_1 .. n_m (old ids)
  uint32_t c0 = 0;                             // chain input node of n_1
  std::vector<std::vector<uint32_t>> cones;    // internal cone nodes of each link (ascending ids)
};

template <class BLD, class LEAF>
struct ChainNet {
  const Graph& g;
  const ChainDef& C;
  BLD& B;
  LEAF leaf;
  std::unordered_map<uint64_t, ChainMap> seg;
  std::unordered_map<uint32_t, uint32_t> val;
  ChainNet(const Graph& g_, const ChainDef& c_, BLD& b_, LEAF l_) : g(g_), C(c_), B(b_), leaf(l_) {}

  ChainMap link_map(uint32_t j) {
    const uint32_t v = C.nodes[j], l = j ? C.nodes[j - 1] : C.c0;
    const std::vector<uint32_t>& in = C.cones[j];
    if (in.size() == 1) {   // simple link: v = AND(l ^ s, y)
      const bool la = (g.a[v] >> 1) == l;
      const uint32_t ll = la ? g.a[v] : g.b[v], y = la ? g.b[v] : g.a[v];
      return {0, leaf(y), ll & 1u, 0u};
    }
    uint32_t f[2];
    for (uint32_t b = 0; b < 2; b++) {
      val.clear();
      auto lit = [&](uint32_t x) -> uint32_t {
        if ((x >> 1) == l) return b ^ (x & 1u);
        auto it = val.find(x >> 1);
        return it != val.end() ? it->second ^ (x & 1u) : leaf(x);
      };
      for (uint32_t y : in) val[y] = B.AND(lit(g.a[y]), lit(g.b[y]));
      f[b] = val[v];
    }
    return from_cofactors(f[0], f[1]);
  }
  ChainMap segment(uint32_t lo, uint32_t hi) {
    const uint64_t key = ((uint64_t)lo << 32) | hi;
    auto it = seg.find(key);
    if (it != seg.end()) return it->second;
    ChainMap r;
    if (lo == hi) {
      r = link_map(lo);
    } else {
      const uint32_t mid = lo + (hi - lo) / 2;
      r = compose_maps(B, segment(lo, mid), segment(mid + 1, hi));
    }
    seg.emplace(key, r);
    return r;
  }
  void cover(uint32_t a, uint32_t b, uint32_t j, std::vector<ChainMap>& parts) {
    if (b <= j) { parts.push_back(segment(a, b)); return; }
    if (a > j) return;
    const uint32_t mid = a + (b - a) / 2;
    cover(a, mid, j, parts);
    cover(mid + 1, b, j, parts);
  }
  // c_j from the chain input's value c0 (every inversion is inside the maps)
  uint32_t tap(uint32_t j, uint32_t c0) {
    std::vector<ChainMap> parts;
    uint32_t size = 1;
    while (size < C.nodes.size()) size <<= 1;
    cover(0, size - 1, j, parts);
    while (parts.size() > 1) {
      std::vector<ChainMap> nx;
      for (size_t k = 0; k + 1 < parts.size(); k += 2) nx.push_back(compose_maps(B, parts[k], parts[k + 1]));
      if (parts.size() & 1) nx.push_back(parts.back());
      parts.swap(nx);
    }
    return apply_map(B, parts[0], c0);
  }
};

template <class BLD, class LEAF>
static ChainNet<BLD, LEAF> make_net(const Graph& g, const ChainDef& c, BLD& b, LEAF l) {
  return ChainNet<BLD, LEAF>(g, c, b, l);
}

static Graph chain_lookahead(const Graph& g, int min_len, int slack, SynthStats& st) {
  const size_t N = g.kind.size();
  const uint32_t kMaxBack = 8, kMaxCone = 32;
  std::vector<uint32_t> refs;
  std::vector<uint8_t> comp, ep;
  ref_counts(g, refs, comp, ep);
  // users (AND fanouts) and reverse depth (longest path to an endpoint)
  std::vector<uint32_t> uoff(N + 1, 0), users;
  for (size_t i = 0; i < N; i++)
    if (g.kind[i] == K_AND) { uoff[(g.a[i] >> 1) + 1]++; uoff[(g.b[i] >> 1) + 1]++; }
  for (size_t i = 0; i < N; i++) uoff[i + 1] += uoff[i];
  users.resize(uoff[N]);
  {
    std::vector<uint32_t> fill(uoff.begin(), uoff.end() - 1);
    for (size_t i = 0; i < N; i++)
      if (g.kind[i] == K_AND) { users[fill[g.a[i] >> 1]++] = (uint32_t)i; users[fill[g.b[i] >> 1]++] = (uint32_t)i; }
  }
  std::vector<uint32_t> rdep(N, 0);
  for (size_t i = N; i-- > 0;)
    for (uint32_t k = uoff[i]; k < uoff[i + 1]; k++) rdep[i] = std::max(rdep[i], rdep[users[k]] + 1);
  auto lvl = [&](uint32_t v) { return g.level[v]; };
  auto crit = [&](uint32_t v) {   // critical (latest) fanin node
    const uint32_t x = g.a[v] >> 1, y = g.b[v] >> 1;
    return lvl(x) >= lvl(y) ? x : y;
  };
  // cone of v above chain input l: the AND nodes with level > level(l); valid
  // if l is reached and every other leaf arrives >= slack levels before l
  std::vector<uint32_t> stamp(N, 0), stack;
  uint32_t cur_stamp = 0;
  auto cone = [&](uint32_t v, uint32_t l, std::vector<uint32_t>* internal) -> bool {
    cur_stamp++;
    stack.assign(1, v);
    stamp[v] = cur_stamp;
    uint32_t n_int = 0;
    bool seen_l = false;
    while (!stack.empty()) {
      const uint32_t x = stack.back();
      stack.pop_back();
      if (x == l) { seen_l = true; continue; }
      if (g.kind[x] != K_AND || lvl(x) <= lvl(l)) {
        if (lvl(x) + (uint32_t)slack > lvl(l)) return false;
        continue;
      }
      if (++n_int > kMaxCone) return false;
      if (internal) internal->push_back(x);
      for (uint32_t f : {g.a[x] >> 1, g.b[x] >> 1})
        if (stamp[f] != cur_stamp) { stamp[f] = cur_stamp; stack.push_back(f); }
    }
    return seen_l;
  };
  // chain input of every AND node: the tightest valid cut along its critical path
  std::vector<int64_t> lin(N, -1);
  for (size_t i = 0; i < N; i++) {
    if (g.kind[i] != K_AND) continue;
    uint32_t l = (uint32_t)i;
    for (uint32_t k = 0; k < kMaxBack; k++) {
      l = crit(l);
      if (g.kind[l] != K_AND) break;
      if (cone((uint32_t)i, l, nullptr)) { lin[i] = l; break; }
    }
  }
  // chain successor of a node: among the links whose chain input it is, the
  // one on the longest path (level + reverse depth), then the longest step
  // (a carry cell's output rather than a node inside its cone)
  std::vector<int64_t> next(N, -1), prev(N, -1);
  auto better = [&](uint32_t i, uint32_t j) {
    const uint32_t pi = lvl(i) + rdep[i], pj = lvl(j) + rdep[j];
    if (pi != pj) return pi > pj;
    if (lvl(i) != lvl(j)) return lvl(i) > lvl(j);
    return i < j;
  };
  for (size_t i = 0; i < N; i++) {
    if (lin[i] < 0) continue;
    const uint32_t l = (uint32_t)lin[i];
    if (next[l] < 0 || better((uint32_t)i, (uint32_t)next[l])) next[l] = (int64_t)i;
  }
  for (size_t i = 0; i < N; i++)
    if (next[i] >= 0) prev[next[i]] = (int64_t)i;
  // old literal -> dry-run literal (old levels are upper bounds of the new ones)
  LevelBuilder LB;
  auto old_leaf = [&](uint32_t x) -> uint32_t {
    if ((x >> 1) == 0) return x & 1u;
    return LevelBuilder::sig(lvl(x >> 1)) ^ (x & 1u);
  };
  std::vector<ChainDef> chains;
  std::vector<int32_t> chain_of(N, -1), pos_of(N, -1);
  for (size_t i = 0; i < N; i++) {
    // a chain starts at a link whose chain input is not a link continued by it
    if (lin[i] < 0 || (prev[i] >= 0 && lin[prev[i]] >= 0)) continue;
    ChainDef C;
    C.c0 = (uint32_t)lin[i];
    for (int64_t v = (int64_t)i; v >= 0; v = next[v]) C.nodes.push_back((uint32_t)v);
    if ((int)C.nodes.size() < min_len) continue;
    uint32_t l = C.c0;
    for (uint32_t v : C.nodes) {
      C.cones.emplace_back();
      cone(v, l, &C.cones.back());
      std::sort(C.cones.back().begin(), C.cones.back().end());
      l = v;
    }
    // dry run: rewrite only if the last tap's level improves
    auto dry = make_net(g, C, LB, old_leaf);
    const uint32_t est = LevelBuilder::level(dry.tap((uint32_t)C.nodes.size() - 1, LevelBuilder::sig(lvl(C.c0))));
    if (est + 2 >= lvl(C.nodes.back())) continue;
    for (size_t j = 0; j < C.nodes.size(); j++) {
      chain_of[C.nodes[j]] = (int32_t)chains.size();
      pos_of[C.nodes[j]] = (int32_t)j;
    }
    chains.push_back(std::move(C));
  }
  // chain nodes that must exist in the new graph (taps): the last node, and
  // any n_j referenced from outside the next link's cone or whose next link's
  // cone has an internal node used from outside that cone
  std::vector<uint8_t> is_tap(N, 0);
  for (auto& C : chains) {
    for (size_t j = 0; j < C.nodes.size(); j++) {
      const uint32_t v = C.nodes[j];
      if (j + 1 == C.nodes.size() || ep[v]) { is_tap[v] = 1; continue; }
      const std::vector<uint32_t>& in = C.cones[j + 1];
      auto refs_from_cone = [&](uint32_t x) {
        uint32_t r = 0;
        for (uint32_t y : in) r += ((g.a[y] >> 1) == x) + ((g.b[y] >> 1) == x);
        return r;
      };
      bool ext = refs[v] > refs_from_cone(v);
      for (uint32_t y : in)
        if (y != C.nodes[j + 1] && (ep[y] || refs[y] > refs_from_cone(y))) ext = true;
      if (ext) is_tap[v] = 1;
    }
  }
  // rebuild in topological order; taps come from each chain's lookahead network
  GraphBuilder B(g);
  std::vector<uint32_t> m(N, 0);
  for (size_t i = 0; i < N; i++)
    if (g.kind[i] != K_AND) m[i] = 2 * (uint32_t)i;
  auto mlit = [&](uint32_t l) { return m[l >> 1] ^ (l & 1u); };
  using Net = decltype(make_net(g, chains[0], B, mlit));
  std::vector<std::unique_ptr<Net>> nets(chains.size());
  for (size_t i = 0; i < N; i++) {
    if (g.kind[i] != K_AND) continue;
    const int c = chain_of[i];
    if (c >= 0) {
      if (is_tap[i]) {
        if (!nets[c]) nets[c].reset(new Net(g, chains[c], B, mlit));
        m[i] = nets[c]->tap((uint32_t)pos_of[i], m[chains[c].c0]);
        st.chain_taps++;
      }
      continue;   // a chain node used only inside the next link's cone is not built
    }
    m[i] = B.AND(mlit(g.a[i]), mlit(g.b[i]));
  }
  st.chains = (uint32_t)chains.size();
  for (auto& C : chains) st.chain_links += (uint32_t)C.nodes.size();
  map_endpoints(g, B.g, m);
  finish_graph(B.g);
  return std::move(B.g);
}

// Compact a graph to its cone of influence (drops unused ANDs, keeps sources).
static Graph prune_graph(const Graph& g) {
  std::vector<uint8_t> live(g.kind.size(), 0);
  auto mark = [&](uint32_t l) { live[l >> 1] = 1; };
  for (auto l : g.flop_next) mark(l);
  for (auto l : g.po) mark(l);
  for (auto& rr : g.rams) for (int p = 0; p < 4; p++) for (int k = 0; k < 32; k++) mark(rr.port[p][k]);
  for (size_t i = g.kind.size(); i-- > 0;)
    if (live[i] && g.kind[i] == K_AND) { live[g.a[i] >> 1] = 1; live[g.b[i] >> 1] = 1; }
  GraphBuilder B(g);
  std::vector<uint32_t> m(g.kind.size(), 0);
  for (size_t i = 0; i < g.kind.size(); i++) {
    if (g.kind[i] != K_AND) { m[i] = 2 * (uint32_t)i; continue; }
    if (!live[i]) continue;
    m[i] = B.AND(m[g.a[i] >> 1] ^ (g.a[i] & 1u), m[g.b[i] >> 1] ^ (g.b[i] & 1u));
  }
  map_endpoints(g, B.g, m);
  finish_graph(B.g);
  return std::move(B.g);
}

static Graph synthesize(const Graph& g, int mode, int chain_min, int chain_slack, SynthStats& st) {
  st.and_in = g.n_and_live;
  st.level_in = g.max_level;
  Graph x = prune_graph(g);
  if (mode >= 1) x = prune_graph(balance_ands(x));
  st.and_balanced = x.n_and_live;
  st.level_balanced = x.max_level;
  if (mode >= 2) x = prune_graph(chain_lookahead(x, chain_min, chain_slack, st));
  st.and_out = x.n_and_live;
  st.level_out = x.max_level;
  return x;
}
