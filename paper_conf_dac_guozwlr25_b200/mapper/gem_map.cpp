// gem_map.cpp -- host-side mapping flow: E-AIG -> VLIW program blob (.gemb).
//
// Follows PAPER.md §III, simplified where SURVEY.md §2 says so:
//   * synthesis (§III-B): the input is already an E-AIG; we only do
//     structural hashing, trivial simplification and cone-of-influence pruning
//     (the commercial depth-optimising synthesiser is out of scope).
//   * partitioning (§III-C): replication-aided (RepCut-style)
//     endpoint clustering.  Endpoints are single flop / PO bits and whole RAM
//     blocks; each partition recomputes the full cone of its endpoints, so
//     partitions never depend on each other inside a cycle.  Clustering
//     is min-hash ordered greedy packing followed by Algorithm 1 merging
//     (P:119-125): try to merge partitions with large overlap, commit if the
//     result is still mappable (here: under the size cap).
//   * multi-stage cut (Fig.5): nodes at a cut level become stage-0
//     endpoints ("cut words") and stage-1 sources.
//   * placement (§III-D, Algorithm 2): iterative layer filling,
//     bottom (1-bit tip, level 13) to top (leaf side), choosing the most
//     timing-critical node (largest reverse depth) of logic level i for
//     a free level-i slot and recursively mapping its fan-in cone into the
//     slot's subtree (bit-mapping primitive); realised values are
//     written out and become leaves of later layers ("remove the nodes
//     already realised ... create a new AIG subgraph").
//   * bitstream generation (§III-E): gem_isa.h encoding.
//
// The mapper shares no code with oracle/.

#include <algorithm>
#include <array>
#include <atomic>
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <cstring>
#include <fstream>
#include <functional>
#include <map>
#include <memory>
#include <set>
#include <mutex>
#include <numeric>
#include <sstream>
#include <stdexcept>
#include <string>
#include <thread>
#include <unordered_map>
#include <unordered_set>
#include <vector>

#include "../csrc/gem_isa.h"

namespace gm {

static thread_local std::string g_err;

// =========================================================== options
struct Options {
  int parts = 0;            // target partition count (0 = auto)
  int part_size = 6000;     // auto target ANDs per partition (paper: 5.7-12.9K, Table I)
  int threads = 0;          // 0 = hardware concurrency
  int leafcap = 320;        // max leaves of one placed root (cost filter)
  int levels = 13;          // deepest boomerang level used per layer (10 = no top levels 11-13)
  int stages = 1;           // 1 or 2 (multi-stage RepCut)
  int cut_level = 0;        // 0 = auto (middle)
  int merge = 1;            // Algorithm 1 merge pass
  int km1 = 8;              // passes of k-way min-cut refinement of the RepCut hypergraph (0 = off)
  int km1_pins = 64;        // hyperedges (shared AND nodes) with more users are left out of the gains
  double km1_slack = 1.1;   // refinement keeps every partition under this x the packing cap
  int key = 0;              // unit order for packing: 0 = min flop index in the cone, 1 = deep-cone
                            // min-hash, 2 = a register's own index (declaration order = module order)
  double merge_cap = 0;     // max merged cone size in ANDs (0 = 2.5 x part_size)
  double merge_ratio = 0.3; // merge only if overlap >= ratio x the smaller cone
  int refine = 3;           // rounds of splitting the costliest partitions (critical path)
  double refine_ratio = 1.35;  // split partitions costing more than this x the median
  int max_parts = 280;      // refinement stops growing the partition count here
  int lanes = 0;            // also emit stream-sliced lane programs (batched streams)
  int lane_words = 16383;   // cap on a lane program's state words (larger partitions are split)
  int max_warps = 8;        // warps that may hold placed roots (8 = all)
  int lane_banks = 1;       // bank-aware placement of lane write-out runs (2: also interior offsets)
  int lane_holes = 32;      // best-fitting holes considered per run
  int lane_k = 4;           // lane mode 2: bank-conflict model for K interleaved groups (K lanes' words
                            // per 16 bytes: lanes of 32/K share one wavefront)
  int lane_m = 1;           // lane mode 2: independent ops per thread and step (1 or 2)
  int words = 0;            // also emit word programs (WRD1, gem_isa.h): the single-stream latency path
  int word_step = 1024;     // word programs: max ops per barrier-separated step
  int word_chain_probe = 0; // analysis: print step counts with per-thread op chains
  int word_local_probe = 0; // analysis: print the share of ops computable before the grid barrier
  int word_sched = 1;       // word programs: 1 = balanced (slack-aware) steps, 0 = greedy ASAP
  int word_fill = GEM_THREADS;  // balanced scheduling: ops per step before slack ops wait
  int word_spread = 0;      // balanced scheduling: every partition spreads over the design depth (measured slower)
  int lane_mode = 2;        // 1: lane program from the boomerang placement ("LANE"); 2: compacted AND
                            // list in barrier-separated steps ("LAN2", gem_isa.h)
  int banks = 1;            // bank-conflict-aware renaming of the state words (rename_state_words)
  int verbose = 0;
  int max_state_words = GEM_MAX_STATE_WORDS;
  double cap_slack = 1.0;
  int synth = 2;            // depth-oriented synthesis (gem_synth.h): 0 strash only, 1 + AND balancing,
                            // 2 + chain lookahead
  int chain_min = 8;        // shortest chain rewritten by the lookahead
  int chain_slack = 2;      // a link's chain edge arrives >= this many levels after its side input
};

static Options parse_opts(const char* s) {
  Options o;
  if (!s) return o;
  std::stringstream ss(s);
  std::string tok;
  while (ss >> tok) {
    size_t eq = tok.find('=');
    if (eq == std::string::npos) throw std::runtime_error("bad option " + tok);
    std::string k = tok.substr(0, eq), v = tok.substr(eq + 1);
    if (k == "parts") o.parts = std::stoi(v);
    else if (k == "part_size") o.part_size = std::stoi(v);
    else if (k == "threads") o.threads = std::stoi(v);
    else if (k == "leafcap") o.leafcap = std::stoi(v);
    else if (k == "levels") o.levels = std::max(5, std::min(13, std::stoi(v)));
    else if (k == "stages") o.stages = std::stoi(v);
    else if (k == "cut_level") o.cut_level = std::stoi(v);
    else if (k == "merge") o.merge = std::stoi(v);
    else if (k == "km1") o.km1 = std::stoi(v);
    else if (k == "km1_pins") o.km1_pins = std::max(2, std::stoi(v));
    else if (k == "km1_slack") o.km1_slack = std::stod(v);
    else if (k == "key") o.key = std::stoi(v);
    else if (k == "merge_cap") o.merge_cap = std::stod(v);
    else if (k == "merge_ratio") o.merge_ratio = std::stod(v);
    else if (k == "verbose") o.verbose = std::stoi(v);
    else if (k == "max_state_words") o.max_state_words = std::stoi(v);
    else if (k == "cap_slack") o.cap_slack = std::stod(v);
    else if (k == "refine") o.refine = std::stoi(v);
    else if (k == "refine_ratio") o.refine_ratio = std::stod(v);
    else if (k == "max_parts") o.max_parts = std::stoi(v);
    else if (k == "lanes") o.lanes = std::stoi(v);
    else if (k == "lane_words") o.lane_words = std::min(16383, std::stoi(v));
    else if (k == "lane_banks") o.lane_banks = std::stoi(v);
    else if (k == "max_warps") o.max_warps = std::max(1, std::min(8, std::stoi(v)));
    else if (k == "lane_holes") o.lane_holes = std::max(1, std::stoi(v));
    else if (k == "lane_mode") o.lane_mode = std::max(1, std::min(2, std::stoi(v)));
    else if (k == "words") o.words = std::stoi(v);
    else if (k == "word_sched") o.word_sched = std::stoi(v);
    else if (k == "word_spread") o.word_spread = std::stoi(v);
    else if (k == "word_fill") o.word_fill = std::max(32, std::min(4 * GEM_THREADS, std::stoi(v)));
    else if (k == "word_local_probe") o.word_local_probe = std::stoi(v);
    else if (k == "word_chain_probe") o.word_chain_probe = std::stoi(v);
    else if (k == "word_step") o.word_step = std::max(32, std::min(4 * GEM_THREADS, std::stoi(v)));
    else if (k == "lane_m") o.lane_m = std::max(1, std::min(2, std::stoi(v)));
    else if (k == "lane_k") o.lane_k = std::stoi(v) >= 4 ? 4 : std::stoi(v) >= 2 ? 2 : 1;
    else if (k == "banks") o.banks = std::stoi(v);
    else if (k == "synth") o.synth = std::stoi(v);
    else if (k == "chain_min") o.chain_min = std::max(2, std::stoi(v));
    else if (k == "chain_slack") o.chain_slack = std::max(1, std::stoi(v));
    else throw std::runtime_error("unknown option " + k);
  }
  if (o.stages < 1 || o.stages > 2) throw std::runtime_error("stages must be 1 or 2");
  if (o.max_state_words > GEM_MAX_STATE_WORDS || o.max_state_words < 64)
    throw std::runtime_error("bad max_state_words");
  return o;
}

// =========================================================== AIGER reader
struct RawRam {
  std::vector<uint64_t> rdata, raddr, waddr, wdata, wbe;
};
struct Raw {
  uint64_t M = 0, I = 0, L = 0, O = 0, A = 0;
  std::vector<uint64_t> lnext;
  std::vector<uint8_t> linit;
  std::vector<uint64_t> outs;
  std::vector<uint64_t> lhs, r0, r1;
  std::vector<RawRam> rams;
};

struct Reader {
  const char* p;
  const char* e;
  bool eof() const { return p >= e; }
  void skip_ws() { while (p < e && (*p == ' ' || *p == '\t' || *p == '\r')) p++; }
  uint64_t num() {
    skip_ws();
    if (p >= e || *p < '0' || *p > '9') throw std::runtime_error("number expected");
    uint64_t x = 0;
    while (p < e && *p >= '0' && *p <= '9') x = x * 10 + (uint64_t)(*p++ - '0');
    return x;
  }
  bool at_eol() { skip_ws(); return p >= e || *p == '\n'; }
  void eol() {
    skip_ws();
    if (p < e && *p != '\n') throw std::runtime_error("end of line expected");
    if (p < e) p++;
  }
  std::string line() {
    const char* s = p;
    while (p < e && *p != '\n') p++;
    std::string r(s, p);
    if (p < e) p++;
    return r;
  }
  uint64_t varint() {
    uint64_t x = 0;
    int sh = 0;
    while (true) {
      if (p >= e) throw std::runtime_error("EOF in binary ANDs");
      uint8_t c = (uint8_t)*p++;
      x |= (uint64_t)(c & 0x7f) << sh;
      if (!(c & 0x80)) return x;
      sh += 7;
      if (sh > 63) throw std::runtime_error("varint overflow");
    }
  }
};

static std::vector<uint64_t> split_nums(const std::string& s) {
  std::vector<uint64_t> r;
  size_t i = 0;
  while (i < s.size()) {
    size_t j = s.find(',', i);
    if (j == std::string::npos) j = s.size();
    r.push_back(std::stoull(s.substr(i, j - i)));
    i = j + 1;
  }
  return r;
}

static Raw read_aiger(const char* data, size_t n) {
  Raw g;
  Reader rd{data, data + n};
  std::string magic;
  while (!rd.eof() && *rd.p != ' ') magic.push_back(*rd.p++);
  bool bin;
  if (magic == "aag") bin = false;
  else if (magic == "aig") bin = true;
  else throw std::runtime_error("not an AIGER file");
  g.M = rd.num(); g.I = rd.num(); g.L = rd.num(); g.O = rd.num(); g.A = rd.num();
  if (!rd.at_eol()) throw std::runtime_error("AIGER B/C/J/F sections are not supported");
  rd.eol();
  if (!bin)
    for (uint64_t i = 0; i < g.I; i++) {
      if (rd.num() != 2 * (i + 1)) throw std::runtime_error("inputs must be 2,4,..");
      rd.eol();
    }
  g.lnext.resize(g.L);
  g.linit.assign(g.L, 0);
  for (uint64_t j = 0; j < g.L; j++) {
    uint64_t cur = 2 * (g.I + 1 + j);
    if (!bin && rd.num() != cur) throw std::runtime_error("latch numbering");
    g.lnext[j] = rd.num();
    if (!rd.at_eol()) {
      uint64_t init = rd.num();
      g.linit[j] = (init == 1) ? 1 : 0;
      if (init != 0 && init != 1 && init != cur) throw std::runtime_error("bad latch init");
    }
    rd.eol();
  }
  g.outs.resize(g.O);
  for (uint64_t k = 0; k < g.O; k++) { g.outs[k] = rd.num(); rd.eol(); }
  g.lhs.resize(g.A); g.r0.resize(g.A); g.r1.resize(g.A);
  if (!bin) {
    for (uint64_t k = 0; k < g.A; k++) {
      g.lhs[k] = rd.num(); g.r0[k] = rd.num(); g.r1[k] = rd.num();
      rd.eol();
    }
  } else {
    for (uint64_t k = 0; k < g.A; k++) {
      uint64_t lhs = 2 * (g.I + g.L + 1 + k);
      uint64_t d0 = rd.varint(), d1 = rd.varint();
      if (d0 > lhs || d1 > lhs - d0) throw std::runtime_error("bad binary delta");
      g.lhs[k] = lhs; g.r0[k] = lhs - d0; g.r1[k] = lhs - d0 - d1;
    }
  }
  bool comments = false;
  while (!rd.eof()) {
    std::string ln = rd.line();
    if (!comments) {
      if (ln == "c" || ln.rfind("c ", 0) == 0) comments = true;
      continue;
    }
    if (ln.rfind("gem-ram ", 0) != 0) continue;
    std::stringstream ss(ln);
    std::string tag, id, f;
    ss >> tag >> id;
    RawRam r;
    while (ss >> f) {
      size_t eq = f.find('=');
      if (eq == std::string::npos) throw std::runtime_error("bad gem-ram");
      std::string k = f.substr(0, eq);
      auto v = split_nums(f.substr(eq + 1));
      if (k == "rdata") r.rdata = v;
      else if (k == "raddr") r.raddr = v;
      else if (k == "waddr") r.waddr = v;
      else if (k == "wdata") r.wdata = v;
      else if (k == "wbe") r.wbe = v;
      else throw std::runtime_error("bad gem-ram key");
    }
    if (r.rdata.size() != 32 || r.raddr.size() != 13 || r.waddr.size() != 13 || r.wdata.size() != 32 ||
        r.wbe.size() != 32)
      throw std::runtime_error("gem-ram port widths must be 32/13/13/32/32");
    g.rams.push_back(r);
  }
  return g;
}

// =========================================================== compact graph
// Node kinds: sources (const, PI, latch, RAM rdata) then ANDs in topological order.
enum : uint8_t { K_CONST = 0, K_SRC = 1, K_AND = 2 };

struct Graph {
  uint32_t n_pi = 0, n_flops = 0, n_po = 0, n_rams = 0;
  std::vector<uint8_t> kind;
  std::vector<uint32_t> a, b;        // AND fanins (compact literals)
  std::vector<uint32_t> gbit;        // sources: region<<27 | word<<5 | bit
  std::vector<uint32_t> level;
  std::vector<uint32_t> flop_next;   // compact literal per flop
  std::vector<uint8_t> flop_init;
  std::vector<uint32_t> po;          // compact literal per PO
  struct Ram { uint32_t port[4][32]; } ;
  std::vector<Ram> rams;             // ports: raddr(13) waddr(13) wdata wbe; missing bits = 0
  uint64_t n_and_live = 0;
  uint32_t max_level = 0;
};

static inline uint32_t mk_gbit(uint32_t region, uint32_t word, uint32_t bit) {
  return (region << 27) | (word << 5) | bit;
}

static Graph build_graph(const Raw& r) {
  Graph g;
  // classify inputs
  std::vector<int64_t> in_ram(r.I, -1), in_bit(r.I, -1);
  for (size_t k = 0; k < r.rams.size(); k++)
    for (int j = 0; j < 32; j++) {
      uint64_t i = r.rams[k].rdata[j];
      if (i >= r.I) throw std::runtime_error("rdata index out of range");
      if (in_ram[i] >= 0) throw std::runtime_error("rdata input owned twice");
      in_ram[i] = (int64_t)k; in_bit[i] = j;
    }
  std::vector<uint32_t> m(r.M + 1, UINT32_MAX);   // orig var -> compact literal
  g.kind.push_back(K_CONST); g.a.push_back(0); g.b.push_back(0); g.gbit.push_back(0); g.level.push_back(0);
  m[0] = 0;
  uint32_t pi = 0;
  for (uint64_t i = 0; i < r.I; i++) {
    uint32_t id = (uint32_t)g.kind.size();
    g.kind.push_back(K_SRC); g.a.push_back(0); g.b.push_back(0); g.level.push_back(0);
    if (in_ram[i] >= 0) g.gbit.push_back(mk_gbit(GEM_R_RD, (uint32_t)in_ram[i], (uint32_t)in_bit[i]));
    else { g.gbit.push_back(mk_gbit(GEM_R_PI, pi / 32, pi % 32)); pi++; }
    m[i + 1] = 2 * id;
  }
  g.n_pi = pi;
  for (uint64_t j = 0; j < r.L; j++) {
    uint32_t id = (uint32_t)g.kind.size();
    g.kind.push_back(K_SRC); g.a.push_back(0); g.b.push_back(0); g.level.push_back(0);
    g.gbit.push_back(mk_gbit(GEM_R_Q, (uint32_t)(j / 32), (uint32_t)(j % 32)));  // external order for now
    m[r.I + 1 + j] = 2 * id;
  }
  // topological order of the original ANDs (Kahn)
  std::vector<int64_t> and_of_var(r.M + 1, -1);
  for (uint64_t k = 0; k < r.A; k++) {
    uint64_t v = r.lhs[k] >> 1;
    if ((r.lhs[k] & 1) || v <= r.I + r.L || v > r.M || and_of_var[v] >= 0)
      throw std::runtime_error("bad AND lhs");
    and_of_var[v] = (int64_t)k;
  }
  std::vector<uint32_t> indeg(r.A, 0);
  std::vector<uint32_t> uoff(r.A + 1, 0);
  for (uint64_t k = 0; k < r.A; k++)
    for (uint64_t l : {r.r0[k], r.r1[k]}) {
      if ((l >> 1) > r.M) throw std::runtime_error("literal out of range");
      int64_t d = and_of_var[l >> 1];
      if (d >= 0) { indeg[k]++; uoff[d + 1]++; }
      else if ((l >> 1) > r.I + r.L) throw std::runtime_error("undefined literal");
    }
  for (uint64_t k = 0; k < r.A; k++) uoff[k + 1] += uoff[k];
  std::vector<uint32_t> users(uoff[r.A]);
  {
    std::vector<uint32_t> fill(uoff.begin(), uoff.end() - 1);
    for (uint64_t k = 0; k < r.A; k++)
      for (uint64_t l : {r.r0[k], r.r1[k]}) {
        int64_t d = and_of_var[l >> 1];
        if (d >= 0) users[fill[d]++] = (uint32_t)k;
      }
  }
  std::vector<uint32_t> q;
  q.reserve(r.A);
  for (uint64_t k = 0; k < r.A; k++) if (!indeg[k]) q.push_back((uint32_t)k);
  std::unordered_map<uint64_t, uint32_t> strash;
  strash.reserve(r.A * 2 + 16);
  for (size_t h = 0; h < q.size(); h++) {
    uint32_t k = q[h];
    uint32_t la = m[r.r0[k] >> 1] ^ (uint32_t)(r.r0[k] & 1);
    uint32_t lb = m[r.r1[k] >> 1] ^ (uint32_t)(r.r1[k] & 1);
    if (la > lb) std::swap(la, lb);
    uint32_t res;
    if (la == 0) res = 0;
    else if (la == 1) res = lb;
    else if (la == lb) res = la;
    else if (la == (lb ^ 1)) res = 0;
    else {
      uint64_t key = ((uint64_t)la << 32) | lb;
      auto it = strash.find(key);
      if (it != strash.end()) res = it->second;
      else {
        uint32_t id = (uint32_t)g.kind.size();
        g.kind.push_back(K_AND); g.a.push_back(la); g.b.push_back(lb); g.gbit.push_back(0);
        g.level.push_back(1 + std::max(g.level[la >> 1], g.level[lb >> 1]));
        res = 2 * id;
        strash.emplace(key, res);
      }
    }
    m[r.lhs[k] >> 1] = res;
    for (uint32_t i = uoff[k]; i < uoff[k + 1]; i++)
      if (--indeg[users[i]] == 0) q.push_back(users[i]);
  }
  if (q.size() != r.A) throw std::runtime_error("combinational loop");
  auto lit = [&](uint64_t l) {
    uint32_t x = m[l >> 1];
    if (x == UINT32_MAX) throw std::runtime_error("undefined literal");
    return x ^ (uint32_t)(l & 1);
  };
  g.n_flops = (uint32_t)r.L;
  g.flop_next.resize(r.L);
  g.flop_init = r.linit;
  for (uint64_t j = 0; j < r.L; j++) g.flop_next[j] = lit(r.lnext[j]);
  g.n_po = (uint32_t)r.O;
  g.po.resize(r.O);
  for (uint64_t k = 0; k < r.O; k++) g.po[k] = lit(r.outs[k]);
  g.n_rams = (uint32_t)r.rams.size();
  for (auto& rr : r.rams) {
    Graph::Ram gr;
    std::memset(&gr, 0, sizeof(gr));
    for (int k = 0; k < 13; k++) gr.port[0][k] = lit(rr.raddr[k]);
    for (int k = 0; k < 13; k++) gr.port[1][k] = lit(rr.waddr[k]);
    for (int k = 0; k < 32; k++) gr.port[2][k] = lit(rr.wdata[k]);
    for (int k = 0; k < 32; k++) gr.port[3][k] = lit(rr.wbe[k]);
    g.rams.push_back(gr);
  }
  // live AND count (cone of influence of all endpoints)
  std::vector<uint8_t> live(g.kind.size(), 0);
  auto mark = [&](uint32_t l) { live[l >> 1] = 1; };
  for (auto l : g.flop_next) mark(l);
  for (auto l : g.po) mark(l);
  for (auto& rr : g.rams) for (int p = 0; p < 4; p++) for (int k = 0; k < 32; k++) mark(rr.port[p][k]);
  for (size_t i = g.kind.size(); i-- > 0;)
    if (live[i] && g.kind[i] == K_AND) { live[g.a[i] >> 1] = 1; live[g.b[i] >> 1] = 1; }
  for (size_t i = 0; i < g.kind.size(); i++)
    if (live[i] && g.kind[i] == K_AND) { g.n_and_live++; g.max_level = std::max(g.max_level, g.level[i]); }
  return g;
}

#include "gem_synth.h"

// =========================================================== partition description
// An output word: destination gid + 32 compact literals (bit k of the word).
struct OutWord {
  uint32_t dst;            // gid (region<<24 | index); RAMP index filled at encode time
  uint32_t lit[32];
};

struct Unit {              // a partitioning unit
  int kind;                // 0 flop bit, 1 PO bit, 2 RAM block, 3 cut bit
  uint32_t idx;            // flop / po / ram / cut index
  uint64_t key;            // locality sort key
};

struct Part {
  int stage = 0;
  std::vector<uint32_t> flops, pos, rams, cuts;   // endpoints owned
  // filled by the layout step
  std::vector<OutWord> outs;
  // filled by mapping
  std::vector<uint32_t> prog;
  std::vector<uint32_t> lane_prog;   // lane-mode program (opt.lanes)
  std::vector<uint32_t> word_prog;   // word program (opt.words; empty if it does not fit)
  uint32_t word_steps = 0, word_ops = 0;
  uint32_t lane_words = 0;
  uint32_t n_layers = 0, n_nodes = 0, state_words = 0, n_leaves = 0, max_level = 0, n_writeouts = 0;
  uint64_t slots_used = 0;
  bool ok = false;
  std::string err;
};

// =========================================================== placement (Algorithm 2)
static inline uint32_t group_width(int k) {      // slots per unit at level k
  if (k <= 5) return 1u << (5 - k);
  if (k <= 10) return 1u << (10 - k);
  return 1u << (13 - k);
}
static inline uint32_t level_slots(int k) { return 8192u >> k; }
static inline uint32_t child_a(int k, uint32_t id) {
  uint32_t g = group_width(k);
  return (id / g) * 2 * g + (id % g);
}
static inline uint32_t child_b(int k, uint32_t id) { return child_a(k, id) + group_width(k); }
static const int kOff[6] = {0, GEM_OFF_L1, GEM_OFF_L2, GEM_OFF_L3, GEM_OFF_L4, GEM_OFF_L5};
// unit (thread for 1..5, warp for 6..10, 0 for 11..13) and packed bit of slot (k,id)
static inline uint32_t slot_unit(int k, uint32_t id) { return k >= 11 ? 0 : id / group_width(k); }
static inline uint32_t slot_bit(int k, uint32_t id) {
  if (k >= 11) return (k == 11 ? 0 : k == 12 ? 4 : 6) + id;
  int kk = k <= 5 ? k : k - 5;
  return (uint32_t)kOff[kk] + id % group_width(k);
}

// packed constant word of a unit (thread: levels 1-5, warp: 6-10, top: 11-13)
static uint32_t pack_unit(int k0, int k1, uint32_t unit, const std::vector<uint8_t>* arr) {
  uint32_t v = 0;
  for (int k = k0; k <= k1; k++) {
    uint32_t g = group_width(k);
    for (uint32_t q = 0; q < g; q++) {
      uint32_t id = unit * g + q;
      if (arr[k][id]) v |= 1u << slot_bit(k, id);
    }
  }
  return v;
}

// per-layer record for the lane-mode encoding
struct LaneLayer {
  std::vector<uint32_t> leaf_sig;                   // 8192 leaves: local signal or UINT32_MAX
  std::vector<std::array<uint32_t, 3>> two, wwo;    // {thread|warp, slot bit, signal}
  std::vector<std::array<uint32_t, 2>> top;         // {slot bit, signal}
  std::vector<uint32_t> cth;                        // 256 x {xa, xb, ob}
  uint32_t cw[8][3];
  uint32_t topc;
};

struct Mapper {
  const Graph& G;
  const Options& opt;
  explicit Mapper(const Graph& g, const Options& o) : G(g), opt(o) {}

  // local graph
  std::vector<uint32_t> cid;          // local -> compact id
  std::vector<uint8_t> is_src;
  std::vector<uint32_t> la, lb;       // local literals
  std::vector<uint32_t> coff, cons;   // consumers CSR
  std::vector<uint8_t> is_ep;         // referenced by an output word
  std::vector<int32_t> loc;           // realised: state bit, or -1

  void map(Part& P, std::vector<int32_t>& scratch) {
    // ---- collect the cone (compact ids), sorted = topological
    std::vector<uint32_t> stack, nodes;
    auto visit = [&](uint32_t c) {
      if (scratch[c] >= 0) return;
      scratch[c] = 0;
      stack.push_back(c);
      while (!stack.empty()) {
        uint32_t x = stack.back();
        stack.pop_back();
        nodes.push_back(x);
        if (G.kind[x] == K_AND)
          for (uint32_t y : {G.a[x] >> 1, G.b[x] >> 1})
            if (scratch[y] < 0) { scratch[y] = 0; stack.push_back(y); }
      }
    };
    visit(0);   // constant always present (padding / constant outputs)
    for (auto& ow : P.outs) for (int k = 0; k < 32; k++) visit(ow.lit[k] >> 1);
    std::sort(nodes.begin(), nodes.end());
    struct Cleanup {
      std::vector<uint32_t>& nodes; std::vector<int32_t>& scratch;
      ~Cleanup() { for (uint32_t c : nodes) scratch[c] = -1; }
    } cleanup{nodes, scratch};
    uint32_t n = (uint32_t)nodes.size();
    for (uint32_t i = 0; i < n; i++) scratch[nodes[i]] = (int32_t)i;
    cid = nodes;
    is_src.assign(n, 0); la.assign(n, 0); lb.assign(n, 0); is_ep.assign(n, 0); loc.assign(n, -1);
    std::vector<uint32_t> cnt(n + 1, 0);
    uint32_t n_and = 0;
    for (uint32_t i = 0; i < n; i++) {
      uint32_t c = nodes[i];
      if (G.kind[c] != K_AND) { is_src[i] = 1; continue; }
      n_and++;
      la[i] = 2 * (uint32_t)scratch[G.a[c] >> 1] | (G.a[c] & 1);
      lb[i] = 2 * (uint32_t)scratch[G.b[c] >> 1] | (G.b[c] & 1);
      cnt[(la[i] >> 1) + 1]++;
      cnt[(lb[i] >> 1) + 1]++;
    }
    coff.assign(n + 1, 0);
    for (uint32_t i = 0; i < n; i++) coff[i + 1] = coff[i] + cnt[i + 1];
    cons.assign(coff[n], 0);
    {
      std::vector<uint32_t> f(coff.begin(), coff.end() - 1);
      for (uint32_t i = 0; i < n; i++)
        if (!is_src[i]) { cons[f[la[i] >> 1]++] = i; cons[f[lb[i] >> 1]++] = i; }
    }
    for (auto& ow : P.outs) for (int k = 0; k < 32; k++) is_ep[(uint32_t)scratch[ow.lit[k] >> 1]] = 1;
    P.n_nodes = n_and;

    // ---- state: word 0 = const 0; gread words next, in ascending global word
    // order so that a warp's 32 port loads fall into few L2 sectors (a2)
    std::vector<uint32_t> gread_src;     // gid per gread
    std::unordered_map<uint32_t, uint32_t> gword;   // gid -> state word
    uint32_t sw_next = 1;
    std::vector<uint32_t> word_live;     // live realised values per state word
    for (uint32_t i = 0; i < n; i++) {
      if (!is_src[i]) continue;
      uint32_t c = nodes[i];
      if (G.kind[c] == K_CONST) continue;
      uint32_t gb = G.gbit[c];
      uint32_t gid = GEM_GID(gb >> 27, (gb >> 5) & 0x3FFFFF);
      if (gword.emplace(gid, 0u).second) gread_src.push_back(gid);
    }
    std::sort(gread_src.begin(), gread_src.end());
    for (uint32_t gid : gread_src) gword[gid] = sw_next++;
    for (uint32_t i = 0; i < n; i++) {
      if (!is_src[i]) continue;
      uint32_t c = nodes[i];
      if (G.kind[c] == K_CONST) { loc[i] = 0; continue; }
      uint32_t gb = G.gbit[c];
      uint32_t gid = GEM_GID(gb >> 27, (gb >> 5) & 0x3FFFFF);
      loc[i] = (int32_t)(gword[gid] * 32 + (gb & 31));
    }
    uint32_t n_gread = sw_next - 1;
    if (sw_next > (uint32_t)opt.max_state_words) { fail(P, "too many gread words"); return; }
    word_live.assign(opt.max_state_words, 0);

    // ---- liveness helpers
    std::vector<uint8_t> mc(n, 0);            // must compute
    auto compute_mc = [&]() {
      for (uint32_t i = n; i-- > 0;) {
        mc[i] = 0;
        if (is_src[i] || loc[i] >= 0) continue;
        if (is_ep[i]) { mc[i] = 1; continue; }
        for (uint32_t j = coff[i]; j < coff[i + 1]; j++)
          if (mc[cons[j]]) { mc[i] = 1; break; }
      }
    };
    auto value_live = [&](uint32_t i) {      // realised i still needed?
      if (is_ep[i]) return true;
      for (uint32_t j = coff[i]; j < coff[i + 1]; j++)
        if (mc[cons[j]]) return true;
      return false;
    };
    compute_mc();
    // live counts for gread words
    std::vector<std::vector<uint32_t>> word_vals(opt.max_state_words);
    for (uint32_t i = 0; i < n; i++)
      if (is_src[i] && loc[i] > 0) word_vals[(uint32_t)loc[i] >> 5].push_back(i);
    std::vector<uint8_t> word_used(opt.max_state_words, 0);
    word_used[0] = 1;
    for (uint32_t w = 1; w < sw_next; w++) word_used[w] = 1;
    std::vector<uint32_t> free_words;
    auto refresh_free = [&]() {
      // a used word becomes free when none of its values is live
      for (uint32_t w = 1; w < (uint32_t)opt.max_state_words; w++) {
        if (!word_used[w]) continue;
        bool live = false;
        for (uint32_t i : word_vals[w]) if (value_live(i)) { live = true; break; }
        if (!live) { word_used[w] = 0; word_vals[w].clear(); free_words.push_back(w); }
      }
    };
    for (uint32_t w = (uint32_t)opt.max_state_words; w-- > sw_next;) free_words.push_back(w);
    refresh_free();
    // keep free words sorted descending so pop_back gives the lowest index
    auto sort_free = [&]() { std::sort(free_words.begin(), free_words.end(), std::greater<uint32_t>()); };
    sort_free();

    std::vector<uint32_t> d(n, 0), rd(n, 0), lf(n, 0);
    std::vector<uint32_t> prog_layers;
    uint32_t n_layers = 0, total_leaves = 0, total_wo = 0, max_state = sw_next;
    uint64_t slots_used = 0;
    // per-layer slot arrays
    std::vector<int32_t> slot[14];
    std::vector<uint8_t> sxa[14], sxb[14], sob[14];
    for (int k = 0; k <= 13; k++) {
      slot[k].assign(level_slots(k), -1);
      sxa[k].assign(level_slots(k), 0); sxb[k].assign(level_slots(k), 0); sob[k].assign(level_slots(k), 0);
    }
    std::vector<int32_t> comp_k(n, -1), comp_id(n, -1);   // one computed copy per node
    std::vector<uint32_t> computed;
    std::vector<uint32_t> thread_leaves(256, 0);
    std::vector<LaneLayer> lane_layers;
    std::vector<uint32_t> lleaf(opt.lanes ? 8192 : 0, UINT32_MAX);

    while (true) {
      // any work left?
      bool any = false;
      for (uint32_t i = 0; i < n; i++) if (mc[i]) { any = true; break; }
      if (!any) break;
      // chunk table limit of the runtime (gem_isa.h GEM_MAX_CHUNKS = layers + 2):
      // a failing partition is split by the caller
      if (n_layers + 2 >= GEM_MAX_CHUNKS) { fail(P, "more than GEM_MAX_CHUNKS - 2 layers"); return; }
      // depth over realised set, reverse depth, leaf cost
      for (uint32_t i = 0; i < n; i++) {
        if (!mc[i]) continue;
        uint32_t a = la[i] >> 1, b = lb[i] >> 1;
        uint32_t da = loc[a] >= 0 ? 0 : d[a], db = loc[b] >= 0 ? 0 : d[b];
        d[i] = 1 + std::max(da, db);
        uint32_t fa = loc[a] >= 0 ? 1 : lf[a], fb = loc[b] >= 0 ? 1 : lf[b];
        lf[i] = std::min<uint32_t>(1u << 24, fa + fb);
      }
      for (uint32_t i = n; i-- > 0;) {
        if (!mc[i]) continue;
        uint32_t r = 0;
        for (uint32_t j = coff[i]; j < coff[i + 1]; j++)
          if (mc[cons[j]]) r = std::max(r, rd[cons[j]] + 1);
        rd[i] = r;
      }
      if (opt.verbose >= 4) {
        uint32_t rem = 0, left = 0, lv1 = 0;
        for (uint32_t i = 0; i < n; i++)
          if (mc[i]) { rem = std::max(rem, d[i] + rd[i]); left++; lv1 += d[i] <= (uint32_t)opt.levels; }
        fprintf(stderr, "gem_map: part %p layer %u: remaining depth %u, %u nodes left (%u within reach)\n",
                (void*)&P, n_layers, rem, left, lv1);
      }
      // candidates per level
      std::vector<uint32_t> cand[14];
      for (uint32_t i = 0; i < n; i++)
        if (mc[i] && d[i] <= (uint32_t)opt.levels) cand[d[i]].push_back(i);
      for (int k = 1; k <= 13; k++)
        std::sort(cand[k].begin(), cand[k].end(), [&](uint32_t x, uint32_t y) {
          if (rd[x] != rd[y]) return rd[x] > rd[y];
          if (lf[x] != lf[y]) return lf[x] < lf[y];
          return x < y;
        });
      // reset slots
      for (int k = 0; k <= 13; k++) {
        std::fill(slot[k].begin(), slot[k].end(), -1);
        std::fill(sxa[k].begin(), sxa[k].end(), 0);
        std::fill(sxb[k].begin(), sxb[k].end(), 0);
        std::fill(sob[k].begin(), sob[k].end(), 0);
      }
      std::fill(thread_leaves.begin(), thread_leaves.end(), 0);
      if (opt.lanes) std::fill(lleaf.begin(), lleaf.end(), UINT32_MAX);
      for (uint32_t i : computed) { comp_k[i] = -1; comp_id[i] = -1; }
      computed.clear();
      uint32_t layer_leaves = 0;

      // recursive placement (explicit stack)
      std::function<void(uint32_t, int, uint32_t)> place_lit;
      std::function<void(uint32_t, int, uint32_t)> place_node = [&](uint32_t x, int k, uint32_t id) {
        // pass-throughs above x down to level d[x]
        while (k > (int)d[x]) {
          slot[k][id] = -2; sob[k][id] = 1;
          id = child_a(k, id);
          k--;
        }
        slot[k][id] = (int32_t)x;
        sxa[k][id] = (uint8_t)(la[x] & 1);
        sxb[k][id] = (uint8_t)(lb[x] & 1);
        if (comp_k[x] < 0) { comp_k[x] = k; comp_id[x] = (int32_t)id; computed.push_back(x); }
        place_lit(la[x], k - 1, child_a(k, id));
        place_lit(lb[x], k - 1, child_b(k, id));
      };
      place_lit = [&](uint32_t l, int k, uint32_t id) {
        uint32_t x = l >> 1;
        if (loc[x] >= 0) {
          while (k > 0) { slot[k][id] = -2; sob[k][id] = 1; id = child_a(k, id); k--; }
          slot[0][id] = loc[x];
          if (opt.lanes) lleaf[id] = x;
          thread_leaves[id >> 5]++;
          layer_leaves++;
        } else {
          place_node(x, k, id);
        }
      };
      // bottom (tip, level 13) to top (leaf side)
      for (int k = opt.levels; k >= 1; k--) {
        if (cand[k].empty()) continue;
        // free slots at level k, interleaved over units to spread leaves
        std::vector<uint32_t> fs;
        uint32_t g = group_width(k), units = level_slots(k) / g;
        std::vector<uint32_t> unit_order(units);
        std::iota(unit_order.begin(), unit_order.end(), 0);
        if (k <= 5) {
          // thread order interleaved across warps, least-loaded first
          std::stable_sort(unit_order.begin(), unit_order.end(), [&](uint32_t a, uint32_t b) {
            if (thread_leaves[a] != thread_leaves[b]) return thread_leaves[a] < thread_leaves[b];
            uint32_t ka = (a % 32) * 8 + a / 32, kb = (b % 32) * 8 + b / 32;
            return ka < kb;
          });
        }
        // max_warps < 8: roots only in the first max_warps warps (a small
        // design's layers then run in one warp: no cross-warp wait per layer)
        if (opt.max_warps < 8) {
          auto warp_of = [&](uint32_t u) { return k <= 5 ? u / 32 : k <= 10 ? u : 0u; };
          unit_order.erase(std::remove_if(unit_order.begin(), unit_order.end(),
                                          [&](uint32_t u) { return k > 10 || warp_of(u) >= (uint32_t)opt.max_warps; }),
                           unit_order.end());
        }
        for (uint32_t q = 0; q < g; q++)
          for (uint32_t u : unit_order)
            if (slot[k][u * g + q] == -1) fs.push_back(u * g + q);
        size_t ci = 0;
        for (uint32_t id : fs) {
          // next admissible candidate
          while (ci < cand[k].size()) {
            uint32_t x = cand[k][ci];
            if (comp_k[x] >= 0) { ci++; continue; }           // already computed in this layer
            if (lf[x] > (uint32_t)opt.leafcap) { ci++; continue; }   // cost filter
            break;
          }
          if (ci >= cand[k].size()) break;
          uint32_t x = cand[k][ci++];
          place_node(x, k, id);

        }
      }
      if (computed.empty()) { fail(P, "empty layer"); return; }
      // ---- write-outs: computed values needed by later layers or endpoints
      std::vector<uint8_t> in_c(0);
      // mark computed set
      std::vector<uint32_t> need_wo;
      for (uint32_t x : computed) {
        bool need = is_ep[x];
        if (!need)
          for (uint32_t j = coff[x]; j < coff[x + 1]; j++) {
            uint32_t c = cons[j];
            if (mc[c] && comp_k[c] < 0) { need = true; break; }
          }
        if (need) need_wo.push_back(x);
      }
      // units with a write-out: thread t (levels 1-5), warp w (6-10), top (11-13)
      std::vector<int32_t> wo_thread(256, -1), wo_warp(8, -1);
      int32_t wo_top = -1;
      auto alloc = [&]() -> int32_t {
        if (free_words.empty()) return -1;
        uint32_t w = free_words.back();
        free_words.pop_back();
        word_used[w] = 1;
        return (int32_t)w;
      };
      for (uint32_t x : need_wo) {
        int k = comp_k[x];
        uint32_t id = (uint32_t)comp_id[x];
        int32_t* tgt = k <= 5 ? &wo_thread[slot_unit(k, id)] : k <= 10 ? &wo_warp[slot_unit(k, id)] : &wo_top;
        if (*tgt < 0) { *tgt = alloc(); total_wo++; }
        if (*tgt < 0) { fail(P, "state overflow"); return; }
        loc[x] = (int32_t)((uint32_t)*tgt * 32 + slot_bit(k, id));
        word_vals[(uint32_t)*tgt].push_back(x);
      }
      if (opt.verbose >= 2) {
        uint32_t nwo = 0;
        for (auto x : wo_thread) nwo += x >= 0;
        for (auto x : wo_warp) nwo += x >= 0;
        uint32_t nmc = 0;
        for (uint32_t i = 0; i < n; i++) nmc += mc[i];
        int topk = 0;
        for (int k = 13; k >= 1 && !topk; k--) for (auto v : slot[k]) if (v >= 0) { topk = k; break; }
        uint32_t maxrd = 0, maxd = 0;
        for (uint32_t i = 0; i < n; i++) if (mc[i]) { maxrd = std::max(maxrd, rd[i]); maxd = std::max(maxd, d[i]); }
        fprintf(stderr, "  part %p layer %u: mc=%u computed=%zu need_wo=%zu wo_words=%u leaves=%u free=%zu top_level=%d "
                "max_rd=%u max_d=%u\n", (void*)&P, n_layers, nmc, computed.size(), need_wo.size(), nwo, layer_leaves,
                free_words.size(), topk, maxrd, maxd);
      }
      // ---- lane-mode record of this layer (same placement, signal-level view)
      if (opt.lanes) {
        LaneLayer LL;
        LL.leaf_sig = lleaf;
        for (uint32_t x : need_wo) {
          int k = comp_k[x];
          uint32_t id = (uint32_t)comp_id[x];
          if (k <= 5) LL.two.push_back({slot_unit(k, id), slot_bit(k, id), x});
          else if (k <= 10) LL.wwo.push_back({slot_unit(k, id), slot_bit(k, id), x});
          else LL.top.push_back({slot_bit(k, id), x});
        }
        LL.cth.resize(256 * 3);
        for (uint32_t t = 0; t < 256; t++) {
          LL.cth[3 * t] = pack_unit(1, 5, t, sxa);
          LL.cth[3 * t + 1] = pack_unit(1, 5, t, sxb);
          LL.cth[3 * t + 2] = pack_unit(1, 5, t, sob);
        }
        for (uint32_t w = 0; w < 8; w++) {
          LL.cw[w][0] = pack_unit(6, 10, w, sxa);
          LL.cw[w][1] = pack_unit(6, 10, w, sxb);
          LL.cw[w][2] = pack_unit(6, 10, w, sob);
        }
        LL.topc = pack_unit(11, 13, 0, sxa) | (pack_unit(11, 13, 0, sxb) << 8) | (pack_unit(11, 13, 0, sob) << 16);
        lane_layers.push_back(std::move(LL));
      }
      // ---- encode the layer
      encode_layer(prog_layers, slot, sxa, sxb, sob, wo_thread, wo_warp, wo_top);
      n_layers++;
      total_leaves += layer_leaves;
      for (int k = 1; k <= 13; k++) for (auto s : slot[k]) if (s != -1) slots_used++;
      // ---- advance: recompute must-compute set, free dead words
      compute_mc();
      refresh_free();
      sort_free();
      uint32_t hi = 0;
      for (uint32_t w = 0; w < (uint32_t)opt.max_state_words; w++) if (word_used[w]) hi = w;
      max_state = std::max(max_state, hi + 1);
    }
    // every endpoint must be realised now
    for (uint32_t i = 0; i < n; i++)
      if (is_ep[i] && loc[i] < 0) { fail(P, "unrealised endpoint"); return; }
    // ---- assemble the partition program
    std::vector<uint32_t>& pr = P.prog;
    pr.assign(PH_WORDS, 0);
    pr[PH_MAGIC] = GEM_PART_MAGIC;
    pr[PH_N_GREAD] = n_gread;
    pr[PH_N_LAYERS] = n_layers;
    pr[PH_N_OUT] = (uint32_t)P.outs.size();
    pr[PH_N_RAM] = (uint32_t)P.rams.size();
    // chunk table: [chunk0 | layers... | out+ram]
    pr[PH_OFF_CHUNKS] = (uint32_t)pr.size();
    pr[PH_N_CHUNKS] = n_layers + 2;
    for (uint32_t k = 0; k < n_layers + 2; k++) pr.push_back(0);
    while (pr.size() % 4) pr.push_back(0);
    pr[PH_OFF_GREAD] = (uint32_t)pr.size();
    for (uint32_t k = 0; k < n_gread; k++) { pr.push_back(gread_src[k]); pr.push_back(k + 1); }
    while (pr.size() % 4) pr.push_back(0);
    pr[PH_OFF_LAYERS] = (uint32_t)pr.size();
    pr[pr[PH_OFF_CHUNKS]] = (uint32_t)pr.size();
    {
      size_t off = 0;
      for (uint32_t l = 0; l < n_layers; l++) {
        pr[pr[PH_OFF_CHUNKS] + 1 + l] = prog_layers[off + LH_WORDS_];
        off += prog_layers[off + LH_WORDS_];
      }
    }
    // record directories (gem_isa.h): layer l+1's into layer l's header, layer 0's into chunk 0
    {
      std::vector<std::array<uint32_t, 4>> dirs(n_layers);
      size_t off = 0;
      for (uint32_t l = 0; l < n_layers; l++) {
        std::array<uint32_t, 4> d{0, 0, 0, 0};
        for (uint32_t w = 0; w < 8; w++) {
          const uint32_t wo = prog_layers[off + LH_WOFF0 + w];
          if (!wo) continue;
          const uint32_t mw = prog_layers[off + wo + 4], mode = mw & 0xFFu, n4 = mw >> 8;
          const uint32_t cls = mode == GEM_WM_DENSE16 ? GEM_DC_DENSE16 : mode == GEM_WM_DENSE ? GEM_DC_DENSE
                               : std::max<uint32_t>(1u, n4);
          if (cls > GEM_DC_DENSE || (mode == GEM_WM_SPARSE && n4 > 8))
            throw std::runtime_error("warp record class not encodable");
          if (wo % 4 || wo >= (1u << 14)) throw std::runtime_error("warp record offset not encodable");
          d[w >> 1] |= GEM_DIR_ENTRY(wo, cls) << (16 * (w & 1));
        }
        dirs[l] = d;
        off += prog_layers[off + LH_WORDS_];
      }
      off = 0;
      for (uint32_t l = 0; l + 1 < n_layers; l++) {
        for (int k = 0; k < 4; k++) prog_layers[off + LH_NEXTDIR + k] = dirs[l + 1][k];
        off += prog_layers[off + LH_WORDS_];
      }
      // chunk 0: the layer-0 directory right before the layer records (after the gread list)
      pr[PH_OFF_DIR0] = (uint32_t)pr.size();
      for (int k = 0; k < 4; k++) pr.push_back(n_layers ? dirs[0][k] : 0u);
      pr[PH_OFF_LAYERS] = (uint32_t)pr.size();
      pr[pr[PH_OFF_CHUNKS]] = (uint32_t)pr.size();
    }
    pr.insert(pr.end(), prog_layers.begin(), prog_layers.end());
    pr[PH_OFF_OUT] = (uint32_t)pr.size();
    uint32_t n_out = (uint32_t)P.outs.size(), n_out_pad = (n_out + 3) & ~3u;
    pr[PH_N_OUT_PAD] = n_out_pad;
    for (uint32_t j = 0; j < n_out_pad; j++) pr.push_back(j < n_out ? P.outs[j].dst : 0);
    for (uint32_t j = 0; j < n_out; j++)
      for (int k = 0; k < 32; k++) {
        uint32_t l = P.outs[j].lit[k];
        uint32_t x = (uint32_t)scratch[l >> 1];
        pr.push_back((uint32_t)loc[x] | ((l & 1) ? GEM_OUT_INV : 0u));
      }
    pr[PH_OFF_RAM] = (uint32_t)pr.size();
    for (uint32_t r : P.rams) { pr.push_back(r); pr.push_back(0); pr.push_back(0); pr.push_back(0); }
    while (pr.size() % 4) pr.push_back(0);
    pr[pr[PH_OFF_CHUNKS] + 1 + n_layers] = (uint32_t)pr.size() - pr[PH_OFF_OUT];
    pr[PH_STATE_WORDS] = max_state;
    if (opt.banks) max_state = rename_state_words(pr, (uint32_t)opt.max_state_words);
    pr[PH_N_LEAVES] = total_leaves;
    pr[PH_N_NODES] = n_and;
    // used-bit mask of every gread word (gem_isa.h: the last ceil4(n_gread)
    // words of the program, outside the chunks; read by GEM_F_ACTIVITY only)
    {
      std::vector<uint32_t> gmask(n_gread, 0u);
      for (uint32_t i = 0; i < n; i++) {
        if (!is_src[i]) continue;
        uint32_t c = nodes[i];
        if (G.kind[c] == K_CONST) continue;
        uint32_t gb = G.gbit[c];
        gmask[gword[GEM_GID(gb >> 27, (gb >> 5) & 0x3FFFFF)] - 1] |= 1u << (gb & 31);
      }
      pr.insert(pr.end(), gmask.begin(), gmask.end());
      while (pr.size() % 4) pr.push_back(0);
    }
    P.n_layers = n_layers;
    P.state_words = max_state;
    P.n_leaves = total_leaves;
    P.n_writeouts = total_wo;
    P.slots_used = slots_used;
    if (opt.lanes && opt.lane_mode == 1 && !encode_lanes(P, lane_layers, gread_src, scratch)) return;
    if (opt.lanes && opt.lane_mode == 2 && !encode_lanes2(P, scratch)) return;
    if (opt.words) encode_words(P, scratch);
    P.ok = true;
  }

  // Bank-conflict-aware bit placement (the paper's placement minimises shared-
  // memory bank conflicts of the permutation).  A
  // state word w lives in bank w mod 32, and one gather LDS (entry j of the 32
  // lanes of a warp) costs as many shared-memory wavefronts as the most
  // crowded bank holds distinct words.  The mapper allocated words by
  // liveness only; this pass renames them with a bijection on [1, M)
  // (M = min(state words, 2048) rounded up to a bank row, so DENSE16 entries
  // stay valid; word 0, the constant, and words >= 2048 keep their index),
  // chosen greedily so that words read together fall into different banks.
  // Renaming a physical word for the whole program is always legal: every
  // read and write of it moves together.  Returns the new state word count.
  static uint32_t rename_state_words(std::vector<uint32_t>& pr, uint32_t max_words) {
    const uint32_t N = pr[PH_STATE_WORDS];
    const uint32_t M = std::min<uint32_t>(N, 2048u);
    // two spare rows per bank give the local search room to move words
    const uint32_t Mp = N <= 2048u ? std::min<uint32_t>({2048u, max_words, ((M + 31u) & ~31u) + 64u}) : 2048u;
    if (M <= 2) return N;
    // ---- access groups (one per warp-wide shared-memory instruction)
    std::vector<std::vector<uint16_t>> groups;
    std::vector<uint16_t> g;
    auto close = [&]() {
      std::sort(g.begin(), g.end());
      g.erase(std::unique(g.begin(), g.end()), g.end());
      if (g.size() > 1) groups.push_back(g);
      g.clear();
    };
    auto add = [&](uint32_t w) { g.push_back((uint16_t)(w < M ? w : 0xFFFFu)); };  // >= M: fixed word
    const uint32_t n_layers = pr[PH_N_LAYERS];
    const uint32_t* ct = pr.data() + pr[PH_OFF_CHUNKS];
    uint32_t L = pr[PH_OFF_LAYERS];
    for (uint32_t l = 0; l < n_layers; l++) {
      for (uint32_t w = 0; w < 8; w++) {
        const uint32_t wo = pr[L + LH_WOFF0 + w];
        if (!wo) continue;
        const uint32_t rec = L + wo, mode = pr[rec + 4] & 0xFFu, n4 = pr[rec + 4] >> 8;
        const uint32_t lv = rec + GEM_WREC_HDR + 128;
        for (uint32_t gg = 0; gg < n4; gg++)
          for (uint32_t c = 0; c < 4; c++) {
            if (mode == GEM_WM_DENSE16) {
              for (uint32_t h = 0; h < 2; h++) {
                for (uint32_t ln = 0; ln < 32; ln++) add(GEM_LEAF16_WORD(pr[lv + (gg * 32 + ln) * 4 + c] >> (16 * h)));
                close();
              }
            } else {
              for (uint32_t ln = 0; ln < 32; ln++) add(GEM_LEAF_WORD(pr[lv + (gg * 32 + ln) * 4 + c]));
              close();
            }
          }
        // thread write-outs (one STS per lane)
        for (uint32_t ln = 0; ln < 32; ln++) {
          const uint32_t x = pr[rec + GEM_WREC_HDR + 4 * ln + 3];
          if (x) add(x);
        }
        close();
      }
      L += ct[1 + l];
    }
    // input ports (32 consecutive entries per STS) and endpoint gathers
    const uint32_t ng = pr[PH_N_GREAD], og = pr[PH_OFF_GREAD];
    for (uint32_t k = 0; k < ng; k++) {
      add(pr[og + 2 * k + 1]);
      if (k % 32 == 31 || k + 1 == ng) close();
    }
    const uint32_t no = pr[PH_N_OUT], oo = pr[PH_OFF_OUT] + pr[PH_N_OUT_PAD];
    for (uint32_t o = 0; o < no; o++) {
      for (uint32_t k = 0; k < 32; k++) add((pr[oo + o * 32 + k] & 0x7FFFFFFFu) >> 5);
      close();
    }
    // ---- greedy bank assignment, busiest words first
    const uint32_t G = (uint32_t)groups.size();
    std::vector<std::vector<uint32_t>> of(M);   // groups of each word
    for (uint32_t k = 0; k < G; k++)
      for (uint16_t w : groups[k])
        if (w != 0xFFFFu) of[w].push_back(k);
    std::vector<uint8_t> cnt((size_t)G * 32, 0), mx(G, 0);
    // word 0 (the constant) is fixed in bank 0; fixed words >= M are ignored
    for (uint32_t k = 0; k < G; k++)
      for (uint16_t w : groups[k])
        if (w == 0) { cnt[(size_t)k * 32] = 1; mx[k] = 1; }
    std::vector<uint32_t> cap(32, 0);
    for (uint32_t p = 1; p < Mp; p++) cap[p & 31]++;
    std::vector<uint32_t> order;
    for (uint32_t w = 1; w < M; w++) order.push_back(w);
    std::stable_sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) { return of[a].size() > of[b].size(); });
    std::vector<int32_t> bank(M, -1);
    bank[0] = 0;
    std::vector<uint32_t> used(32, 0);
    for (uint32_t w : order) {
      int best = -1;
      uint64_t best_key = UINT64_MAX;
      for (uint32_t b = 0; b < 32; b++) {
        if (used[b] >= cap[b]) continue;
        uint32_t delta = 0, load = 0;
        for (uint32_t k : of[w]) {
          const uint32_t c = cnt[(size_t)k * 32 + b];
          if (c + 1u > mx[k]) delta++;
          load += c;
        }
        const uint64_t key = ((uint64_t)delta << 40) | ((uint64_t)load << 16) | used[b];
        if (key < best_key) { best_key = key; best = (int)b; }
      }
      bank[w] = best;
      used[best]++;
      for (uint32_t k : of[w]) {
        uint8_t& c = cnt[(size_t)k * 32 + best];
        c++;
        mx[k] = std::max(mx[k], c);
      }
    }
    // ---- local search: move a word to the bank that lowers the wavefront count
    auto regroup_max = [&](uint32_t k) {
      uint8_t m = 0;
      for (uint32_t b = 0; b < 32; b++) m = std::max(m, cnt[(size_t)k * 32 + b]);
      mx[k] = m;
    };
    for (int pass = 0; pass < 4; pass++) {
      uint32_t moved = 0;
      for (uint32_t w : order) {
        const uint32_t a = (uint32_t)bank[w];
        if (of[w].empty()) continue;
        for (uint32_t k : of[w]) { cnt[(size_t)k * 32 + a]--; regroup_max(k); }
        // cost of w's groups with w in bank b = sum of maxima + #groups where b becomes the max
        auto cost_in = [&](uint32_t b) {
          int32_t c = 0;
          for (uint32_t k : of[w]) c += mx[k] + ((cnt[(size_t)k * 32 + b] + 1u > mx[k]) ? 1 : 0);
          return c;
        };
        int best = (int)a;
        int32_t best_cost = cost_in(a);
        for (uint32_t b = 0; b < 32; b++) {
          if (b == a || used[b] >= cap[b]) continue;
          const int32_t c = cost_in(b);
          if (c < best_cost) { best_cost = c; best = (int)b; }
        }
        for (uint32_t k : of[w]) {
          uint8_t& c = cnt[(size_t)k * 32 + best];
          c++;
          mx[k] = std::max(mx[k], c);
        }
        if ((uint32_t)best != a) { used[a]--; used[best]++; bank[w] = best; moved++; }
      }
      if (!moved) break;
    }
    // ---- physical words: bank b's logical words take the free rows of bank b in order
    std::vector<uint32_t> next_row(32, 0);
    for (uint32_t b = 0; b < 32; b++) next_row[b] = b == 0 ? 1u : 0u;
    std::vector<uint32_t> phys(M, 0);
    uint32_t hi = 0;
    for (uint32_t w = 1; w < M; w++) {
      const uint32_t b = (uint32_t)bank[w];
      phys[w] = next_row[b]++ * 32 + b;
      hi = std::max(hi, phys[w]);
    }
    auto R = [&](uint32_t w) -> uint32_t { return w < M ? phys[w] : w; };
    // ---- rewrite every word reference
    L = pr[PH_OFF_LAYERS];
    for (uint32_t l = 0; l < n_layers; l++) {
      if (pr[L + LH_FLAGS] & GEM_LF_USES_TOP) pr[L + LH_TOPWO] = R(pr[L + LH_TOPWO]);
      for (uint32_t w = 0; w < 8; w++) {
        const uint32_t wo = pr[L + LH_WOFF0 + w];
        if (!wo) continue;
        const uint32_t rec = L + wo, mode = pr[rec + 4] & 0xFFu, n4 = pr[rec + 4] >> 8;
        if (pr[rec + 3]) pr[rec + 3] = R(pr[rec + 3]);
        for (uint32_t ln = 0; ln < 32; ln++) {
          uint32_t& x = pr[rec + GEM_WREC_HDR + 4 * ln + 3];
          if (x) x = R(x);
        }
        const uint32_t lv = rec + GEM_WREC_HDR + 128;
        for (uint32_t k = 0; k < n4 * 128; k++) {
          uint32_t& e = pr[lv + k];
          if (mode == GEM_WM_DENSE16) {
            uint32_t out = 0;
            for (uint32_t h = 0; h < 2; h++) {
              const uint32_t x = (e >> (16 * h)) & 0xFFFFu;
              out |= ((x & 31u) | (R(GEM_LEAF16_WORD(x)) << 5)) << (16 * h);
            }
            e = out;
          } else {
            e = (e & 0xFFFFu) | (R(GEM_LEAF_WORD(e)) << 18);
          }
        }
      }
      L += ct[1 + l];
    }
    for (uint32_t k = 0; k < ng; k++) pr[og + 2 * k + 1] = R(pr[og + 2 * k + 1]);
    for (uint32_t k = 0; k < no * 32; k++) {
      uint32_t& e = pr[oo + k];
      const uint32_t src = e & 0x7FFFFFFFu;
      e = (e & GEM_OUT_INV) | (R(src >> 5) << 5) | (src & 31u);
    }
    const uint32_t NS = std::max(N, hi + 1);
    pr[PH_STATE_WORDS] = NS;
    return NS;
  }

  // Lane program (gem_isa.h "Lane mode"): allocate one lane word per live signal
  // (interval allocation over layers) and encode the recorded layers.
  bool encode_lanes(Part& P, const std::vector<LaneLayer>& LLs, const std::vector<uint32_t>& gread_src,
                    const std::vector<int32_t>& scratch) {
    (void)gread_src;
    const uint32_t n = (uint32_t)cid.size();
    const int32_t INF = 1 << 30;
    const uint32_t L = (uint32_t)LLs.size();
    std::vector<int32_t> last(n, -1);
    for (uint32_t l = 0; l < L; l++)
      for (uint32_t x : LLs[l].leaf_sig)
        if (x != UINT32_MAX) last[x] = std::max<int32_t>(last[x], (int32_t)l);
    for (uint32_t i = 0; i < n; i++) if (is_ep[i]) last[i] = INF;
    std::vector<int32_t> word(n, -1), birth(n, 0);
    word[0] = 0;   // local node 0 is the constant
    // free-interval allocator (first fit, coalescing); word 0 reserved
    std::map<uint32_t, uint32_t> freeiv;   // start -> length
    const uint32_t kMaxWords = (uint32_t)opt.lane_words;   // leaf entries hold byte offsets (word * 4) in 16 bits
    freeiv[1] = kMaxWords - 1;
    uint32_t max_word = 1;
    std::vector<std::vector<uint32_t>> die(L + 1);
    // best fit among the holes below the allocated extent; the open tail
    // (the interval reaching kMaxWords) only when no hole is large enough
    auto take = [&](uint32_t k) -> int64_t {
      auto best = freeiv.end();
      for (auto it = freeiv.begin(); it != freeiv.end(); ++it) {
        if (it->second < k) continue;
        const bool tail = it->first + it->second >= kMaxWords;
        if (best == freeiv.end()) { best = it; continue; }
        const bool btail = best->first + best->second >= kMaxWords;
        if ((btail && !tail) || (btail == tail && it->second < best->second)) best = it;
      }
      if (best == freeiv.end()) return -1;
      uint32_t st = best->first, len = best->second;
      freeiv.erase(best);
      if (len > k) freeiv[st + k] = len - k;
      max_word = std::max(max_word, st + k);
      return st;
    };
    auto give = [&](uint32_t w) {
      auto nx = freeiv.lower_bound(w);
      uint32_t st = w, len = 1;
      if (nx != freeiv.end() && nx->first == w + 1) { len += nx->second; nx = freeiv.erase(nx); }
      if (nx != freeiv.begin()) {
        auto pv = std::prev(nx);
        if (pv->first + pv->second == w) { st = pv->first; len += pv->second; freeiv.erase(pv); }
      }
      freeiv[st] = len;
    };
    // Bank-aware placement (lane_banks=1): a leaf load of the lane kernel is one
    // LDS.K per (layer, warp, leaf position) over the 32 lanes; with K = 2
    // each half-warp's 16 lanes read 8-byte words, conflict-free when their
    // lane words differ mod 16.  reads[x] lists the (instruction, half-warp)
    // groups that read signal x; occ counts the words already placed per group
    // and residue.  Runs are placed at the offset (within the few best-fitting
    // holes, or the tail) that adds the fewest same-residue readers.
    const bool banks = opt.lane_banks != 0;
    std::vector<std::vector<uint32_t>> reads(banks ? n : 0);
    std::vector<uint8_t> occ;
    if (banks) {
      for (uint32_t l = 0; l < L; l++)
        for (uint32_t id = 0; id < 8192; id++) {
          const uint32_t x = LLs[l].leaf_sig[id];
          if (x == UINT32_MAX || x == 0) continue;
          const uint32_t warp = id >> 10, lane = (id >> 5) & 31, pos = id & 31;
          reads[x].push_back(((l * 8 + warp) * 32 + pos) * 2 + (lane >> 4));
        }
      occ.assign((size_t)L * 8 * 32 * 2 * 16, 0);
    }
    auto bind = [&](uint32_t x, uint32_t w) {
      word[x] = (int32_t)w;
      if (last[x] >= 0 && last[x] < (int32_t)L) die[last[x]].push_back(w);
      if (banks)
        for (uint32_t g : reads[x]) { uint8_t& o = occ[(size_t)g * 16 + (w & 15)]; if (o < 255) o++; }
    };
    auto run_cost = [&](const std::vector<std::pair<uint32_t, uint32_t>>& v, uint32_t b) {
      uint32_t c = 0;
      for (size_t k = 0; k < v.size(); k++)
        for (uint32_t g : reads[v[k].second]) c += occ[(size_t)g * 16 + ((b + k) & 15)];
      return c;
    };
    // place a run: best (cost, hole size, address) over the lane_holes best-fitting holes
    // (all 16 residues each) and the tail; only holes, if any fits
    auto take_banked = [&](const std::vector<std::pair<uint32_t, uint32_t>>& v) -> int64_t {
      const uint32_t k = (uint32_t)v.size();
      std::vector<std::pair<uint32_t, uint32_t>> holes;   // (len, start)
      uint32_t tail_st = 0, tail_len = 0;
      for (auto& iv : freeiv) {
        if (iv.second < k) continue;
        if (iv.first + iv.second >= kMaxWords) { tail_st = iv.first; tail_len = iv.second; continue; }
        holes.push_back({iv.second, iv.first});
      }
      std::vector<std::pair<uint32_t, uint32_t>> cands;
      if (!holes.empty()) {
        const size_t nh = std::min<size_t>((size_t)opt.lane_holes, holes.size());
        std::partial_sort(holes.begin(), holes.begin() + nh, holes.end());
        holes.resize(nh);
        cands = holes;
      } else if (tail_len >= k) {
        cands.push_back({tail_len, tail_st});
      } else {
        return -1;
      }
      uint64_t best = UINT64_MAX;
      uint32_t bst = 0, bb = 0;
      for (auto& c : cands) {
        // interior offsets fragment the hole: only where it is large (mode 2)
        // or never (mode 1: choose among holes only)
        const uint32_t nb = opt.lane_banks == 1 ? 1u : std::min<uint32_t>(16, c.first - k + 1);
        for (uint32_t o = 0; o < nb; o++) {
          const uint64_t key = ((uint64_t)run_cost(v, c.second + o) << 40) | ((uint64_t)c.first << 16) | o;
          if (key < best) { best = key; bst = c.second; bb = c.second + o; }
        }
      }
      // split the interval [bst, bst+len) around [bb, bb+k)
      const uint32_t len = freeiv[bst];
      freeiv.erase(bst);
      if (bb > bst) freeiv[bst] = bb - bst;
      if (bb + k < bst + len) freeiv[bb + k] = bst + len - (bb + k);
      max_word = std::max(max_word, bb + k);
      return bb;
    };
    // sources take the first lane words in port-list order (entry k -> word
    // k + 1).  The list is sorted by global bit (a warp's port loads stay
    // coalesced); with lane_banks, each aligned block of 16 entries -- the same
    // addresses whichever lane loads them -- is permuted so its sources get
    // the word residues that add the fewest same-residue readers.
    std::vector<uint32_t> srcs;
    for (uint32_t i = 1; i < n; i++)
      if (is_src[i]) srcs.push_back(i);
    std::stable_sort(srcs.begin(), srcs.end(), [&](uint32_t x, uint32_t y) {
      const uint32_t gx = G.gbit[cid[x]], gy = G.gbit[cid[y]];
      const uint64_t kx = ((uint64_t)(gx >> 27) << 32) | (((gx >> 5) & 0x3FFFFF) * 32 + (gx & 31));
      const uint64_t ky = ((uint64_t)(gy >> 27) << 32) | (((gy >> 5) & 0x3FFFFF) * 32 + (gy & 31));
      return kx < ky;
    });
    if (banks) {
      for (size_t b0 = 0; b0 < srcs.size(); b0 += 16) {
        const size_t b1 = std::min(srcs.size(), b0 + 16);
        std::vector<uint32_t> blk(srcs.begin() + b0, srcs.begin() + b1), out(b1 - b0, UINT32_MAX);
        std::stable_sort(blk.begin(), blk.end(), [&](uint32_t x, uint32_t y) { return reads[x].size() > reads[y].size(); });
        for (uint32_t x : blk) {
          size_t best = SIZE_MAX;
          uint32_t bc = UINT32_MAX;
          for (size_t j = 0; j < out.size(); j++) {
            if (out[j] != UINT32_MAX) continue;
            const uint32_t wj = (uint32_t)(b0 + j + 1);
            uint32_t c = 0;
            for (uint32_t g : reads[x]) c += occ[(size_t)g * 16 + (wj & 15)];
            if (c < bc) { bc = c; best = j; }
          }
          out[best] = x;
          const uint32_t wb = (uint32_t)(b0 + best + 1);
          for (uint32_t g : reads[x]) { uint8_t& o = occ[(size_t)g * 16 + (wb & 15)]; if (o < 255) o++; }
        }
        std::copy(out.begin(), out.end(), srcs.begin() + b0);
      }
      std::fill(occ.begin(), occ.end(), 0);   // rebuilt by bind below
    }
    for (uint32_t x : srcs) {
      int64_t w = take(1);
      if (w < 0) { fail(P, "lane state overflow"); return false; }
      bind(x, (uint32_t)w);
    }
    // per layer: unit -> (mask, base)
    struct UnitWo { uint32_t mask = 0, base = 0; };
    std::vector<std::array<UnitWo, 256>> th(L);
    std::vector<std::array<UnitWo, 8>> wa(L);
    std::vector<UnitWo> tp(L);
    for (uint32_t l = 0; l < L; l++) {
      if (l > 0)
        for (uint32_t w : die[l - 1]) give(w);
      // group write-outs by unit, consecutive words in slot-bit order
      std::map<uint32_t, std::vector<std::pair<uint32_t, uint32_t>>> units;   // key: kind<<16 | unit
      for (auto& e : LLs[l].two) units[(0u << 16) | e[0]].push_back({e[1], e[2]});
      for (auto& e : LLs[l].wwo) units[(1u << 16) | e[0]].push_back({e[1], e[2]});
      for (auto& e : LLs[l].top) units[(2u << 16)].push_back({e[0], e[1]});
      // larger runs first (they are the hardest to place in holes)
      std::vector<std::pair<const uint32_t, std::vector<std::pair<uint32_t, uint32_t>>>*> order;
      for (auto& kv : units) order.push_back(&kv);
      std::stable_sort(order.begin(), order.end(), [](auto* x, auto* y) { return x->second.size() > y->second.size(); });
      for (auto* kvp : order) {
        auto& kv = *kvp;
        auto& v = kv.second;
        std::sort(v.begin(), v.end());
        uint32_t kind = kv.first >> 16, unit = kv.first & 0xFFFF;
        UnitWo u;
        // thread units write two runs (gem_isa.h): level-1 slots (bits < 16)
        // and levels 2-5 (bits >= 16), so shorter runs fit the holes
        const size_t split = kind == 0 ? (size_t)(std::lower_bound(v.begin(), v.end(), std::make_pair(16u, 0u)) - v.begin())
                                       : v.size();
        for (int part = 0; part < (kind == 0 ? 2 : 1); part++) {
          std::vector<std::pair<uint32_t, uint32_t>> r(part == 0 ? v.begin() : v.begin() + split,
                                                       part == 0 ? v.begin() + split : v.end());
          uint32_t b0 = 0;
          if (!r.empty()) {
            int64_t base = banks ? take_banked(r) : take((uint32_t)r.size());
            if (base < 0) { fail(P, "lane state overflow"); return false; }
            b0 = (uint32_t)base;
            for (size_t k = 0; k < r.size(); k++) {
              u.mask |= 1u << r[k].first;
              bind(r[k].second, b0 + (uint32_t)k);
              birth[r[k].second] = (int32_t)l;
            }
          }
          if (kind == 0) u.base |= b0 << (16 * part);
          else u.base = b0;
        }
        if (kind == 0) th[l][unit] = u;
        else if (kind == 1) wa[l][unit] = u;
        else tp[l] = u;
      }
    }
    if (opt.verbose >= 3) {
      // peak number of simultaneously live lane words vs the allocated extent
      uint32_t peak = 0;
      for (uint32_t l = 0; l < L; l++) {
        uint32_t live = 0;
        for (uint32_t i = 0; i < n; i++)
          if (word[i] > 0 && birth[i] <= (int32_t)l && last[i] >= (int32_t)l) live++;
        peak = std::max(peak, live);
      }
      fprintf(stderr, "lane part: n=%u srcs=%zu layers=%u max_word=%u peak_live=%u\n", n, srcs.size(), L, max_word,
              peak);
    }
    if (max_word >= kMaxWords) { fail(P, "lane state overflow"); return false; }
    auto lw = [&](uint32_t x) -> uint32_t {
      if (word[x] < 0)
        throw std::runtime_error("lane: signal without a word (local " + std::to_string(x) + ")");
      return (uint32_t)word[x];
    };
    std::vector<uint32_t>& pr = P.lane_prog;
    pr.assign(LPH_WORDS, 0);
    pr[LPH_MAGIC] = GEM_LANE_MAGIC;
    pr[LPH_N_LAYERS] = L;
    pr[LPH_N_OUT] = (uint32_t)P.outs.size() * 32;
    pr[LPH_N_RAM] = (uint32_t)P.rams.size();
    pr[LPH_LANE_WORDS] = (max_word + 3) & ~3u;
    pr[LPH_OFF_CHUNKS] = (uint32_t)pr.size();
    pr[LPH_N_CHUNKS] = L + 2;
    for (uint32_t k = 0; k < L + 2; k++) pr.push_back(0);
    while (pr.size() % 4) pr.push_back(0);
    pr[LPH_OFF_LAYERS] = (uint32_t)pr.size();   // chunk 0 = header + chunk table
    pr[pr[LPH_OFF_CHUNKS]] = (uint32_t)pr.size();
    for (uint32_t l = 0; l < L; l++) {
      const LaneLayer& LL = LLs[l];
      size_t base = pr.size();
      pr.resize(base + LLH_WORDS, 0);
      uint32_t active = 0;
      for (uint32_t t = 0; t < 256; t++) if (th[l][t].mask) active |= 1u << (t / 32);
      for (uint32_t w = 0; w < 8; w++) if (wa[l][w].mask) active |= 1u << w;
      for (uint32_t id = 0; id < 8192; id++) if (LL.leaf_sig[id] != UINT32_MAX) active |= 1u << (id >> 10);
      const bool uses_top = tp[l].mask != 0;
      pr[base + LLH_FLAGS] = active | (uses_top ? GEM_LF_USES_TOP : 0u);
      pr[base + LLH_TOPC] = LL.topc;
      pr[base + LLH_TOPWO] = tp[l].mask | (tp[l].base << 8);
      for (uint32_t w = 0; w < 8; w++) {
        if (!(active >> w & 1)) continue;
        pr[base + LLH_WOFF0 + w] = (uint32_t)(pr.size() - base);
        pr.push_back(LL.cw[w][0]); pr.push_back(LL.cw[w][1]); pr.push_back(LL.cw[w][2]);
        pr.push_back(wa[l][w].mask); pr.push_back(wa[l][w].base);
        pr.push_back(0); pr.push_back(0); pr.push_back(0);
        for (uint32_t ln = 0; ln < 32; ln++) {
          uint32_t t = w * 32 + ln;
          // byte-spread constants (gem_isa.h): slot bit b -> bit 8*(b&3) + 7 - (b>>2), so the
          // kernel makes each mask with one shift per 4 slots and one PRMT sign-replicate
          auto spread = [](uint32_t c) {
            uint32_t r = 0;
            for (uint32_t q = 0; q < 31; q++) r |= ((c >> q) & 1u) << (8 * (q & 3) + 7 - (q >> 2));
            return r;
          };
          pr.push_back(spread(LL.cth[3 * t])); pr.push_back(spread(LL.cth[3 * t + 1]));
          pr.push_back(spread(LL.cth[3 * t + 2]));
          pr.push_back(th[l][t].mask);
        }
        for (uint32_t g = 0; g < 4; g++)
          for (uint32_t ln = 0; ln < 32; ln++)
            for (uint32_t k = 0; k < 4; k++) {
              uint32_t e = 0;
              for (uint32_t h = 0; h < 2; h++) {
                uint32_t pos = 8 * g + 2 * k + h, id = (w * 32 + ln) * 32 + pos;
                uint32_t x = LL.leaf_sig[id];
                e |= (x == UINT32_MAX ? 0u : 4u * lw(x)) << (16 * h);
              }
              pr.push_back(e);
            }
        for (uint32_t ln = 0; ln < 32; ln++) pr.push_back(th[l][w * 32 + ln].base);
      }
      pr[base + LLH_WORDS_] = (uint32_t)(pr.size() - base);
      pr[pr[LPH_OFF_CHUNKS] + 1 + l] = pr[base + LLH_WORDS_];
    }
    // next-layer header copies (LLH_NEXT)
    {
      size_t off = pr[LPH_OFF_LAYERS];
      for (uint32_t l = 0; l < L; l++) {
        const size_t nx = off + pr[off + LLH_WORDS_];
        for (int k = 0; k < 12; k++) pr[off + LLH_NEXT + k] = (l + 1 < L) ? pr[nx + k] : 0u;
        off = nx;
      }
    }
    pr[LPH_OFF_OUT] = (uint32_t)pr.size();
    for (auto& ow : P.outs) {
      uint32_t reg = GEM_GID_REGION(ow.dst), idx = GEM_GID_INDEX(ow.dst);
      for (int k = 0; k < 32; k++) {
        uint32_t l = ow.lit[k];
        uint32_t x = (uint32_t)scratch[l >> 1];
        pr.push_back((reg << 24) | (idx * 32 + (uint32_t)k));
        pr.push_back(lw(x) | ((l & 1) ? GEM_OUT_INV : 0u));
      }
    }
    pr[LPH_OFF_RAM] = (uint32_t)pr.size();
    for (uint32_t r : P.rams) { pr.push_back(r); pr.push_back(0); pr.push_back(0); pr.push_back(0); }
    while (pr.size() % 4) pr.push_back(0);
    pr[pr[LPH_OFF_CHUNKS] + 1 + L] = (uint32_t)pr.size() - pr[LPH_OFF_OUT];
    // input-port list last: read from global memory by the kernel, not streamed
    pr[LPH_OFF_GREAD] = (uint32_t)pr.size();
    uint32_t ng = 0;
    for (uint32_t x : srcs) {
      uint32_t gb = G.gbit[cid[x]];
      // one word per entry: the destination lane word is implicit (entry k ->
      // lane word k + 1: the sources took the first words, in this order)
      if (lw(x) != ng + 1) throw std::runtime_error("lane: source words not consecutive");
      pr.push_back(((gb >> 27) << 24) | (((gb >> 5) & 0x3FFFFF) * 32 + (gb & 31)));
      ng++;
    }
    pr[LPH_N_GREAD] = ng;
    while (pr.size() % 4) pr.push_back(0);
    P.lane_words = pr[LPH_LANE_WORDS];
    return true;
  }

  // Compacted lane program ("LAN2", gem_isa.h): the partition's ANDs list-
  // scheduled into steps of <= 256 (critical path first), lane words
  // allocated by liveness, ops of a step assigned to threads and destination
  // words chosen so that each half-warp's 16 operand / destination residues
  // (mod 16) collide as little as possible.
  bool encode_lanes2(Part& P, const std::vector<int32_t>& scratch) {
    const uint32_t n = (uint32_t)cid.size();
    const uint32_t kMaxWords = (uint32_t)opt.lane_words;
    // one LDS/STS of K interleaved groups moves 4K bytes per lane: a wavefront
    // (128 bytes) serves kHalf = 32/K lanes, conflict-free when their words
    // differ mod kHalf
    const uint32_t kStep = GEM_LANE2_STEP * (uint32_t)opt.lane_m, kHalf = 32u / (uint32_t)opt.lane_k,
                   kGroups = kStep / kHalf;
    // sources: port-list order (sorted by global bit: a warp's port loads stay coalesced)
    std::vector<uint32_t> srcs;
    for (uint32_t i = 1; i < n; i++)
      if (is_src[i]) srcs.push_back(i);
    std::stable_sort(srcs.begin(), srcs.end(), [&](uint32_t x, uint32_t y) {
      const uint32_t gx = G.gbit[cid[x]], gy = G.gbit[cid[y]];
      const uint64_t kx = ((uint64_t)(gx >> 27) << 32) | (((gx >> 5) & 0x3FFFFF) * 32 + (gx & 31));
      const uint64_t ky = ((uint64_t)(gy >> 27) << 32) | (((gy >> 5) & 0x3FFFFF) * 32 + (gy & 31));
      return kx < ky;
    });
    if (srcs.size() + 1 >= kMaxWords) { fail(P, "lane state overflow"); return false; }
    // ---- list scheduling: an op is ready one step after its last operand
    std::vector<uint32_t> rd(n, 0), pend(n, 0), step_of(n, 0);
    for (uint32_t i = n; i-- > 0;)
      for (uint32_t j = coff[i]; j < coff[i + 1]; j++) rd[i] = std::max(rd[i], rd[cons[j]] + 1);
    std::vector<uint32_t> ready;   // max-heap on (rd, -id)
    auto prio = [&](uint32_t x, uint32_t y) { return rd[x] != rd[y] ? rd[x] < rd[y] : x > y; };
    uint32_t n_ops = 0;
    for (uint32_t i = 0; i < n; i++) {
      if (is_src[i]) continue;
      n_ops++;
      pend[i] = (uint32_t)(!is_src[la[i] >> 1]) + (uint32_t)(!is_src[lb[i] >> 1]);
      if ((la[i] >> 1) == (lb[i] >> 1) && !is_src[la[i] >> 1]) pend[i] = 1;
      if (!pend[i]) ready.push_back(i);
    }
    std::make_heap(ready.begin(), ready.end(), prio);
    std::vector<std::vector<uint32_t>> steps;
    std::vector<uint32_t> next_ready;
    uint32_t done = 0;
    while (done < n_ops) {
      if (ready.empty()) throw std::runtime_error("lane2: scheduling stalled");
      steps.emplace_back();
      auto& st = steps.back();
      while (!ready.empty() && st.size() < kStep) {
        std::pop_heap(ready.begin(), ready.end(), prio);
        st.push_back(ready.back());
        ready.pop_back();
      }
      next_ready.clear();
      for (uint32_t x : st) {
        step_of[x] = (uint32_t)steps.size() - 1;
        done++;
        for (uint32_t j = coff[x]; j < coff[x + 1]; j++) {
          const uint32_t c = cons[j];
          if (j > coff[x] && cons[j - 1] == c) continue;   // both fanins from x: counted once
          if (--pend[c] == 0) next_ready.push_back(c);
        }
      }
      for (uint32_t c : next_ready) { ready.push_back(c); std::push_heap(ready.begin(), ready.end(), prio); }
    }
    const uint32_t S = (uint32_t)steps.size();
    // ---- last reading step of every value (endpoints: live to the end)
    const uint32_t INF = UINT32_MAX;
    std::vector<uint32_t> last(n, 0);
    for (uint32_t i = 0; i < n; i++) {
      if (is_ep[i]) { last[i] = INF; continue; }
      for (uint32_t j = coff[i]; j < coff[i + 1]; j++) last[i] = std::max(last[i], step_of[cons[j]]);
    }
    // ---- future-read residue budgets: bud[(s * 2 + side) * kHalf + r] = operands of
    // step s (side 0 = A, 1 = B) already placed at word residue r.  A value's word
    // residue is chosen where its future readers' steps have the fewest, so the
    // operands of every step spread over the residues (conflict-free groups).
    std::vector<uint16_t> bud((size_t)S * 2 * kHalf, 0);
    auto readers_cost = [&](uint32_t x, uint32_t r) {
      uint32_t c = 0;
      for (uint32_t j = coff[x]; j < coff[x + 1]; j++) {
        const uint32_t y = cons[j];
        c += bud[((size_t)step_of[y] * 2 + ((la[y] >> 1) == x ? 0u : 1u)) * kHalf + r];
      }
      return c;
    };
    auto add_readers = [&](uint32_t x, uint32_t r) {
      for (uint32_t j = coff[x]; j < coff[x + 1]; j++) {
        const uint32_t y = cons[j];
        bud[((size_t)step_of[y] * 2 + ((la[y] >> 1) == x ? 0u : 1u)) * kHalf + r]++;
      }
    };
    // ---- words: 0 = constant, 1..n_src = ports (entry k -> word k+1); within each
    // aligned block of kHalf entries (the same lines whichever lane loads them,
    // and consecutive words for the port stores) the sources are permuted onto
    // the residues their readers need most
    for (size_t b0 = 0; b0 < srcs.size(); b0 += kHalf) {
      const size_t b1 = std::min(srcs.size(), b0 + kHalf);
      std::vector<uint32_t> blk(srcs.begin() + b0, srcs.begin() + b1), out(b1 - b0, UINT32_MAX);
      std::stable_sort(blk.begin(), blk.end(), [&](uint32_t x, uint32_t y) { return coff[x + 1] - coff[x] > coff[y + 1] - coff[y]; });
      for (uint32_t x : blk) {
        size_t best = 0;
        uint32_t bc = UINT32_MAX;
        for (size_t j = 0; j < out.size(); j++) {
          if (out[j] != UINT32_MAX) continue;
          const uint32_t c = readers_cost(x, (uint32_t)(b0 + j + 1) % kHalf);
          if (c < bc) { bc = c; best = j; }
        }
        out[best] = x;
        add_readers(x, (uint32_t)(b0 + best + 1) % kHalf);
      }
      std::copy(out.begin(), out.end(), srcs.begin() + b0);
    }
    std::vector<int32_t> word(n, -1);
    word[0] = 0;
    std::vector<std::set<uint32_t>> freew(kHalf);
    uint32_t top = 1, max_word = 1;
    for (uint32_t x : srcs) { word[x] = (int32_t)top++; }
    max_word = top;
    std::vector<std::vector<uint32_t>> die(S + 1);
    for (uint32_t x : srcs)
      if (last[x] != INF) die[last[x]].push_back((uint32_t)word[x]);
    auto alloc = [&](uint32_t res) -> uint32_t {   // lowest free word of residue res (or a fresh one)
      uint32_t best = UINT32_MAX;
      if (!freew[res].empty()) best = *freew[res].begin();
      // a fresh word of this residue at the top (may also open lower residues)
      uint32_t fresh = top + ((res + kHalf - (top % kHalf)) % kHalf);
      if (best != UINT32_MAX && best < fresh) { freew[res].erase(freew[res].begin()); return best; }
      for (uint32_t w = top; w < fresh; w++) freew[w % kHalf].insert(w);
      top = fresh + 1;
      return fresh;
    };
    auto lw = [&](uint32_t l) -> uint32_t {
      const int32_t w = word[l >> 1];
      if (w < 0) throw std::runtime_error("lane2: operand without a word");
      return (uint32_t)w;
    };
    std::vector<uint32_t>& pr = P.lane_prog;
    pr.assign(LPH_WORDS, 0);
    pr[LPH_MAGIC] = GEM_LANE2_MAGIC;
    pr[LPH_N_LAYERS] = S;
    pr[LPH_N_OPS] = n_ops;
    pr[LPH_OPS_PER_THREAD] = (uint32_t)opt.lane_m;
    pr[LPH_N_OUT] = (uint32_t)P.outs.size() * 32;
    pr[LPH_N_RAM] = (uint32_t)P.rams.size();
    pr[LPH_OFF_CHUNKS] = (uint32_t)pr.size();
    pr[LPH_N_CHUNKS] = 1;
    pr.push_back(0);
    while (pr.size() % 4) pr.push_back(0);
    pr[LPH_OFF_LAYERS] = (uint32_t)pr.size();
    pr.resize(pr.size() + (size_t)S * kStep * 2, 0);
    uint32_t* ops = pr.data() + pr[LPH_OFF_LAYERS];
    std::vector<std::array<uint8_t, 32>> ca(kGroups), cb(kGroups), cd(kGroups);
    std::vector<uint32_t> fill(kGroups);
    for (uint32_t s = 0; s < S; s++) {
      // words last read before step s are free (the barrier separates the read and the write)
      if (s > 0)
        for (uint32_t w : die[s - 1]) freew[w % kHalf].insert(w);
      for (uint32_t g = 0; g < kGroups; g++) { ca[g].fill(0); cb[g].fill(0); cd[g].fill(0); fill[g] = 0; }
      auto& st = steps[s];
      // critical ops first
      std::stable_sort(st.begin(), st.end(), [&](uint32_t x, uint32_t y) { return rd[x] > rd[y]; });
      // Operand residues: an op is an edge (A residue, B residue) of a bipartite
      // multigraph; a proper edge colouring puts ops of distinct A and distinct
      // B residues in each colour class, i.e. conflict-free wavefronts.  König:
      // max-degree colours suffice (alternating-path recolouring); colour c ->
      // group c when there are at most kGroups colours, the rest fall back to
      // the greedy choice below.
      std::vector<int32_t> pref(st.size(), -1);
      {
        const uint32_t n_e = (uint32_t)st.size();
        std::array<uint32_t, 64> deg{};
        for (uint32_t x : st) { deg[lw(la[x]) % kHalf]++; deg[kHalf + lw(lb[x]) % kHalf]++; }
        uint32_t C = 0;
        for (uint32_t v = 0; v < 2 * kHalf; v++) C = std::max(C, deg[v]);
        std::vector<int32_t> at((size_t)2 * kHalf * C, -1), col(n_e, -1);   // at[v*C + c] = edge
        auto U = [&](uint32_t e) { return lw(la[st[e]]) % kHalf; };
        auto V = [&](uint32_t e) { return kHalf + lw(lb[st[e]]) % kHalf; };
        for (uint32_t e = 0; e < n_e; e++) {
          const uint32_t u = U(e), v = V(e);
          uint32_t a = 0, bcol = 0;
          while (at[(size_t)u * C + a] >= 0) a++;
          while (at[(size_t)v * C + bcol] >= 0) bcol++;
          if (at[(size_t)v * C + a] >= 0) {
            // flip the a/b alternating path from v (a bipartite path never returns to u)
            std::vector<uint32_t> path;
            uint32_t w = v, cc = a;
            while (at[(size_t)w * C + cc] >= 0) {
              const uint32_t f = (uint32_t)at[(size_t)w * C + cc];
              path.push_back(f);
              w = (U(f) == w) ? V(f) : U(f);
              cc = (cc == a) ? bcol : a;
            }
            for (uint32_t f : path) { at[(size_t)U(f) * C + col[f]] = -1; at[(size_t)V(f) * C + col[f]] = -1; }
            for (uint32_t f : path) {
              col[f] = col[f] == (int32_t)a ? (int32_t)bcol : (int32_t)a;
              at[(size_t)U(f) * C + col[f]] = (int32_t)f;
              at[(size_t)V(f) * C + col[f]] = (int32_t)f;
            }
          }
          col[e] = (int32_t)a;
          at[(size_t)u * C + a] = (int32_t)e;
          at[(size_t)v * C + a] = (int32_t)e;
        }
        if (C <= kGroups)
          for (uint32_t e = 0; e < n_e; e++) pref[e] = col[e];
        else {
          // the kGroups largest colour classes keep their group
          std::vector<std::pair<uint32_t, uint32_t>> sz(C);
          for (uint32_t c = 0; c < C; c++) sz[c] = {0u, c};
          for (uint32_t e = 0; e < n_e; e++) sz[col[e]].first++;
          std::sort(sz.begin(), sz.end(), std::greater<std::pair<uint32_t, uint32_t>>());
          std::vector<int32_t> gmap(C, -1);
          for (uint32_t k = 0; k < kGroups; k++) gmap[sz[k].second] = (int32_t)k;
          for (uint32_t e = 0; e < n_e; e++) pref[e] = gmap[col[e]];
        }
      }
      // operand words already read by each group (a repeated word is a broadcast, no conflict)
      std::vector<std::array<uint32_t, 32>> gwa(kGroups), gwb(kGroups);
      for (uint32_t ei = 0; ei < st.size(); ei++) {
        const uint32_t x = st[ei];
        const uint32_t wa = lw(la[x]), wb = lw(lb[x]);
        const uint32_t ra = wa % kHalf, rb = wb % kHalf;
        // group (kHalf lanes = one wavefront) with room and the fewest distinct
        // same-residue operand words (the colouring's group when it has room)
        uint32_t bg = 0, bc = UINT32_MAX;
        if (pref[ei] >= 0 && fill[pref[ei]] < kHalf) { bg = (uint32_t)pref[ei]; bc = 0; }
        for (uint32_t g = 0; g < kGroups && bc; g++) {
          if (fill[g] == kHalf) continue;
          uint32_t xa = 0, xb = 0;
          bool da = false, db = false;
          for (uint32_t k = 0; k < fill[g]; k++) {
            da |= gwa[g][k] == wa; db |= gwb[g][k] == wb;
          }
          if (!da) xa = ca[g][ra];
          if (!db) xb = cb[g][rb];
          const uint32_t c = 4u * (xa + xb) + fill[g] / 8;
          if (c < bc) { bc = c; bg = g; }
        }
        {
          bool da = false, db = false;
          for (uint32_t k = 0; k < fill[bg]; k++) { da |= gwa[bg][k] == wa; db |= gwb[bg][k] == wb; }
          gwa[bg][fill[bg]] = wa;
          gwb[bg][fill[bg]] = wb;
          if (da) ca[bg][ra]--;   // (undone by the increment below: a repeated word adds no wavefront)
          if (db) cb[bg][rb]--;
        }
        // destination residue: least used by the group's stores, then the fewest
        // future readers' operands at that residue, then a free (low) word
        uint32_t bres = 0;
        uint64_t bkey = UINT64_MAX;
        for (uint32_t r = 0; r < kHalf; r++) {
          const uint64_t fw = freew[r].empty() ? 0xFFFFFFull : *freew[r].begin();
          const uint64_t key = ((uint64_t)cd[bg][r] << 56) | ((uint64_t)std::min<uint32_t>(readers_cost(x, r), 0xFFFFFF) << 24) | fw;
          if (key < bkey) { bkey = key; bres = r; }
        }
        const uint32_t w = alloc(bres);
        add_readers(x, w % kHalf);
        ca[bg][ra]++; cb[bg][rb]++; cd[bg][w % kHalf]++;
        const uint32_t t = bg * kHalf + fill[bg]++;
        word[x] = (int32_t)w;
        max_word = std::max(max_word, w + 1);
        if (last[x] != INF) die[std::max(last[x], s)].push_back(w);
        ops[((size_t)s * kStep + t) * 2] = GEM_LANE2_OP_X(lw(la[x]), la[x] & 1u, lw(lb[x]), lb[x] & 1u);
        ops[((size_t)s * kStep + t) * 2 + 1] = w;
      }
      if (max_word >= kMaxWords) { fail(P, "lane state overflow"); return false; }
    }
    pr[LPH_LANE_WORDS] = (max_word + 3) & ~3u;
    pr[LPH_OFF_OUT] = (uint32_t)pr.size();
    for (auto& ow : P.outs) {
      const uint32_t reg = GEM_GID_REGION(ow.dst), idx = GEM_GID_INDEX(ow.dst);
      for (int k = 0; k < 32; k++) {
        const uint32_t l = ow.lit[k];
        const uint32_t x = (uint32_t)scratch[l >> 1];
        pr.push_back((reg << 24) | (idx * 32 + (uint32_t)k));
        pr.push_back(lw(2 * x) | ((l & 1) ? GEM_OUT_INV : 0u));
      }
    }
    pr[LPH_OFF_RAM] = (uint32_t)pr.size();
    for (uint32_t r : P.rams) { pr.push_back(r); pr.push_back(0); pr.push_back(0); pr.push_back(0); }
    while (pr.size() % 4) pr.push_back(0);
    pr[LPH_OFF_GREAD] = (uint32_t)pr.size();
    for (uint32_t x : srcs) {
      const uint32_t gb = G.gbit[cid[x]];
      pr.push_back(((gb >> 27) << 24) | (((gb >> 5) & 0x3FFFFF) * 32 + (gb & 31)));
    }
    pr[LPH_N_GREAD] = (uint32_t)srcs.size();
    while (pr.size() % 4) pr.push_back(0);
    pr[pr[LPH_OFF_CHUNKS]] = (uint32_t)pr.size();
    P.lane_words = pr[LPH_LANE_WORDS];
    if (opt.verbose >= 3)
      fprintf(stderr, "lane2 part: ops=%u steps=%u (fill %.2f) srcs=%zu words=%u\n", n_ops, S,
              n_ops / (double)(S * kStep), srcs.size(), max_word);
    return true;
  }

  // Word program ("WRD1", gem_isa.h): the single-stream path.  One signal per
  // shared-memory word; the partition's ANDs list-scheduled (critical path
  // first, as LAN2) into steps of <= word_step ops separated by one block
  // barrier, stored compactly.  Within a step, ops are placed in warp-sized
  // rounds (slot j -> thread j % 256, lane j % 32) so that a round's operand
  // words fall into distinct banks where the ready list allows it, and each
  // op's destination word is allocated (by liveness) in bank j % 32, so a
  // round's 32 stores are conflict-free.  Leaves P.word_prog empty when the
  // live words exceed GEM_WORD_MAX_WORDS (the blob then has no word programs).
  void encode_words(Part& P, const std::vector<int32_t>& scratch) {
    P.word_prog.clear();
    const uint32_t n = (uint32_t)cid.size();
    const uint32_t kStep = (uint32_t)opt.word_step;
    std::vector<uint32_t> srcs;
    for (uint32_t i = 1; i < n; i++)
      if (is_src[i]) srcs.push_back(i);
    std::stable_sort(srcs.begin(), srcs.end(), [&](uint32_t x, uint32_t y) {
      const uint32_t gx = G.gbit[cid[x]], gy = G.gbit[cid[y]];
      const uint64_t kx = ((uint64_t)(gx >> 27) << 32) | (((gx >> 5) & 0x3FFFFF) * 32 + (gx & 31));
      const uint64_t ky = ((uint64_t)(gy >> 27) << 32) | (((gy >> 5) & 0x3FFFFF) * 32 + (gy & 31));
      return kx < ky;
    });
    if (srcs.size() + 1 >= GEM_WORD_MAX_WORDS) return;
    // ---- list scheduling (an op is ready one step after its last operand)
    std::vector<uint32_t> rd(n, 0), pend(n, 0), step_of(n, 0);
    for (uint32_t i = n; i-- > 0;)
      for (uint32_t j = coff[i]; j < coff[i + 1]; j++) rd[i] = std::max(rd[i], rd[cons[j]] + 1);
    std::vector<uint32_t> ready;
    auto prio = [&](uint32_t x, uint32_t y) { return rd[x] != rd[y] ? rd[x] < rd[y] : x > y; };
    uint32_t n_ops = 0;
    for (uint32_t i = 0; i < n; i++) {
      if (is_src[i]) continue;
      n_ops++;
      pend[i] = (uint32_t)(!is_src[la[i] >> 1]) + (uint32_t)(!is_src[lb[i] >> 1]);
      if ((la[i] >> 1) == (lb[i] >> 1) && !is_src[la[i] >> 1]) pend[i] = 1;
      if (!pend[i]) ready.push_back(i);
    }
    std::make_heap(ready.begin(), ready.end(), prio);
    std::vector<std::vector<uint32_t>> steps;
    std::vector<uint32_t> next_ready;
    uint32_t done = 0;
    // balanced scheduling (word_sched=1): an op with slack need not run in the
    // first step it is ready in.  Steps are as many as the critical path (Lc =
    // 1 + max rd over ops); op x must run by step Lc - 1 - rd[x] (its ALAP
    // step).  Each step takes every ready op at its deadline, then fills up to
    // one round (256 ops) with the ready ops of least slack; only a step whose
    // deadlines exceed that goes wide.  Fewer capacity-bound wide steps, same
    // number of steps.
    uint32_t Lc = 0;
    for (uint32_t i = 0; i < n; i++)
      if (!is_src[i]) Lc = std::max(Lc, rd[i] + 1);
    // one stage: every partition may use as many steps as the deepest one has
    // (the design's depth); a shallow partition with many ops then spreads
    // them thinner instead of running extra rounds in fewer steps -- the cycle
    // is the slowest partition's, and an extra round costs more than a step
    if (opt.word_spread && opt.stages == 1) Lc = std::max(Lc, G.max_level + 1);
    while (done < n_ops) {
      if (ready.empty()) throw std::runtime_error("words: scheduling stalled");
      steps.emplace_back();
      auto& st = steps.back();
      if (opt.word_sched) {
        const uint32_t s = (uint32_t)steps.size() - 1;
        // ready ops by deadline (ALAP step = Lc - 1 - rd), most urgent first
        std::sort(ready.begin(), ready.end(), [&](uint32_t x, uint32_t y) { return rd[x] != rd[y] ? rd[x] > rd[y] : x < y; });
        size_t take = 0;
        while (take < ready.size() && take < kStep && Lc - 1 - rd[ready[take]] <= s) take++;   // due now
        const size_t fill = std::max<size_t>(take, std::min<size_t>((size_t)opt.word_fill, kStep));
        while (take < ready.size() && take < fill) take++;
        st.assign(ready.begin(), ready.begin() + (ptrdiff_t)take);
        ready.erase(ready.begin(), ready.begin() + (ptrdiff_t)take);
        std::make_heap(ready.begin(), ready.end(), prio);
      }
      while (!opt.word_sched && !ready.empty() && st.size() < kStep) {
        std::pop_heap(ready.begin(), ready.end(), prio);
        st.push_back(ready.back());
        ready.pop_back();
      }
      next_ready.clear();
      for (uint32_t x : st) {
        step_of[x] = (uint32_t)steps.size() - 1;
        done++;
        for (uint32_t j = coff[x]; j < coff[x + 1]; j++) {
          const uint32_t c = cons[j];
          if (j > coff[x] && cons[j - 1] == c) continue;
          if (--pend[c] == 0) next_ready.push_back(c);
        }
      }
      for (uint32_t c : next_ready) { ready.push_back(c); std::push_heap(ready.begin(), ready.end(), prio); }
    }
    if (opt.word_local_probe) {
      // analysis only: ops whose cone reads only this partition's own flop
      // words, its own RAMs' read data and PIs ("local": computable right after
      // the partition's own commit, before the grid barrier completes) -- the
      // work a split-phase barrier (arrive, local steps, wait) could hide
      std::unordered_set<uint32_t> own_q, own_rd;
      for (auto& ow : P.outs)
        if (GEM_GID_REGION(ow.dst) == GEM_R_Q) own_q.insert(GEM_GID_INDEX(ow.dst));
      for (uint32_t r : P.rams) own_rd.insert(r);
      std::vector<uint8_t> local(n, 1);
      uint32_t n_local = 0, n_and_ops = 0, src_local = 0, src_all = 0;
      for (uint32_t i = 0; i < n; i++) {
        if (is_src[i]) {
          if (G.kind[cid[i]] == K_CONST) { local[i] = 1; continue; }
          const uint32_t gb = G.gbit[cid[i]], reg = gb >> 27, w = (gb >> 5) & 0x3FFFFF;
          local[i] = reg == GEM_R_PI || (reg == GEM_R_Q && own_q.count(w)) || (reg == GEM_R_RD && own_rd.count(w));
          src_all++;
          src_local += local[i];
          continue;
        }
        local[i] = local[la[i] >> 1] && local[lb[i] >> 1];
        n_and_ops++;
        n_local += local[i];
      }
      // steps of the local sub-schedule (ops only waiting for local ops)
      uint32_t local_steps = 0;
      for (uint32_t x = 0; x < n; x++)
        if (!is_src[x] && local[x]) local_steps = std::max(local_steps, step_of[x] + 1);
      uint32_t first_remote = UINT32_MAX;
      for (uint32_t x = 0; x < n; x++)
        if (!is_src[x] && !local[x]) first_remote = std::min(first_remote, step_of[x]);
      fprintf(stderr, "words local probe: ops %u local %u (%.2f) ports %u local %u steps %zu first remote-dependent step %u last local step %u\n",
              n_and_ops, n_local, n_and_ops ? (double)n_local / n_and_ops : 0.0, src_all, src_local, steps.size(),
              first_remote, local_steps);
    }
    if (opt.word_chain_probe) {
      // analysis only: steps if a thread could run a chain of up to L ops in one
      // narrow step (op k+1 takes op k's result from a register, its other
      // operand from an earlier step)
      for (uint32_t L : {2u, 4u, 8u}) {
        std::vector<int32_t> d2(n, -1);
        std::vector<uint32_t> pend2(n, 0), rdy;
        uint32_t left = 0;
        for (uint32_t i = 0; i < n; i++) {
          if (is_src[i]) continue;
          d2[i] = INT32_MAX;
          left++;
        }
        auto avail = [&](uint32_t c, int32_t s) { return d2[c] < s; };
        int32_t s = 0;
        while (left) {
          rdy.clear();
          for (uint32_t i = 0; i < n; i++)
            if (d2[i] == INT32_MAX && avail(la[i] >> 1, s) && avail(lb[i] >> 1, s)) rdy.push_back(i);
          std::stable_sort(rdy.begin(), rdy.end(), [&](uint32_t x, uint32_t y) { return rd[x] > rd[y]; });
          const bool wide = rdy.size() > 256;
          if (rdy.size() > (wide ? kStep : 256u)) rdy.resize(wide ? kStep : 256u);
          for (uint32_t x : rdy) { d2[x] = s; left--; }
          if (!wide)
            for (uint32_t x : rdy) {
              uint32_t cur = x;
              for (uint32_t k = 1; k < L; k++) {
                uint32_t best = UINT32_MAX;
                for (uint32_t j = coff[cur]; j < coff[cur + 1]; j++) {
                  const uint32_t y = cons[j];
                  if (d2[y] != INT32_MAX) continue;
                  const uint32_t o = (la[y] >> 1) == cur ? (lb[y] >> 1) : (la[y] >> 1);
                  if (o != cur && !avail(o, s)) continue;
                  if (best == UINT32_MAX || rd[y] > rd[best]) best = y;
                }
                if (best == UINT32_MAX) break;
                d2[best] = s;
                left--;
                cur = best;
              }
            }
          s++;
        }
        fprintf(stderr, "words chain probe: L=%u steps %d (plain %zu)\n", L, s, steps.size());
      }
    }
    const uint32_t S = (uint32_t)steps.size();
    const uint32_t INF = UINT32_MAX;
    std::vector<uint32_t> last(n, 0);
    for (uint32_t i = 0; i < n; i++) {
      if (is_ep[i]) { last[i] = INF; continue; }
      for (uint32_t j = coff[i]; j < coff[i + 1]; j++) last[i] = std::max(last[i], step_of[cons[j]]);
    }
    // ---- future-read bank budgets (as LAN2): bud[(s * 2 + side) * 32 + r] =
    // operands of step s (side 0 = A, 1 = B) already placed in bank r.  A
    // value's bank is chosen where its readers' steps have the fewest, so the
    // operands of every step spread over the banks (fewer conflict replays).
    std::vector<uint16_t> bud((size_t)S * 2 * 32, 0);
    auto readers_cost = [&](uint32_t x, uint32_t r) {
      uint32_t c = 0;
      for (uint32_t j = coff[x]; j < coff[x + 1]; j++) {
        const uint32_t y = cons[j];
        c += bud[((size_t)step_of[y] * 2 + ((la[y] >> 1) == x ? 0u : 1u)) * 32 + r];
      }
      return c;
    };
    auto add_readers = [&](uint32_t x, uint32_t r) {
      for (uint32_t j = coff[x]; j < coff[x + 1]; j++) {
        const uint32_t y = cons[j];
        uint16_t& b = bud[((size_t)step_of[y] * 2 + ((la[y] >> 1) == x ? 0u : 1u)) * 32 + r];
        b = (uint16_t)std::min<uint32_t>(b + 1u, 0xFFFFu);
      }
    };
    // ---- words: 0 = constant, 1..n_src = ports (permuted within aligned blocks
    // of 32 onto the banks their readers need most; a warp still loads the same
    // 32 entries), then by liveness with a bank choice
    for (size_t b0 = 0; b0 < srcs.size(); b0 += 32) {
      const size_t b1 = std::min(srcs.size(), b0 + 32);
      std::vector<uint32_t> blk(srcs.begin() + b0, srcs.begin() + b1), out(b1 - b0, UINT32_MAX);
      std::stable_sort(blk.begin(), blk.end(), [&](uint32_t x, uint32_t y) { return coff[x + 1] - coff[x] > coff[y + 1] - coff[y]; });
      for (uint32_t x : blk) {
        size_t best = 0;
        uint32_t bc = UINT32_MAX;
        for (size_t j = 0; j < out.size(); j++) {
          if (out[j] != UINT32_MAX) continue;
          const uint32_t c = readers_cost(x, (uint32_t)(b0 + j + 1) % 32);
          if (c < bc) { bc = c; best = j; }
        }
        out[best] = x;
        add_readers(x, (uint32_t)(b0 + best + 1) % 32);
      }
      std::copy(out.begin(), out.end(), srcs.begin() + b0);
    }
    std::vector<int32_t> word(n, -1);
    word[0] = 0;
    uint32_t top = 1;
    for (uint32_t x : srcs) word[x] = (int32_t)top++;
    std::vector<std::set<uint32_t>> freew(32);
    std::vector<std::vector<uint32_t>> die(S + 1);
    for (uint32_t x : srcs)
      if (last[x] != INF) die[last[x]].push_back((uint32_t)word[x]);
    auto alloc = [&](uint32_t res) -> uint32_t {
      if (!freew[res].empty()) {
        const uint32_t w = *freew[res].begin();
        freew[res].erase(freew[res].begin());
        return w;
      }
      const uint32_t fresh = top + ((res + 32 - (top % 32)) % 32);
      for (uint32_t w = top; w < fresh; w++) freew[w % 32].insert(w);
      top = fresh + 1;
      return fresh;
    };
    auto lw = [&](uint32_t l) -> uint32_t {
      const int32_t w = word[l >> 1];
      if (w < 0) throw std::runtime_error("words: operand without a word");
      return (uint32_t)w;
    };
    std::vector<uint32_t> step_start(S + 1, 0), ops;
    ops.reserve((size_t)n_ops * 2);
    uint32_t max_step = 0;
    for (uint32_t s = 0; s < S; s++) {
      if (s > 0)
        for (uint32_t w : die[s - 1]) freew[w % 32].insert(w);
      step_start[s] = (uint32_t)(ops.size() / 2);
      auto& st = steps[s];
      max_step = std::max<uint32_t>(max_step, (uint32_t)st.size());
      std::stable_sort(st.begin(), st.end(), [&](uint32_t x, uint32_t y) { return rd[x] > rd[y]; });
      // rounds of 32 slots (one warp's LDS): take the first remaining op (in
      // priority order) whose A and B banks the round does not use yet (a word
      // already in the round is a broadcast, free); if none, the op adding the
      // fewest same-bank words
      std::vector<uint32_t> rem(st.begin(), st.end()), order;
      order.reserve(st.size());
      while (!rem.empty()) {
        uint8_t cntA[32] = {0}, cntB[32] = {0};
        std::vector<uint32_t> wA, wB;   // words already in the round
        const size_t take = std::min<size_t>(32, rem.size());
        for (size_t k = 0; k < take; k++) {
          size_t pick = 0;
          uint32_t best = UINT32_MAX;
          for (size_t c = 0; c < rem.size() && best; c++) {
            const uint32_t x = rem[c], a = lw(la[x]), b = lw(lb[x]);
            const bool inA = std::find(wA.begin(), wA.end(), a) != wA.end();
            const bool inB = std::find(wB.begin(), wB.end(), b) != wB.end();
            const uint32_t cost = (inA ? 0u : cntA[a % 32]) + (inB ? 0u : cntB[b % 32]);
            if (cost < best) { best = cost; pick = c; }
          }
          const uint32_t x = rem[pick];
          rem.erase(rem.begin() + (ptrdiff_t)pick);
          const uint32_t a = lw(la[x]), b = lw(lb[x]);
          if (std::find(wA.begin(), wA.end(), a) == wA.end()) { wA.push_back(a); cntA[a % 32]++; }
          if (std::find(wB.begin(), wB.end(), b) == wB.end()) { wB.push_back(b); cntB[b % 32]++; }
          order.push_back(x);
        }
      }
      uint32_t used = 0;   // banks already stored to by the op's warp (32 slots)
      for (uint32_t j = 0; j < (uint32_t)order.size(); j++) {
        const uint32_t x = order[j];
        const uint32_t a = lw(la[x]), b = lw(lb[x]);
        if (j % 32 == 0) used = 0;
        // a bank no other op of this warp stores to (conflict-free STS), the
        // one whose future readers have the fewest operands there, then the
        // lowest free word
        uint32_t bres = 0;
        uint64_t bkey = UINT64_MAX;
        for (uint32_t r = 0; r < 32; r++) {
          if ((used >> r) & 1u) continue;
          const uint64_t fw = freew[r].empty() ? 0xFFFFFFull : *freew[r].begin();
          const uint64_t key = ((uint64_t)std::min<uint32_t>(readers_cost(x, r), 0xFFFFFF) << 24) | fw;
          if (key < bkey) { bkey = key; bres = r; }
        }
        used |= 1u << bres;
        add_readers(x, bres);
        const uint32_t w = alloc(bres);
        word[x] = (int32_t)w;
        if (last[x] != INF) die[std::max(last[x], s)].push_back(w);
        ops.push_back((a * 4 | (la[x] & 1u)) | ((b * 4 | (lb[x] & 1u)) << 16));
        ops.push_back(w * 4);
      }
      if (top >= GEM_WORD_MAX_WORDS) return;
    }
    step_start[S] = (uint32_t)(ops.size() / 2);
    std::vector<uint32_t>& pr = P.word_prog;
    pr.assign(WPH_WORDS, 0);
    pr[WPH_MAGIC] = GEM_WORD_MAGIC;
    pr[WPH_N_GREAD] = (uint32_t)srcs.size();
    pr[WPH_N_STEPS] = S;
    pr[WPH_N_OPS] = n_ops;
    pr[WPH_N_OUT] = (uint32_t)P.outs.size();
    pr[WPH_N_RAM] = (uint32_t)P.rams.size();
    pr[WPH_STATE_WORDS] = (top + 3) & ~3u;
    pr[WPH_MAX_STEP_OPS] = max_step;
    pr[WPH_OFF_STEPS] = (uint32_t)pr.size();
    pr.insert(pr.end(), step_start.begin(), step_start.end());
    while (pr.size() % 4) pr.push_back(0);
    pr[WPH_OFF_OPS] = (uint32_t)pr.size();
    pr.insert(pr.end(), ops.begin(), ops.end());
    while (pr.size() % 4) pr.push_back(0);
    pr[WPH_OFF_OUT] = (uint32_t)pr.size();
    for (auto& ow : P.outs) pr.push_back(ow.dst);
    for (auto& ow : P.outs)
      for (int k = 0; k < 32; k++) {
        const uint32_t l = ow.lit[k];
        pr.push_back(lw(2 * (uint32_t)scratch[l >> 1]) * 4 | (l & 1u));
      }
    while (pr.size() % 4) pr.push_back(0);
    pr[WPH_OFF_RAM] = (uint32_t)pr.size();
    for (uint32_t r : P.rams) { pr.push_back(r); pr.push_back(0); pr.push_back(0); pr.push_back(0); }
    pr[WPH_OFF_GREAD] = (uint32_t)pr.size();
    for (uint32_t x : srcs) {
      const uint32_t gb = G.gbit[cid[x]];
      pr.push_back(((gb >> 27) << 24) | (((gb >> 5) & 0x3FFFFF) * 32 + (gb & 31)));
    }
    while (pr.size() % 4) pr.push_back(0);
    pr[WPH_PROG_LEN] = (uint32_t)pr.size();
    P.word_steps = S;
    P.word_ops = n_ops;
    if (opt.verbose >= 3)
      fprintf(stderr, "words part: ops=%u steps=%u max_step=%u srcs=%zu words=%u\n", n_ops, S, max_step,
              srcs.size(), top);
  }

  void fail(Part& P, const char* why) {
    P.ok = false;
    P.err = why;
    for (uint32_t c : cid) (void)c;
  }

  // Layer record encoding (gem_isa.h).  A warp whose fullest lane has more than
  // kDenseMin leaves uses the DENSE gather (32 entries per lane, entry index =
  // leaf position, 4 instructions per entry); otherwise SPARSE (explicit
  // positions, fewer entries).
  static constexpr uint32_t kDenseMin = 18;
  static void encode_layer(std::vector<uint32_t>& out, std::vector<int32_t>* slot, std::vector<uint8_t>* sxa,
                           std::vector<uint8_t>* sxb, std::vector<uint8_t>* sob,
                           const std::vector<int32_t>& wo_thread, const std::vector<int32_t>& wo_warp,
                           int32_t wo_top) {
    size_t base = out.size();
    out.resize(base + LH_WORDS, 0);
    // leaves per thread: (state bit, position)
    std::vector<std::vector<std::pair<uint32_t, uint32_t>>> leaves(256);
    for (uint32_t id = 0; id < 8192; id++)
      if (slot[0][id] >= 0) leaves[id >> 5].push_back({(uint32_t)slot[0][id], id & 31});
    uint32_t active = 0;
    uint32_t niter[8] = {0};
    for (uint32_t w = 0; w < 8; w++) {
      for (uint32_t l = 0; l < 32; l++) niter[w] = std::max<uint32_t>(niter[w], (uint32_t)leaves[w * 32 + l].size());
      bool act = niter[w] > 0 || wo_warp[w] >= 0;
      for (uint32_t l = 0; l < 32; l++) act = act || wo_thread[w * 32 + l] >= 0;
      if (act) active |= 1u << w;
    }
    auto pack = [&](int k0, int k1, uint32_t unit, const std::vector<uint8_t>* arr) {
      uint32_t v = 0;
      for (int k = k0; k <= k1; k++) {
        uint32_t g = group_width(k);
        for (uint32_t q = 0; q < g; q++) {
          uint32_t id = unit * g + q;
          if (arr[k][id]) v |= 1u << slot_bit(k, id);
        }
      }
      return v;
    };
    bool uses_top = wo_top >= 0;
    out[base + LH_FLAGS] = active | (uses_top ? GEM_LF_USES_TOP : 0u);
    out[base + LH_TOPC] = pack(11, 13, 0, sxa) | (pack(11, 13, 0, sxb) << 8) | (pack(11, 13, 0, sob) << 16);
    out[base + LH_TOPWO] = uses_top ? (uint32_t)wo_top : 0u;
    for (uint32_t w = 0; w < 8; w++) {
      if (!(active >> w & 1)) continue;
      out[base + LH_WOFF0 + w] = (uint32_t)(out.size() - base);
      const bool dense = niter[w] > kDenseMin;
      bool small_words = true;
      for (uint32_t l = 0; l < 32; l++)
        for (auto& x : leaves[w * 32 + l]) small_words = small_words && (x.first >> 5) < 2048;
      const bool d16 = dense && small_words;
      const uint32_t n4 = d16 ? 4u : dense ? 8u : std::max<uint32_t>(1u, (niter[w] + 3) / 4);
      out.push_back(pack(6, 10, w, sxa));
      out.push_back(pack(6, 10, w, sxb));
      out.push_back(pack(6, 10, w, sob));
      out.push_back(wo_warp[w] >= 0 ? (uint32_t)wo_warp[w] : 0u);
      out.push_back((d16 ? GEM_WM_DENSE16 : dense ? GEM_WM_DENSE : GEM_WM_SPARSE) | (n4 << 8));
      out.push_back(0); out.push_back(0); out.push_back(0);
      for (uint32_t l = 0; l < 32; l++) {
        uint32_t t = w * 32 + l;
        out.push_back(pack(1, 5, t, sxa));
        out.push_back(pack(1, 5, t, sxb));
        out.push_back(pack(1, 5, t, sob));
        out.push_back(wo_thread[t] >= 0 ? (uint32_t)wo_thread[t] : 0u);
      }
      for (uint32_t g = 0; g < n4; g++)
        for (uint32_t l = 0; l < 32; l++) {
          auto& lv = leaves[w * 32 + l];
          for (uint32_t c = 0; c < 4; c++) {
            uint32_t j = 4 * g + c, e = 0;
            if (d16) {
              for (uint32_t h = 0; h < 2; h++) {
                uint32_t jj = 8 * g + 2 * c + h;
                for (auto& x : lv)
                  if (x.second == jj) e |= GEM_LEAF16(x.first >> 5, x.first & 31, jj) << (16 * h);
              }
            } else if (dense) {
              for (auto& x : lv)
                if (x.second == j) e = GEM_LEAF_DENSE(x.first >> 5, x.first & 31, j);
            } else if (j < lv.size()) {
              e = GEM_LEAF(lv[j].first >> 5, lv[j].first & 31, lv[j].second);
            }
            out.push_back(e);
          }
        }
    }
    out[base + LH_WORDS_] = (uint32_t)(out.size() - base);
  }
};

// Estimated SM clocks for one cycle of a partition program (cost model fitted to
// B200 phase measurements: fixed per-layer latency + per-16-byte leaf group).
static uint32_t part_cost(const uint32_t* pr) {
  const double kItem = 6000.0, kLayer = 1900.0, kGroup = 12.0, kGread = 2.0, kOut = 20.0;
  double c = kItem + kGread * pr[PH_N_GREAD] + kOut * pr[PH_N_OUT];
  const uint32_t* L = pr + pr[PH_OFF_LAYERS];
  for (uint32_t l = 0; l < pr[PH_N_LAYERS]; l++) {
    uint32_t groups = 0;
    for (uint32_t w = 0; w < 8; w++)
      if (L[LH_WOFF0 + w]) groups += L[L[LH_WOFF0 + w] + 4] >> 8;
    c += kLayer + kGroup * groups;
    L += L[LH_WORDS_];
  }
  return (uint32_t)std::min(c, 4.0e9);
}

// =========================================================== partitioning
struct Design {
  Graph G;
  SynthStats synth;                 // depth-oriented synthesis report (gem_synth.h)
  std::vector<uint32_t> ext_gbit;   // source locations before the internal flop layout
  Options opt;
  std::vector<Part> parts;
  uint32_t q_words = 0, po_words = 0, cut_words = 0, n_stages = 1;
  std::vector<int64_t> q_ext_of_int, po_ext_of_int;   // internal bit -> external index / -1
  std::vector<uint32_t> cut_lit;                      // cut index -> compact literal
};

static uint64_t mix64(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return x;
}

// min-hash cone signatures: sig(n) = min(h(n), sig(a), sig(b))
static std::vector<uint64_t> cone_minhash(const Graph& G, uint64_t seed) {
  size_t N = G.kind.size();
  std::vector<uint64_t> s(N);
  for (size_t i = 0; i < N; i++) {
    uint64_t h = mix64(i * 0x9E3779B97F4A7C15ull + seed);
    if (G.kind[i] == K_AND) h = std::min(h, std::min(s[G.a[i] >> 1], s[G.b[i] >> 1]));
    else if (G.kind[i] == K_CONST) h = UINT64_MAX;
    s[i] = h;
  }
  return s;
}

static void partition(Design& D) {
  const Graph& G = D.G;
  const Options& opt = D.opt;
  size_t N = G.kind.size();
  // stage assignment of nodes: stage 1 nodes have level > cut
  uint32_t cut = 0;
  if (opt.stages == 2) {
    cut = opt.cut_level ? (uint32_t)opt.cut_level : std::max<uint32_t>(1, G.max_level / 2);
  }
  // ---- units
  std::vector<Unit> units;
  // Locality key of a unit: the smallest flop (state) index in its cone --
  // logic that reads the same registers sits in the same module -- with a
  // cone min-hash as tie breaker.
  auto s0 = cone_minhash(G, 1);
  std::vector<uint32_t> mflop(N, UINT32_MAX);
  for (size_t i = 0; i < N; i++) {
    if (G.kind[i] == K_SRC) {
      uint32_t gb = G.gbit[i];
      if ((gb >> 27) == GEM_R_Q) mflop[i] = ((gb >> 5) & 0x3FFFFF) * 32 + (gb & 31);
      else if ((gb >> 27) == GEM_R_RD) mflop[i] = 0x7FFFFFFFu + ((gb >> 5) & 0x3FFFFF);
    } else if (G.kind[i] == K_AND) {
      mflop[i] = std::min(mflop[G.a[i] >> 1], mflop[G.b[i] >> 1]);
    }
  }
  // key 1: min-hash over the endpoint's *deep* cone (nodes below a third of the
  // depth): endpoints whose deep logic coincides -- one module's registers --
  // sort together, whatever registers of neighbouring modules they also read
  std::vector<uint64_t> sdeep;
  if (opt.key == 1) {
    sdeep.assign(N, UINT64_MAX);
    const uint32_t thr = std::max<uint32_t>(1, G.max_level / 3);
    for (size_t i = 0; i < N; i++) {
      if (G.kind[i] != K_AND) continue;
      uint64_t h = G.level[i] >= thr ? mix64(i * 0x9E3779B97F4A7C15ull + 11) : UINT64_MAX;
      sdeep[i] = std::min(h, std::min(sdeep[G.a[i] >> 1], sdeep[G.b[i] >> 1]));
    }
  }
  auto key_of = [&](uint32_t lit) -> uint64_t {
    uint32_t x = lit >> 1;
    if (opt.key == 1 && sdeep[x] != UINT64_MAX) return sdeep[x] >> 1;
    if (opt.key == 1) return (1ull << 63) | ((uint64_t)mflop[x] << 31) | (s0[x] >> 33);
    return ((uint64_t)mflop[x] << 32) | (s0[x] >> 32);
  };
  std::vector<uint32_t> cut_nodes;            // compact ids that are stage-0 endpoints
  std::vector<int32_t> cut_of(N, -1);
  if (opt.stages == 2) {
    // cut nodes: level <= cut with a consumer above the cut, or an endpoint above... (endpoints
    // deeper than the cut are stage-1 units; shallow endpoints stay stage-0 units)
    std::vector<uint8_t> live(N, 0);
    for (auto l : G.flop_next) live[l >> 1] = 1;
    for (auto l : G.po) live[l >> 1] = 1;
    for (auto& rr : G.rams) for (int p = 0; p < 4; p++) for (int k = 0; k < 32; k++) live[rr.port[p][k] >> 1] = 1;
    for (size_t i = N; i-- > 0;)
      if (live[i] && G.kind[i] == K_AND) { live[G.a[i] >> 1] = 1; live[G.b[i] >> 1] = 1; }
    for (size_t i = 0; i < N; i++) {
      if (!live[i] || G.kind[i] != K_AND || G.level[i] <= cut) continue;
      for (uint32_t y : {G.a[i] >> 1, G.b[i] >> 1})
        if (G.kind[y] == K_AND && G.level[y] <= cut && cut_of[y] < 0) {
          cut_of[y] = (int32_t)cut_nodes.size();
          cut_nodes.push_back(y);
        }
    }
  }
  auto ep_stage = [&](uint32_t lit) -> int {
    if (opt.stages == 1) return 0;
    uint32_t x = lit >> 1;
    return (G.kind[x] == K_AND && G.level[x] > cut) ? 1 : 0;
  };
  for (uint32_t j = 0; j < G.n_flops; j++)
    units.push_back({0, j, opt.key == 2 ? ((uint64_t)j << 32) : key_of(G.flop_next[j])});
  for (uint32_t j = 0; j < G.n_po; j++) units.push_back({1, j, key_of(G.po[j])});
  for (uint32_t r = 0; r < G.n_rams; r++) {
    uint64_t k = UINT64_MAX;
    for (int p = 0; p < 4; p++) for (int b = 0; b < 32; b++) k = std::min(k, key_of(G.rams[r].port[p][b]));
    units.push_back({2, r, k});
  }
  for (uint32_t c = 0; c < cut_nodes.size(); c++) units.push_back({3, c, key_of(2 * cut_nodes[c])});
  // unit stage
  auto unit_stage = [&](const Unit& u) -> int {
    if (opt.stages == 1) return 0;
    if (u.kind == 0) return ep_stage(G.flop_next[u.idx]);
    if (u.kind == 1) return ep_stage(G.po[u.idx]);
    if (u.kind == 3) return 0;
    int s = 0;
    for (int p = 0; p < 4; p++) for (int b = 0; b < 32; b++) s = std::max(s, ep_stage(G.rams[u.idx].port[p][b]));
    return s;
  };
  // sources of a stage-1 cone: cut nodes act as leaves
  auto is_leaf_for = [&](uint32_t x, int stage) {
    if (G.kind[x] != K_AND) return true;
    return stage == 1 && cut_of[x] >= 0;
  };
  auto unit_lits = [&](const Unit& u, std::vector<uint32_t>& out) {
    out.clear();
    if (u.kind == 0) out.push_back(G.flop_next[u.idx]);
    else if (u.kind == 1) out.push_back(G.po[u.idx]);
    else if (u.kind == 2) { for (int p = 0; p < 4; p++) for (int b = 0; b < 32; b++) out.push_back(G.rams[u.idx].port[p][b]); }
    else out.push_back(2 * cut_nodes[u.idx]);
  };
  for (int stage = 0; stage < opt.stages; stage++) {
    std::vector<Unit> su;
    for (auto& u : units) if (unit_stage(u) == stage) su.push_back(u);
    std::stable_sort(su.begin(), su.end(), [](const Unit& a, const Unit& b) { return a.key < b.key; });
    // cone sizes in stage terms; greedy sequential packing with a size cap
    std::vector<uint32_t> stamp(N, 0);
    uint32_t cur_stamp = 0;
    std::vector<uint32_t> st;
    std::vector<uint32_t> lits;
    auto add_cone = [&](const Unit& u) -> uint32_t {
      uint32_t added = 0;
      unit_lits(u, lits);
      for (uint32_t l : lits) {
        uint32_t x = l >> 1;
        if (stamp[x] == cur_stamp) continue;
        stamp[x] = cur_stamp;
        st.push_back(x);
        while (!st.empty()) {
          uint32_t y = st.back(); st.pop_back();
          if (is_leaf_for(y, stage)) continue;
          added++;
          for (uint32_t z : {G.a[y] >> 1, G.b[y] >> 1})
            if (stamp[z] != cur_stamp) { stamp[z] = cur_stamp; st.push_back(z); }
        }
      }
      return added;
    };
    // total stage work estimate
    uint64_t stage_ands = 0;
    {
      cur_stamp++;
      for (auto& u : su) stage_ands += add_cone(u);
    }
    int target = opt.parts > 0 ? opt.parts : (int)std::max<uint64_t>(1, (G.n_and_live + opt.part_size / 2) / opt.part_size);
    if (opt.stages == 2) target = std::max(1, target / 2);
    target = std::max(1, std::min<int>(target, (int)su.size()));
    // a cap below typical single-unit cones would leave every unit alone (and
    // re-traverse each full cone): start from >= 3x the median unit cone
    double med = 0;
    {
      std::vector<uint32_t> sz;
      for (size_t i = 0; i < su.size(); i += std::max<size_t>(1, su.size() / 256)) {
        cur_stamp++;
        sz.push_back(add_cone(su[i]));
      }
      if (!sz.empty()) {
        std::nth_element(sz.begin(), sz.begin() + sz.size() / 2, sz.end());
        med = sz[sz.size() / 2];
      }
    }
    double cap = std::max<double>({64.0, 4.0 * (double)stage_ands / target * opt.cap_slack, 3.0 * med});
    // unit cones (CSR over su) and node users: the RepCut hypergraph (one
    // hyperedge per AND node over the units whose cone contains it)
    const uint32_t nu = (uint32_t)su.size();
    std::vector<uint32_t> uoff(nu + 1, 0), unodes, users;
    const bool need_cones = opt.km1 > 0;
    if (need_cones) {
      for (uint32_t i = 0; i < nu; i++) {
        cur_stamp++;
        unit_lits(su[i], lits);
        for (uint32_t l : lits) {
          uint32_t x = l >> 1;
          if (stamp[x] == cur_stamp) continue;
          stamp[x] = cur_stamp;
          st.push_back(x);
          while (!st.empty()) {
            uint32_t y = st.back(); st.pop_back();
            if (is_leaf_for(y, stage)) continue;
            unodes.push_back(y);
            for (uint32_t z : {G.a[y] >> 1, G.b[y] >> 1})
              if (stamp[z] != cur_stamp) { stamp[z] = cur_stamp; st.push_back(z); }
          }
        }
        uoff[i + 1] = (uint32_t)unodes.size();
      }
      users.assign(N, 0);
      for (uint32_t x : unodes) users[x]++;
    }
    auto shared = [&](uint32_t x) { return users[x] >= 2 && users[x] <= (uint32_t)opt.km1_pins; };
    auto pack = [&](double pcap, std::vector<std::vector<uint32_t>>& out) {
      out.clear();
      cur_stamp++;
      uint64_t size = 0;
      for (uint32_t i = 0; i < su.size(); i++) {
        // try adding to the current group
        if (out.empty()) out.emplace_back();
        uint32_t add = add_cone(su[i]);
        if (!out.back().empty() && size + add > pcap) {
          // start a new group containing unit i
          out.emplace_back();
          cur_stamp++;
          size = add_cone(su[i]);
          out.back().push_back(i);
        } else {
          size += add;
          out.back().push_back(i);
        }
      }
    };
    // cap search: the group count as a function of the cap is not monotone
    // (below the size of typical shared cones every unit ends up alone), so
    // keep the iteration whose count is closest to the target
    std::vector<std::vector<uint32_t>> groups, best_groups;   // indices into su
    double best_err = 1e300, best_cap = cap;
    for (int iter = 0; iter < 6; iter++) {
      pack(cap, groups);
      const double ratio = (double)groups.size() / target;
      if (opt.verbose >= 1)
        fprintf(stderr, "gem_map: stage %d packing iter %d cap %.0f -> %zu groups (target %d)\\n", stage, iter, cap,
                groups.size(), target);
      const double err = std::fabs(std::log(ratio));
      if (err < best_err) { best_err = err; best_cap = cap; best_groups = groups; }
      if (ratio > 0.85 && ratio < 1.2) break;
      cap *= std::max(0.5, std::min(2.0, ratio > 3.0 ? 1.5 : ratio));
    }
    groups.swap(best_groups);
    cap = best_cap;
    // ---- min-cut refinement (the partitioner of P:105/P:117, RepCut [17]):
    // the RepCut hypergraph has one vertex per unit (endpoint) and one
    // hyperedge per AND node, spanning the units whose cone contains it; a
    // node is replicated in every partition that holds one of its units, so
    // the replication cost is the connectivity-minus-one (km1) metric
    // sum_x (lambda(x) - 1).  k-way FM-style passes move single units to the
    // partition that lowers km1 most (gain = the unit's shared nodes that leave
    // its partition minus those new to the target), keeping every partition's
    // cone under km1_slack x the packing cap.  Nodes with one user move with
    // their unit; nodes with more than km1_pins users (shallow, wide logic that
    // every partition needs anyway) are left out of the gains.
    if (opt.km1 > 0 && groups.size() > 1) {
      // per shared node: (partition, count) slots, at most `users` of them
      std::vector<uint32_t> noff(N + 1, 0);
      for (size_t x = 0; x < N; x++) noff[x + 1] = noff[x] + ((users[x] >= 2 && users[x] <= (uint32_t)opt.km1_pins) ? users[x] : 0);
      std::vector<uint32_t> npart(noff[N], UINT32_MAX), ncnt(noff[N], 0);
      std::vector<uint8_t> nlen(N, 0);
      std::vector<uint32_t> part_of(nu, 0);
      const uint32_t ng = (uint32_t)groups.size();
      for (uint32_t g = 0; g < ng; g++) for (uint32_t i : groups[g]) part_of[i] = g;
      auto slot = [&](uint32_t x, uint32_t P) -> int64_t {
        for (uint32_t k = 0; k < nlen[x]; k++) if (npart[noff[x] + k] == P) return noff[x] + k;
        return -1;
      };
      auto add = [&](uint32_t x, uint32_t P) {
        int64_t k = slot(x, P);
        if (k < 0) { k = noff[x] + nlen[x]++; npart[k] = P; ncnt[k] = 0; }
        ncnt[k]++;
      };
      auto remove = [&](uint32_t x, uint32_t P) {
        const int64_t k = slot(x, P);
        if (--ncnt[k] == 0) {
          const uint32_t last = noff[x] + --nlen[x];
          npart[k] = npart[last]; ncnt[k] = ncnt[last];
        }
      };
      // partition sizes: exact cones (private + shared + wide nodes)
      std::vector<uint64_t> psize(ng, 0);
      {
        std::vector<uint32_t> mark(N, UINT32_MAX);
        for (uint32_t g = 0; g < ng; g++)
          for (uint32_t i : groups[g])
            for (uint32_t k = uoff[i]; k < uoff[i + 1]; k++) {
              const uint32_t x = unodes[k];
              if (mark[x] != g) { mark[x] = g; psize[g]++; }
            }
      }
      for (uint32_t i = 0; i < nu; i++)
        for (uint32_t k = uoff[i]; k < uoff[i + 1]; k++)
          if (shared(unodes[k])) add(unodes[k], part_of[i]);
      // from here on a unit needs only its shared nodes and its private count
      std::vector<uint32_t> upriv(nu, 0);
      {
        std::vector<uint32_t> off2(nu + 1, 0), sh;
        sh.reserve(unodes.size() / 4);
        for (uint32_t i = 0; i < nu; i++) {
          for (uint32_t k = uoff[i]; k < uoff[i + 1]; k++) {
            const uint32_t x = unodes[k];
            if (users[x] == 1) upriv[i]++;
            else if (shared(x)) sh.push_back(x);
          }
          off2[i + 1] = (uint32_t)sh.size();
        }
        uoff.swap(off2);
        unodes.swap(sh);
      }
      auto km1_cost = [&]() {
        uint64_t c = 0;
        for (size_t x = 0; x < N; x++) if (nlen[x]) c += nlen[x] - 1;
        return c;
      };
      const uint64_t before = km1_cost();
      uint64_t rep_before = 0;
      for (uint32_t g = 0; g < ng; g++) rep_before += psize[g];
      const double pcap = cap * opt.km1_slack;
      std::vector<uint32_t> have(ng, 0), touched;
      std::vector<uint32_t> order(nu);
      std::iota(order.begin(), order.end(), 0);
      uint64_t moves_total = 0;
      for (int pass = 0; pass < opt.km1; pass++) {
        uint64_t moves = 0;
        // deterministic shuffle per pass
        for (uint32_t i = nu; i > 1; i--) std::swap(order[i - 1], order[mix64(pass * 1000003ull + i) % i]);
        for (uint32_t i : order) {
          const uint32_t A = part_of[i];
          if (groups[A].size() <= 1) continue;
          uint32_t n_sh = 0, loss = 0;
          const uint32_t priv = upriv[i];
          touched.clear();
          for (uint32_t k = uoff[i]; k < uoff[i + 1]; k++) {
            const uint32_t x = unodes[k];
            n_sh++;
            for (uint32_t q = 0; q < nlen[x]; q++) {
              const uint32_t P = npart[noff[x] + q];
              if (P == A) { if (ncnt[noff[x] + q] == 1) loss++; continue; }
              if (!have[P]++) touched.push_back(P);
            }
          }
          int64_t best_gain = 0;
          uint32_t best = UINT32_MAX;
          for (uint32_t P : touched) {
            const int64_t gain = (int64_t)loss - (int64_t)(n_sh - have[P]);
            const double new_size = (double)psize[P] + priv + (n_sh - have[P]);
            if (new_size > pcap) continue;
            if (gain > best_gain || (gain == best_gain && gain > 0 && P < best)) { best_gain = gain; best = P; }
          }
          for (uint32_t P : touched) have[P] = 0;
          if (best == UINT32_MAX) continue;
          // commit the move A -> best (sizes: wide nodes are assumed present in both)
          psize[A] -= priv + loss;
          psize[best] += priv + (uint64_t)((int64_t)loss - best_gain);   // = shared nodes new to `best`
          for (uint32_t k = uoff[i]; k < uoff[i + 1]; k++) { remove(unodes[k], A); add(unodes[k], best); }
          part_of[i] = best;
          auto& ga = groups[A];
          ga.erase(std::find(ga.begin(), ga.end(), i));
          groups[best].push_back(i);
          moves++;
        }
        moves_total += moves;
        if (moves * 200 < nu) break;   // converged (< 0.5% of the units moved)
      }
      for (auto& g : groups) std::sort(g.begin(), g.end());
      std::vector<std::vector<uint32_t>> kept;
      for (auto& g : groups) if (!g.empty()) kept.push_back(std::move(g));
      groups.swap(kept);
      if (opt.verbose >= 1) {
        uint64_t pins = 0;
        for (size_t x = 0; x < N; x++) if (shared((uint32_t)x)) pins += users[x];
        fprintf(stderr, "gem_map: stage %d km1 refinement: %llu moves, km1 %llu -> %llu (%llu pins, %zu groups)\n",
                stage, (unsigned long long)moves_total, (unsigned long long)before, (unsigned long long)km1_cost(),
                (unsigned long long)pins, groups.size());
      }
      (void)rep_before;
    }
    // ---- Algorithm 1: after the excessive partitioning above,
    // visit partitions largest first; sort the unvisited ones by cone overlap
    // with p (large to small) and merge q into p if the result stays mappable.
    // "Mappable" here: the merged cone stays under merge_cap ANDs (the width /
    // state check proper runs in the mapper, which splits a partition that
    // does not fit), and the overlap is a real saving (>= merge_ratio of the
    // smaller cone) -- merging disjoint logic would only lengthen layers.
    if (opt.merge && groups.size() > 1) {
      const size_t ng = groups.size();
      std::vector<std::vector<uint32_t>> cone(ng);
      for (size_t gi = 0; gi < ng; gi++) {
        cur_stamp++;
        for (uint32_t i : groups[gi]) {
          unit_lits(su[i], lits);
          for (uint32_t l : lits) {
            uint32_t x = l >> 1;
            if (stamp[x] == cur_stamp) continue;
            stamp[x] = cur_stamp;
            st.push_back(x);
            while (!st.empty()) {
              uint32_t y = st.back(); st.pop_back();
              if (is_leaf_for(y, stage)) continue;
              cone[gi].push_back(y);
              for (uint32_t z : {G.a[y] >> 1, G.b[y] >> 1})
                if (stamp[z] != cur_stamp) { stamp[z] = cur_stamp; st.push_back(z); }
            }
          }
        }
        std::sort(cone[gi].begin(), cone[gi].end());
      }
      // inverted index node -> groups (CSR)
      std::vector<uint32_t> cnt(N + 1, 0);
      for (size_t gi = 0; gi < ng; gi++) for (uint32_t x : cone[gi]) cnt[x + 1]++;
      for (size_t i = 0; i < N; i++) cnt[i + 1] += cnt[i];
      std::vector<uint32_t> inv(cnt[N]);
      {
        std::vector<uint32_t> f(cnt.begin(), cnt.end() - 1);
        for (size_t gi = 0; gi < ng; gi++) for (uint32_t x : cone[gi]) inv[f[x]++] = (uint32_t)gi;
      }
      const double cap = opt.merge_cap > 0 ? opt.merge_cap : 2.5 * opt.part_size;
      std::vector<int32_t> owner(ng);          // group -> current merged partition
      std::iota(owner.begin(), owner.end(), 0);
      std::vector<uint8_t> visited(ng, 0);
      std::vector<size_t> order(ng);
      std::iota(order.begin(), order.end(), 0);
      std::stable_sort(order.begin(), order.end(), [&](size_t a, size_t b) { return cone[a].size() > cone[b].size(); });
      std::vector<uint32_t> ov(ng, 0);
      size_t merges = 0;
      for (size_t p : order) {
        if (visited[p]) continue;
        visited[p] = 1;
        // overlap of p's (growing) cone with every unvisited original group
        std::vector<uint32_t> touched;
        for (uint32_t x : cone[p])
          for (uint32_t k = cnt[x]; k < cnt[x + 1]; k++) {
            const uint32_t q = inv[k];
            if (visited[q]) continue;
            if (!ov[q]++) touched.push_back(q);
          }
        std::sort(touched.begin(), touched.end(), [&](uint32_t a, uint32_t b) {
          return ov[a] != ov[b] ? ov[a] > ov[b] : a < b;
        });
        for (uint32_t q : touched) {
          const uint32_t o = ov[q];
          if (visited[q]) continue;
          const size_t a = cone[p].size(), b = cone[q].size();
          if (o < opt.merge_ratio * std::min(a, b) || a + b - o > cap) continue;
          // commit: p absorbs q (units and cone); overlaps with q's new nodes are not re-counted
          std::vector<uint32_t> u;
          u.reserve(a + b - o);
          std::set_union(cone[p].begin(), cone[p].end(), cone[q].begin(), cone[q].end(), std::back_inserter(u));
          cone[p].swap(u);
          groups[p].insert(groups[p].end(), groups[q].begin(), groups[q].end());
          groups[q].clear();
          cone[q].clear();
          cone[q].shrink_to_fit();
          visited[q] = 1;
          merges++;
        }
        for (uint32_t q : touched) ov[q] = 0;
      }
      std::vector<std::vector<uint32_t>> kept;
      for (auto& g : groups) if (!g.empty()) { std::sort(g.begin(), g.end()); kept.push_back(std::move(g)); }
      groups.swap(kept);
      if (opt.verbose >= 1)
        fprintf(stderr, "gem_map: stage %d Algorithm 1 merged %zu pairs -> %zu groups\n", stage, merges, groups.size());
    }
    for (auto& grp : groups) {
      Part P;
      P.stage = stage;
      for (uint32_t i : grp) {
        const Unit& u = su[i];
        if (u.kind == 0) P.flops.push_back(u.idx);
        else if (u.kind == 1) P.pos.push_back(u.idx);
        else if (u.kind == 2) P.rams.push_back(u.idx);
        else P.cuts.push_back(u.idx);
      }
      D.parts.push_back(std::move(P));
    }
  }
  D.n_stages = (uint32_t)opt.stages;
  D.cut_lit.resize(cut_nodes.size());
  for (size_t c = 0; c < cut_nodes.size(); c++) D.cut_lit[c] = 2 * cut_nodes[c];
  // stage-1 sources: cut nodes are read from the CUT region; rewrite graph view
  // by giving cut nodes a gbit (the Mapper treats nodes with gbit as sources
  // only in stage 1, see layout()).
  (void)cut;
}

// internal layout: each partition owns whole internal words for its flops / POs / cuts
static void layout(Design& D) {
  Graph& G = D.G;
  uint32_t qw = 0, pw = 0, cw = 0;
  D.q_ext_of_int.clear();
  D.po_ext_of_int.clear();
  std::vector<uint32_t> q_int_of_ext(G.n_flops), cut_int(D.cut_lit.size());
  for (auto& P : D.parts) {
    auto words = [](size_t n) { return (uint32_t)((n + 31) / 32); };
    for (size_t k = 0; k < P.flops.size(); k++) q_int_of_ext[P.flops[k]] = qw * 32 + (uint32_t)k;
    for (size_t k = 0; k < P.cuts.size(); k++) cut_int[P.cuts[k]] = cw * 32 + (uint32_t)k;
    for (uint32_t w = 0; w < words(P.flops.size()); w++)
      for (int b = 0; b < 32; b++) {
        size_t k = w * 32 + b;
        D.q_ext_of_int.push_back(k < P.flops.size() ? (int64_t)P.flops[k] : -1);
      }
    for (uint32_t w = 0; w < words(P.pos.size()); w++)
      for (int b = 0; b < 32; b++) {
        size_t k = w * 32 + b;
        D.po_ext_of_int.push_back(k < P.pos.size() ? (int64_t)P.pos[k] : -1);
      }
    qw += words(P.flops.size());
    pw += words(P.pos.size());
    cw += words(P.cuts.size());
  }
  D.q_words = qw; D.po_words = pw; D.cut_words = cw;
  // rewrite latch source locations to the internal layout
  if (D.ext_gbit.empty()) D.ext_gbit = G.gbit;
  for (size_t i = 0; i < G.kind.size(); i++) {
    if (G.kind[i] != K_SRC) continue;
    uint32_t gb = D.ext_gbit[i];
    if ((gb >> 27) == GEM_R_Q) {
      uint32_t ext = ((gb >> 5) & 0x3FFFFF) * 32 + (gb & 31);
      uint32_t in = q_int_of_ext[ext];
      G.gbit[i] = mk_gbit(GEM_R_Q, in / 32, in % 32);
    }
  }
  // output words per partition
  uint32_t qbase = 0, pbase = 0, cbase = 0;
  for (auto& P : D.parts) {
    P.outs.clear();
    auto emit = [&](uint32_t region, uint32_t base, const std::vector<uint32_t>& idx,
                    const std::function<uint32_t(uint32_t)>& lit_of) {
      uint32_t nw = (uint32_t)((idx.size() + 31) / 32);
      for (uint32_t w = 0; w < nw; w++) {
        OutWord o;
        o.dst = GEM_GID(region, base + w);
        for (int b = 0; b < 32; b++) {
          size_t k = w * 32 + b;
          o.lit[b] = k < idx.size() ? lit_of(idx[k]) : 0u;
        }
        P.outs.push_back(o);
      }
      return nw;
    };
    qbase += emit(GEM_R_Q, qbase, P.flops, [&](uint32_t j) { return G.flop_next[j]; });
    pbase += emit(GEM_R_PO, pbase, P.pos, [&](uint32_t j) { return G.po[j]; });
    cbase += emit(GEM_R_CUT, cbase, P.cuts, [&](uint32_t c) { return D.cut_lit[c]; });
    for (uint32_t r = 0; r < P.rams.size(); r++)
      for (int p = 0; p < 4; p++) {
        OutWord o;
        o.dst = GEM_GID(GEM_R_RAMP, r * 4 + p);
        for (int b = 0; b < 32; b++) o.lit[b] = G.rams[P.rams[r]].port[p][b];
        P.outs.push_back(o);
      }
  }
  D.cut_lit.clear();
  // cut nodes become CUT-region sources for stage-1 partitions: remember them
  D.cut_lit.resize(cut_int.size());
  for (size_t c = 0; c < cut_int.size(); c++) D.cut_lit[c] = cut_int[c];
}

// =========================================================== top level
struct Blob {
  std::vector<uint32_t> w;
};

static Blob compile(const char* data, size_t n, const char* opts) {
  auto t0 = std::chrono::steady_clock::now();
  Design D;
  D.opt = parse_opts(opts);
  auto tick = [&](const char* what) {
    if (D.opt.verbose) {
      static thread_local auto last = std::chrono::steady_clock::now();
      auto now = std::chrono::steady_clock::now();
      fprintf(stderr, "gem_map: %-10s %8.0f ms\n", what, std::chrono::duration<double, std::milli>(now - last).count());
      last = now;
    }
  };
  tick("start");
  Raw raw = read_aiger(data, n);
  tick("parse");
  D.G = build_graph(raw);
  raw = Raw();
  tick("strash");
  D.G = synthesize(D.G, D.opt.synth, D.opt.chain_min, D.opt.chain_slack, D.synth);
  tick("synth");
  if (D.opt.verbose)
    fprintf(stderr, "gem_map: synth ANDs %llu -> %llu (balanced %llu), levels %u -> %u (balanced %u), "
            "%u chains / %u links / %u taps\n", (unsigned long long)D.synth.and_in, (unsigned long long)D.synth.and_out,
            (unsigned long long)D.synth.and_balanced, D.synth.level_in, D.synth.level_out, D.synth.level_balanced,
            D.synth.chains, D.synth.chain_links, D.synth.chain_taps);
  partition(D);
  tick("partition");
  // remember which compact nodes are cut nodes (stage-1 leaves) before layout rewrites cut_lit
  std::vector<uint32_t> cut_nodes;
  for (auto& P : D.parts) (void)P;
  {
    // cut_lit holds compact literals at this point
    for (auto l : D.cut_lit) cut_nodes.push_back(l >> 1);
  }
  std::vector<uint32_t> cut_compact = D.cut_lit;   // compact literals of cut nodes
  auto t1 = std::chrono::steady_clock::now();
  int nth = D.opt.threads > 0 ? D.opt.threads : (int)std::max(1u, std::thread::hardware_concurrency());
  // deep-cone signature: min-hash over the nodes deeper than a third of the depth
  std::vector<uint64_t> dsig(D.G.kind.size(), UINT64_MAX);
  {
    const uint32_t thr = std::max<uint32_t>(1, D.G.max_level / 3);
    for (size_t i = 0; i < D.G.kind.size(); i++) {
      if (D.G.kind[i] != K_AND) continue;
      uint64_t h = D.G.level[i] >= thr ? mix64(i * 0x9E3779B97F4A7C15ull + 7) : UINT64_MAX;
      dsig[i] = std::min(h, std::min(dsig[D.G.a[i] >> 1], dsig[D.G.b[i] >> 1]));
    }
  }
  int refine_round = 0;
  for (int attempt = 0;; attempt++) {
    D.cut_lit = cut_compact;
    layout(D);   // cut_lit now holds internal cut bit indices
    // Stage-1 partitions see cut nodes as sources: a graph view where cut
    // nodes are K_SRC with a CUT-region location.
    Graph G1;
    bool two = D.n_stages == 2;
    if (two) {
      G1 = D.G;
      for (size_t c = 0; c < cut_nodes.size(); c++) {
        uint32_t x = cut_nodes[c];
        uint32_t in = D.cut_lit[c];
        G1.kind[x] = K_SRC;
        G1.gbit[x] = mk_gbit(GEM_R_CUT, in / 32, in % 32);
      }
    }
    std::atomic<size_t> next{0};
    std::vector<std::thread> th;
    for (int t = 0; t < nth; t++)
      th.emplace_back([&]() {
        std::vector<int32_t> scratch(D.G.kind.size(), -1);
        while (true) {
          size_t i = next++;
          if (i >= D.parts.size()) break;
          Part& P = D.parts[i];
          Mapper M(P.stage == 1 ? G1 : D.G, D.opt);
          try {
            M.map(P, scratch);
          } catch (const std::exception& e) {
            P.ok = false;
            P.err = e.what();
          }
        }
      });
    for (auto& x : th) x.join();
    // split partitions that did not fit (state overflow) and retry
    std::vector<Part> next_parts;
    bool any_fail = false;
    std::string last_err;
    for (size_t i = 0; i < D.parts.size(); i++) {
      Part& P = D.parts[i];
      if (P.ok) { next_parts.push_back(std::move(P)); continue; }
      any_fail = true;
      last_err = P.err;
      size_t n_units = P.flops.size() + P.pos.size() + P.rams.size() + P.cuts.size();
      if (n_units <= 1 || attempt >= 12)
        throw std::runtime_error("mapping partition " + std::to_string(i) + " failed: " + P.err);
      Part A, B;
      A.stage = B.stage = P.stage;
      auto half = [](const std::vector<uint32_t>& v, std::vector<uint32_t>& a, std::vector<uint32_t>& b) {
        size_t h = (v.size() + 1) / 2;
        a.assign(v.begin(), v.begin() + h);
        b.assign(v.begin() + h, v.end());
      };
      // keep unit kinds together where possible: split the largest list
      half(P.flops, A.flops, B.flops);
      half(P.pos, A.pos, B.pos);
      half(P.cuts, A.cuts, B.cuts);
      half(P.rams, A.rams, B.rams);
      for (Part* X : {&A, &B})
        if (X->flops.size() + X->pos.size() + X->rams.size() + X->cuts.size()) next_parts.push_back(std::move(*X));
    }
    D.parts = std::move(next_parts);
    if (!any_fail && refine_round < D.opt.refine && D.parts.size() > 1) {
      // critical-path refinement: split the costliest partitions along the
      // deep-cone signature (units sharing deep logic stay together)
      std::vector<uint32_t> cost(D.parts.size());
      for (size_t i = 0; i < D.parts.size(); i++) cost[i] = part_cost(D.parts[i].prog.data());
      std::vector<uint32_t> sorted = cost;
      std::sort(sorted.begin(), sorted.end());
      const double med = sorted[sorted.size() / 2];
      std::vector<Part> out;
      size_t n_split = 0;
      for (size_t i = 0; i < D.parts.size(); i++) {
        Part& P = D.parts[i];
        size_t n_units = P.flops.size() + P.pos.size() + P.rams.size() + P.cuts.size();
        if (cost[i] > D.opt.refine_ratio * med && n_units > 1 &&
            D.parts.size() + n_split < (size_t)D.opt.max_parts) {
          // all units ordered by deep signature, then halved
          std::vector<std::pair<uint64_t, std::pair<int, uint32_t>>> us;
          for (auto j : P.flops) us.push_back({dsig[D.G.flop_next[j] >> 1], {0, j}});
          for (auto j : P.pos) us.push_back({dsig[D.G.po[j] >> 1], {1, j}});
          for (auto j : P.rams) us.push_back({dsig[D.G.rams[j].port[3][0] >> 1], {2, j}});
          for (auto j : P.cuts) us.push_back({dsig[cut_compact[j] >> 1], {3, j}});
          std::stable_sort(us.begin(), us.end(), [](auto& a, auto& b) { return a.first < b.first; });
          Part A, B;
          A.stage = B.stage = P.stage;
          for (size_t k = 0; k < us.size(); k++) {
            Part& X = k < (us.size() + 1) / 2 ? A : B;
            auto u = us[k].second;
            (u.first == 0 ? X.flops : u.first == 1 ? X.pos : u.first == 2 ? X.rams : X.cuts).push_back(u.second);
          }
          out.push_back(std::move(A));
          out.push_back(std::move(B));
          n_split++;
        } else {
          out.push_back(std::move(P));
        }
      }
      refine_round++;
      if (n_split) {
        D.parts = std::move(out);
        for (auto& P : D.parts) { P.prog.clear(); P.ok = false; }
        if (D.opt.verbose)
          fprintf(stderr, "gem_map: refine %d: split %zu partitions (median cost %.0f) -> %zu\n", refine_round,
                  n_split, med, D.parts.size());
        continue;
      }
      D.parts = std::move(out);
    }
    if (!any_fail) break;
    for (auto& P : D.parts) { P.prog.clear(); P.ok = false; }
    if (D.opt.verbose) fprintf(stderr, "gem_map: retry %d with %zu partitions (%s)\n", attempt + 1, D.parts.size(), last_err.c_str());
  }
  // drop partitions with no endpoints (possible after splitting)
  auto t2 = std::chrono::steady_clock::now();
  // ---- assemble blob
  Blob B;
  auto& w = B.w;
  w.assign(GH_N_WORDS, 0);
  uint32_t np = (uint32_t)D.parts.size();
  w[GH_MAGIC] = GEM_MAGIC;
  w[GH_VERSION] = GEM_VERSION;
  w[GH_N_PI] = D.G.n_pi;
  w[GH_N_PO] = D.G.n_po;
  w[GH_N_FLOPS] = D.G.n_flops;
  w[GH_N_RAMS] = D.G.n_rams;
  w[GH_N_PARTS] = np;
  w[GH_N_STAGES] = D.n_stages;
  w[GH_PI_WORDS] = (D.G.n_pi + 31) / 32;
  w[GH_PO_WORDS] = D.po_words;
  w[GH_Q_WORDS] = D.q_words;
  w[GH_CUT_WORDS] = D.cut_words;
  // gate evals (reading U14): live ANDs of the design before depth-oriented
  // synthesis and replication; the synthesised count and depths ride along
  w[GH_N_AND_LO] = (uint32_t)D.synth.and_in;
  w[GH_N_AND_HI] = (uint32_t)(D.synth.and_in >> 32);
  w[GH_N_AND_SYNTH_LO] = (uint32_t)D.G.n_and_live;
  w[GH_N_AND_SYNTH_HI] = (uint32_t)(D.G.n_and_live >> 32);
  w[GH_LEVELS_IN] = D.synth.level_in;
  w[GH_SYNTH_CHAINS] = D.synth.chains;
  uint64_t mapped = 0, leaves = 0, slots = 0;
  uint32_t maxl = 0, maxs = 0, tl = 0, two_ = 0, maxout = 0;
  for (auto& P : D.parts) {
    mapped += P.n_nodes; leaves += P.n_leaves; slots += P.slots_used;
    maxl = std::max(maxl, P.n_layers); maxs = std::max(maxs, P.state_words); tl += P.n_layers;
    two_ += P.n_writeouts; maxout = std::max<uint32_t>(maxout, (uint32_t)P.outs.size());
  }
  w[GH_N_AND_MAPPED_LO] = (uint32_t)mapped;
  w[GH_N_AND_MAPPED_HI] = (uint32_t)(mapped >> 32);
  w[GH_MAX_LAYERS] = maxl;
  w[GH_MAX_STATE_WORDS] = maxs;
  w[GH_TOTAL_LAYERS] = tl;
  w[GH_TOTAL_LEAVES_LO] = (uint32_t)leaves;
  w[GH_TOTAL_LEAVES_HI] = (uint32_t)(leaves >> 32);
  w[GH_MAX_LEVELS] = D.G.max_level;
  w[GH_TOTAL_WRITEOUTS] = two_;
  w[GH_MAX_OUT] = maxout;
  w[GH_SLOTS_USED_LO] = (uint32_t)slots;
  w[GH_SLOTS_USED_HI] = (uint32_t)(slots >> 32);
  // part table
  w[GH_OFF_PARTS] = (uint32_t)w.size();
  size_t part_tab = w.size();
  w.resize(w.size() + (size_t)np * GP_WORDS, 0);
  // stage list: prefix offsets [n_stages+1] then part ids
  w[GH_OFF_STAGES] = (uint32_t)w.size();
  {
    std::vector<std::vector<uint32_t>> by(D.n_stages);
    for (uint32_t i = 0; i < np; i++) by[D.parts[i].stage].push_back(i);
    uint32_t acc = 0;
    for (uint32_t s = 0; s < D.n_stages; s++) { w.push_back(acc); acc += (uint32_t)by[s].size(); }
    w.push_back(acc);
    for (uint32_t s = 0; s < D.n_stages; s++) for (auto i : by[s]) w.push_back(i);
  }
  // flop init (internal layout) + permutation tables
  w[GH_OFF_FLOP_INIT] = (uint32_t)w.size();
  {
    size_t base = w.size();
    w.resize(base + D.q_words, 0);
    for (size_t b = 0; b < D.q_ext_of_int.size(); b++) {
      int64_t e = D.q_ext_of_int[b];
      if (e >= 0 && D.G.flop_init[(size_t)e]) w[base + b / 32] |= 1u << (b % 32);
    }
    // q_ext_of_int [q_words*32] then po_ext_of_int [po_words*32] (0xFFFFFFFF = padding)
    for (auto e : D.q_ext_of_int) w.push_back(e < 0 ? 0xFFFFFFFFu : (uint32_t)e);
    for (auto e : D.po_ext_of_int) w.push_back(e < 0 ? 0xFFFFFFFFu : (uint32_t)e);
  }
  while (w.size() % 4) w.push_back(0);
  w[GH_OFF_PROG] = (uint32_t)w.size();
  uint64_t prog = 0;
  uint32_t max_chunk = 0, max_prog = 0;
  for (uint32_t i = 0; i < np; i++) {
    auto& P = D.parts[i];
    w[part_tab + i * GP_WORDS + GP_STAGE] = (uint32_t)P.stage;
    w[part_tab + i * GP_WORDS + GP_PROG_OFF] = (uint32_t)prog;
    w[part_tab + i * GP_WORDS + GP_PROG_LEN] = (uint32_t)P.prog.size();
    w[part_tab + i * GP_WORDS + GP_N_LAYERS] = P.n_layers;
    {
      const uint32_t* pr = P.prog.data();
      uint32_t mc = 0;
      for (uint32_t k = 0; k < pr[PH_N_CHUNKS]; k++) mc = std::max(mc, pr[pr[PH_OFF_CHUNKS] + k]);
      w[part_tab + i * GP_WORDS + GP_CHUNK0] = pr[pr[PH_OFF_CHUNKS]];
      w[part_tab + i * GP_WORDS + GP_CHUNK1] = pr[PH_N_CHUNKS] > 1 ? pr[pr[PH_OFF_CHUNKS] + 1] : 0;
      w[part_tab + i * GP_WORDS + GP_CHUNK2] = pr[PH_N_CHUNKS] > 2 ? pr[pr[PH_OFF_CHUNKS] + 2] : 0;
      w[part_tab + i * GP_WORDS + GP_MAX_CHUNK] = mc;
      w[part_tab + i * GP_WORDS + GP_COST] = part_cost(pr);
      max_chunk = std::max(max_chunk, mc);
      max_prog = std::max<uint32_t>(max_prog, (uint32_t)P.prog.size());
    }
    w.insert(w.end(), P.prog.begin(), P.prog.end());
    prog += P.prog.size();
    while (prog % 4) { w.push_back(0); prog++; }
  }
  w[GH_MAX_CHUNK_WORDS] = max_chunk;
  w[GH_MAX_PROG_WORDS] = max_prog;
  if (D.opt.lanes) {
    w[GH_HAS_LANES] = 1;
    w[GH_OFF_LANE_PROG] = (uint32_t)w.size();
    uint64_t lp = 0;
    uint32_t lmc = 0, lmw = 0;
    for (uint32_t i = 0; i < np; i++) {
      auto& P = D.parts[i];
      const uint32_t* pr = P.lane_prog.data();
      w[part_tab + i * GP_WORDS + GP_LANE_OFF] = (uint32_t)lp;
      w[part_tab + i * GP_WORDS + GP_LANE_LEN] = (uint32_t)P.lane_prog.size();
      w[part_tab + i * GP_WORDS + GP_LANE_CHUNK0] = pr[pr[LPH_OFF_CHUNKS]];
      w[part_tab + i * GP_WORDS + GP_LANE_CHUNK1] = pr[LPH_N_CHUNKS] > 1 ? pr[pr[LPH_OFF_CHUNKS] + 1] : 0;
      w[part_tab + i * GP_WORDS + GP_LANE_CHUNK2] = pr[LPH_N_CHUNKS] > 2 ? pr[pr[LPH_OFF_CHUNKS] + 2] : 0;
      w[part_tab + i * GP_WORDS + GP_LANE_WORDS] = P.lane_words;
      for (uint32_t k = 0; k < pr[LPH_N_CHUNKS]; k++) lmc = std::max(lmc, pr[pr[LPH_OFF_CHUNKS] + k]);
      lmw = std::max(lmw, P.lane_words);
      w.insert(w.end(), P.lane_prog.begin(), P.lane_prog.end());
      lp += P.lane_prog.size();
      while (lp % 4) { w.push_back(0); lp++; }
    }
    w[GH_LANE_PROG_WORDS_LO] = (uint32_t)lp;
    w[GH_LANE_PROG_WORDS_HI] = (uint32_t)(lp >> 32);
    w[GH_LANE_MAX_CHUNK_WORDS] = lmc;
    w[GH_LANE_MAX_WORDS] = lmw;
    uint32_t mr = 0;
    for (auto& P : D.parts) mr = std::max<uint32_t>(mr, (uint32_t)P.rams.size());
    w[GH_MAX_RAMS_PART] = mr;
  }
  // word programs (WRD1): only if every partition has one (else the runtime
  // stays on the bit-packed path)
  if (D.opt.words && std::all_of(D.parts.begin(), D.parts.end(), [](const Part& P) { return !P.word_prog.empty(); })) {
    while (w.size() % 4) w.push_back(0);
    w[GH_HAS_WORDS] = 1;
    w[GH_OFF_WORD_PROG] = (uint32_t)w.size();
    uint64_t wp = 0, wops = 0;
    uint32_t mst = 0, mpw = 0, msteps = 0, tsteps = 0;
    for (uint32_t i = 0; i < np; i++) {
      auto& P = D.parts[i];
      w[part_tab + i * GP_WORDS + GP_WORD_OFF] = (uint32_t)wp;
      mst = std::max(mst, P.word_prog[WPH_STATE_WORDS]);
      mpw = std::max<uint32_t>(mpw, (uint32_t)P.word_prog.size());
      msteps = std::max(msteps, P.word_steps);
      tsteps += P.word_steps;
      wops += P.word_ops;
      w.insert(w.end(), P.word_prog.begin(), P.word_prog.end());
      wp += P.word_prog.size();
    }
    w[GH_WORD_PROG_WORDS_LO] = (uint32_t)wp;
    w[GH_WORD_PROG_WORDS_HI] = (uint32_t)(wp >> 32);
    w[GH_WORD_MAX_STATE] = mst;
    w[GH_WORD_MAX_PROG] = mpw;
    w[GH_WORD_MAX_STEPS] = msteps;
    w[GH_WORD_OPS_LO] = (uint32_t)wops;
    w[GH_WORD_OPS_HI] = (uint32_t)(wops >> 32);
    w[GH_WORD_TOTAL_STEPS] = tsteps;
    uint32_t mr = 0;
    for (auto& P : D.parts) mr = std::max<uint32_t>(mr, (uint32_t)P.rams.size());
    w[GH_MAX_RAMS_PART] = std::max(w[GH_MAX_RAMS_PART], mr);
  } else if (D.opt.words && D.opt.verbose) {
    fprintf(stderr, "gem_map: no word programs (a partition exceeds %u live words)\n", (unsigned)GEM_WORD_MAX_WORDS);
  }
  w[GH_PROG_WORDS_LO] = (uint32_t)prog;
  w[GH_PROG_WORDS_HI] = (uint32_t)(prog >> 32);
  w[GH_TOTAL_WORDS_LO] = (uint32_t)w.size();
  w[GH_TOTAL_WORDS_HI] = (uint32_t)((uint64_t)w.size() >> 32);
  auto t3 = std::chrono::steady_clock::now();
  if (D.opt.verbose) {
    auto ms = [](auto a, auto b) { return std::chrono::duration<double, std::milli>(b - a).count(); };
    fprintf(stderr, "gem_map: %u parts, %u stages, n_and=%llu mapped=%llu max_layers=%u total_layers=%u "
            "leaves=%llu prog=%.2f MB  (partition %.0f ms, place %.0f ms, asm %.0f ms)\n",
            np, D.n_stages, (unsigned long long)D.G.n_and_live, (unsigned long long)mapped, maxl, tl,
            (unsigned long long)leaves, prog * 4.0 / 1e6, ms(t0, t1), ms(t1, t2), ms(t2, t3));
  }
  return B;
}

}  // namespace gm

// =========================================================== C ABI
extern "C" {

const char* gem_map_last_error(void) { return gm::g_err.c_str(); }

int gem_compile(const void* eaig, size_t n, const char* opts, void** blob, size_t* nbytes) {
  if (!eaig || !blob || !nbytes) { gm::g_err = "null argument"; return -1; }
  try {
    gm::Blob B = gm::compile((const char*)eaig, n, opts);
    size_t bytes = B.w.size() * 4;
    void* p = std::malloc(bytes);
    if (!p) { gm::g_err = "out of memory"; return -4; }
    std::memcpy(p, B.w.data(), bytes);
    *blob = p;
    *nbytes = bytes;
    return 0;
  } catch (const std::exception& e) {
    gm::g_err = e.what();
    return -2;
  }
}

int gem_compile_file(const char* path, const char* opts, void** blob, size_t* nbytes) {
  std::ifstream f(path, std::ios::binary);
  if (!f) { gm::g_err = std::string("cannot open ") + path; return -1; }
  std::string data((std::istreambuf_iterator<char>(f)), std::istreambuf_iterator<char>());
  return gem_compile(data.data(), data.size(), opts, blob, nbytes);
}

void gem_free_blob(void* blob) { std::free(blob); }

}  // extern "C"
