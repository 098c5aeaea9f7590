// oracle.cpp -- TEST INFRASTRUCTURE ONLY.  Plain, slow, obviously-correct CPU
// simulator of a synchronous extended AIG (E-AIG).  Only tests/,
// __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
// may load this library.  It shares no code, header, table or helper with the
// mapper or the CUDA path (paper_conf_dac_guozwlr25_b200/).
//
// What it computes (the plain definition):
//   cycle-accurate, zero-delay, 2-state simulation of a synchronous E-AIG with
//   one implicit clock -- PAPER.md P:41-47 (§II: compile, then execute with
//   stimuli, measured in simulated cycles), P:73 (§III-A: E-AIG = AND, INVERT,
//   D flip-flops, RAM blocks), P:93 (§III-B: RAM block = 13-bit address x
//   32-bit data), P:241 (§IV: RAM blocks are synchronous), P:247 (§V: 2-state).
// Readings where the paper is silent (U5-U12):
//   U5  flop init 0 unless AIGER init 1; "uninitialised" -> 0
//   U7  one read + one write port, registered read (data visible next cycle)
//   U8  read-during-write to the same address returns OLD data (read-first)
//   U9  per-bit write enable wbe[32]
//   U10 RAM contents start at 0
//   U11 POs sampled after combinational evaluation, before the clock edge
//   U12 one PI vector per cycle, applied before evaluation
//
// Algorithm, per cycle t, in this order:
//   1. v[0]=0; PI i -> stim[t][i]; RAM r rdata input k -> bit k of RD_r;
//      latch j -> Q_j
//   2. every AND n in a topological order (Kahn): v[n] = L(a_n) & L(b_n),
//      L(l) = v[l>>1] ^ (l&1)
//   3. PO[t][o] = L(out_o)
//   4. Qn_j = L(next_j)
//   5. per RAM r: ra, wa, wd, be assembled LSB-first from their literals;
//      RDn_r = M_r[ra] (before the write); M_r[wa] = (M_r[wa] & ~be) | (wd & be)
//   6. Q <- Qn, RD <- RDn
//   7. optional recording of Q(t+1) (full vector) and its digest
//      d_t = sum_w rotl64(zext64(word_w), w mod 64) * (2w+1) mod 2^64
//
// Batched variant ("lanes"): identical per-lane semantics with one uint64 per
// node carrying 64 independent stimulus streams.

#include <algorithm>
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <fstream>
#include <sstream>
#include <stdexcept>
#include <string>
#include <vector>
#include <thread>
#include <atomic>

namespace {

const int kAddrBits = 13;
const int kDataBits = 32;
const uint32_t kRamWords = 1u << kAddrBits;

struct Ram {
  std::vector<uint64_t> rdata_input;  // 32 AIGER input indices
  std::vector<uint64_t> raddr, waddr, wdata, wbe;  // literals
};

struct Oracle {
  uint64_t M = 0, I = 0, L = 0, O = 0, A = 0;
  std::vector<uint64_t> latch_next;
  std::vector<uint8_t> latch_init;
  std::vector<uint64_t> outputs;
  std::vector<uint64_t> and_lhs, and_a, and_b;  // as parsed (lhs literal, inputs)
  std::vector<Ram> rams;
  // derived
  std::vector<int64_t> input_pi;        // input index -> PI index, or -1
  std::vector<int64_t> input_ram;       // input index -> RAM index, or -1
  std::vector<int64_t> input_rambit;    // input index -> data bit, or -1
  uint64_t n_pi = 0;
  std::vector<uint64_t> topo;           // AND indices in topological order
  // single-stream state
  std::vector<uint8_t> v;               // value per variable
  std::vector<uint8_t> Q;
  std::vector<uint32_t> RD;
  std::vector<std::vector<uint32_t>> MEM;
  // batched state: groups of 64 lanes
  uint64_t n_groups = 0;
  std::vector<std::vector<uint64_t>> gQ;            // [group][latch]
  std::vector<std::vector<uint32_t>> gRD;           // [group][ram*64 + lane]
  std::vector<std::vector<uint32_t>> gMEM;          // [group][(ram*64+lane)*8192 + addr]
};

thread_local std::string g_err;

// ---------------------------------------------------------------- parsing
uint64_t read_uint_token(std::istream& in) {
  std::string tok;
  if (!(in >> tok)) throw std::runtime_error("unexpected end of file");
  for (char c : tok)
    if (c < '0' || c > '9') throw std::runtime_error("bad number '" + tok + "'");
  return std::stoull(tok);
}

uint64_t read_varint(std::istream& in) {
  uint64_t x = 0;
  int shift = 0;
  while (true) {
    int ch = in.get();
    if (ch == EOF) throw std::runtime_error("unexpected EOF in binary AND section");
    x |= (uint64_t)(ch & 0x7f) << shift;
    if (!(ch & 0x80)) break;
    shift += 7;
    if (shift > 63) throw std::runtime_error("varint overflow");
  }
  return x;
}

std::vector<uint64_t> parse_list(const std::string& s) {
  std::vector<uint64_t> out;
  std::stringstream ss(s);
  std::string item;
  while (std::getline(ss, item, ',')) {
    if (item.empty()) throw std::runtime_error("empty list item");
    for (char c : item)
      if (c < '0' || c > '9') throw std::runtime_error("bad list item '" + item + "'");
    out.push_back(std::stoull(item));
  }
  return out;
}

void parse_ram_line(Oracle& o, const std::string& line) {
  std::stringstream ss(line);
  std::string tag, id;
  ss >> tag >> id;
  Ram r;
  std::string field;
  int seen = 0;
  while (ss >> field) {
    size_t eq = field.find('=');
    if (eq == std::string::npos) throw std::runtime_error("bad gem-ram field " + field);
    std::string key = field.substr(0, eq);
    std::vector<uint64_t> vals = parse_list(field.substr(eq + 1));
    if (key == "rdata") { r.rdata_input = vals; seen |= 1; }
    else if (key == "raddr") { r.raddr = vals; seen |= 2; }
    else if (key == "waddr") { r.waddr = vals; seen |= 4; }
    else if (key == "wdata") { r.wdata = vals; seen |= 8; }
    else if (key == "wbe") { r.wbe = vals; seen |= 16; }
    else throw std::runtime_error("unknown gem-ram field " + key);
  }
  if (seen != 31) throw std::runtime_error("gem-ram line misses a field");
  if (r.rdata_input.size() != (size_t)kDataBits || r.raddr.size() != (size_t)kAddrBits ||
      r.waddr.size() != (size_t)kAddrBits || r.wdata.size() != (size_t)kDataBits ||
      r.wbe.size() != (size_t)kDataBits)
    throw std::runtime_error("gem-ram port width mismatch (need 32/13/13/32/32)");
  o.rams.push_back(r);
}

void parse_file(Oracle& o, const char* path) {
  std::ifstream in(path, std::ios::binary);
  if (!in) throw std::runtime_error(std::string("cannot open ") + path);
  std::string fmt;
  in >> fmt;
  bool binary;
  if (fmt == "aag") binary = false;
  else if (fmt == "aig") binary = true;
  else throw std::runtime_error("bad AIGER magic '" + fmt + "'");
  o.M = read_uint_token(in);
  o.I = read_uint_token(in);
  o.L = read_uint_token(in);
  o.O = read_uint_token(in);
  o.A = read_uint_token(in);
  // reject B C J F extensions: the header line must end here
  {
    std::string rest;
    std::getline(in, rest);
    for (char c : rest)
      if (c != ' ' && c != '\r' && c != '\t')
        throw std::runtime_error("AIGER 1.9 B/C/J/F sections are not supported");
  }
  if (o.M < o.I + o.L + o.A) throw std::runtime_error("M < I+L+A");
  std::vector<uint64_t> input_lit(o.I);
  if (!binary) {
    for (uint64_t i = 0; i < o.I; i++) {
      input_lit[i] = read_uint_token(in);
      if (input_lit[i] != 2 * (i + 1))
        throw std::runtime_error("inputs must be numbered 1..I (var order I, L, A)");
    }
  }
  o.latch_next.resize(o.L);
  o.latch_init.assign(o.L, 0);
  for (uint64_t j = 0; j < o.L; j++) {
    std::string line;
    std::getline(in, line);
    if (line.empty()) { j--; if (!in) throw std::runtime_error("EOF in latches"); continue; }
    std::stringstream ls(line);
    uint64_t cur = 2 * (o.I + 1 + j);
    if (!binary) {
      uint64_t c;
      ls >> c;
      if (c != cur) throw std::runtime_error("latches must be numbered I+1..I+L");
    }
    uint64_t nxt;
    if (!(ls >> nxt)) throw std::runtime_error("bad latch line");
    o.latch_next[j] = nxt;
    uint64_t init;
    if (ls >> init) {
      if (init == 0) o.latch_init[j] = 0;
      else if (init == 1) o.latch_init[j] = 1;
      else if (init == cur) o.latch_init[j] = 0;   // uninitialised -> 0 (U5)
      else throw std::runtime_error("bad latch init");
    }
  }
  o.outputs.resize(o.O);
  for (uint64_t k = 0; k < o.O; k++) o.outputs[k] = read_uint_token(in);
  o.and_lhs.resize(o.A);
  o.and_a.resize(o.A);
  o.and_b.resize(o.A);
  if (!binary) {
    for (uint64_t k = 0; k < o.A; k++) {
      o.and_lhs[k] = read_uint_token(in);
      o.and_a[k] = read_uint_token(in);
      o.and_b[k] = read_uint_token(in);
    }
  } else {
    // consume the newline after the last output (outputs were read as tokens;
    // with no outputs the latch/header getline already consumed it)
    if (o.O > 0) {
      int ch = in.get();
      while (ch == '\r' || ch == ' ') ch = in.get();
      if (ch != '\n') throw std::runtime_error("expected newline before binary ANDs");
    }
    for (uint64_t k = 0; k < o.A; k++) {
      uint64_t lhs = 2 * (o.I + o.L + 1 + k);
      uint64_t d0 = read_varint(in), d1 = read_varint(in);
      if (d0 > lhs) throw std::runtime_error("bad delta");
      uint64_t r0 = lhs - d0;
      if (d1 > r0) throw std::runtime_error("bad delta");
      o.and_lhs[k] = lhs;
      o.and_a[k] = r0;
      o.and_b[k] = r0 - d1;
    }
  }
  // symbol table and comments
  std::string line;
  bool in_comment = false;
  while (std::getline(in, line)) {
    if (!in_comment) {
      if (line == "c" || line.rfind("c ", 0) == 0) { in_comment = true; continue; }
      continue;  // symbol table entries are ignored
    }
    if (line.rfind("gem-ram ", 0) == 0) parse_ram_line(o, line);
  }
}

// ---------------------------------------------------------------- validation + order
void validate_and_order(Oracle& o) {
  const uint64_t maxlit = 2 * o.M + 1;
  auto chk = [&](uint64_t lit, const char* what) {
    if (lit > maxlit) throw std::runtime_error(std::string("literal out of range in ") + what);
  };
  for (auto x : o.latch_next) chk(x, "latch");
  for (auto x : o.outputs) chk(x, "output");
  std::vector<int64_t> and_of_var(o.M + 1, -1);
  for (uint64_t k = 0; k < o.A; k++) {
    chk(o.and_a[k], "and");
    chk(o.and_b[k], "and");
    uint64_t lhs = o.and_lhs[k];
    if (lhs & 1) throw std::runtime_error("AND lhs must be even");
    uint64_t var = lhs >> 1;
    if (var <= o.I + o.L || var > o.M) throw std::runtime_error("AND lhs out of range");
    if (and_of_var[var] >= 0) throw std::runtime_error("AND variable defined twice");
    and_of_var[var] = (int64_t)k;
  }
  // any literal must be a constant, an input, a latch or a defined AND
  auto defined = [&](uint64_t lit) {
    uint64_t var = lit >> 1;
    return var <= o.I + o.L || and_of_var[var] >= 0;
  };
  for (uint64_t k = 0; k < o.A; k++)
    if (!defined(o.and_a[k]) || !defined(o.and_b[k])) throw std::runtime_error("undefined AND input");
  for (auto x : o.latch_next) if (!defined(x)) throw std::runtime_error("undefined latch next");
  for (auto x : o.outputs) if (!defined(x)) throw std::runtime_error("undefined output");
  // RAMs
  o.input_ram.assign(o.I, -1);
  o.input_rambit.assign(o.I, -1);
  for (size_t r = 0; r < o.rams.size(); r++) {
    const Ram& ram = o.rams[r];
    for (int k = 0; k < kDataBits; k++) {
      uint64_t inp = ram.rdata_input[k];
      if (inp >= o.I) throw std::runtime_error("RAM rdata index out of range");
      if (o.input_ram[inp] >= 0) throw std::runtime_error("RAM rdata input owned twice");
      o.input_ram[inp] = (int64_t)r;
      o.input_rambit[inp] = k;
    }
    for (auto* v : {&ram.raddr, &ram.waddr, &ram.wdata, &ram.wbe})
      for (auto x : *v) { chk(x, "ram port"); if (!defined(x)) throw std::runtime_error("undefined RAM port"); }
  }
  o.input_pi.assign(o.I, -1);
  o.n_pi = 0;
  for (uint64_t i = 0; i < o.I; i++)
    if (o.input_ram[i] < 0) o.input_pi[i] = (int64_t)o.n_pi++;
  // Kahn's topological sort of the ANDs
  std::vector<uint32_t> indeg(o.A, 0);
  std::vector<std::vector<uint64_t>> users(o.A);
  for (uint64_t k = 0; k < o.A; k++) {
    for (uint64_t lit : {o.and_a[k], o.and_b[k]}) {
      int64_t d = and_of_var[lit >> 1];
      if (d >= 0) { indeg[k]++; users[(uint64_t)d].push_back(k); }
    }
  }
  std::vector<uint64_t> queue;
  for (uint64_t k = 0; k < o.A; k++) if (indeg[k] == 0) queue.push_back(k);
  o.topo.clear();
  o.topo.reserve(o.A);
  for (size_t h = 0; h < queue.size(); h++) {
    uint64_t k = queue[h];
    o.topo.push_back(k);
    for (uint64_t u : users[k]) if (--indeg[u] == 0) queue.push_back(u);
  }
  if (o.topo.size() != o.A) throw std::runtime_error("combinational loop");
}

// ---------------------------------------------------------------- single stream
inline uint8_t val(const Oracle& o, uint64_t lit) { return (uint8_t)(o.v[lit >> 1] ^ (lit & 1)); }

void reset_state(Oracle& o) {
  o.v.assign(o.M + 1, 0);
  o.Q.assign(o.L, 0);
  for (uint64_t j = 0; j < o.L; j++) o.Q[j] = o.latch_init[j];
  o.RD.assign(o.rams.size(), 0);
  o.MEM.assign(o.rams.size(), std::vector<uint32_t>(kRamWords, 0));
}

uint64_t digest_words(const uint32_t* w, uint64_t nw) {
  uint64_t d = 0;
  for (uint64_t i = 0; i < nw; i++) {
    uint64_t x = (uint64_t)w[i];
    unsigned r = (unsigned)(i % 64);
    uint64_t rot = r ? ((x << r) | (x >> (64 - r))) : x;
    d += rot * (2 * i + 1);
  }
  return d;
}

void run_cycles(Oracle& o, const uint32_t* stim, uint64_t cycles, uint32_t* po, uint32_t* st,
                uint64_t* dig) {
  const uint64_t piw = (o.n_pi + 31) / 32, pow_ = (o.O + 31) / 32, qw = (o.L + 31) / 32;
  std::vector<uint8_t> Qn(o.L);
  std::vector<uint32_t> RDn(o.rams.size());
  std::vector<uint32_t> qwords(qw);
  for (uint64_t t = 0; t < cycles; t++) {
    // 1. sources
    o.v[0] = 0;
    for (uint64_t i = 0; i < o.I; i++) {
      uint8_t b;
      if (o.input_pi[i] >= 0) {
        uint64_t p = (uint64_t)o.input_pi[i];
        b = (uint8_t)((stim[t * piw + p / 32] >> (p % 32)) & 1u);
      } else {
        b = (uint8_t)((o.RD[(uint64_t)o.input_ram[i]] >> o.input_rambit[i]) & 1u);
      }
      o.v[1 + i] = b;
    }
    for (uint64_t j = 0; j < o.L; j++) o.v[1 + o.I + j] = o.Q[j];
    // 2. ANDs in topological order
    for (uint64_t k : o.topo) o.v[o.and_lhs[k] >> 1] = (uint8_t)(val(o, o.and_a[k]) & val(o, o.and_b[k]));
    // 3. outputs before the edge
    if (po) {
      uint32_t* row = po + t * pow_;
      for (uint64_t w = 0; w < pow_; w++) row[w] = 0;
      for (uint64_t k = 0; k < o.O; k++) row[k / 32] |= (uint32_t)val(o, o.outputs[k]) << (k % 32);
    }
    // 4. next state
    for (uint64_t j = 0; j < o.L; j++) Qn[j] = val(o, o.latch_next[j]);
    // 5. RAMs: read first, then write
    for (size_t r = 0; r < o.rams.size(); r++) {
      const Ram& ram = o.rams[r];
      uint32_t ra = 0, wa = 0, wd = 0, be = 0;
      for (int k = 0; k < kAddrBits; k++) ra |= (uint32_t)val(o, ram.raddr[k]) << k;
      for (int k = 0; k < kAddrBits; k++) wa |= (uint32_t)val(o, ram.waddr[k]) << k;
      for (int k = 0; k < kDataBits; k++) wd |= (uint32_t)val(o, ram.wdata[k]) << k;
      for (int k = 0; k < kDataBits; k++) be |= (uint32_t)val(o, ram.wbe[k]) << k;
      RDn[r] = o.MEM[r][ra];
      o.MEM[r][wa] = (o.MEM[r][wa] & ~be) | (wd & be);
    }
    // 6. commit
    o.Q = Qn;
    for (size_t r = 0; r < o.rams.size(); r++) o.RD[r] = RDn[r];
    // 7. record Q(t+1)
    if (st || dig) {
      for (uint64_t w = 0; w < qw; w++) qwords[w] = 0;
      for (uint64_t j = 0; j < o.L; j++) qwords[j / 32] |= (uint32_t)o.Q[j] << (j % 32);
      if (st) std::memcpy(st + t * qw, qwords.data(), qw * 4);
      if (dig) dig[t] = digest_words(qwords.data(), qw);
    }
  }
}

// ---------------------------------------------------------------- multi-threaded baseline
// SURVEY §8(d) "also time an nproc-thread variant (OpenMP over the ANDs of each
// level)": the same cycle as run_cycles, with step 2 evaluated level by level
// (level = 1 + max level of the AND's AND fan-ins; every AND of a level depends
// only on earlier levels, so a level is any-order).  Runs of consecutive levels
// too small to share (< kParMin ANDs) are evaluated by thread 0 alone, so
// threads meet at a barrier only around the wide levels.  Steps 1 and 3-7 are
// thread 0's.  Test infrastructure / CPU baseline only, like the rest of oracle/.
struct SpinBarrier {
  std::atomic<uint32_t> count{0}, gen{0};
  uint32_t n;
  explicit SpinBarrier(uint32_t n_) : n(n_) {}
  void wait() {
    const uint32_t g = gen.load(std::memory_order_acquire);
    if (count.fetch_add(1, std::memory_order_acq_rel) + 1 == n) {
      count.store(0, std::memory_order_relaxed);
      gen.store(g + 1, std::memory_order_release);
    } else {
      while (gen.load(std::memory_order_acquire) == g) std::this_thread::yield();
    }
  }
};

void run_cycles_mt(Oracle& o, const uint32_t* stim, uint64_t cycles, uint32_t* po, uint32_t nth) {
  const uint64_t kParMin = 4096;
  // levels
  std::vector<uint32_t> lvl_of_var(o.M + 1, 0), lvl(o.A, 0);
  uint32_t max_lvl = 0;
  for (uint64_t k : o.topo) {
    const uint32_t la = lvl_of_var[o.and_a[k] >> 1], lb = lvl_of_var[o.and_b[k] >> 1];
    lvl[k] = 1 + std::max(la, lb);
    lvl_of_var[o.and_lhs[k] >> 1] = lvl[k];
    max_lvl = std::max(max_lvl, lvl[k]);
  }
  std::vector<std::vector<uint64_t>> by_lvl(max_lvl + 1);
  for (uint64_t k : o.topo) by_lvl[lvl[k]].push_back(k);
  // segments: {parallel?, ANDs in evaluation order}
  std::vector<std::pair<bool, std::vector<uint64_t>>> seg;
  for (uint32_t l = 1; l <= max_lvl; l++) {
    const bool par = by_lvl[l].size() >= kParMin && nth > 1;
    if (seg.empty() || par || seg.back().first)
      seg.push_back({par, {}});
    auto& v = seg.back().second;
    v.insert(v.end(), by_lvl[l].begin(), by_lvl[l].end());
  }
  const uint64_t piw = (o.n_pi + 31) / 32, pow_ = (o.O + 31) / 32;
  std::vector<uint8_t> Qn(o.L);
  std::vector<uint32_t> RDn(o.rams.size());
  SpinBarrier bar(nth);
  auto worker = [&](uint32_t tid) {
    for (uint64_t t = 0; t < cycles; t++) {
      if (tid == 0) {
        o.v[0] = 0;
        for (uint64_t i = 0; i < o.I; i++) {
          uint8_t b;
          if (o.input_pi[i] >= 0) {
            uint64_t p = (uint64_t)o.input_pi[i];
            b = (uint8_t)((stim[t * piw + p / 32] >> (p % 32)) & 1u);
          } else {
            b = (uint8_t)((o.RD[(uint64_t)o.input_ram[i]] >> o.input_rambit[i]) & 1u);
          }
          o.v[1 + i] = b;
        }
        for (uint64_t j = 0; j < o.L; j++) o.v[1 + o.I + j] = o.Q[j];
      }
      for (auto& sg : seg) {
        if (sg.first) {
          bar.wait();
          const uint64_t n = sg.second.size(), a = n * tid / nth, b = n * (tid + 1) / nth;
          for (uint64_t q = a; q < b; q++) {
            const uint64_t k = sg.second[q];
            o.v[o.and_lhs[k] >> 1] = (uint8_t)(val(o, o.and_a[k]) & val(o, o.and_b[k]));
          }
          bar.wait();
        } else if (tid == 0) {
          for (uint64_t k : sg.second) o.v[o.and_lhs[k] >> 1] = (uint8_t)(val(o, o.and_a[k]) & val(o, o.and_b[k]));
        }
      }
      if (tid == 0) {
        if (po) {
          uint32_t* row = po + t * pow_;
          for (uint64_t w = 0; w < pow_; w++) row[w] = 0;
          for (uint64_t k = 0; k < o.O; k++) row[k / 32] |= (uint32_t)val(o, o.outputs[k]) << (k % 32);
        }
        for (uint64_t j = 0; j < o.L; j++) Qn[j] = val(o, o.latch_next[j]);
        for (size_t r = 0; r < o.rams.size(); r++) {
          const Ram& ram = o.rams[r];
          uint32_t ra = 0, wa = 0, wd = 0, be = 0;
          for (int k = 0; k < kAddrBits; k++) ra |= (uint32_t)val(o, ram.raddr[k]) << k;
          for (int k = 0; k < kAddrBits; k++) wa |= (uint32_t)val(o, ram.waddr[k]) << k;
          for (int k = 0; k < kDataBits; k++) wd |= (uint32_t)val(o, ram.wdata[k]) << k;
          for (int k = 0; k < kDataBits; k++) be |= (uint32_t)val(o, ram.wbe[k]) << k;
          RDn[r] = o.MEM[r][ra];
          o.MEM[r][wa] = (o.MEM[r][wa] & ~be) | (wd & be);
        }
        o.Q = Qn;
        for (size_t r = 0; r < o.rams.size(); r++) o.RD[r] = RDn[r];
      }
    }
  };
  std::vector<std::thread> th;
  for (uint32_t i = 1; i < nth; i++) th.emplace_back(worker, i);
  worker(0);
  for (auto& x : th) x.join();
}

// ---------------------------------------------------------------- 64-lane batches
inline uint64_t lval(const std::vector<uint64_t>& v, uint64_t lit) {
  return v[lit >> 1] ^ ((lit & 1) ? ~0ull : 0ull);
}

void lanes_reset(Oracle& o, uint64_t groups) {
  o.n_groups = groups;
  o.gQ.assign(groups, std::vector<uint64_t>(o.L, 0));
  for (uint64_t g = 0; g < groups; g++)
    for (uint64_t j = 0; j < o.L; j++) o.gQ[g][j] = o.latch_init[j] ? ~0ull : 0ull;
  o.gRD.assign(groups, std::vector<uint32_t>(o.rams.size() * 64, 0));
  o.gMEM.assign(groups, std::vector<uint32_t>(o.rams.size() * 64 * (size_t)kRamWords, 0));
}

// stim: [64 lanes][cycles][piw] for this group; outputs with the same lane-major layout
void lanes_run_group(Oracle& o, uint64_t g, uint64_t lanes, const uint32_t* stim, uint64_t cycles,
                     uint32_t* po, uint64_t* dig) {
  const uint64_t piw = (o.n_pi + 31) / 32, pow_ = (o.O + 31) / 32, qw = (o.L + 31) / 32;
  std::vector<uint64_t> v(o.M + 1, 0);
  std::vector<uint64_t>& Q = o.gQ[g];
  std::vector<uint32_t>& RD = o.gRD[g];
  std::vector<uint32_t>& MEM = o.gMEM[g];
  std::vector<uint64_t> Qn(o.L);
  std::vector<uint32_t> RDn(o.rams.size() * 64);
  std::vector<uint32_t> qwords(qw);
  for (uint64_t t = 0; t < cycles; t++) {
    v[0] = 0;
    for (uint64_t i = 0; i < o.I; i++) {
      uint64_t x = 0;
      for (uint64_t l = 0; l < lanes; l++) {
        uint64_t b;
        if (o.input_pi[i] >= 0) {
          uint64_t p = (uint64_t)o.input_pi[i];
          b = (stim[(l * cycles + t) * piw + p / 32] >> (p % 32)) & 1u;
        } else {
          b = (RD[(uint64_t)o.input_ram[i] * 64 + l] >> o.input_rambit[i]) & 1u;
        }
        x |= b << l;
      }
      v[1 + i] = x;
    }
    for (uint64_t j = 0; j < o.L; j++) v[1 + o.I + j] = Q[j];
    for (uint64_t k : o.topo) v[o.and_lhs[k] >> 1] = lval(v, o.and_a[k]) & lval(v, o.and_b[k]);
    if (po) {
      for (uint64_t l = 0; l < lanes; l++) {
        uint32_t* row = po + (l * cycles + t) * pow_;
        for (uint64_t w = 0; w < pow_; w++) row[w] = 0;
        for (uint64_t k = 0; k < o.O; k++)
          row[k / 32] |= (uint32_t)((lval(v, o.outputs[k]) >> l) & 1u) << (k % 32);
      }
    }
    for (uint64_t j = 0; j < o.L; j++) Qn[j] = lval(v, o.latch_next[j]);
    for (size_t r = 0; r < o.rams.size(); r++) {
      const Ram& ram = o.rams[r];
      for (uint64_t l = 0; l < lanes; l++) {
        uint32_t ra = 0, wa = 0, wd = 0, be = 0;
        for (int k = 0; k < kAddrBits; k++) ra |= (uint32_t)((lval(v, ram.raddr[k]) >> l) & 1u) << k;
        for (int k = 0; k < kAddrBits; k++) wa |= (uint32_t)((lval(v, ram.waddr[k]) >> l) & 1u) << k;
        for (int k = 0; k < kDataBits; k++) wd |= (uint32_t)((lval(v, ram.wdata[k]) >> l) & 1u) << k;
        for (int k = 0; k < kDataBits; k++) be |= (uint32_t)((lval(v, ram.wbe[k]) >> l) & 1u) << k;
        uint32_t* mem = &MEM[(r * 64 + l) * (size_t)kRamWords];
        RDn[r * 64 + l] = mem[ra];
        mem[wa] = (mem[wa] & ~be) | (wd & be);
      }
    }
    Q = Qn;
    RD = RDn;
    if (dig) {
      for (uint64_t l = 0; l < lanes; l++) {
        for (uint64_t w = 0; w < qw; w++) qwords[w] = 0;
        for (uint64_t j = 0; j < o.L; j++) qwords[j / 32] |= (uint32_t)((Q[j] >> l) & 1u) << (j % 32);
        dig[l * cycles + t] = digest_words(qwords.data(), qw);
      }
    }
  }
}

}  // namespace

// ====================================================================== C API
extern "C" {

const char* orc_last_error(void) { return g_err.c_str(); }

void* orc_load(const char* path) {
  try {
    Oracle* o = new Oracle();
    try {
      parse_file(*o, path);
      validate_and_order(*o);
      reset_state(*o);
    } catch (...) {
      delete o;
      throw;
    }
    return o;
  } catch (const std::exception& e) {
    g_err = e.what();
    return nullptr;
  }
}

void orc_free(void* h) { delete (Oracle*)h; }

// out[0..7] = I, L, O, A, n_pi, n_rams, M, 0
int orc_info(void* h, uint64_t* out) {
  Oracle* o = (Oracle*)h;
  out[0] = o->I; out[1] = o->L; out[2] = o->O; out[3] = o->A;
  out[4] = o->n_pi; out[5] = o->rams.size(); out[6] = o->M; out[7] = 0;
  return 0;
}

int orc_reset(void* h) { reset_state(*(Oracle*)h); return 0; }

int orc_get_state(void* h, uint32_t* words) {
  Oracle* o = (Oracle*)h;
  uint64_t qw = (o->L + 31) / 32;
  for (uint64_t w = 0; w < qw; w++) words[w] = 0;
  for (uint64_t j = 0; j < o->L; j++) words[j / 32] |= (uint32_t)o->Q[j] << (j % 32);
  return 0;
}

int orc_set_state(void* h, const uint32_t* words) {
  Oracle* o = (Oracle*)h;
  for (uint64_t j = 0; j < o->L; j++) o->Q[j] = (uint8_t)((words[j / 32] >> (j % 32)) & 1u);
  return 0;
}

int orc_get_ram(void* h, uint32_t r, uint32_t* words) {
  Oracle* o = (Oracle*)h;
  if (r >= o->rams.size()) { g_err = "bad ram id"; return -1; }
  std::memcpy(words, o->MEM[r].data(), kRamWords * 4);
  return 0;
}

int orc_set_ram(void* h, uint32_t r, const uint32_t* words) {
  Oracle* o = (Oracle*)h;
  if (r >= o->rams.size()) { g_err = "bad ram id"; return -1; }
  std::memcpy(o->MEM[r].data(), words, kRamWords * 4);
  return 0;
}

int orc_get_rd(void* h, uint32_t* rd) {
  Oracle* o = (Oracle*)h;
  for (size_t r = 0; r < o->rams.size(); r++) rd[r] = o->RD[r];
  return 0;
}

// stim [cycles][ceil(n_pi/32)]; po [cycles][ceil(O/32)]; st [cycles][ceil(L/32)]; dig [cycles]
int orc_run(void* h, const uint32_t* stim, uint64_t cycles, uint32_t* po, uint32_t* st, uint64_t* dig,
            double* seconds) {
  try {
    Oracle* o = (Oracle*)h;
    auto t0 = std::chrono::steady_clock::now();
    run_cycles(*o, stim, cycles, po, st, dig);
    auto t1 = std::chrono::steady_clock::now();
    if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
    return 0;
  } catch (const std::exception& e) {
    g_err = e.what();
    return -1;
  }
}

int orc_run_mt(void* h, const uint32_t* stim, uint64_t cycles, uint32_t* po, uint32_t threads, double* seconds) {
  try {
    Oracle* o = (Oracle*)h;
    auto t0 = std::chrono::steady_clock::now();
    run_cycles_mt(*o, stim, cycles, po, std::max<uint32_t>(1, threads));
    auto t1 = std::chrono::steady_clock::now();
    if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
    return 0;
  } catch (const std::exception& e) {
    g_err = e.what();
    return -1;
  }
}

int orc_lanes_reset(void* h, uint64_t groups) {
  lanes_reset(*(Oracle*)h, groups);
  return 0;
}

// group g, `lanes` (<=64) active lanes; stim [lanes][cycles][piw]; po [lanes][cycles][pow];
// dig [lanes][cycles]
int orc_lanes_run(void* h, uint64_t g, uint64_t lanes, const uint32_t* stim, uint64_t cycles,
                  uint32_t* po, uint64_t* dig, double* seconds) {
  Oracle* o = (Oracle*)h;
  if (g >= o->n_groups || lanes == 0 || lanes > 64) { g_err = "bad lane group"; return -1; }
  auto t0 = std::chrono::steady_clock::now();
  lanes_run_group(*o, g, lanes, stim, cycles, po, dig);
  auto t1 = std::chrono::steady_clock::now();
  if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
  return 0;
}

int orc_lanes_get_state(void* h, uint64_t g, uint64_t lane, uint32_t* words) {
  Oracle* o = (Oracle*)h;
  if (g >= o->n_groups || lane >= 64) { g_err = "bad lane"; return -1; }
  uint64_t qw = (o->L + 31) / 32;
  for (uint64_t w = 0; w < qw; w++) words[w] = 0;
  for (uint64_t j = 0; j < o->L; j++)
    words[j / 32] |= (uint32_t)((o->gQ[g][j] >> lane) & 1u) << (j % 32);
  return 0;
}

// RAM block r of lane `lane` in 64-lane group g (state access only, no arithmetic)
int orc_lanes_get_ram(void* h, uint64_t g, uint64_t lane, uint32_t r, uint32_t* words) {
  Oracle* o = (Oracle*)h;
  if (g >= o->n_groups || lane >= 64 || r >= o->rams.size()) { g_err = "bad lane ram"; return -1; }
  const uint32_t* m = &o->gMEM[g][(r * 64 + lane) * (size_t)kRamWords];
  for (int k = 0; k < kRamWords; k++) words[k] = m[k];
  return 0;
}

int orc_lanes_set_ram(void* h, uint64_t g, uint64_t lane, uint32_t r, const uint32_t* words) {
  Oracle* o = (Oracle*)h;
  if (g >= o->n_groups || lane >= 64 || r >= o->rams.size()) { g_err = "bad lane ram"; return -1; }
  uint32_t* m = &o->gMEM[g][(r * 64 + lane) * (size_t)kRamWords];
  for (int k = 0; k < kRamWords; k++) m[k] = words[k];
  return 0;
}

uint64_t orc_digest(const uint32_t* words, uint64_t nw) { return digest_words(words, nw); }

}  // extern "C"
