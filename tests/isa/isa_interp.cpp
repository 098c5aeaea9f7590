// isa_interp.cpp -- TEST TOOL: executes a .gemb program on the CPU by the ISA
// *definition* in gem_isa.h (slot by slot, level by level), to check the
// mapper against the oracle without a GPU.  It is not the oracle (it knows
// partitions/layers) and not a product fallback (nothing in the package loads
// it).  Hazard checks: a layer's write-out targets must not be read by the
// same layer's gathers, and state word 0 is never written.
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "../../paper_conf_dac_guozwlr25_b200/csrc/gem_isa.h"

namespace {
thread_local std::string g_err;

struct Interp {
  std::vector<uint32_t> w;
  uint32_t n_parts, n_stages, q_words, po_words, cut_words, pi_words, n_rams, n_flops, n_po;
  const uint32_t* parts;
  const uint32_t* stages;
  const uint32_t* prog;
  const uint32_t* flop_init;
  const uint32_t* q_ext;
  const uint32_t* po_ext;
  std::vector<uint32_t> Q[2], RD[2], CUT;
  std::vector<std::vector<uint32_t>> MEM;
  uint64_t cycle = 0;
};

static inline uint32_t gw(int k) { return k <= 5 ? 1u << (5 - k) : k <= 10 ? 1u << (10 - k) : 1u << (13 - k); }
static inline uint32_t sbit(int k, uint32_t id) {
  static const int off[6] = {0, 0, 16, 24, 28, 30};
  if (k >= 11) return (k == 11 ? 0 : k == 12 ? 4 : 6) + id;
  int kk = k <= 5 ? k : k - 5;
  return (uint32_t)off[kk] + id % gw(k);
}

int run_part(Interp& I, uint32_t p, uint64_t t, const uint32_t* stim, uint32_t* po_row) {
  const uint32_t* pt = I.parts + p * GP_WORDS;
  const uint32_t* pr = I.prog + pt[GP_PROG_OFF];
  if (pr[PH_MAGIC] != GEM_PART_MAGIC) { g_err = "bad part magic"; return -1; }
  uint32_t cur = (uint32_t)(I.cycle & 1), nxt = cur ^ 1;
  std::vector<uint32_t> S(GEM_MAX_STATE_WORDS, 0);
  std::vector<uint8_t> written(GEM_MAX_STATE_WORDS, 0);
  // gread
  const uint32_t* gr = pr + pr[PH_OFF_GREAD];
  for (uint32_t k = 0; k < pr[PH_N_GREAD]; k++) {
    uint32_t gid = gr[2 * k], dst = gr[2 * k + 1];
    uint32_t reg = GEM_GID_REGION(gid), idx = GEM_GID_INDEX(gid), v;
    if (reg == GEM_R_PI) v = stim[idx];
    else if (reg == GEM_R_Q) v = I.Q[cur][idx];
    else if (reg == GEM_R_RD) v = I.RD[cur][idx];
    else if (reg == GEM_R_CUT) v = I.CUT[idx];
    else { g_err = "bad gread region"; return -1; }
    if (dst == 0 || dst >= GEM_MAX_STATE_WORDS) { g_err = "bad gread dst"; return -1; }
    S[dst] = v;
  }
  // layers
  const uint32_t* L = pr + pr[PH_OFF_LAYERS];
  std::vector<uint8_t> val[14];
  for (int k = 0; k <= 13; k++) val[k].assign(8192u >> k, 0);
  // record directory of the current layer (gem_isa.h): chunk 0 for layer 0,
  // then the previous layer's LH_NEXTDIR words -- read the way the kernel does
  uint32_t dir[4];
  for (int k = 0; k < 4; k++) dir[k] = pr[pr[PH_OFF_DIR0] + k];
  for (uint32_t l = 0; l < pr[PH_N_LAYERS]; l++) {
    uint32_t flags = L[LH_FLAGS];
    uint32_t topc = L[LH_TOPC];
    uint32_t lane_c[256][4];
    uint32_t warp_c[8][4];
    std::memset(lane_c, 0, sizeof(lane_c));
    std::memset(warp_c, 0, sizeof(warp_c));
    for (int k = 0; k <= 13; k++) std::fill(val[k].begin(), val[k].end(), 0);
    std::vector<uint8_t> read(GEM_MAX_STATE_WORDS, 0);
    for (uint32_t wp = 0; wp < 8; wp++) {
      const uint32_t de = (dir[wp >> 1] >> (16 * (wp & 1))) & 0xFFFFu, cls = de >> 12;
      if (((flags >> wp) & 1) != (cls != 0)) { g_err = "directory / active-warp mismatch"; return -1; }
      if (!((flags >> wp) & 1)) continue;
      const uint32_t* rec = L + 4 * (de & 0xFFFu);
      if (rec != L + L[LH_WOFF0 + wp]) { g_err = "directory offset mismatch"; return -1; }
      const uint32_t mode = cls == GEM_DC_DENSE16 ? GEM_WM_DENSE16 : cls == GEM_DC_DENSE ? GEM_WM_DENSE : GEM_WM_SPARSE;
      const uint32_t n4 = cls == GEM_DC_DENSE16 ? 4u : cls == GEM_DC_DENSE ? 8u : cls;
      if (rec[4] != (mode | (n4 << 8))) { g_err = "directory class / record mode mismatch"; return -1; }
      for (int c = 0; c < 4; c++) warp_c[wp][c] = rec[c];
      for (uint32_t ln = 0; ln < 32; ln++)
        for (int c = 0; c < 4; c++) lane_c[wp * 32 + ln][c] = rec[GEM_WREC_HDR + ln * 4 + c];
      const uint32_t* lv = rec + GEM_WREC_HDR + 128;
      for (uint32_t g = 0; g < n4; g++)
        for (uint32_t ln = 0; ln < 32; ln++)
          for (uint32_t c = 0; c < 4; c++) {
            uint32_t e = lv[(g * 32 + ln) * 4 + c];
            if (mode == GEM_WM_DENSE16) {
              for (uint32_t h = 0; h < 2; h++) {
                uint32_t x = (e >> (16 * h)) & 0xFFFFu, word = GEM_LEAF16_WORD(x), rot = x & 31u;
                uint32_t pos = 8 * g + 2 * c + h;
                read[word] = 1;
                uint32_t s = S[word];
                uint32_t rs = rot ? ((s << rot) | (s >> (32 - rot))) : s;
                val[0][(wp * 32 + ln) * 32 + pos] |= (uint8_t)((rs >> pos) & 1u);
              }
              continue;
            }
            uint32_t word = GEM_LEAF_WORD(e), rot = GEM_LEAF_ROT(e);
            uint32_t pos = mode == GEM_WM_DENSE ? 4 * g + c : GEM_LEAF_POS(e);
            if (word >= GEM_MAX_STATE_WORDS) { g_err = "leaf word out of range"; return -1; }
            read[word] = 1;
            uint32_t s = S[word];
            uint32_t rs = rot ? ((s << rot) | (s >> (32 - rot))) : s;   // rotl: bit b -> (b+rot)%32
            val[0][(wp * 32 + ln) * 32 + pos] |= (uint8_t)((rs >> pos) & 1u);
          }
    }
    for (int k = 1; k <= 13; k++) {
      uint32_t g = gw(k);
      for (uint32_t id = 0; id < (8192u >> k); id++) {
        uint32_t ca = (id / g) * 2 * g + id % g, cb = ca + g;
        uint32_t xa, xb, ob, b = sbit(k, id);
        if (k <= 5) { uint32_t t = id / g; xa = lane_c[t][0]; xb = lane_c[t][1]; ob = lane_c[t][2]; }
        else if (k <= 10) { uint32_t wq = id / g; xa = warp_c[wq][0]; xb = warp_c[wq][1]; ob = warp_c[wq][2]; }
        else { xa = topc & 0xFF; xb = (topc >> 8) & 0xFF; ob = (topc >> 16) & 0xFF; }
        uint32_t A = val[k - 1][ca] ^ ((xa >> b) & 1u);
        uint32_t B = (val[k - 1][cb] ^ ((xb >> b) & 1u)) | ((ob >> b) & 1u);
        val[k][id] = (uint8_t)(A & B);
      }
    }
    // write-outs (after all gathers of the layer)
    auto wo = [&](uint32_t dst, int k0, int k1, uint32_t unit) -> int {
      if (!dst) return 0;
      if (dst >= GEM_MAX_STATE_WORDS) { g_err = "bad write-out"; return -1; }
      if (read[dst]) { g_err = "write-out target read in the same layer"; return -1; }
      if (written[dst] == 2) { g_err = "two write-outs to one word in a layer"; return -1; }
      uint32_t v = 0;
      for (int k = k0; k <= k1; k++) {
        uint32_t g = gw(k);
        for (uint32_t q = 0; q < g; q++) v |= (uint32_t)val[k][unit * g + q] << sbit(k, unit * g + q);
      }
      S[dst] = v;
      written[dst] = 2;
      return 0;
    };
    for (uint32_t t = 0; t < 256; t++) if (wo(lane_c[t][3], 1, 5, t)) return -1;
    for (uint32_t wq = 0; wq < 8; wq++) if (wo(warp_c[wq][3], 6, 10, wq)) return -1;
    if (flags & GEM_LF_USES_TOP) if (wo(L[LH_TOPWO], 11, 13, 0)) return -1;
    for (auto& x : written) if (x == 2) x = 1;
    for (int k = 0; k < 4; k++) dir[k] = L[LH_NEXTDIR + k];
    L += L[LH_WORDS_];
  }
  // outputs
  const uint32_t* od = pr + pr[PH_OFF_OUT];
  const uint32_t* os = od + pr[PH_N_OUT_PAD];
  uint32_t ramp[GEM_MAX_RAMS_PER_PART * 4];
  std::memset(ramp, 0, sizeof(ramp));
  for (uint32_t j = 0; j < pr[PH_N_OUT]; j++) {
    uint32_t v = 0;
    for (int b = 0; b < 32; b++) {
      uint32_t e = os[j * 32 + b];
      uint32_t src = e & 0x7FFFFFFFu;
      v |= (((S[src >> 5] >> (src & 31)) & 1u) ^ (e >> 31)) << b;
    }
    uint32_t reg = GEM_GID_REGION(od[j]), idx = GEM_GID_INDEX(od[j]);
    if (reg == GEM_R_Q) I.Q[nxt][idx] = v;
    else if (reg == GEM_R_PO) po_row[idx] = v;
    else if (reg == GEM_R_CUT) I.CUT[idx] = v;
    else if (reg == GEM_R_RAMP) ramp[idx] = v;
    else { g_err = "bad out region"; return -1; }
  }
  const uint32_t* rr = pr + pr[PH_OFF_RAM];
  for (uint32_t r = 0; r < pr[PH_N_RAM]; r++) {
    uint32_t id = rr[4 * r];
    uint32_t ra = ramp[4 * r + 0] & 0x1FFF, wa = ramp[4 * r + 1] & 0x1FFF;
    uint32_t wd = ramp[4 * r + 2], be = ramp[4 * r + 3];
    I.RD[nxt][id] = I.MEM[id][ra];
    I.MEM[id][wa] = (I.MEM[id][wa] & ~be) | (wd & be);
  }
  (void)t;
  return 0;
}

// ------------------------------------------------------------------ lane mode
// 32 streams per lane word.  Global lane state: Q_lane[2][q_bits], RD_lane[2][rams*32],
// CUT_lane[cut_bits]; MEM per stream.
struct LaneSim {
  std::vector<uint32_t> Q[2], RD[2], CUT;
  std::vector<std::vector<uint32_t>> MEM;   // [stream*n_rams + ram][8192]
};

int run_lane_part(Interp& I, LaneSim& Ls, uint32_t p, const uint32_t* pi_lane /* [pi_bits] */,
                  uint32_t* po_lane /* [po_bits] */) {
  const uint32_t* pt = I.parts + p * GP_WORDS;
  const uint32_t* lane_base = I.w.data() + I.w[GH_OFF_LANE_PROG];
  const uint32_t* pr = lane_base + pt[GP_LANE_OFF];
  const bool v2 = pr[LPH_MAGIC] == GEM_LANE2_MAGIC;
  if (pr[LPH_MAGIC] != GEM_LANE_MAGIC && !v2) { g_err = "bad lane magic"; return -1; }
  uint32_t cur = (uint32_t)(I.cycle & 1), nxt = cur ^ 1;
  std::vector<uint32_t> S(pr[LPH_LANE_WORDS] + 1, 0);
  const uint32_t* gr = pr + pr[LPH_OFF_GREAD];
  for (uint32_t k = 0; k < pr[LPH_N_GREAD]; k++) {
    uint32_t gid = gr[k], dst = k + 1;
    uint32_t reg = gid >> 24, b = gid & 0xFFFFFF, v;
    if (reg == GEM_R_PI) v = pi_lane[b];
    else if (reg == GEM_R_Q) v = Ls.Q[cur][b];
    else if (reg == GEM_R_RD) v = Ls.RD[cur][b];
    else if (reg == GEM_R_CUT) v = Ls.CUT[b];
    else { g_err = "bad lane gread"; return -1; }
    if (dst == 0 || dst >= S.size()) { g_err = "bad lane gread dst"; return -1; }
    S[dst] = v;
  }
  const uint32_t* L = pr + pr[LPH_OFF_LAYERS];
  if (v2) {
    // compacted program (gem_isa.h "LAN2"): every op of a step reads the state
    // as it was before the step; a step's destinations are written after all
    // of its reads (and must not be read within the step)
    std::vector<std::pair<uint32_t, uint32_t>> wr;
    std::vector<uint8_t> written(S.size(), 0);
    const uint32_t M = pr[LPH_OPS_PER_THREAD] ? pr[LPH_OPS_PER_THREAD] : 1u;
    for (uint32_t st = 0; st < pr[LPH_N_LAYERS]; st++) {
      wr.clear();
      const uint32_t* ops = L + (size_t)st * GEM_LANE2_STEP * M * 2;
      for (uint32_t t = 0; t < GEM_LANE2_STEP * M; t++) {
        const uint32_t x = ops[2 * t], y = ops[2 * t + 1];
        if (!y) continue;
        const uint32_t a = x & 0x3FFFu, b = (x >> 16) & 0x3FFFu;
        if (a >= S.size() || b >= S.size() || y >= S.size()) { g_err = "lane2 op word out of range"; return -1; }
        const uint32_t va = S[a] ^ (((x >> 14) & 1u) ? ~0u : 0u), vb = S[b] ^ (((x >> 30) & 1u) ? ~0u : 0u);
        wr.push_back({y, va & vb});
      }
      for (auto& e : wr) {
        if (written[e.first] == 1 + (st & 1) ) { g_err = "lane2 destination written twice in a step"; return -1; }
        written[e.first] = (uint8_t)(1 + (st & 1));
      }
      for (uint32_t t = 0; t < GEM_LANE2_STEP * M; t++) {
        const uint32_t x = ops[2 * t];
        if (!ops[2 * t + 1]) continue;
        if (written[x & 0x3FFFu] == 1 + (st & 1) || written[(x >> 16) & 0x3FFFu] == 1 + (st & 1)) {
          g_err = "lane2 op reads a word written in the same step";
          return -1;
        }
      }
      for (auto& e : wr) S[e.first] = e.second;
      for (auto& e : wr) written[e.first] = 0;
    }
  }
  std::vector<uint32_t> val[14];
  for (uint32_t l = 0; !v2 && l < pr[LPH_N_LAYERS]; l++) {
    for (int k = 0; k <= 13; k++) val[k].assign(8192u >> k, 0);
    uint32_t flags = L[LLH_FLAGS], topc = L[LLH_TOPC];
    uint32_t lane_c[256][3];
    uint32_t warp_c[8][3];
    std::memset(lane_c, 0, sizeof(lane_c));
    std::memset(warp_c, 0, sizeof(warp_c));
    std::vector<std::pair<uint32_t, uint32_t>> wo;   // (slot id global (k<<16|id), word)
    std::vector<uint8_t> read(S.size(), 0);
    for (uint32_t wp = 0; wp < 8; wp++) {
      if (!((flags >> wp) & 1)) continue;
      const uint32_t* rec = L + L[LLH_WOFF0 + wp];
      for (int c = 0; c < 3; c++) warp_c[wp][c] = rec[c];
      for (uint32_t ln = 0; ln < 32; ln++)
        for (int c = 0; c < 3; c++) lane_c[wp * 32 + ln][c] = rec[GEM_LWREC_HDR + ln * 4 + c];
      const uint32_t* lv = rec + GEM_LWREC_HDR + 128;
      for (uint32_t g = 0; g < 4; g++)
        for (uint32_t ln = 0; ln < 32; ln++)
          for (uint32_t k = 0; k < 4; k++) {
            uint32_t e = lv[(g * 32 + ln) * 4 + k];
            for (uint32_t h = 0; h < 2; h++) {
              uint32_t word = ((e >> (16 * h)) & 0xFFFFu) >> 2, pos = 8 * g + 2 * k + h;
              if (((e >> (16 * h)) & 3u) != 0) { g_err = "lane leaf offset not word aligned"; return -1; }
              if (word >= S.size()) { g_err = "lane leaf out of range"; return -1; }
              read[word] = 1;
              val[0][(wp * 32 + ln) * 32 + pos] = 0;
              // stash the word in a separate array: val arrays hold bits for packed mode; here words
            }
          }
    }
    // word-valued slots
    std::vector<uint32_t> wv[14];
    for (int k = 0; k <= 13; k++) wv[k].assign(8192u >> k, 0);
    for (uint32_t wp = 0; wp < 8; wp++) {
      if (!((flags >> wp) & 1)) continue;
      const uint32_t* rec = L + L[LLH_WOFF0 + wp];
      const uint32_t* lv = rec + GEM_LWREC_HDR + 128;
      for (uint32_t g = 0; g < 4; g++)
        for (uint32_t ln = 0; ln < 32; ln++)
          for (uint32_t k = 0; k < 4; k++) {
            uint32_t e = lv[(g * 32 + ln) * 4 + k];
            for (uint32_t h = 0; h < 2; h++) {
              uint32_t word = ((e >> (16 * h)) & 0xFFFFu) >> 2, pos = 8 * g + 2 * k + h;
              wv[0][(wp * 32 + ln) * 32 + pos] = S[word];
            }
          }
    }
    for (int k = 1; k <= 13; k++) {
      uint32_t gwid = gw(k);
      for (uint32_t id = 0; id < (8192u >> k); id++) {
        uint32_t ca = (id / gwid) * 2 * gwid + id % gwid, cb = ca + gwid;
        uint32_t xa, xb, ob, b = sbit(k, id);
        if (k <= 5) {
          // lane-mode levels 1-5: slot bit b sits at bit 8*(b&3) + 7 - (b>>2) (gem_isa.h)
          auto un = [](uint32_t c) {
            uint32_t r = 0;
            for (uint32_t q = 0; q < 31; q++) r |= ((c >> (8 * (q & 3) + 7 - (q >> 2))) & 1u) << q;
            return r;
          };
          uint32_t t = id / gwid; xa = un(lane_c[t][0]); xb = un(lane_c[t][1]); ob = un(lane_c[t][2]);
        }
        else if (k <= 10) { uint32_t wq = id / gwid; xa = warp_c[wq][0]; xb = warp_c[wq][1]; ob = warp_c[wq][2]; }
        else { xa = topc & 0xFF; xb = (topc >> 8) & 0xFF; ob = (topc >> 16) & 0xFF; }
        uint32_t XA = ((xa >> b) & 1u) ? ~0u : 0u, XB = ((xb >> b) & 1u) ? ~0u : 0u, OB = ((ob >> b) & 1u) ? ~0u : 0u;
        wv[k][id] = (wv[k - 1][ca] ^ XA) & ((wv[k - 1][cb] ^ XB) | OB);
      }
    }
    // write-outs: slot bit -> slot id within the unit
    auto slot_of = [&](int unit_kind, uint32_t unit, uint32_t bit, int& k_out, uint32_t& id_out) {
      static const int off[6] = {0, 0, 16, 24, 28, 30};
      if (unit_kind == 2) {   // top
        if (bit < 4) { k_out = 11; id_out = bit; } else if (bit < 6) { k_out = 12; id_out = bit - 4; }
        else { k_out = 13; id_out = 0; }
        return;
      }
      int kk = bit < 16 ? 1 : bit < 24 ? 2 : bit < 28 ? 3 : bit < 30 ? 4 : 5;
      uint32_t q = bit - (uint32_t)off[kk];
      k_out = unit_kind == 0 ? kk : kk + 5;
      id_out = unit * gw(k_out) + q;
    };
    // thread units (kind 0) write two runs: level-1 slots (bits 0-15) from the
    // low 16 bits of base, levels 2-5 (bits 16-30) from the high 16 bits
    auto do_wo = [&](int kind, uint32_t unit, uint32_t mask, uint32_t base) -> int {
      for (uint32_t bit = 0; bit < 31; bit++) {
        if (!((mask >> bit) & 1u)) continue;
        uint32_t word = base + (uint32_t)__builtin_popcount(mask & ((1u << bit) - 1u));
        if (kind == 0)
          word = bit < 16 ? (base & 0xFFFFu) + (uint32_t)__builtin_popcount(mask & ((1u << bit) - 1u))
                          : (base >> 16) + (uint32_t)__builtin_popcount(mask & ((1u << bit) - 1u) & 0xFFFF0000u);
        if (word == 0 || word >= S.size()) { g_err = "bad lane write-out"; return -1; }
        if (read[word]) { g_err = "lane write-out target read in the same layer"; return -1; }
        int k; uint32_t id;
        slot_of(kind, unit, bit, k, id);
        wo.push_back({word, wv[k][id]});
      }
      return 0;
    };
    for (uint32_t wp = 0; wp < 8; wp++) {
      if (!((flags >> wp) & 1)) continue;
      const uint32_t* rec = L + L[LLH_WOFF0 + wp];
      for (uint32_t ln = 0; ln < 32; ln++)
        if (do_wo(0, wp * 32 + ln, rec[GEM_LWREC_HDR + ln * 4 + 3], rec[GEM_LWREC_BASE + ln])) return -1;
      if (do_wo(1, wp, rec[3], rec[4])) return -1;
    }
    if (do_wo(2, 0, L[LLH_TOPWO] & 0x7F, L[LLH_TOPWO] >> 8)) return -1;
    for (auto& x : wo) S[x.first] = x.second;
    L += L[LLH_WORDS_];
  }
  // outputs
  const uint32_t* od = pr + pr[LPH_OFF_OUT];
  std::vector<uint32_t> ramp(GEM_MAX_RAMS_PER_PART * 4 * 32, 0);
  for (uint32_t j = 0; j < pr[LPH_N_OUT]; j++) {
    uint32_t dst = od[2 * j], src = od[2 * j + 1];
    uint32_t v = S[src & 0xFFFF] ^ ((src >> 31) ? ~0u : 0u);
    uint32_t reg = dst >> 24, b = dst & 0xFFFFFF;
    if (reg == GEM_R_Q) Ls.Q[nxt][b] = v;
    else if (reg == GEM_R_PO) po_lane[b] = v;
    else if (reg == GEM_R_CUT) Ls.CUT[b] = v;
    else if (reg == GEM_R_RAMP) ramp[b] = v;
    else { g_err = "bad lane out"; return -1; }
  }
  const uint32_t* rr = pr + pr[LPH_OFF_RAM];
  for (uint32_t r = 0; r < pr[LPH_N_RAM]; r++) {
    uint32_t id = rr[4 * r];
    for (uint32_t st = 0; st < 32; st++) {
      auto num = [&](uint32_t port, int bits) {
        uint32_t v = 0;
        for (int k = 0; k < bits; k++) v |= ((ramp[(r * 4 + port) * 32 + k] >> st) & 1u) << k;
        return v;
      };
      uint32_t ra = num(0, 13), wa = num(1, 13), wd = num(2, 32), be = num(3, 32);
      auto& M = Ls.MEM[st * I.n_rams + id];
      uint32_t old = M[ra];
      M[wa] = (M[wa] & ~be) | (wd & be);
      for (int k = 0; k < 32; k++) {
        uint32_t& word = Ls.RD[nxt][id * 32 + k];
        word = (word & ~(1u << st)) | (((old >> k) & 1u) << st);
      }
    }
  }
  return 0;
}

// ------------------------------------------------------------------ word mode
// gem_isa.h "WRD1": one signal per word (bit 0), steps of independent ops.
// Hazard checks: an op of step s reads no word written in step s, a word is
// written at most once per step, word 0 is never written.
int run_word_part(Interp& I, uint32_t p, const uint32_t* stim, uint32_t* po_row) {
  const uint32_t* pt = I.parts + p * GP_WORDS;
  const uint32_t* pr = I.w.data() + I.w[GH_OFF_WORD_PROG] + pt[GP_WORD_OFF];
  if (pr[WPH_MAGIC] != GEM_WORD_MAGIC) { g_err = "bad word magic"; return -1; }
  uint32_t cur = (uint32_t)(I.cycle & 1), nxt = cur ^ 1;
  std::vector<uint32_t> S(pr[WPH_STATE_WORDS], 0);
  std::vector<uint32_t> wstep(S.size(), 0xFFFFFFFFu);
  const uint32_t* gr = pr + pr[WPH_OFF_GREAD];
  for (uint32_t k = 0; k < pr[WPH_N_GREAD]; k++) {
    const uint32_t reg = gr[k] >> 24, bit = gr[k] & 0xFFFFFFu, wi = bit >> 5;
    uint32_t v;
    if (reg == GEM_R_PI) v = stim[wi];
    else if (reg == GEM_R_Q) v = I.Q[cur][wi];
    else if (reg == GEM_R_RD) v = I.RD[cur][wi];
    else if (reg == GEM_R_CUT) v = I.CUT[wi];
    else { g_err = "bad word gread region"; return -1; }
    if (1 + k >= S.size()) { g_err = "word gread outside the state"; return -1; }
    S[1 + k] = (v >> (bit & 31)) & 1u;
  }
  const uint32_t* stp = pr + pr[WPH_OFF_STEPS];
  const uint32_t* ops = pr + pr[WPH_OFF_OPS];
  std::vector<std::pair<uint32_t, uint32_t>> wr;
  for (uint32_t s = 0; s < pr[WPH_N_STEPS]; s++) {
    wr.clear();
    for (uint32_t i = stp[s]; i < stp[s + 1]; i++) {
      const uint32_t x = ops[2 * i], y = ops[2 * i + 1];
      const uint32_t a = (x & 0xFFFCu) >> 2, b = ((x >> 16) & 0xFFFCu) >> 2, d = y >> 2;
      if (a >= S.size() || b >= S.size() || d >= S.size() || d == 0 || (y & 3u)) { g_err = "word op out of range"; return -1; }
      if (wstep[a] == s || wstep[b] == s) { g_err = "word op reads a word written in the same step"; return -1; }
      if (wstep[d] == s) { g_err = "word written twice in a step"; return -1; }
      wstep[d] = s;
      wr.push_back({d, ((S[a] ^ x) & (S[b] ^ (x >> 16))) & 1u});
    }
    for (uint32_t i = stp[s]; i < stp[s + 1]; i++) {
      const uint32_t x = ops[2 * i];
      if (wstep[(x & 0xFFFCu) >> 2] == s || wstep[((x >> 16) & 0xFFFCu) >> 2] == s) {
        g_err = "word op reads a word written in the same step";
        return -1;
      }
    }
    for (auto& e : wr) S[e.first] = e.second;
  }
  const uint32_t n_out = pr[WPH_N_OUT];
  const uint32_t* od = pr + pr[WPH_OFF_OUT];
  const uint32_t* os = od + n_out;
  uint32_t ramp[GEM_MAX_RAMS_PER_PART * 4];
  std::memset(ramp, 0, sizeof(ramp));
  for (uint32_t j = 0; j < n_out; j++) {
    uint32_t v = 0;
    for (int b = 0; b < 32; b++) {
      const uint32_t e = os[j * 32 + b];
      if (((e & 0xFFFCu) >> 2) >= S.size()) { g_err = "word output out of range"; return -1; }
      v |= ((S[(e & 0xFFFCu) >> 2] ^ e) & 1u) << b;
    }
    uint32_t reg = GEM_GID_REGION(od[j]), idx = GEM_GID_INDEX(od[j]);
    if (reg == GEM_R_Q) I.Q[nxt][idx] = v;
    else if (reg == GEM_R_PO) po_row[idx] = v;
    else if (reg == GEM_R_CUT) I.CUT[idx] = v;
    else if (reg == GEM_R_RAMP) ramp[idx] = v;
    else { g_err = "bad word out region"; return -1; }
  }
  const uint32_t* rr = pr + pr[WPH_OFF_RAM];
  for (uint32_t r = 0; r < pr[WPH_N_RAM]; r++) {
    uint32_t id = rr[4 * r];
    uint32_t ra = ramp[4 * r + 0] & 0x1FFF, wa = ramp[4 * r + 1] & 0x1FFF;
    uint32_t wd = ramp[4 * r + 2], be = ramp[4 * r + 3];
    I.RD[nxt][id] = I.MEM[id][ra];
    I.MEM[id][wa] = (I.MEM[id][wa] & ~be) | (wd & be);
  }
  return 0;
}
}  // namespace

extern "C" {
const char* isa_last_error(void) { return g_err.c_str(); }

void* isa_load(const void* blob, size_t nbytes) {
  Interp* I = new Interp();
  I->w.assign((const uint32_t*)blob, (const uint32_t*)blob + nbytes / 4);
  const uint32_t* h = I->w.data();
  if (h[GH_MAGIC] != GEM_MAGIC) { g_err = "bad magic"; delete I; return nullptr; }
  I->n_parts = h[GH_N_PARTS]; I->n_stages = h[GH_N_STAGES];
  I->q_words = h[GH_Q_WORDS]; I->po_words = h[GH_PO_WORDS]; I->cut_words = h[GH_CUT_WORDS];
  I->pi_words = h[GH_PI_WORDS]; I->n_rams = h[GH_N_RAMS]; I->n_flops = h[GH_N_FLOPS]; I->n_po = h[GH_N_PO];
  I->parts = h + h[GH_OFF_PARTS];
  I->stages = h + h[GH_OFF_STAGES];
  I->prog = h + h[GH_OFF_PROG];
  I->flop_init = h + h[GH_OFF_FLOP_INIT];
  I->q_ext = I->flop_init + I->q_words;
  I->po_ext = I->q_ext + (size_t)I->q_words * 32;
  for (int b = 0; b < 2; b++) { I->Q[b].assign(I->q_words, 0); I->RD[b].assign(I->n_rams, 0); }
  for (uint32_t w = 0; w < I->q_words; w++) I->Q[0][w] = I->flop_init[w];
  I->CUT.assign(I->cut_words, 0);
  I->MEM.assign(I->n_rams, std::vector<uint32_t>(GEM_RAM_WORDS, 0));
  return I;
}

void isa_free(void* h) { delete (Interp*)h; }

// 32 streams in lane mode: stim [32][cycles][pi_words]; po_ext [32][cycles][ceil(n_po/32)];
// q_ext [32][cycles][ceil(n_flops/32)]
int isa_run_lanes(void* h, const uint32_t* stim, uint64_t cycles, uint32_t* po_ext, uint32_t* q_ext_tr) {
  Interp& I = *(Interp*)h;
  if (!I.w[GH_HAS_LANES]) { g_err = "blob has no lane programs"; return -1; }
  LaneSim Ls;
  for (int b = 0; b < 2; b++) { Ls.Q[b].assign(I.q_words * 32, 0); Ls.RD[b].assign(I.n_rams * 32, 0); }
  for (uint32_t bit = 0; bit < I.q_words * 32; bit++)
    Ls.Q[0][bit] = ((I.flop_init[bit / 32] >> (bit % 32)) & 1u) ? ~0u : 0u;
  Ls.CUT.assign(I.cut_words * 32, 0);
  Ls.MEM.assign((size_t)32 * I.n_rams, std::vector<uint32_t>(GEM_RAM_WORDS, 0));
  uint32_t pwe = (I.n_po + 31) / 32, qwe = (I.n_flops + 31) / 32;
  std::vector<uint32_t> pi_lane(I.pi_words * 32), po_lane(I.po_words * 32);
  uint64_t c0 = I.cycle;
  for (uint64_t t = 0; t < cycles; t++) {
    for (uint32_t b = 0; b < I.pi_words * 32; b++) {
      uint32_t v = 0;
      for (uint32_t st = 0; st < 32; st++)
        v |= ((stim[(st * cycles + t) * I.pi_words + b / 32] >> (b % 32)) & 1u) << st;
      pi_lane[b] = v;
    }
    std::fill(po_lane.begin(), po_lane.end(), 0);
    for (uint32_t s = 0; s < I.n_stages; s++)
      for (uint32_t k = I.stages[s]; k < I.stages[s + 1]; k++)
        if (run_lane_part(I, Ls, I.stages[I.n_stages + 1 + k], pi_lane.data(), po_lane.data())) return -1;
    I.cycle++;
    uint32_t cur = (uint32_t)(I.cycle & 1);
    for (uint32_t st = 0; st < 32; st++) {
      uint32_t* row = po_ext + (st * cycles + t) * pwe;
      std::memset(row, 0, pwe * 4);
      for (uint32_t b = 0; b < I.po_words * 32; b++) {
        uint32_t e = I.po_ext[b];
        if (e == 0xFFFFFFFFu) continue;
        row[e / 32] |= ((po_lane[b] >> st) & 1u) << (e % 32);
      }
      if (q_ext_tr) {
        uint32_t* qr = q_ext_tr + (st * cycles + t) * qwe;
        std::memset(qr, 0, qwe * 4);
        for (uint32_t b = 0; b < I.q_words * 32; b++) {
          uint32_t e = I.q_ext[b];
          if (e == 0xFFFFFFFFu) continue;
          qr[e / 32] |= ((Ls.Q[cur][b] >> st) & 1u) << (e % 32);
        }
      }
    }
  }
  (void)c0;
  return 0;
}

// stim [cycles][pi_words] ; po_ext [cycles][ceil(n_po/32)] ; q_ext [cycles][ceil(n_flops/32)] (nullable)
static int isa_run_impl(void* h, const uint32_t* stim, uint64_t cycles, uint32_t* po_ext, uint32_t* q_ext_tr,
                        bool words) {
  Interp& I = *(Interp*)h;
  if (words && !I.w[GH_HAS_WORDS]) { g_err = "blob has no word programs"; return -1; }
  std::vector<uint32_t> po_int(I.po_words);
  uint32_t pwe = (I.n_po + 31) / 32, qwe = (I.n_flops + 31) / 32;
  for (uint64_t t = 0; t < cycles; t++) {
    std::fill(po_int.begin(), po_int.end(), 0);
    for (uint32_t s = 0; s < I.n_stages; s++)
      for (uint32_t k = I.stages[s]; k < I.stages[s + 1]; k++) {
        uint32_t p = I.stages[I.n_stages + 1 + k];
        if (words ? run_word_part(I, p, stim + t * I.pi_words, po_int.data())
                  : run_part(I, p, t, stim + t * I.pi_words, po_int.data()))
          return -1;
      }
    I.cycle++;
    uint32_t cur = (uint32_t)(I.cycle & 1);
    if (po_ext) {
      uint32_t* row = po_ext + t * pwe;
      std::memset(row, 0, pwe * 4);
      for (uint32_t b = 0; b < I.po_words * 32; b++) {
        uint32_t e = I.po_ext[b];
        if (e == 0xFFFFFFFFu) continue;
        row[e / 32] |= ((po_int[b / 32] >> (b % 32)) & 1u) << (e % 32);
      }
    }
    if (q_ext_tr) {
      uint32_t* row = q_ext_tr + t * qwe;
      std::memset(row, 0, qwe * 4);
      for (uint32_t b = 0; b < I.q_words * 32; b++) {
        uint32_t e = I.q_ext[b];
        if (e == 0xFFFFFFFFu) continue;
        row[e / 32] |= ((I.Q[cur][b / 32] >> (b % 32)) & 1u) << (e % 32);
      }
    }
  }
  return 0;
}
int isa_run(void* h, const uint32_t* stim, uint64_t cycles, uint32_t* po_ext, uint32_t* q_ext_tr) {
  return isa_run_impl(h, stim, cycles, po_ext, q_ext_tr, false);
}
int isa_run_words(void* h, const uint32_t* stim, uint64_t cycles, uint32_t* po_ext, uint32_t* q_ext_tr) {
  return isa_run_impl(h, stim, cycles, po_ext, q_ext_tr, true);
}
}
