// gem_isa.h -- the VLIW program ("bitstream") format executed by the sm_100a
// interpreter kernel and produced by the mapper.  Product-path header: it is
// NOT shared with oracle/ (the oracle knows nothing about partitions, layers
// or this ISA).
//
// Paper background:
//   P:73  one logic partition = one Boolean processor core = one thread block
//   P:85  boomerang executor layer: permute (gather) 8192 state bits, then fold
//         them with bitwise AND + XOR constants down to one bit ("14" bit-vectors
//         = 8192 leaves + 13 AND levels; reading U1)
//   P:180 VLIW instructions consumed by 256 threads with coalesced wide loads
//   P:196 init instruction (layer count, RAM count, state size), global-read
//         instructions (input ports, once per cycle), interleaved permutation +
//         fold-constant instructions with XOR.A, XOR.B, OR.B per thread
//
// This build's own encoding (the paper's Fig. 7 bit layout is not available):
//
//  * Partition state S: up to GEM_MAX_STATE_WORDS u32 words in shared memory.
//    Word 0 is the constant-0 word and is never written.
//  * A layer = one 8192-leaf, 13-level boomerang over 256 threads:
//      - thread t gathers leaf word t (32 leaves) from S (sparse leaf list),
//      - levels 1-5 fold the word inside the thread (16,8,4,2,1 slots),
//      - a warp ballot collects the 32 level-5 bits; levels 6-10 fold that
//        word inside the warp (16,8,4,2,1 slots),
//      - levels 11-13 fold the 8 warp bits (4,2,1 slots) in one thread.
//    Slot op (readings U2/U3):  out = (A ^ xa) & ((B ^ xb) | ob)
//    At level k inside a group with g slots per unit, slot q takes A = slot q
//    and B = slot q+g of the level below (same unit).
//  * Packed slot words: a thread's level-1..5 slot values (and constants) are
//    packed as bits [0,16) L1, [16,24) L2, [24,28) L3, [28,30) L4, [30] L5;
//    the warp's levels 6..10 use the same offsets; top levels 11,12,13 use
//    bits [0,4), [4,6), [6].
//  * Write-out (reading U4): a thread (warp, top) may store its packed slot
//    word into one free state word; the mapper tracks which bits are live.
//
// Program blob (.gemb), all little-endian u32 words:
//   GembHeader | part table | stage list | flop init | program area
#pragma once
#include <stdint.h>

#define GEM_MAGIC 0x424d4547u   /* "GEMB" */
#define GEM_VERSION 1u
#define GEM_THREADS 256         /* thread block of 256 threads */
#define GEM_WARPS 8
#define GEM_LEAVES 8192         /* 8,192 bits per boomerang layer */
#define GEM_LEVELS 13
#define GEM_MAX_STATE_WORDS 8192  /* 256 Kbit state (32 KB of shared memory) */
#define GEM_RAM_ABITS 13
#define GEM_RAM_WORDS 8192
#define GEM_MAX_RAMS_PER_PART 32
#define GEM_MAX_CHUNKS 256      /* chunks per partition program (= layers + 2)      */

/* global word regions (gid = region << 24 | index) */
#define GEM_R_PI 0u     /* gread source: PI word of the current cycle        */
#define GEM_R_Q 1u      /* gread: flop word of Q_cur;  out: flop word of Q_next */
#define GEM_R_RD 2u     /* gread: registered RAM read data RD_cur[ram]        */
#define GEM_R_CUT 3u    /* gread/out: stage-cut word (multi-stage)     */
#define GEM_R_PO 4u     /* out: PO word of the current cycle                  */
#define GEM_R_RAMP 5u   /* out: RAM port staging word (ram_local*4 + port)    */
#define GEM_GID(region, idx) (((uint32_t)(region) << 24) | (uint32_t)(idx))
#define GEM_GID_REGION(g) ((g) >> 24)
#define GEM_GID_INDEX(g) ((g) & 0xFFFFFFu)

/* RAM port staging order */
#define GEM_PORT_RADDR 0
#define GEM_PORT_WADDR 1
#define GEM_PORT_WDATA 2
#define GEM_PORT_WBE 3

/* output-gather source entry: bit index into S, bit 31 = invert */
#define GEM_OUT_INV 0x80000000u

/* leaf entry (gather of one state bit b of word w into leaf position p):
 *   bits [0,5)   rot = (p - b) mod 32   -> rotl(S[w], rot) puts bit b at p
 *                (a funnel shift uses the low 5 bits of the entry directly)
 *   bits [8,13)  p (SPARSE warps only; DENSE warps use entry index = p):
 *                rotl(1, entry >> 8) is the position mask
 *   bits [16,32) byte offset of S[w] (w*4; S sits at shared-memory offset 0),
 *                so the load address is entry >> 16
 * Padding entries are 0: they read S[0] == 0.                                  */
#define GEM_LEAF(word, bit, pos) \
  ((((uint32_t)(pos) - (uint32_t)(bit)) & 31u) | ((uint32_t)(pos) << 8) | ((uint32_t)(word) << 18))
#define GEM_LEAF_DENSE(word, bit, pos) ((((uint32_t)(pos) - (uint32_t)(bit)) & 31u) | ((uint32_t)(word) << 18))
#define GEM_LEAF_WORD(e) ((uint32_t)(e) >> 18)
/* 16-bit dense entry (DENSE16 warps, state words < 2048): rot | word << 5;
 * u32 k of a lane's group g holds entries 8g+2k (low half) and 8g+2k+1 (high). */
#define GEM_LEAF16(word, bit, pos) ((((uint32_t)(pos) - (uint32_t)(bit)) & 31u) | ((uint32_t)(word) << 5))
#define GEM_LEAF16_WORD(h) (((h) >> 5) & 0x7FFu)
#define GEM_LEAF_ROT(e) ((e) & 31u)
#define GEM_LEAF_POS(e) (((e) >> 8) & 31u)

/* packed slot-word bit offsets for levels 1..5 of a group */
#define GEM_OFF_L1 0
#define GEM_OFF_L2 16
#define GEM_OFF_L3 24
#define GEM_OFF_L4 28
#define GEM_OFF_L5 30

/* blob header (64 words) */
enum {
  GH_MAGIC = 0, GH_VERSION, GH_N_PI, GH_N_PO, GH_N_FLOPS, GH_N_RAMS, GH_N_PARTS, GH_N_STAGES,
  GH_MAX_STATE_WORDS, GH_MAX_LAYERS, GH_PI_WORDS, GH_PO_WORDS, GH_Q_WORDS, GH_CUT_WORDS,
  GH_N_AND_LO, GH_N_AND_HI, GH_N_AND_MAPPED_LO, GH_N_AND_MAPPED_HI, GH_TOTAL_LAYERS,
  GH_TOTAL_LEAVES_LO, GH_TOTAL_LEAVES_HI, GH_OFF_PARTS, GH_OFF_STAGES, GH_OFF_FLOP_INIT,
  GH_OFF_PROG, GH_PROG_WORDS_LO, GH_PROG_WORDS_HI, GH_MAX_LEVELS, GH_TOTAL_WRITEOUTS,
  GH_MAX_OUT, GH_TOTAL_WORDS_LO, GH_TOTAL_WORDS_HI, GH_SLOTS_USED_LO, GH_SLOTS_USED_HI,
  GH_MAX_CHUNK_WORDS, GH_MAX_PROG_WORDS,
  GH_HAS_LANES, GH_OFF_LANE_PROG, GH_LANE_PROG_WORDS_LO, GH_LANE_PROG_WORDS_HI, GH_LANE_MAX_CHUNK_WORDS,
  GH_LANE_MAX_WORDS, GH_MAX_RAMS_PART,
  GH_N_AND_SYNTH_LO, GH_N_AND_SYNTH_HI,  /* live ANDs after depth-oriented synthesis (GH_N_AND: before) */
  GH_LEVELS_IN,                         /* logic depth before synthesis (GH_MAX_LEVELS: after)       */
  GH_SYNTH_CHAINS,                      /* chains rewritten by the lookahead                          */
  GH_HAS_WORDS, GH_OFF_WORD_PROG, GH_WORD_PROG_WORDS_LO, GH_WORD_PROG_WORDS_HI,   /* word programs (WRD1) */
  GH_WORD_MAX_STATE, GH_WORD_MAX_PROG, GH_WORD_MAX_STEPS, GH_WORD_OPS_LO, GH_WORD_OPS_HI, GH_WORD_TOTAL_STEPS,
  GH_N_WORDS = 64
};

/* part table entry */
enum {
  GP_STAGE = 0, GP_PROG_OFF, GP_PROG_LEN, GP_N_LAYERS, GP_CHUNK0, GP_MAX_CHUNK, GP_CHUNK1, GP_CHUNK2,
  GP_COST, GP_LANE_OFF, GP_LANE_LEN, GP_LANE_CHUNK0, GP_LANE_CHUNK1, GP_LANE_CHUNK2, GP_LANE_WORDS,
  GP_WORD_OFF /* word program offset in the WRD1 section (GH_HAS_WORDS) */,
  GP_WORDS = 16
};
/* GP_COST: mapper's estimate of one cycle of the partition in SM clocks (used by
 * the runtime's longest-processing-time work-list scheduling). */
/* GP_CHUNK1/2: sizes of chunks 1 and 2 (0 if absent) so the first three chunks of
 * the next work item can be prefetched before its chunk table has arrived. */

/* A partition program is a sequence of "chunks" streamed into shared memory by
 * TMA bulk copies (cp.async.bulk, 16-byte granules): chunk 0 = header + chunk
 * table + gread list, chunks 1..n_layers = one layer record each, chunk
 * n_layers+1 = output + RAM sections.  The chunk table (PH_OFF_CHUNKS) holds
 * the word size of every chunk (all multiples of 4 words).  After the last
 * chunk, the program's final ceil4(n_gread) words hold the used-bit mask of
 * every gread word (entry order; read only by GEM_F_ACTIVITY, row f3).      */
/* partition program header (16 words) */
enum {
  PH_MAGIC = 0, PH_N_GREAD, PH_N_LAYERS, PH_N_OUT, PH_N_RAM, PH_STATE_WORDS, PH_OFF_GREAD,
  PH_OFF_LAYERS, PH_OFF_OUT, PH_OFF_RAM, PH_N_LEAVES, PH_N_NODES, PH_N_OUT_PAD, PH_OFF_CHUNKS,
  PH_N_CHUNKS, PH_OFF_DIR0, PH_WORDS = 16
};
#define GEM_PART_MAGIC 0x54524150u  /* "PART" */

/* layer header (16 words) followed by one record per active warp:
 *   [LH_WORDS_] layer size in words, [LH_FLAGS] active-warp mask | USES_TOP,
 *   [LH_TOPC] top constants, [LH_TOPWO] top write-out word,
 *   [LH_WOFF0 + w] word offset of warp w's record from the layer start (0 = inactive)
 * warp record:
 *   [0..3]  wxa, wxb, wob, wwo           (levels 6-10 constants, write-out)
 *   [4]     mode (GEM_WM_DENSE / GEM_WM_SPARSE) | n4 << 8   (n4 = uint4 leaf groups per lane)
 *   [5..7]  reserved
 *   [8..136) lane constants: uint4 {xa, xb, ob, wo} per lane (levels 1-5)
 *   [136..) leaves: [n4][32 lanes] x uint4 (4 entries per lane per group)
 * DENSE warps have n4 = 8 and entry j of a lane fills leaf position j.        */
enum {
  LH_WORDS_ = 0, LH_FLAGS, LH_TOPC, LH_TOPWO, LH_WOFF0 /* ..LH_WOFF0+7 */, LH_NEXTDIR = 12 /* ..15 */,
  LH_WORDS = 16
};
/* Record directory of a layer: 8 u16 entries (warp w in half w&1 of word w>>1),
 *   bits [0,12)  warp record offset from the layer start / 4 (words)
 *   bits [12,16) record class GEM_DC_* (0 = warp inactive; SPARSE n4 = class)
 * Layer l's header holds the directory of layer l+1 (LH_NEXTDIR, zeros after
 * the last layer); layer 0's directory sits in chunk 0 at PH_OFF_DIR0.  A warp
 * therefore knows where its next record lies before that record's layer is
 * read, and issues all of its record loads at once (no dependent load chain). */
/* classes 1..8: SPARSE with n4 = class */
#define GEM_DC_DENSE16 9u
#define GEM_DC_DENSE 10u
#define GEM_DIR_ENTRY(woff, cls) ((((uint32_t)(woff) >> 2) & 0xFFFu) | ((uint32_t)(cls) << 12))
#define GEM_LF_USES_TOP 0x100u   /* flags bit 8; bits [0,8) = active warp mask */
#define GEM_WM_SPARSE 0u
#define GEM_WM_DENSE 1u     /* 32 u32 entries per lane (n4 = 8)                  */
#define GEM_WM_DENSE16 2u   /* 32 u16 entries per lane (n4 = 4)                  */
#define GEM_WREC_HDR 8
#define GEM_WARP_REC_WORDS(n4) (GEM_WREC_HDR + 32 * 4 + 128 * (n4))

/* output section: dst gid [n_out_pad] then src [n_out][32]
 * RAM section: per owned RAM 4 words {ram_id, 0, 0, 0}; its ports are staged by
 * outputs with region GEM_R_RAMP index = local*4 + port.                       */

/* ---------------------------------------------------------------------------
 * Lane mode (stream-sliced execution of the same placement, optional: mapper
 * option lanes=1).  For a group of 32 independent stimulus streams every
 * signal is one 32-bit "lane word" (bit s = stream s), so one pass over a
 * layer evaluates it for 32 streams: leaves are whole lane words (no bit
 * extraction) and each gate slot is two LOP3 on words.  Same layers, same
 * slots, same packed constants as the bit-packed program; only signal storage
 * differs (one lane word per live signal, allocated by liveness).
 *
 * Global lane layout (per 32-stream group g, n_groups words per row):
 *   Q_lane[2][q_words*32][G], RD_lane[2][n_rams*32][G], CUT_lane[cut_words*32][G],
 *   PI_lane[cycle][pi_words*32][G], PO_lane[cycle][po_words*32][G]
 * gid_l = region << 24 | bit index (RAMP: (ram_local*4 + port)*32 + bit).
 *
 * Lane partition program: header (16) | chunk table | layers | out+ram | gread
 *   (chunks: 0 = header + table, 1..L = layers, L+1 = out+ram; the gread list
 *   is read from global memory)
 *   gread: one u32 gid_l per entry; entry k is stored to lane word k + 1
 *   layer: header (32 words) {size, flags, topc, top_mask | top_base << 8, woff[8], 0 x4,
 *          next layer's first 12 words, 0 x4}
 *          warp record (GEM_LWREC_WORDS words):
 *            [0..5)    wxa, wxb, wob, wmask, wbase       (levels 6-10)
 *            [8..136)  lane constants uint4 {xa, xb, ob, mask}  (levels 1-5; xa/xb/ob
 *                      byte-spread: slot bit b at bit 8*(b&3) + 7 - (b>>2), so
 *                      prmt(c << (b>>2), sign-replicate byte b&3) is its mask;
 *                      mask keeps slot-bit order)
 *            [136..648) leaves: [4 groups][32 lanes] uint4 (32 u16 lane-word byte offsets w*4
 *                       per lane, entry 8g+2k low half, 8g+2k+1 high half)
 *            [648..680) per-lane write-out base words: level-1 slots (bits 0-15) from the
 *                       low 16 bits, levels 2-5 (bits 16-30) from the high 16 bits
 *   Write-outs: a unit (thread / warp / top) stores the slots whose bits are set
 *   in its mask, in slot-bit order, to consecutive lane words from its base:
 *   slot b -> base + popc(mask & ((1 << b) - 1)); thread units write two such
 *   runs (levels 1 and 2-5, bases in the low / high half of the base word).
 *   out:   uint2 {dst gid_l, src lane word | GEM_OUT_INV}
 *   ram:   4 words per owned RAM {ram_id, 0, 0, 0}
 * Lane word 0 is the constant 0.                                            */
#define GEM_LANE_MAGIC 0x454E414Cu  /* "LANE" */
#define GEM_LANE_STREAMS 32
enum {
  LPH_MAGIC = 0, LPH_N_GREAD, LPH_N_LAYERS, LPH_N_OUT, LPH_N_RAM, LPH_LANE_WORDS, LPH_OFF_GREAD,
  LPH_OFF_LAYERS, LPH_OFF_OUT, LPH_OFF_RAM, LPH_OFF_CHUNKS, LPH_N_CHUNKS, LPH_N_OPS /* LAN2: AND ops */,
  LPH_OPS_PER_THREAD /* LAN2: M ops per thread and step (0 = 1) */, LPH_R14, LPH_R15, LPH_WORDS = 16
};
/* lane layer header: [0,12) this layer {size, flags, topc, topwo, woff[8]};
 * [16,28) a copy of the NEXT layer's [0,12) (zeros after the last layer), so
 * the kernel knows layer l+1's record addresses while it runs layer l and all
 * of its record loads issue at once (no header -> offset -> record chain) */
enum { LLH_WORDS_ = 0, LLH_FLAGS, LLH_TOPC, LLH_TOPWO, LLH_WOFF0 /* ..+7 */, LLH_NEXT = 16, LLH_WORDS = 32 };
#define GEM_LWREC_HDR 8
#define GEM_LWREC_LEAVES (GEM_LWREC_HDR + 128)
#define GEM_LWREC_BASE (GEM_LWREC_HDR + 128 + 512)
#define GEM_LWREC_WORDS (GEM_LWREC_BASE + 32)

/* ---------------------------------------------------------------------------
 * Lane mode, compacted program (magic "LAN2", mapper lane_mode=2, the default).
 * The boomerang placement evaluates every slot of every layer, 8191 per
 * layer, of which C5 uses 42% as real ANDs (the rest are pass-throughs, empty
 * slots and tree-expanded copies); with whole lane words in shared memory a
 * signal needs no bit permutation and no fan-out duplication, so the lane
 * program is the partition's AND list itself, list-scheduled into STEPS of at
 * most 256 independent ANDs (one per thread) separated by a block barrier:
 *   header (LPH_*, LPH_N_LAYERS = n_steps, LPH_OFF_LAYERS = op array)
 *   gread:  one u32 gid_l per entry, entry k -> lane word k + 1 (as "LANE")
 *   ops:    [n_steps][M][256] uint2 {x, y} (M = LPH_OPS_PER_THREAD, 1 or 2), thread
 *           t of step s runs ops (s*M + j)*256 + t, j < M:
 *             x = a | ia << 14 | b << 16 | ib << 30   (lane words < 16384)
 *             y = destination lane word (0 = no op)
 *           result(y) = (S[a] ^ -ia) & (S[b] ^ -ib); operands were written in
 *           earlier steps; a destination is never read in the same step.
 *   out, ram: as "LANE".
 * Words are allocated by liveness (free after the last reading step) with
 * the destination residues of each half-warp chosen apart (LDS.64/STS.64 of
 * two interleaved 32-stream groups are conflict-free when the 16 lanes of a
 * half-warp touch different word residues mod 16).                        */
#define GEM_LANE2_MAGIC 0x324E414Cu  /* "LAN2" */
#define GEM_LANE2_STEP 256
#define GEM_LANE2_OP_X(a, ia, b, ib) \
  ((uint32_t)(a) | ((uint32_t)(ia) << 14) | ((uint32_t)(b) << 16) | ((uint32_t)(ib) << 30))

/* ---------------------------------------------------------------------------
 * Word programs ("WRD1", mapper option words=1): the single-stream latency
 * path.  One stream, one signal per 32-bit shared-memory word (bit 0 = value,
 * bits 1-31 don't-care).  The bit-packed boomerang layer buys 32x
 * gates per instruction, which a batched or throughput-bound run needs; a
 * single stream is bound by the latency of the partition's logic chain
 * instead, and a word-level step -- every thread one or
 * more independent ANDs, one block barrier -- costs ~1/10 of a boomerang
 * layer while a layer advances the critical path by ~6 levels.  The program
 * is the partition's AND list list-scheduled (critical path first) into
 * barrier-separated steps of at most `word_step` ops; steps are stored
 * compactly (op i of step s at index step_start[s] + i; thread t runs ops
 * t, t + 256, ... of the step).
 *   header (WPH_*) | step starts [n_steps + 1] | ops [n_ops] uint2 |
 *   out dst gid [n_out] | out src [n_out][32] | ram [n_ram][4] | gread [n_gread]
 *   op: x = (a_byte | ia) | (b_byte | ib) << 16, y = dst_byte
 *       (a_byte, b_byte, dst_byte: word * 4 < 65536; ia / ib = operand
 *       inversion in bit 0 of the byte offset, which is 4-aligned)
 *       S[y] = (S[a] ^ ia) & (S[b] ^ ib)   (bit 0)
 *   out src: byte offset of the endpoint's word | inv (bit 0); bit k of
 *       output word o = (S[src[o][k] & ~3] ^ src[o][k]) & 1; a padding bit reads
 *       word 0 (constant 0)
 *   gread: region << 24 | global bit (word = bit >> 5); entry k -> word 1 + k
 *   ram: {ram_id, 0, 0, 0}, ports staged by outputs with region GEM_R_RAMP
 * Word 0 is the constant 0.  Words are allocated by liveness (a word last
 * read in step s is rewritten from step s + 1 on, after the barrier).       */
#define GEM_WORD_MAGIC 0x31445257u  /* "WRD1" */
#define GEM_WORD_MAX_WORDS 16384    /* byte offsets fit 16 bits */
enum {
  WPH_MAGIC = 0, WPH_N_GREAD, WPH_N_STEPS, WPH_N_OPS, WPH_N_OUT, WPH_N_RAM, WPH_STATE_WORDS, WPH_OFF_STEPS,
  WPH_OFF_OPS, WPH_OFF_OUT, WPH_OFF_RAM, WPH_OFF_GREAD, WPH_PROG_LEN, WPH_MAX_STEP_OPS, WPH_R14, WPH_R15,
  WPH_WORDS = 16
};
