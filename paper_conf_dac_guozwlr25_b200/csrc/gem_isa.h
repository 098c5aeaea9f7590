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
#define GEM_MAX_STATE_WORDS 2048  /* 64 Kbit state (16-bit leaf indices) */
#define GEM_RAM_ABITS 13
#define GEM_RAM_WORDS 8192
#define GEM_MAX_RAMS_PER_PART 32

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

/* leaf entry: bits [0,16) = state bit index, bits [16,21) = leaf position */
#define GEM_LEAF(src, pos) ((uint32_t)(src) | ((uint32_t)(pos) << 16))

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
  GH_N_WORDS = 64
};

/* part table entry (4 words) */
enum { GP_STAGE = 0, GP_PROG_OFF, GP_PROG_LEN, GP_N_LAYERS, GP_WORDS = 4 };

/* partition program header (16 words) */
enum {
  PH_MAGIC = 0, PH_N_GREAD, PH_N_LAYERS, PH_N_OUT, PH_N_RAM, PH_STATE_WORDS, PH_OFF_GREAD,
  PH_OFF_LAYERS, PH_OFF_OUT, PH_OFF_RAM, PH_N_LEAVES, PH_N_NODES, PH_N_OUT_PAD, PH_R13,
  PH_R14, PH_R15, PH_WORDS = 16
};
#define GEM_PART_MAGIC 0x54524150u  /* "PART" */

/* layer header (16 words) followed by one record per active warp:
 *   wconst[4] = {wxa, wxb, wob, wwo}
 *   lane[32][4] = {xa, xb, ob, wo}         (uint4 per lane)
 *   leaves[n_iter][32]                      (lane-minor, coalesced)       */
enum {
  LH_WORDS_ = 0, LH_FLAGS, LH_TOPC, LH_TOPWO, LH_NITER0 /* ..LH_NITER0+7 */, LH_WORDS = 16
};
#define GEM_LF_USES_TOP 0x100u   /* flags bit 8; bits [0,8) = active warp mask */
#define GEM_WARP_REC_WORDS(n_iter) (4 + 32 * 4 + 32 * (n_iter))

/* output section: dst gid [n_out_pad] then src [n_out][32]
 * RAM section: per owned RAM 4 words {ram_id, 0, 0, 0}; its ports are staged by
 * outputs with region GEM_R_RAMP index = local*4 + port.                       */
