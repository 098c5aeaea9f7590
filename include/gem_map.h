/* gem_map.h -- C ABI of libgemmap, the host-side GEM mapping flow.
 *
 * Maps a synchronous extended AIG (§III-A: ANDs, inverters,
 * D flip-flops, 13-bit x 32-bit RAM blocks) onto the virtual VLIW
 * Boolean processor: replication-aided partitioning (§III-C, P:103-125,
 * Algorithm 1), timing-driven boomerang-layer placement (§III-D,
 * P:127-156, Algorithm 2) and bitstream generation (§III-E).
 *
 * Input: a `.eaig` file = AIGER 1.9 (aag or aig) with `gem-ram` comment
 * records.  Output: a `.gemb` program blob
 * (layout in paper_conf_dac_guozwlr25_b200/csrc/gem_isa.h) for
 * gem_load_program().
 *
 * opts: space separated key=value pairs, e.g. "parts=148 stages=2 threads=8":
 *   partitioning: parts, part_size, max_parts, key, km1, km1_pins, km1_slack,
 *     merge, merge_cap, merge_ratio, refine, refine_ratio, stages (1|2),
 *     cut_level;
 *   synthesis: synth (0 strash, 1 + AND balancing, 2 + chain
 *     lookahead), chain_min, chain_slack;
 *   boomerang layers: levels, leafcap, max_warps, banks, max_state_words,
 *     cap_slack;
 *   lane programs (batched streams): lanes=1, lane_mode, lane_k, lane_m,
 *     lane_words, lane_banks, lane_holes;
 *   word programs (the single-stream path, gem_isa.h WRD1): words=1,
 *     word_step (ops per step, <= 1024), word_sched (1 balanced, 0 ASAP),
 *     word_fill, word_spread, word_chain_probe (analysis output only);
 *   threads, verbose.
 *   A blob gets word programs only if every partition's fits in 16K state
 *   words; the runtime then also needs them to fit in shared memory.
 *
 * Ownership: *blob is malloc'ed by the library; release with gem_free_blob().
 * Errors: 0 on success; -1 bad argument / unreadable file, -2 parse or mapping
 * failure, -4 out of memory; gem_map_last_error() gives a thread-local message.
 */
#ifndef GEM_MAP_H
#define GEM_MAP_H
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

int gem_compile(const void* eaig, size_t nbytes, const char* opts, void** blob, size_t* blob_bytes);
int gem_compile_file(const char* path, const char* opts, void** blob, size_t* blob_bytes);
void gem_free_blob(void* blob);
const char* gem_map_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* GEM_MAP_H */
