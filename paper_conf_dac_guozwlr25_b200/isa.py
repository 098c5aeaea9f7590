"""Read-only view of a `.gemb` header (field names from csrc/gem_isa.h)."""
from __future__ import annotations

import dataclasses

import numpy as np

GH = ["MAGIC", "VERSION", "N_PI", "N_PO", "N_FLOPS", "N_RAMS", "N_PARTS", "N_STAGES",
      "MAX_STATE_WORDS", "MAX_LAYERS", "PI_WORDS", "PO_WORDS", "Q_WORDS", "CUT_WORDS",
      "N_AND_LO", "N_AND_HI", "N_AND_MAPPED_LO", "N_AND_MAPPED_HI", "TOTAL_LAYERS",
      "TOTAL_LEAVES_LO", "TOTAL_LEAVES_HI", "OFF_PARTS", "OFF_STAGES", "OFF_FLOP_INIT",
      "OFF_PROG", "PROG_WORDS_LO", "PROG_WORDS_HI", "MAX_LEVELS", "TOTAL_WRITEOUTS",
      "MAX_OUT", "TOTAL_WORDS_LO", "TOTAL_WORDS_HI", "SLOTS_USED_LO", "SLOTS_USED_HI",
      "MAX_CHUNK_WORDS", "MAX_PROG_WORDS", "HAS_LANES", "OFF_LANE_PROG", "LANE_PROG_WORDS_LO",
      "LANE_PROG_WORDS_HI", "LANE_MAX_CHUNK_WORDS", "LANE_MAX_WORDS", "MAX_RAMS_PART",
      "N_AND_SYNTH_LO", "N_AND_SYNTH_HI", "LEVELS_IN", "SYNTH_CHAINS",
      "HAS_WORDS", "OFF_WORD_PROG", "WORD_PROG_WORDS_LO", "WORD_PROG_WORDS_HI", "WORD_MAX_STATE",
      "WORD_MAX_PROG", "WORD_MAX_STEPS", "WORD_OPS_LO", "WORD_OPS_HI", "WORD_TOTAL_STEPS"]
GP_WORDS = 16   # csrc/gem_isa.h GP_WORDS
GEM_MAGIC = 0x424D4547
SLOTS_PER_LAYER = 8191


@dataclasses.dataclass
class BlobInfo:
    n_pi: int
    n_po: int
    n_flops: int
    n_rams: int
    n_parts: int
    n_stages: int
    max_state_words: int
    max_layers: int
    total_layers: int
    q_words: int
    po_words: int
    cut_words: int
    n_and: int
    n_and_mapped: int
    total_leaves: int
    max_levels: int
    program_bytes: int
    blob_bytes: int
    slots_used: int
    part_layers: list
    max_chunk_words: int = 0
    max_prog_words: int = 0
    part_cost: list = None
    part_stage: list = None
    n_and_synth: int = 0
    levels_in: int = 0
    synth_chains: int = 0
    lane_ops: int = 0          # LAN2 lane programs: AND ops over all partitions (0 otherwise)
    lane_steps: int = 0
    has_words: bool = False    # word programs (WRD1, the single-stream path)
    word_max_steps: int = 0    # steps of the deepest word program (the critical step chain)
    word_total_steps: int = 0
    word_ops: int = 0
    word_program_bytes: int = 0
    word_max_state: int = 0
    word_part_steps: list = None   # steps of each partition's word program

    def stage_max_word_steps(self) -> list:
        """Deepest word program (steps) of each stage: the critical step chain."""
        out = [0] * max(1, self.n_stages)
        for st, ns in zip(self.part_stage or [], self.word_part_steps or []):
            out[st] = max(out[st], ns)
        return out

    def stage_max_layers(self) -> list:
        """Deepest partition (layers) of each stage: a lower bound on the layers
        a cycle's critical path executes."""
        out = [0] * max(1, self.n_stages)
        for st, nl in zip(self.part_stage or [], self.part_layers):
            out[st] = max(out[st], nl)
        return out

    @property
    def replication(self) -> float:
        """RepCut replication over the synthesised graph."""
        return self.n_and_mapped / max(1, self.n_and_synth or self.n_and) - 1.0

    @property
    def synth_growth(self) -> float:
        """AND gates added by depth-oriented synthesis, relative."""
        return (self.n_and_synth or self.n_and) / max(1, self.n_and) - 1.0

    @property
    def slot_util(self) -> float:
        return self.n_and / max(1, self.total_layers * SLOTS_PER_LAYER)

    @property
    def bytes_per_and(self) -> float:
        return self.program_bytes / max(1, self.n_and)

    def as_dict(self) -> dict:
        d = dataclasses.asdict(self)
        d.pop("part_layers")
        d.pop("part_cost", None)
        d.pop("part_stage", None)
        d.pop("word_part_steps", None)
        d.update(replication=self.replication, synth_growth=self.synth_growth, slot_util=self.slot_util,
                 bytes_per_and=self.bytes_per_and,
                 levels_per_layer=self.max_levels / max(1, self.max_layers))
        return d


def blob_info(blob: bytes) -> BlobInfo:
    w = np.frombuffer(blob, dtype=np.uint32)
    h = {k: int(w[i]) for i, k in enumerate(GH)}
    if h["MAGIC"] != GEM_MAGIC:
        raise ValueError("not a .gemb blob")
    u64 = lambda k: h[k + "_LO"] | (h[k + "_HI"] << 32)
    np_ = h["N_PARTS"]
    pt = w[h["OFF_PARTS"]:h["OFF_PARTS"] + GP_WORDS * np_].reshape(np_, GP_WORDS)
    word_part_steps = []
    if h["HAS_WORDS"]:
        for p in range(np_):
            wp = h["OFF_WORD_PROG"] + int(pt[p, 15])
            word_part_steps.append(int(w[wp + 2]))
    lane_ops = lane_steps = 0
    if h["HAS_LANES"]:
        for p in range(np_):
            lp = h["OFF_LANE_PROG"] + int(pt[p, 9])
            if int(w[lp]) == 0x324E414C:   # "LAN2"
                lane_steps += int(w[lp + 2])
                lane_ops += int(w[lp + 12])
    return BlobInfo(n_pi=h["N_PI"], n_po=h["N_PO"], n_flops=h["N_FLOPS"], n_rams=h["N_RAMS"],
                    n_parts=np_, n_stages=h["N_STAGES"], max_state_words=h["MAX_STATE_WORDS"],
                    max_layers=h["MAX_LAYERS"], total_layers=h["TOTAL_LAYERS"], q_words=h["Q_WORDS"],
                    po_words=h["PO_WORDS"], cut_words=h["CUT_WORDS"], n_and=u64("N_AND"),
                    n_and_mapped=u64("N_AND_MAPPED"), total_leaves=u64("TOTAL_LEAVES"),
                    max_levels=h["MAX_LEVELS"], program_bytes=4 * u64("PROG_WORDS"),
                    blob_bytes=len(blob), slots_used=u64("SLOTS_USED"), part_layers=pt[:, 3].tolist(),
                    max_chunk_words=h["MAX_CHUNK_WORDS"], max_prog_words=h["MAX_PROG_WORDS"],
                    part_cost=pt[:, 8].tolist(), part_stage=pt[:, 0].tolist(),
                    n_and_synth=u64("N_AND_SYNTH"), levels_in=h["LEVELS_IN"], synth_chains=h["SYNTH_CHAINS"],
                    lane_ops=lane_ops, lane_steps=lane_steps, has_words=bool(h["HAS_WORDS"]),
                    word_max_steps=h["WORD_MAX_STEPS"], word_total_steps=h["WORD_TOTAL_STEPS"],
                    word_ops=u64("WORD_OPS"), word_program_bytes=4 * u64("WORD_PROG_WORDS"),
                    word_max_state=h["WORD_MAX_STATE"], word_part_steps=word_part_steps)
