"""Seeded synthetic inputs (netlists + stimuli) shared by the oracle and the CUDA path.

Holds no simulation arithmetic (task rule ③): only structure drawing and
serialisation.
"""
from .aig import AigBuilder, Netlist, RamBlock, write_eaig  # noqa: F401
from .netlists import build_config, build_c1, netlist_path  # noqa: F401
from .stimulus import stimulus, stimulus_streams, pack_bits, unpack_bits, splitmix64  # noqa: F401
