"""GEM (DAC'25) hot path, B200-native: mapper -> VLIW bitstream -> sm_100a interpreter.

  mapping.compile_file(eaig)  -> .gemb blob       (native C++ mapper)
  gem.Simulator(blob, ...)    -> libgem C-ABI     (CUDA sm_100a kernels)
"""
