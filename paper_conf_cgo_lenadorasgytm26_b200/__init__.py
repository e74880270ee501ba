"""B200-native GRANII hot path (Lenadora et al., CGO'26).

Submodules:
  granii  -- ctypes binding of include/granii.h (libgranii.so; CUDA required)
  model   -- multi-layer driver (per-layer selection, training step)
  synth   -- seeded synthetic inputs (shared with the oracle tests)
  build   -- nvcc build of libgranii.so for sm_100a
The binding is imported lazily so `synth` and `build` work without the library.
"""
__all__ = ["granii", "model", "synth", "build"]
