"""B200-native MEM extraction (GPUMEM's hot path, Abu-Doleh et al., IPDPSW 2014).

Submodules:
  gpumem  - thin ctypes binding over the C ABI in include/gpumem.h (libgpumem.so);
            importing it fails loudly if the CUDA library is missing.
  dist    - one-process-per-GPU query sharding with NCCL gather (torch.distributed).
  synth   - seeded synthetic genome pairs (inputs only; no method arithmetic).

Nothing is imported eagerly so that `synth` is usable without the CUDA library.
"""
__all__ = ["gpumem", "dist", "synth"]
