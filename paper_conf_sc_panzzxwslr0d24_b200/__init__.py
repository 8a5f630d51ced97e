"""RecFlex hot path, B200-native: fused heterogeneous-schedule embedding-bag forward.

Submodules (imported lazily so that input generation does not load CUDA):
  synth   -- seeded synthetic inputs (shared with the tests' oracle side)
  _lib    -- ctypes binding of the C ABI in include/recflex.h (librecflex.so)
  plan    -- Python Plan wrapper (torch tensors in, same C-ABI names underneath)
  shard   -- table-wise sharding + pooled-output all-to-all (torch.distributed)
"""
__all__ = ['synth', 'plan', 'shard']
