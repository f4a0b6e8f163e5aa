"""DUET on B200: multi-branch inference after coarse-grained subgraph partitioning, scheduled
across CUDA-stream / GPU slots (BASELINE.json north_star).

The product is libduet.so (C ABI, include/duet.h); `duet` is its thin ctypes binding.
`workloads` / `inputs` only describe and generate seeded synthetic inputs.
"""
