"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This package holds NO arithmetic of the method (no data-usage, PCIe or
kernel-time math).  It only produces:

* skeleton descriptions (plain Python dicts: arrays, kernels, regions,
  per-(kernel, transformation) characteristics) shaped like the paper's
  workloads (HotSpot, SRAD, CFD, Stassuij, vector add; §IV-B,
  P:L153-167, and the vector-add example P:L57-59);
* candidate records (SoA ``skx, nx, ny, iters``) from a counter-based
  SplitMix64 generator, closed form per index so any shard regenerates its
  own slice.

Both ``oracle/oracle.py`` and ``paper_conf_ipps_boyermk13_b200`` marshal these
dicts into their OWN C structs independently.
"""
