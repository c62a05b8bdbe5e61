"""es200 -- B200-native placement-invariant EST gradient aggregation
(EasyScale, SC '23).  See DESIGN.md.

  es          : ctypes binding of libes (include/es.h), same names as the C ABI
  aggregator  : torch-facing per-rank wrapper (workspace, streams, generator mirror)
  workloads   : seeded synthetic inputs (no method arithmetic)
"""
__all__ = ["es", "aggregator", "workloads"]
