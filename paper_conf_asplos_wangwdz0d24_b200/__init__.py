"""B200-native RAP fused DLRM input preprocessing (ASPLOS '24, Wang et al.).

The product is the C-ABI library ``librap.so`` (include/rap.h) built from
``csrc/``; :mod:`.rap` is its thin ctypes binding and :mod:`.synth` the seeded
synthetic workload generator.  There is no CPU fallback: importing
:mod:`.rap` without the built library raises.
"""
