"""B200-native IPsec ESP outbound hot path of NBA (EuroSys'15).

See DESIGN.md.  The compute path is libnba_ipsec.so (CUDA, sm_100a) behind the
C ABI in include/nba_ipsec.h; ``nba_ipsec`` is a thin ctypes binding.
"""
