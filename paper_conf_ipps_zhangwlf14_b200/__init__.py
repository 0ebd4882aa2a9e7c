"""B200-native (sm_100a) hot path of cuBLASTP: hit detection, two-hit filter and
X-drop ungapped extension behind the C-ABI libblastp.so (include/blastp.h).

``blastp``  -- ctypes binding (same names as the C-ABI)
``dist``    -- one process per GPU: subject-range shards + NCCL HSP gather
``build``   -- nvcc build of libblastp.so for sm_100a
``cli``     -- FASTA command line (queries x database -> HSP table)
"""
__all__ = ["blastp", "dist", "build", "cli"]
