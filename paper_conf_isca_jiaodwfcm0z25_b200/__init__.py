"""B200-native CKKS Hybrid key-switching (the hot path of Neo, ISCA'25) behind a C-ABI.

libneo.so (csrc/, built for sm_100a by build.py) does all the arithmetic; neo.py is the
ctypes binding.  PyTorch provides device memory, streams and process groups only.
"""
from .neo import (Context, EvalKey, NeoError, neo_automorphism, neo_bconv, neo_hmult,  # noqa: F401
                  neo_hrot, neo_intt, neo_keyswitch, neo_ntt, neo_rescale, neo_tensor)
