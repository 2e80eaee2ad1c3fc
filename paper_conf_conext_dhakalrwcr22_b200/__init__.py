"""paper_conf_conext_dhakalrwcr22_b200 -- B200-native batched ORB extraction + tracking
descriptor matching (the data-parallel hot path of SLAM-Share's GPU tracking, Dhakal et
al., CoNEXT'22, §4.2.1).

The product is libss.so (csrc/, C ABI in include/ss.h); ``ss`` is its ctypes binding and
``pipeline`` a torch-buffer convenience layer.  Nothing here imports ``oracle/``.
"""
from . import ss  # noqa: F401
from .ss import (SSError, ss_create, ss_destroy, ss_last_error, ss_match_projection,  # noqa: F401
                 ss_orb_extract, ss_orb_params_init)

__all__ = ["ss", "SSError", "ss_create", "ss_destroy", "ss_last_error", "ss_match_projection",
           "ss_orb_extract", "ss_orb_params_init"]
