"""paper_conf_dac_liuy25_b200 — B200-native exhaustive-simulation CEC hot path (Liu & Young, DAC 2025).

  capi      ctypes binding of include/cec.h (libcec.so: sm_100a kernels + C++ host driver)
  driver    host policy above the ABI: P/G/L routing by support size, cut enumeration (Eq. 1)
            for local checks, merge loop

The package never imports oracle/ (test infrastructure) and has no CPU compute fallback.
"""
from . import capi  # noqa: F401  (raises ImportError if libcec.so was not built)
from .capi import (  # noqa: F401
    CEC_BAD_CUT, CEC_EQUIVALENT, CEC_NO_CEX, CEC_NOT_EQUIVALENT, CEC_UNDECIDED, CecError, Context,
)
