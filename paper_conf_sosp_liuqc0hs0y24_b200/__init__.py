"""B200-native nested-recurrence wavefront (FractalTensor, SOSP'24 hot path).

The product is libft.so (C ABI, include/ft.h) built from csrc/ for sm_100a; `ft` is its thin
ctypes binding.  This package never imports oracle/ (the CPU test oracle).
"""
from . import ft  # noqa: F401
from .ft import dilated_rnn, grid_rnn, stacked_lstm, stacked_rnn  # noqa: F401
