"""paper_conf_ppopp_xiaja20_b200 -- spec-k speculative FSM execution with parallel merge on B200.

The product is the C-ABI library ``libfsmspec.so`` (include/fsmspec.h) built from ``csrc/``;
``fsmspec`` is its thin ctypes binding and ``dist`` the multi-GPU shard merge over
torch.distributed.  Method: Xia, Jiang & Agrawal, PPoPP'20.
"""
from .fsmspec import FSM, FsmError, SymbolError, lookback_table, map_compose  # noqa: F401
