"""paper_conf_sosp_songz0c23_b200 -- B200-native UGache factored embedding extraction.

The product is ``libugache.so`` (C ABI in ``include/ugache.h``, sm_100a kernels in
``csrc/``); this package is its thin Python binding:

* :mod:`._abi`   -- ctypes declarations, one per C entry point (same names);
* :mod:`.ugache` -- ``UGache`` (init / peers / fill / extract / stats), host-only
  ``solve`` / ``build_placement``;
* :mod:`.dist`   -- torch.distributed control plane (IPC-handle exchange, barriers);
* :mod:`.build`  -- nvcc build of the library (sm_100a).
"""
from .ugache import (UGache, build_placement, connect_in_process, fill_host_tier,  # noqa: F401
                     host_tier_rows, make_config, model_time, solve)

__all__ = ["UGache", "solve", "build_placement", "make_config", "connect_in_process",
           "fill_host_tier", "host_tier_rows", "model_time"]
