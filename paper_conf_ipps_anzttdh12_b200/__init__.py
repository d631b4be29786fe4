"""paper_conf_ipps_anzttdh12_b200 — block-asynchronous relaxation async-(k) on B200 (sm_100a).

The product is ``libbar.so`` (C ABI in ``include/bar.h``, CUDA kernels in ``csrc/``);
``bar`` is its ctypes binding. Import ``paper_conf_ipps_anzttdh12_b200.bar`` to use it
(the import fails loudly if the library has not been built — there is no CPU path).
"""

__all__ = ["bar"]
