"""b2cl: OpenCL 1.2 memory objects, samplers and bulk copies, native on B200.

The product is the C-ABI shared library ``libb2cl.so`` (entry points declared
in ``include/b2cl_cl.h`` and ``include/b2cl_ext.h``), built from ``csrc/``.
``paper_conf_sc_kimdjjl15_b200.cl`` is the thin ctypes binding with the same
names.  Importing this package does not load the library; the first call
through ``cl`` does, and raises if the library is missing.
"""
