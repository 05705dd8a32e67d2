"""B200-native MPI-derived-datatype pack/unpack and GPU<->GPU non-contiguous
transfer (Wu et al., HPDC'16).  The product is libdt.so (C-ABI, include/dt.h);
``dt`` is its thin ctypes binding."""
from . import dt  # noqa: F401
from .dt import DTError, Type, from_recipe, pack, unpack  # noqa: F401
