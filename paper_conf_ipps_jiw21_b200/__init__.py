"""B200-native CTXBack: per-thread-block context save at a flashback-point and
restore-and-replay on resume (Ji & Wang, IPDPS 2021), for sm_100a.

The product is the C-ABI library ``libctxb.so`` (include/ctxb.h); this
package is its thin ctypes binding (argument marshalling only).  There is no
CPU fallback: importing the binding fails loudly when the library is absent.
"""
from .ctxb import *  # noqa: F401,F403
from .ctxb import __all__  # noqa: F401
