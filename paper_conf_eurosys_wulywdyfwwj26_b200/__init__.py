"""B200-native GROUTER data-passing hot path (EuroSys '26, Wu et al.).

``libgrouter.so`` (C ABI in ``include/grouter.h``) + sm_100a kernels; this
package only holds the sources, the in-tree build and a thin ctypes binding
(``grouter``).  See DESIGN.md.
"""
from . import grouter  # noqa: F401

__all__ = ["grouter"]
