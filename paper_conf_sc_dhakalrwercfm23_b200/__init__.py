"""B200-native multiplexed small-function runtime (Dhakal et al., SC-W 2023).

The product is libmx.so (include/mx.h): partitions = CUDA green contexts over
8-SM groups + HBM quota arenas, a C++ dispatcher per GPU, and sm_100a kernels
for the two invocation types (LLM greedy decode, IP-emulator MPNN). This
package is its thin ctypes binding (`mx`) plus reporting helpers.
"""
from . import mx  # noqa: F401
