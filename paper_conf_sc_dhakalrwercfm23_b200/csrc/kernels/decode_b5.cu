// decode_kernel<B> instantiation for B = 5
#include "decode_impl.cuh"

MX_DECODE_INSTANTIATE(5)
