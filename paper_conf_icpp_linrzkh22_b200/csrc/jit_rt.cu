// jit_rt.cu — device functions the JIT-generated partition kernels call
// (compiled to PTX at build time and prepended to every generated module):
// the generic any-width op path (variable wide shifts, rare cases) and the
// check-mode digest accumulation.
#include "device_ops.cuh"

using namespace rtlsim;

extern "C" __device__ __noinline__ void rtl_exec_wide(uint32_t *sm, const WideRec *rec, uint32_t lane) {
  exec_wide(sm, rec, lane);
}

// digest[s] ^= mix64(key << 32 | v) for the calling stimulus lane (check mode)
extern "C" __device__ __noinline__ void rtl_dig(unsigned long long *slot, uint32_t key, uint32_t v) {
  atomicXor(slot, mix64(((unsigned long long)key << 32) | v));
}
