// k_main_inst.cu -- one instantiation of the persistent kernel per translation
// unit, selected by -DRCM_KBPS=<min blocks per SM> -DRCM_KMB=<0 chain | 1 multi-batch | 2 leveled>.
// build.py compiles the variants in parallel and links them with rcm.cu, which
// looks the kernels up through the host accessors defined here.
#include "rcm_main.cuh"

#ifndef RCM_KBPS
#define RCM_KBPS 2
#endif
#ifndef RCM_KMB
#define RCM_KMB 0
#endif

#define RCM_CAT2(a, b, c) rcm_kmain_ptr_##a##_##b
#define RCM_CAT(a, b) RCM_CAT2(a, b, 0)

extern "C" const void* RCM_CAT(RCM_KBPS, RCM_KMB)() {
  return (const void*)rcm::k_main<RCM_KBPS, RCM_KMB>;
}
