// count_np.cu -- the counting kernels of ONE accumulator class NP
// (compiled once per NP in {1,2,4,8,16} with -DFSGC_NPV=NP; count.cu picks
// the kernel of a pass by its pattern count).
#include "count_dev.cuh"

#ifndef FSGC_NPV
#error "compile with -DFSGC_NPV=<1|2|4|8|16>"
#endif
#define FSGC_CAT2(a, b) a##b
#define FSGC_CAT(a, b) FSGC_CAT2(a, b)

// which: 0 vertex, 1 edge, 2 general core, 3 / 4 triangle core (warp / block
// tables), 5 / 6 the same on the Z-term path only
const void* FSGC_CAT(fsgc_np_kernel_, FSGC_NPV)(int which) {
    switch (which) {
        case 0: return (const void*)vertex_core_kernel<FSGC_NPV>;
        case 1: return (const void*)edge_fc_kernel<FSGC_NPV>;
        case 2: return (const void*)core_kernel<FSGC_NPV>;
        case 3: return (const void*)list_warp_kernel<1, FSGC_NPV>;
        case 4: return (const void*)list_block_kernel<1, FSGC_NPV>;
        case 5: return (const void*)list_warp_kernel<2, FSGC_NPV>;
        default: return (const void*)list_block_kernel<2, FSGC_NPV>;
    }
}

int FSGC_CAT(fsgc_np_init_, FSGC_NPV)() { return dev_consts_init(); }
